// pt_scene.h -- device image of a path-tracing scene (config 4), written by
// sr_scene_build (bvh.cpp) and read by the pathtrace kernels.
//
//   [PtHeader][PtNode x n_nodes][PtTri x n_tris][PtMat x n_mats]
//
// PtNode is a four-wide BVH node (128 bytes, two lines): its four children's
// boxes as rows of four (lo.x of children 0-3, lo.y, ..., hi.z -- one 128-bit
// load per row), then per child ref / count: ref >= 0 with count 0 = inner node
// index; count > 0 = leaf of `count` (1..8) triangles starting at `ref`;
// ref < 0 = empty slot (its box is empty, never hit).  The tree is the binary
// SAH tree collapsed: a node takes its two binary children and keeps opening
// the inner child of largest surface area until it has four (the wide BVH of
// Wald et al. 2008 / Ylitie et al. 2017), so a ray needs about half the
// dependent node fetches of the binary tree.  Triangles are stored in BVH
// order with the edge vectors precomputed (e1 = v1 - v0, e2 = v2 - v0,
// binary32, the same two subtractions the oracle performs) and their original
// index, which the closest-hit tie-break uses.
#pragma once
#include <cstdint>

namespace sr {

constexpr uint32_t kPtMagic = 0x34525054u;  // "TPR4"
constexpr uint32_t kPtWide = 4;             // children per node
constexpr uint32_t kPtLeafMax = 8;          // triangles per leaf
// a traversal-stack entry is an inner node index (>= 0) or a leaf, ~(first << 3 | (count - 1))
constexpr uint32_t kPtLeafFirstMax = 1u << 28;

struct PtHeader {
  uint32_t magic, n_nodes, n_tris, n_mats;
  uint64_t off_nodes, off_tris, off_mats, bytes;
  float cam[16];      // eye, forward, right, up, tan(fov/2), aspect
  uint32_t stack_need;  // deepest traversal stack any ray can need (entries)
  uint32_t pad[3];
};
static_assert(sizeof(PtHeader) == 128, "PtHeader layout");

struct PtNode {
  float lox[4], loy[4], loz[4], hix[4], hiy[4], hiz[4];
  int32_t ref[4], cnt[4];
};
static_assert(sizeof(PtNode) == 128, "PtNode layout");

struct PtTri {
  float v0[3], e1[3], e2[3];
  uint32_t id, mat, pad;
};
static_assert(sizeof(PtTri) == 48, "PtTri layout");

struct PtMat {
  float kind, r, g, b, er, eg, eb, ior;
};
static_assert(sizeof(PtMat) == 32, "PtMat layout");

}  // namespace sr
