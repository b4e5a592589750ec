// pt_scene.h -- device image of a path-tracing scene (config 4), written by
// sr_scene_build (bvh.cpp) and read by the pathtrace kernels.
//
//   [PtHeader][PtNode x n_nodes][PtTri x n_tris][PtMat x n_mats]
//
// PtNode holds BOTH children's boxes (one 64-byte line per visit, the
// two-wide layout of Aila & Laine; the boxes interleaved per axis): child ref >= 0 with count 0 = inner node
// index; count > 0 = leaf of `count` triangles starting at `ref`; count 0 and
// ref < 0 = empty slot.  Triangles are stored in BVH order with the edge
// vectors precomputed (e1 = v1 - v0, e2 = v2 - v0, binary32, the same two
// subtractions the oracle performs) and their original index, which the
// closest-hit tie-break uses.
#pragma once
#include <cstdint>

namespace sr {

constexpr uint32_t kPtMagic = 0x53525054u;  // "TPRS"

struct PtHeader {
  uint32_t magic, n_nodes, n_tris, n_mats;
  uint64_t off_nodes, off_tris, off_mats, bytes;
  float cam[16];      // eye, forward, right, up, tan(fov/2), aspect
  uint32_t stack_need;  // deepest traversal stack any ray can need (entries)
  uint32_t pad[3];
};
static_assert(sizeof(PtHeader) == 128, "PtHeader layout");

// lo[a][c] / hi[a][c]: child c's box on axis a -- the two children interleaved per
// axis, so one f32x2 operation computes an axis' slab distance for both children
struct PtNode {
  float lo[3][2], hi[3][2];
  int32_t ref0, cnt0, ref1, cnt1;
};
static_assert(sizeof(PtNode) == 64, "PtNode layout");

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
