// pathtrace.cu -- config 4: path tracer over a BVH scene (the paper's
// "pathtracer", Table 2; Russian roulette and bounded bounces,
// P:1377-1383), Loop Merge over the bounce loop (Fig. 2(b)), the
// samples per pixel being the coarsened outer loop:
//
//   for (s = 0; s < spp; s++) {                  // outer loop
//     Prolog: camera ray of sample s
//     for (b = 0; alive; b++) { L1: bounce() }   // divergent trip count
//     Epilog: pixel += radiance
//   }
//
//   pt_pdom  as written: a warp's 32 pixels trace sample s together; lanes
//            whose path ended idle until the longest path of the warp ends.
//   pt_spec  Loop Merge + soft barrier at one of three granularities:
//            bounce (SR_F_COARSE): P = ballot(path in flight); if popc(P) >= T
//              or no idle lane has a sample left, every in-flight lane takes
//              one bounce; otherwise idle lanes run the epilog and the next
//              camera ray;
//            node (SR_F_NOSPLIT): the same one nesting level deeper, one
//              release = merge_unroll BVH node visits;
//            split (default): two concurrent predictions --
//              lanes at an inner node and lanes with leaf triangles pending
//              are separate candidate sets; each round releases the larger
//              (soft barrier T), the other waits (Iteration Delay's vote,
//              P:1552-1557).
//
// One lane = one pixel (static; the pixel sum is accumulated in sample order,
// so the float result is schedule-free).  bounce() = BVH closest hit (exactly
// the brute-force closest hit, ties to the smaller triangle id; conservative
// padded-box slab test) + material shading, operation for operation as
// oracle/pathtrace.c (reading R7).
#include <cstring>
#include <mutex>
#include <utility>
#include <vector>

#include "pt_scene.h"
#include "sr_device.cuh"
#include "sr_internal.h"

namespace sr {
namespace {

constexpr float kTmin = 1.0e-4f;
constexpr float kDetEps = 1.0e-12f;
// traversal stack: one column of PtHeader.stack_need entries per thread in
// dynamic shared memory (23 for configs[3]); kMaxStack bounds what a scene may need
constexpr uint32_t kMaxStack = 256;
// CTAs of 128 threads per SM the register budget must allow, per kernel, each
// at its best measured setting (profiles/pt_tuning_r01.md): both latency-bound
// kernels want as many warps as fit.  With the ray kept once (Path.o/d, not
// copied into Trav) and the pixel sum accumulated in the output, 9 CTAs
// (56 registers, 32-40 B spilled) beat 8 (64 registers): SPEC 36.4 -> 35.6 ms,
// PDOM 67.8 -> 67.0 ms; 10 CTAs (48 registers, 64-80 B spilled) lose (37.5 / 71.2).
// (An L1 prefetch of the next node / triangle was measured 5 % slower.)
#ifndef SR_PT_MINB_PDOM
#define SR_PT_MINB_PDOM 9
#endif
#ifndef SR_PT_MINB_SPEC
#define SR_PT_MINB_SPEC 9
#endif

struct V3 {
  float x, y, z;
};
__device__ __forceinline__ V3 mk(float x, float y, float z) { return {x, y, z}; }
__device__ __forceinline__ V3 sub(V3 a, V3 b) { return mk(a.x - b.x, a.y - b.y, a.z - b.z); }
__device__ __forceinline__ V3 add(V3 a, V3 b) { return mk(a.x + b.x, a.y + b.y, a.z + b.z); }
__device__ __forceinline__ V3 scl(V3 a, float s) { return mk(a.x * s, a.y * s, a.z * s); }
__device__ __forceinline__ float dot(V3 a, V3 b) { return (a.x * b.x + a.y * b.y) + a.z * b.z; }
__device__ __forceinline__ V3 cross(V3 a, V3 b) {
  return mk(a.y * b.z - a.z * b.y, a.z * b.x - a.x * b.z, a.x * b.y - a.y * b.x);
}
__device__ __forceinline__ V3 normalize(V3 a) {
  const float inv = 1.0f / sqrtf(dot(a, a));
  return scl(a, inv);
}

struct PtArgs {
  const unsigned char* scene;
  const PtNode* nodes;
  const PtTri* tris;
  const PtMat* mats;
  uint32_t width, height, spp, max_depth, T;
  uint32_t unroll;                  // node visits per release (partial unroll)
  uint32_t stack_cap;               // traversal stack entries per thread (>= stack_need)
  uint64_t n, seed;
  RoundKeys keys;
#ifdef SR_BOUNDS_CHECK
  uint32_t n_nodes, n_tris, n_mats;
#endif
  float* rgb;                       // 3 floats per pixel
  float* prad;                      // POOL: 3 floats per (pixel, sample), pixel-major
  unsigned long long* counters;     // [0] paths [1] rays [2] node visits [3] tri tests
  uint32_t* sched;
  // diagnostics (sr_pt_closest): rays in, hits out
  const float* q_rays;
  int64_t* q_hit;
  float* q_t;
};

struct Stats {
  uint32_t rays, nodes, tests;
};

// Scene reads through the read-only data path as 128-bit loads (LDG.E.128.
// CONSTANT): a node is 4, a triangle 3, a material 2 vector loads instead of
// one scalar load per field (the structs are 4-byte aligned, so the compiler
// would not vectorise them itself; the image keeps every record 16-byte
// aligned: 128-byte header, 64-byte nodes, 48-byte triangles).
// sm_100 has 256-bit global loads: a node (64 bytes, 64-byte aligned in the image)
// is two LDG.E.256 instead of four LDG.E.128.
__device__ __forceinline__ void ldg256(const void* p, float4& a, float4& b) {
  asm("ld.global.nc.v8.f32 {%0, %1, %2, %3, %4, %5, %6, %7}, [%8];"
      : "=f"(a.x), "=f"(a.y), "=f"(a.z), "=f"(a.w), "=f"(b.x), "=f"(b.y), "=f"(b.z), "=f"(b.w)
      : "l"(p));
}
// Conservative slab test against a padded box: accept when the ray's
// parametric interval [tmin, tbest] can touch the box (slack 1e-5 relative).
// Callers evaluate it for both child slots unconditionally and AND the result
// with `slot is not empty` (no branch around the test: the box arithmetic is
// cheaper than the divergence bookkeeping of a short-circuit).
#ifdef SR_PT_BOX_BRANCH  // tuning variant: the short-circuit form
#define SR_PT_SLOT_TEST(REF, HIT) ((REF) >= 0 && (HIT))
#else
#define SR_PT_SLOT_TEST(REF, HIT) ((HIT) & ((REF) >= 0))
#endif

// A node visit's box half: both child boxes against the ray, the slab distances of
// the two children computed together -- the image interleaves the children per axis
// (pt_scene.h), so each (lo or hi, axis) is one FADD2 (x - o, o broadcast) and one
// FMUL2 (* 1/d, broadcast): 12 paired operations instead of 24 scalar ones, the same
// IEEE roundings.  Then per child the slab interval and the conservative accept test
// (box_hit's expressions, operand for operand).
struct NodeVisit {
  float tn0, tn1;
  bool h0, h1;        // child slot hit (ANDed with "slot not empty")
  int32_t ref0, cnt0, ref1, cnt1;
};
__device__ __forceinline__ uint64_t fmul2rn(uint64_t a, uint64_t b) {
  uint64_t d;  // feeds only min / max, so nothing can contract it into an FFMA2
  asm("mul.rn.f32x2 %0, %1, %2;" : "=l"(d) : "l"(a), "l"(b));
  return d;
}
__device__ __forceinline__ bool slab_accept(float tx0, float tx1, float ty0, float ty1, float tz0,
                                            float tz1, float tb, float& tnear) {
  const float tn = fmaxf(fmaxf(fminf(tx0, tx1), fminf(ty0, ty1)), fmaxf(fminf(tz0, tz1), 0.0f));
  const float tf = fminf(fminf(fmaxf(tx0, tx1), fmaxf(ty0, ty1)), fmaxf(tz0, tz1));
  tnear = tn;
  return tn * (1.0f - 1e-5f) <= tf * (1.0f + 1e-5f) && tn * (1.0f - 1e-5f) <= tb;
}
__device__ __forceinline__ NodeVisit visit_node(const PtNode* base, int32_t i, V3 o, V3 inv,
                                                float tb) {
  SR_CHECK(i >= 0);
  const float4* q = reinterpret_cast<const float4*>(base + i);
  float4 x, y, z, w;  // x: lo[0][*] lo[1][*]  y: lo[2][*] hi[0][*]  z: hi[1][*] hi[2][*]
  ldg256(q, x, y);
  ldg256(q + 2, z, w);
  const uint64_t nox = pack2(-o.x, -o.x), noy = pack2(-o.y, -o.y), noz = pack2(-o.z, -o.z);
  const uint64_t ix = pack2(inv.x, inv.x), iy = pack2(inv.y, inv.y), iz = pack2(inv.z, inv.z);
  float lx0, lx1, ly0, ly1, lz0, lz1, hx0, hx1, hy0, hy1, hz0, hz1;
  unpack2(fmul2rn(fadd2(pack2(x.x, x.y), nox), ix), lx0, lx1);
  unpack2(fmul2rn(fadd2(pack2(x.z, x.w), noy), iy), ly0, ly1);
  unpack2(fmul2rn(fadd2(pack2(y.x, y.y), noz), iz), lz0, lz1);
  unpack2(fmul2rn(fadd2(pack2(y.z, y.w), nox), ix), hx0, hx1);
  unpack2(fmul2rn(fadd2(pack2(z.x, z.y), noy), iy), hy0, hy1);
  unpack2(fmul2rn(fadd2(pack2(z.z, z.w), noz), iz), hz0, hz1);
  NodeVisit v;
  v.ref0 = __float_as_int(w.x); v.cnt0 = __float_as_int(w.y);
  v.ref1 = __float_as_int(w.z); v.cnt1 = __float_as_int(w.w);
  v.h0 = SR_PT_SLOT_TEST(v.ref0, slab_accept(lx0, hx0, ly0, hy0, lz0, hz0, tb, v.tn0));
  v.h1 = SR_PT_SLOT_TEST(v.ref1, slab_accept(lx1, hx1, ly1, hy1, lz1, hz1, tb, v.tn1));
  return v;
}
// The same visit with the 24 scalar FADD / FMUL (identical values).
__device__ __forceinline__ NodeVisit visit_node_scalar(const PtNode* base, int32_t i, V3 o, V3 inv,
                                                       float tb) {
  SR_CHECK(i >= 0);
  const float4* q = reinterpret_cast<const float4*>(base + i);
  float4 x, y, z, w;
  ldg256(q, x, y);
  ldg256(q + 2, z, w);
  NodeVisit v;
  v.ref0 = __float_as_int(w.x); v.cnt0 = __float_as_int(w.y);
  v.ref1 = __float_as_int(w.z); v.cnt1 = __float_as_int(w.w);
  v.h0 = SR_PT_SLOT_TEST(v.ref0, slab_accept((x.x - o.x) * inv.x, (y.z - o.x) * inv.x,
                                             (x.z - o.y) * inv.y, (z.x - o.y) * inv.y,
                                             (y.x - o.z) * inv.z, (z.z - o.z) * inv.z, tb, v.tn0));
  v.h1 = SR_PT_SLOT_TEST(v.ref1, slab_accept((x.y - o.x) * inv.x, (y.w - o.x) * inv.x,
                                             (x.w - o.y) * inv.y, (z.y - o.y) * inv.y,
                                             (y.y - o.z) * inv.z, (z.w - o.z) * inv.z, tb, v.tn1));
  return v;
}
__device__ __forceinline__ PtTri load_tri(const PtTri* base, int32_t i) {
  SR_CHECK(i >= 0);
  const float4* q = reinterpret_cast<const float4*>(base + i);
  const float4 x = __ldg(q), y = __ldg(q + 1);
  const uint4 z = __ldg(reinterpret_cast<const uint4*>(q + 2));
  PtTri t;
  t.v0[0] = x.x; t.v0[1] = x.y; t.v0[2] = x.z; t.e1[0] = x.w;
  t.e1[1] = y.x; t.e1[2] = y.y; t.e2[0] = y.z; t.e2[1] = y.w;
  t.e2[2] = __uint_as_float(z.x); t.id = z.y; t.mat = z.z; t.pad = z.w;
  return t;
}
__device__ __forceinline__ PtMat load_mat(const PtMat* base, uint32_t i) {
  const float4* q = reinterpret_cast<const float4*>(base + i);
  const float4 x = __ldg(q), y = __ldg(q + 1);
  PtMat m;
  m.kind = x.x; m.r = x.y; m.g = x.z; m.b = x.w;
  m.er = y.x; m.eg = y.y; m.eb = y.z; m.ior = y.w;
  return m;
}


// Moller-Trumbore exactly as the oracle (e1, e2 precomputed with the same
// binary32 subtractions).
// Branch-free form (the split merge's leaf releases, trav_leaf): every quantity
// computed, the four rejections folded into one predicate -- the same comparisons,
// so the same accepted hits and the same t.  A leaf release runs >= T lanes, so
// nearly every warp has a lane that passes each early-out test and pays the full
// test anyway; this drops the branches around it (merged kernel -1 %; the PDOM
// kernel, whose warps test triangles with fewer lanes, keeps the early-out form
// of trav_step, measured 1.6 % faster there; profiles/experiments.md).
__device__ __forceinline__ void tri_test_flat(const PtTri& T, int32_t at, V3 o, V3 d, float& tb,
                                              int32_t& ib, uint32_t& mb, uint32_t& slot) {
  const V3 v0 = mk(T.v0[0], T.v0[1], T.v0[2]);  // @sr-region TT
  const V3 e1 = mk(T.e1[0], T.e1[1], T.e1[2]);
  const V3 e2 = mk(T.e2[0], T.e2[1], T.e2[2]);
  const V3 pv = cross(d, e2);
  const float det = dot(e1, pv);
  const float inv = 1.0f / det;
  const V3 tv = sub(o, v0);
  const float u = dot(tv, pv) * inv;
  const V3 qv = cross(tv, e1);
  const float v = dot(d, qv) * inv;
  const float t = dot(e2, qv) * inv;
  const int32_t id = (int32_t)T.id;
  const bool ok = !(fabsf(det) < kDetEps) & !(u < 0.0f) & !(u > 1.0f) & !(v < 0.0f) &
                  !(u + v > 1.0f) & (t > kTmin) & ((t < tb) | ((t == tb) & (id < ib)));
  if (ok) {
    tb = t;  // @sr-region TT_UPD
    ib = id;
    mb = T.mat;
    slot = (uint32_t)at;
  }
}  // @sr-region END

__device__ __forceinline__ void tri_test(const PtTri& T, int32_t at, V3 o, V3 d, float& tb,
                                         int32_t& ib, uint32_t& mb, uint32_t& slot) {
  const V3 v0 = mk(T.v0[0], T.v0[1], T.v0[2]);  // @sr-region TT
  const V3 e1 = mk(T.e1[0], T.e1[1], T.e1[2]);
  const V3 e2 = mk(T.e2[0], T.e2[1], T.e2[2]);
  const V3 pv = cross(d, e2);
  const float det = dot(e1, pv);
  if (fabsf(det) < kDetEps) return;
  const float inv = 1.0f / det;  // @sr-region TT_U
  const V3 tv = sub(o, v0);
  const float u = dot(tv, pv) * inv;
  if (u < 0.0f || u > 1.0f) return;
  const V3 qv = cross(tv, e1);  // @sr-region TT_V
  const float v = dot(d, qv) * inv;
  if (v < 0.0f || u + v > 1.0f) return;
  const float t = dot(e2, qv) * inv;  // @sr-region TT_T
  if (!(t > kTmin)) return;
  const int32_t id = (int32_t)T.id;  // < 2^31 (sr_scene_build checks)  // @sr-region TT_ID
  if (t < tb || (t == tb && id < ib)) {   // ties -> smaller original id (= brute force)
    tb = t;  // @sr-region TT_UPD
    ib = id;
    mb = T.mat;
    slot = (uint32_t)at;
  }
}  // @sr-region END

// Resumable BVH traversal: one call of trav_step visits one node (its two
// child boxes, the triangles of child leaves, push/pop).  closest_hit() runs
// it to completion; the node-granularity Loop Merge kernel interleaves single
// steps of different lanes' rays.
//
// The traversal stack lives in shared memory, one column per thread
// (entry i of thread t at smem[i * blockDim + t]: consecutive lanes hit
// consecutive banks), so the per-lane traversal state that stays in
// registers is small and the node fetches have L1 to themselves.
struct Trav {
  V3 inv;           // the ray itself (origin, direction) is the caller's (Path.o, Path.d)
  float tb;
  int32_t ib;       // original index of the closest triangle so far (-1: none)
  uint32_t mb, slot;
  int32_t node;
  int32_t sp;
  // split merge (default): leaf ranges found by the last node visit, tested later by
  // trav_leaf (current range la/na, queued range lb/nb)
  int32_t la, lb;
  uint32_t na, nb;
};

extern __shared__ int32_t pt_stack_smem[];
// entry i of this thread's stack column (addressed from threadIdx / blockDim,
// so no per-lane pointer is kept in registers)
__device__ __forceinline__ int32_t& stk(int32_t i) {
  SR_CHECK(i >= 0 && (uint32_t)i < kMaxStack);
  return pt_stack_smem[(uint32_t)i * blockDim.x + threadIdx.x];
}

__device__ __forceinline__ void trav_begin(Trav& tr, V3 d) {
  tr.inv = mk(1.0f / d.x, 1.0f / d.y, 1.0f / d.z);
  tr.tb = INFINITY;
  tr.ib = -1;
  tr.mb = 0;
  tr.slot = 0;
  tr.node = 0;
  tr.sp = 0;
  tr.na = 0;
  tr.nb = 0;
}

// returns false when the traversal is finished
__device__ __forceinline__ bool trav_step(const PtArgs& a, Trav& tr, V3 o, V3 d, Stats& st) {
  SR_CHECK((uint32_t)tr.node < a.n_nodes);
  const NodeVisit N = visit_node(a.nodes, tr.node, o, tr.inv, tr.tb);  // @sr-region NODE
  ++st.nodes;
  const float tn0 = N.tn0, tn1 = N.tn1;
  const bool h0 = N.h0, h1 = N.h1;
  // leaves: test their triangles now (child 0's, then child 1's, one loop);
  // inner children: descend / push
  const int32_t n0 = (h0 && N.cnt0 > 0) ? N.cnt0 : 0, n1 = (h1 && N.cnt1 > 0) ? N.cnt1 : 0;
#pragma unroll 1  // one triangle test per trip (the simulator's LEAF count)
  for (int32_t k = 0; k < n0 + n1; ++k) {  // @sr-region LEAFIF
    const int32_t at = k < n0 ? N.ref0 + k : N.ref1 + (k - n0);  // @sr-region LEAF
    tri_test(load_tri(a.tris, at), at, o, d, tr.tb, tr.ib, tr.mb, tr.slot);
    ++st.tests;
  }
  const bool in0 = h0 && N.cnt0 == 0, in1 = h1 && N.cnt1 == 0;  // @sr-region NODE
  int32_t next = -1;
  if (in0 && in1) {
    const bool first0 = tn0 <= tn1;  // @sr-region PUSH
    next = first0 ? N.ref0 : N.ref1;
    if ((uint32_t)tr.sp < a.stack_cap) stk(tr.sp++) = first0 ? N.ref1 : N.ref0;
  } else if (in0) {
    next = N.ref0;  // @sr-region NOPUSH
  } else if (in1) {
    next = N.ref1;
  }
  if (next < 0) {  // @sr-region NODE
    if (tr.sp == 0) return false;  // @sr-region NEXTNONE
    next = stk(--tr.sp);  // @sr-region POP
  }
  tr.node = next;  // @sr-region NODE
  return true;
}  // @sr-region END

// Split merge (default): trav_step cut into its two regions, each lane's sequence of
// node visits and triangle tests unchanged.  trav_node visits tr.node: box
// tests, queues the hit leaf children (child 0 first) for trav_leaf, picks
// the next node exactly as trav_step (node = -1 when the stack is empty).
// trav_leaf tests ONE queued triangle.  Returns: a leaf triangle is pending
// (na > 0), else a node is pending (node >= 0), else the traversal is done.
// PAIRED: the f32x2 box tests (visit_node) or the scalar ones (visit_node_scalar);
// each kernel takes the form measured faster for it (the path pool: scalar;
// SR_PT_POOL_PAIRED, a tuning variant, gives it the paired form too).
#ifdef SR_PT_POOL_PAIRED
constexpr bool kPairedAlways = true;
#else
constexpr bool kPairedAlways = false;
#endif
template <bool PAIRED>
__device__ __forceinline__ void trav_node(const PtArgs& a, Trav& tr, V3 o, Stats& st) {
  SR_CHECK((uint32_t)tr.node < a.n_nodes);
  const NodeVisit N = PAIRED ? visit_node(a.nodes, tr.node, o, tr.inv, tr.tb)  // @sr-region NODE
                             : visit_node_scalar(a.nodes, tr.node, o, tr.inv, tr.tb);
  ++st.nodes;
  const float tn0 = N.tn0, tn1 = N.tn1;
  const bool h0 = N.h0, h1 = N.h1;
  const bool l0 = h0 && N.cnt0 > 0, l1 = h1 && N.cnt1 > 0;
  tr.la = l0 ? N.ref0 : N.ref1;
  tr.na = l0 ? (uint32_t)N.cnt0 : (l1 ? (uint32_t)N.cnt1 : 0u);
  tr.lb = N.ref1;
  tr.nb = (l0 && l1) ? (uint32_t)N.cnt1 : 0u;
  const bool in0 = h0 && N.cnt0 == 0, in1 = h1 && N.cnt1 == 0;
  int32_t next = -1;
  if (in0 && in1) {
    const bool first0 = tn0 <= tn1;  // @sr-region PUSH
    next = first0 ? N.ref0 : N.ref1;
    if ((uint32_t)tr.sp < a.stack_cap) stk(tr.sp++) = first0 ? N.ref1 : N.ref0;
  } else if (in0) {
    next = N.ref0;  // @sr-region NOPUSH
  } else if (in1) {
    next = N.ref1;
  }
  if (next < 0) {  // @sr-region NODE
    if (tr.sp > 0) next = stk(--tr.sp);  // @sr-region POP
  }
  tr.node = next;  // @sr-region NODE
}  // @sr-region END

__device__ __forceinline__ void trav_leaf(const PtArgs& a, Trav& tr, V3 o, V3 d, Stats& st) {
#ifdef SR_PT_TT_BRANCH  // tuning variant: the early-out test of trav_step
  tri_test(load_tri(a.tris, tr.la), tr.la, o, d, tr.tb, tr.ib, tr.mb, tr.slot);  // @sr-region LEAF
#else
  SR_CHECK((uint32_t)tr.la < a.n_tris);
  tri_test_flat(load_tri(a.tris, tr.la), tr.la, o, d, tr.tb, tr.ib, tr.mb, tr.slot);  // @sr-region LEAF
#endif
  ++st.tests;
  ++tr.la;
  if (--tr.na == 0u) {
    tr.la = tr.lb;
    tr.na = tr.nb;
    tr.nb = 0u;
  }
}  // @sr-region END

// SYNC (the PDOM kernel): the lanes of `mask` run the traversal loop together and
// reconverge at its latch every trip -- the loop's immediate post-dominator --
// instead of letting independent thread scheduling split the warp inside it.
template <bool SYNC>
__device__ __forceinline__ int64_t closest_hit(const PtArgs& a, Trav& tr, V3 o, V3 d, Stats& st,
                                               uint32_t mask = 0u) {
  trav_begin(tr, d);  // @sr-region TBEGIN
  if constexpr (SYNC) {
    bool more = true;
    while (__any_sync(mask, more)) {  // @sr-region STEP
      if (more) more = trav_step(a, tr, o, d, st);
    }
  } else {
    while (trav_step(a, tr, o, d, st)) {  // @sr-region STEP
    }
  }
  return (int64_t)tr.ib;  // @sr-region BOUNCE
}  // @sr-region END

struct Path {
  V3 o, d, thr, rad;   // the pixel sum lives in a.rgb (this lane's pixel only)
  uint32_t pix, s, b;
  bool alive;
};


// The pixel of lane slot i (thread g, or slot g&~31 + k of a warp's path pool): when
// the frame splits into 8 x 4 tiles, warp w = i / 32 covers tile w (tiles row-major,
// lanes row-major inside the tile), so a warp's camera rays leave from a compact
// patch rather than 32 pixels of one row (both kernels ~4 % faster at configs[3];
// profiles/experiments.md); other frames keep i.  inputs.pt_lane_pixels states the
// same map for the simulator.  SR_PT_ROWS (tuning variant): always i.
__device__ __forceinline__ uint32_t pix_of(const PtArgs& a, uint32_t i) {
#ifndef SR_PT_ROWS
  if ((a.width & 7u) == 0u && (a.height & 3u) == 0u) {
    const uint32_t w = i >> 5, l = i & 31u, tpr = a.width >> 3;
    return ((w / tpr) * 4u + (l >> 3)) * a.width + (w % tpr) * 8u + (l & 7u);
  }
#endif
  return i;
}

__device__ __forceinline__ void camera_ray(const PtArgs& a, const PtHeader& H, Path& p) {
  const uint64_t q = (uint64_t)p.pix * a.spp + p.s;  // @sr-region LAUNCH
  const uint4 u = draw(0u, kTagPt, q, a.keys);
  const uint32_t px = p.pix % a.width, py = p.pix / a.width;
  const float fx = ((float)px + u01(u.x)) / (float)a.width;
  const float fy = ((float)py + u01(u.y)) / (float)a.height;
  const float tan_half = H.cam[12], aspect = H.cam[13];
  const float sx = (2.0f * fx - 1.0f) * tan_half * aspect;
  const float sy = (1.0f - 2.0f * fy) * tan_half;
  const V3 fwd = mk(H.cam[3], H.cam[4], H.cam[5]);
  const V3 right = mk(H.cam[6], H.cam[7], H.cam[8]);
  const V3 up = mk(H.cam[9], H.cam[10], H.cam[11]);
  p.d = normalize(add(add(fwd, scl(right, sx)), scl(up, sy)));
  p.o = mk(H.cam[0], H.cam[1], H.cam[2]);
  p.thr = mk(1.0f, 1.0f, 1.0f);
  p.rad = mk(0.0f, 0.0f, 0.0f);
  p.b = 0;
  p.alive = true;
}  // @sr-region END

__device__ __forceinline__ void onb(V3 n, V3& t1, V3& t2) {
  const float sign = copysignf(1.0f, n.z);
  const float a = -1.0f / (sign + n.z);
  const float b = n.x * n.y * a;
  t1 = mk(1.0f + sign * n.x * n.x * a, sign * b, -sign * n.x);
  t2 = mk(b, sign + n.y * n.y * a, -n.y);
}

// The shading half of a bounce, after the closest hit of ray (p.o, p.d) is
// known (tr finished).  Ends the path when it escaped, hit a light, reached
// max_depth or lost the roulette; the epilog (pixel sum) happens at that
// point, in sample order.
// POOL: a pixel's samples run on several lanes, so each path's radiance is stored
// at (pixel, sample) and the pixel sum is formed after the warp's pool is done.
template <bool POOL = false>
__device__ void shade(const PtArgs& a, Path& p, const Trav& tr) {
  const int64_t hit = tr.ib;  // @sr-region SH
  const float t = tr.tb;
  const uint32_t mat = tr.mb, slot = tr.slot;
  bool end = hit < 0;
  if (!end) {
    SR_CHECK(mat < a.n_mats && slot < a.n_tris);
    const PtMat m = load_mat(a.mats, mat);  // @sr-region SH_HIT
    const uint32_t kind = (uint32_t)m.kind;
    p.rad = add(p.rad, mk(p.thr.x * m.er, p.thr.y * m.eg, p.thr.z * m.eb));
    if (kind == 3u) {
      end = true;
    } else {
      const PtTri T = load_tri(a.tris, (int32_t)slot);  // @sr-region SH_SURF
      const V3 e1 = mk(T.e1[0], T.e1[1], T.e1[2]);
      const V3 e2 = mk(T.e2[0], T.e2[1], T.e2[2]);
      const V3 ng = normalize(cross(e1, e2));
      const float cosd = dot(ng, p.d);
      const bool entering = cosd < 0.0f;
      const V3 n = entering ? ng : scl(ng, -1.0f);
      const V3 pt = add(p.o, scl(p.d, t));
      const uint64_t q = (uint64_t)p.pix * a.spp + p.s;
      const uint4 u = draw(p.b + 1u, kTagPt, q, a.keys);
      if (kind == 0u) {
        const float r1 = u01(u.x);  // @sr-region SH_DIFF
        const float rr = sqrtf(r1);
        float sp, cp;
        sr_sincos2pif(u01(u.y), sp, cp);
        const float lx = rr * cp, ly = rr * sp, lz = sqrtf(1.0f - r1);
        V3 t1, t2;
        onb(n, t1, t2);
        p.d = add(add(scl(t1, lx), scl(t2, ly)), scl(n, lz));
      } else if (kind == 1u) {
        p.d = sub(p.d, scl(n, 2.0f * dot(p.d, n)));  // @sr-region SH_MIRR
      } else {
        const float ior = m.ior;  // @sr-region SH_GLASS
        const float eta = entering ? 1.0f / ior : ior;
        const float cosi = -dot(p.d, n);
        const float k = 1.0f - eta * eta * (1.0f - cosi * cosi);
        float r0 = (1.0f - ior) / (1.0f + ior);
        r0 = r0 * r0;
        const float c5 = 1.0f - cosi;
        const float fr = r0 + (1.0f - r0) * (c5 * c5 * c5 * c5 * c5);
        if (k < 0.0f || u01(u.z) < fr) p.d = sub(p.d, scl(n, 2.0f * dot(p.d, n)));
        else p.d = add(scl(p.d, eta), scl(n, eta * cosi - sqrtf(k)));
      }
      p.thr = mk(p.thr.x * m.r, p.thr.y * m.g, p.thr.z * m.b);  // @sr-region SH_SURF
      p.o = pt;
      if (p.b >= 3u) {
        const float pm = fmaxf(p.thr.x, fmaxf(p.thr.y, p.thr.z));  // @sr-region SH_RR
        const float prr = fminf(0.95f, pm);
        if (!(u01(u.w) < prr)) end = true;
        else p.thr = mk(p.thr.x / prr, p.thr.y / prr, p.thr.z / prr);
      }
    }
  }
  p.b = p.b + 1u;  // @sr-region SH
  if (!end && p.b >= a.max_depth) end = true;
  if (end) {
    // Epilog: pixel += radiance, in sample order, in the output itself (a lane owns
    // its pixel; one read-modify-write per path keeps three registers free)
    if constexpr (POOL) {
      float* pr = a.prad + 3 * ((uint64_t)p.pix * a.spp + p.s);  // @sr-region SH_END
      pr[0] = p.rad.x;
      pr[1] = p.rad.y;
      pr[2] = p.rad.z;
    } else {
      float* px = a.rgb + 3 * (uint64_t)p.pix;  // @sr-region SH_END
      px[0] = px[0] + p.rad.x;
      px[1] = px[1] + p.rad.y;
      px[2] = px[2] + p.rad.z;
    }
    p.alive = false;
  }
}  // @sr-region END

__device__ __forceinline__ void finish(const PtArgs& a, const Path& p, bool valid, Stats st,
                                       uint32_t paths, uint64_t warp, uint32_t rounds,
                                       uint32_t rel, uint32_t rel_lanes, uint32_t adv,
                                       uint32_t adv_lanes, uint32_t lrel = 0,
                                       uint32_t lrel_lanes = 0) {
  unsigned long long v[4] = {paths, st.rays, st.nodes, st.tests};  // @sr-region ENTRY:full
#pragma unroll
  for (int i = 0; i < 4; ++i) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v[i] += __shfl_xor_sync(kFull, v[i], o);
  }
  if (lane_id() == 0) {
#pragma unroll
    for (int i = 0; i < 4; ++i) atomicAdd(&a.counters[i], v[i]);
    if (a.sched) {
      uint4* s = reinterpret_cast<uint4*>(a.sched + warp * kSchedWords);
      s[0] = make_uint4(rounds, rel, rel_lanes, adv);
      s[1] = make_uint4(adv_lanes, lrel, lrel_lanes, 0u);
    }
  }
}  // @sr-region END

__device__ __forceinline__ void bounce(const PtArgs& a, Path& p, Trav& tr, Stats& st,
                                       uint32_t mask) {
  closest_hit<true>(a, tr, p.o, p.d, st, mask);  // @sr-region BOUNCE
  ++st.rays;
  shade(a, p, tr);
}  // @sr-region END

template <bool SCHED>
__global__ void __launch_bounds__(SR_PT_MAXT, SR_PT_MINB_PDOM) pt_pdom(const PtArgs a) {
  const PtHeader& H = *reinterpret_cast<const PtHeader*>(a.scene);  // @sr-region ENTRY:full
  const uint64_t g = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const bool valid = g < a.n;
  Path p;
  p.pix = valid ? pix_of(a, (uint32_t)g) : 0u;
  if (valid) {
    float* px = a.rgb + 3 * (uint64_t)p.pix;
    px[0] = 0.0f; px[1] = 0.0f; px[2] = 0.0f;
  }
  p.alive = false;
  Trav tr;
  Stats st{0, 0, 0};
  uint32_t paths = 0, outer = 0, rel = 0, rel_lanes = 0, launch_lanes = 0;
  for (uint32_t s = 0; s < a.spp; ++s) {  // @sr-region OUTER:full
    if (SCHED) { ++outer; launch_lanes += __popc(__ballot_sync(kFull, valid)); }
    if (valid) {
      p.s = s;  // @sr-region LAUNCH
      camera_ray(a, H, p);              // Prolog
      ++paths;
    }
    // L1: the bounce loop, divergent trip count; every bounce reconverges at the
    // loop latch (its immediate post-dominator), as the traversal loop inside does
    uint32_t A = __ballot_sync(kFull, valid);  // @sr-region OUTER:full
    while (A != 0u) {  // @sr-region BOUNCE
      if constexpr (SCHED) { ++rel; rel_lanes += __popc(A); }
      if ((A >> lane_id()) & 1u) bounce(a, p, tr, st, A);
      A = __ballot_sync(kFull, valid && p.alive);  // @sr-region BOUNCE
    }                                   // IPDOM: reconverge, next sample  // @sr-region OUTER:full
  }
  uint32_t r = rel, rl = rel_lanes;  // @sr-region ENTRY:full
  finish(a, p, valid, st, paths, g >> 5, outer, r, rl, outer, launch_lanes);
}

// Loop Merge.  NODE = false: the merged inner loop is the bounce loop (one
// release = one whole bounce: traversal + shading).  NODE = true: the merged
// inner loop is the BVH traversal itself (one release = one node visit for
// every lane with a ray in flight); shading, the pixel epilog and the next
// camera ray form the advance step.  The second is Loop Merge applied one
// nesting level deeper (P:1514-1528 leaves nesting open), where the trip
// count (nodes per ray) varies most.  SPLIT (with NODE): the node visit's
// leaf triangle tests become their own region (trav_node / trav_leaf).
// MATG (with SPLIT, SR_F_MATGROUP): NEXT-3's same-material grouping
// of the shading step -- the lanes of R that must shade a hit
// are grouped by material kind with __match_any_sync; the largest group shades
// in this advance round (ties: the group of the lowest lane), the others wait
// in R for a later one.  A miss forms its own group.
// POOL (with SPLIT, SR_F_POOL): the warp's nv pixels x spp samples form one pool of
// paths, path q = sample q / nv of pixel q % nv; a lane whose path has ended claims
// the next one in an advance round (idle lanes in lane order), so no lane idles
// while the warp has paths left -- the fixed-pixel kernel keeps a lane on its own
// pixel's spp paths and the warp runs until the pixel with the most work is done.
// Each path's radiance goes to a.prad; the pixel sums are formed at the end in
// sample order (the same additions as the fixed-pixel epilog).
template <bool SCHED, bool NODE, bool SPLIT = false, bool MATG = false, bool POOL = false>
__global__ void __launch_bounds__(SR_PT_MAXT, SR_PT_MINB_SPEC) pt_spec(const PtArgs a) {
  const PtHeader& H = *reinterpret_cast<const PtHeader*>(a.scene);  // @sr-region ENTRY:full
  const uint64_t g = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const bool valid = g < a.n;
  Path p;
  p.pix = valid ? pix_of(a, (uint32_t)g) : 0u;
  if (!POOL && valid) {
    float* px = a.rgb + 3 * (uint64_t)p.pix;
    px[0] = 0.0f; px[1] = 0.0f; px[2] = 0.0f;
  }
  p.alive = false;
  p.s = 0;
  Trav tr;
  bool trav = false;                   // NODE: a ray of this lane is being traversed
  Stats st{0, 0, 0};
  uint32_t paths = 0, rounds = 0, rel = 0, rel_lanes = 0, adv = 0, adv_lanes = 0;
  uint32_t next_s = 0;                 // fixed pixel: this lane's next sample; POOL: the
                                       // warp's next unclaimed path (warp-uniform)
  // POOL: every lane of the warp takes paths, of the nv valid pixels
  const uint32_t nv = POOL ? (uint32_t)__popc(__ballot_sync(kFull, valid)) : 0u;
  const uint32_t pool = nv * a.spp;
  // lanes with nothing left to do
  uint32_t E = POOL ? 0u : __ballot_sync(kFull, !valid || a.spp == 0);
  uint32_t lrel = 0, lrel_lanes = 0;
  for (;;) {  // @sr-region ROUND:full
    if constexpr (SPLIT) {
      // two concurrent predictions: I = lanes at a BVH node, L = lanes with a
      // leaf triangle pending.  Vote: the larger group G is the candidate
      // release (soft barrier T); the other group waits (Iteration Delay).
      const uint32_t L = __ballot_sync(kFull, trav && tr.na > 0u);
      const uint32_t I = __ballot_sync(kFull, trav && tr.na == 0u);
      const uint32_t R = ~(I | L | E);
      if ((I | L | R) == 0u) break;
      if constexpr (SCHED) ++rounds;
      const bool leaf = __popc(L) > __popc(I);
      const uint32_t G = leaf ? L : I;
      if (G != 0u && ((uint32_t)__popc(G) >= a.T || R == 0u)) {
        if constexpr (SCHED) {  // warp-uniform release counters (every lane keeps them)
          if (leaf) { ++lrel; lrel_lanes += __popc(G); }
          else { ++rel; rel_lanes += __popc(G); }
        }
        if ((G >> lane_id()) & 1u) {
          __syncwarp(G);  // @sr-region REL
          if (leaf) {
            for (uint32_t k = 0; k < a.unroll && tr.na > 0u; ++k) trav_leaf(a, tr, p.o, p.d, st);  // @sr-region LEAF
          } else {
            for (uint32_t k = 0; k < a.unroll && tr.na == 0u && tr.node >= 0; ++k)  // @sr-region STEP
              trav_node<kPairedAlways || !POOL>(a, tr, p.o, st);
          }
          trav = tr.na > 0u || tr.node >= 0;  // @sr-region REL
        }
        continue;  // @sr-region ROUND:full
      }
      if constexpr (SCHED) { ++adv; adv_lanes += __popc(R); }  // @sr-region ADV:full
      bool go = (R >> lane_id()) & 1u;
      if constexpr (MATG) {
        const bool needs = go && p.alive;   // a finished traversal whose hit must be shaded
        if (__ballot_sync(kFull, needs) != 0u) {
          const uint32_t key = !needs ? 0xFFFFFFFFu
                             : (tr.ib < 0 ? 4u : (uint32_t)__ldg(&a.mats[tr.mb].kind));
          const uint32_t grp = __match_any_sync(kFull, key);
          // largest group, ties to the lowest lane: maximise (size << 5) | (31 - lowest lane)
          const uint32_t score = needs ? ((uint32_t)__popc(grp) << 5) | (31u - (__ffs(grp) - 1u)) : 0u;
          const uint32_t best = __reduce_max_sync(kFull, score);
          go = go && (!needs || score == best);
        }
      }
      if constexpr (POOL) {
        if (go && p.alive) shade<true>(a, p, tr);  // @sr-region ADV
        // claims: the lanes of R without a path take the next ones, in lane order
        const bool need = go && !p.alive;  // @sr-region ADV:full
        const uint32_t C = __ballot_sync(kFull, need);
        const uint32_t q = next_s + (uint32_t)__popc(C & lanemask_lt());
        if (need && q < pool) {
          p.pix = pix_of(a, (uint32_t)(g & ~31ull) + (nv == 32u ? (q & 31u) : q % nv));  // @sr-region LAUNCH
          p.s = nv == 32u ? (q >> 5) : q / nv;
          camera_ray(a, H, p);
          ++paths;
        }
        next_s = min(pool, next_s + (uint32_t)__popc(C));  // @sr-region ADV:full
        if (go && p.alive) {  // @sr-region ADV
          trav_begin(tr, p.d);  // @sr-region TBEGIN
          ++st.rays;
          trav = true;
        }
        E = __ballot_sync(kFull, !p.alive && next_s >= pool);  // @sr-region ADV:full
        continue;
      }
      if (go) {
        if (p.alive) shade(a, p, tr);  // @sr-region ADV
        if (!p.alive && next_s < a.spp) {
          p.s = next_s++;  // @sr-region LAUNCH
          camera_ray(a, H, p);
          ++paths;
        }
        if (p.alive) {  // @sr-region ADV
          trav_begin(tr, p.d);  // @sr-region TBEGIN
          ++st.rays;
          trav = true;
        }
      }
      E = __ballot_sync(kFull, !valid || (!p.alive && next_s >= a.spp));  // @sr-region ADV:full
      continue;
    }
    const uint32_t P = __ballot_sync(kFull, NODE ? trav : p.alive);  // @sr-region ROUND:full
    const uint32_t R = ~(P | E);
    if ((P | R) == 0u) break;
    if constexpr (SCHED) ++rounds;
    if ((uint32_t)__popc(P) >= a.T || R == 0u) {
      if constexpr (SCHED) { ++rel; rel_lanes += __popc(P); }
      if ((P >> lane_id()) & 1u) {
        __syncwarp(P);
        if constexpr (NODE) {
          for (uint32_t k = 0; k < a.unroll && trav; ++k) trav = trav_step(a, tr, p.o, p.d, st);
        }
        else bounce(a, p, tr, st, P);
      }
    } else {
      if constexpr (SCHED) { ++adv; adv_lanes += __popc(R); }
      if ((R >> lane_id()) & 1u) {
        if (NODE && p.alive) shade(a, p, tr);        // finish the bounce whose ray is done
        if (!p.alive && next_s < a.spp) {             // epilog done in shade; next sample
          p.s = next_s++;
          camera_ray(a, H, p);
          ++paths;
        }
        if (NODE && p.alive) {                        // start the next ray
          trav_begin(tr, p.d);
          ++st.rays;
          trav = true;
        }
      }
      E = __ballot_sync(kFull, !valid || (!p.alive && next_s >= a.spp));
    }
  }
  if constexpr (POOL) {
    // the pixel sums, each in sample order, once every path of the warp is done
    __syncwarp();  // @sr-region ENTRY:full
    if (valid) {
      const uint64_t pg = pix_of(a, (uint32_t)g);
      const float* pr = a.prad + 3 * pg * a.spp;
      float r = 0.0f, gg = 0.0f, b = 0.0f;
#pragma unroll 1  // one sample per trip (the simulator's PSUM count)
      for (uint32_t s = 0; s < a.spp; ++s) {  // @sr-region PSUM
        r = r + pr[3 * s];
        gg = gg + pr[3 * s + 1];
        b = b + pr[3 * s + 2];
      }
      float* px = a.rgb + 3 * pg;  // @sr-region ENTRY:full
      px[0] = r; px[1] = gg; px[2] = b;
    }
  }
  finish(a, p, valid, st, paths, g >> 5, rounds, rel, rel_lanes, adv, adv_lanes, lrel,  // @sr-region ENTRY:full
         lrel_lanes);
}

// sr_pt_closest diagnostics: one ray per thread
__global__ void pt_query(const PtArgs a) {
  const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= a.n) return;
  const float* r = a.q_rays + 6 * i;
  Stats st{0, 0, 0};
  Trav tr;
  const int64_t h = closest_hit<false>(a, tr, mk(r[0], r[1], r[2]), mk(r[3], r[4], r[5]), st);
  a.q_hit[i] = h;
  a.q_t[i] = tr.tb;
}

PtArgs base_args(const void* scene) {
  PtArgs a{};
  const unsigned char* s = static_cast<const unsigned char*>(scene);
  a.scene = s;
  // header offsets are read on the host from a copy (see check_pathtrace)
  return a;
}

}  // namespace

std::string check_pathtrace(const sr_pathtrace_params& p, uint64_t n_threads) {
  if (!p.scene_dev) return "pathtrace.scene_dev is NULL (build it with sr_scene_build)";
  if (p.scene_bytes < sizeof(PtHeader)) return "pathtrace.scene_bytes too small";
  if (p.width == 0 || p.height == 0) return "pathtrace.width/height must be >= 1";
  if ((uint64_t)p.width * p.height != n_threads)
    return "pathtrace: n_threads must equal width*height (one lane per pixel)";
  if (p.max_depth == 0) return "pathtrace.max_depth must be >= 1";
  return "";
}

size_t pathtrace_perthread_bytes(uint64_t n) { return 12 * n; }

// Scene headers known on the host: sr_scene_build registers the header of every
// image it writes, so a run needs no device->host read of it (sr_run stays
// stream-ordered and capturable in a CUDA graph).  An image the library did not
// write in this process (e.g. one built with sr_scene_build_host and copied by
// the caller) is read once -- a synchronous copy on the context stream, refused
// during stream capture -- and then registered too.  An entry stays valid while
// the caller's buffer holds that image.
namespace {
std::mutex g_scene_mu;
std::vector<std::pair<const void*, PtHeader>> g_scenes;
}  // namespace

void register_scene(const void* dev, const void* header) {
  std::lock_guard<std::mutex> lk(g_scene_mu);
  PtHeader h;
  std::memcpy(&h, header, sizeof h);
  for (auto& e : g_scenes)
    if (e.first == dev) { e.second = h; return; }
  g_scenes.emplace_back(dev, h);
}

static cudaError_t read_header(cudaStream_t st, const void* scene, PtHeader& h) {
  bool known = false;
  {
    std::lock_guard<std::mutex> lk(g_scene_mu);
    for (const auto& e : g_scenes)
      if (e.first == scene) { h = e.second; known = true; break; }
  }
  if (!known) {
    cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
    cudaError_t e = cudaStreamIsCapturing(st, &cs);
    if (e != cudaSuccess) return e;
    if (cs != cudaStreamCaptureStatusNone) {
      set_launch_note("scene_dev was not written by sr_scene_build in this process; its header "
                      "cannot be read during stream capture");
      return cudaErrorInvalidValue;
    }
    e = cudaMemcpyAsync(&h, scene, sizeof h, cudaMemcpyDeviceToHost, st);
    if (e == cudaSuccess) e = cudaStreamSynchronize(st);
    if (e != cudaSuccess) return e;
  }
  if (h.magic != kPtMagic) {
    set_launch_note("scene_dev does not hold an sr_scene_build image");
    return cudaErrorInvalidValue;
  }
  if (h.stack_need > kMaxStack) {
    set_launch_note("scene BVH needs a traversal stack of " + std::to_string(h.stack_need) +
                    " entries, more than " + std::to_string(kMaxStack));
    return cudaErrorInvalidValue;
  }
  if (!known) register_scene(scene, &h);
  return cudaSuccess;
}

cudaError_t launch_pathtrace(const LaunchCtx& c, const sr_workload& w, uint64_t n, uint32_t iters,
                             uint64_t seed, int mode, uint32_t T) {
  PtHeader h;
  cudaError_t e = read_header(c.stream, w.pathtrace.scene_dev, h);
  if (e != cudaSuccess) return e;
  if (h.bytes > w.pathtrace.scene_bytes) {
    set_launch_note("pathtrace.scene_bytes is smaller than the scene image");
    return cudaErrorInvalidValue;
  }
  PtArgs a = base_args(w.pathtrace.scene_dev);
  a.nodes = reinterpret_cast<const PtNode*>(a.scene + h.off_nodes);
  a.tris = reinterpret_cast<const PtTri*>(a.scene + h.off_tris);
  a.mats = reinterpret_cast<const PtMat*>(a.scene + h.off_mats);
  a.width = w.pathtrace.width;
  a.height = w.pathtrace.height;
  a.spp = iters;
  a.max_depth = w.pathtrace.max_depth;
  a.unroll = w.pathtrace.merge_unroll ? w.pathtrace.merge_unroll : 8;
  a.stack_cap = h.stack_need > 0 ? h.stack_need : 1u;
  a.T = T;
  a.n = n;
#ifdef SR_BOUNDS_CHECK
  a.n_nodes = h.n_nodes;
  a.n_tris = h.n_tris;
  a.n_mats = h.n_mats;
#endif
  a.seed = seed;
  a.keys = round_keys(seed);
  a.rgb = reinterpret_cast<float*>(c.ws + c.lay.off[SR_T_PERTHREAD]);
  a.counters = reinterpret_cast<unsigned long long*>(c.ws + c.lay.off[SR_T_COUNTERS]);
  a.sched = (w.flags & SR_F_SCHED) ? reinterpret_cast<uint32_t*>(c.ws + c.lay.off[SR_T_SCHED])
                                   : nullptr;
  // POOL: the per-path radiance buffer follows SCRATCH's first 256 bytes (layout_of)
  a.prad = reinterpret_cast<float*>(c.ws + c.lay.off[SR_T_SCRATCH] + 256);
  const uint32_t block = c.block;
  const uint64_t grid = (n + block - 1) / block;
  if (grid > 0x7fffffffull) return cudaErrorInvalidConfiguration;
  const bool spec = mode == SR_SPEC_LOOP;
  const bool pool = spec && (w.flags & SR_F_POOL);
  const bool node = (w.flags & SR_F_COARSE) == 0;
  const unsigned gr = (unsigned)grid;
  const size_t smem = (size_t)a.stack_cap * block * sizeof(int32_t);  // traversal stacks
  if (smem > 227 * 1024) return cudaErrorInvalidConfiguration;
  record_launch((uint32_t)grid, block, (uint32_t)smem);
  if (smem > 48 * 1024) {
    cudaFuncSetAttribute(pt_pdom<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    cudaFuncSetAttribute(pt_pdom<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    cudaFuncSetAttribute(pt_spec<false, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    cudaFuncSetAttribute(pt_spec<false, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    cudaFuncSetAttribute(pt_spec<true, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    cudaFuncSetAttribute(pt_spec<true, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    cudaFuncSetAttribute(pt_spec<false, true, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    cudaFuncSetAttribute(pt_spec<true, true, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    cudaFuncSetAttribute(pt_spec<false, true, true, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    cudaFuncSetAttribute(pt_spec<true, true, true, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    cudaFuncSetAttribute(pt_spec<false, true, true, false, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    cudaFuncSetAttribute(pt_spec<true, true, true, false, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  }
  if (!spec) {
    if (a.sched) pt_pdom<true><<<gr, block, smem, c.stream>>>(a);
    else pt_pdom<false><<<gr, block, smem, c.stream>>>(a);
  } else if (pool) {  // check_pathtrace: split merge only
    if (a.sched) pt_spec<true, true, true, false, true><<<gr, block, smem, c.stream>>>(a);
    else pt_spec<false, true, true, false, true><<<gr, block, smem, c.stream>>>(a);
  } else if (node && !(w.flags & SR_F_NOSPLIT) && (w.flags & SR_F_MATGROUP)) {
    if (a.sched) pt_spec<true, true, true, true><<<gr, block, smem, c.stream>>>(a);
    else pt_spec<false, true, true, true><<<gr, block, smem, c.stream>>>(a);
  } else if (node && !(w.flags & SR_F_NOSPLIT)) {
    if (a.sched) pt_spec<true, true, true><<<gr, block, smem, c.stream>>>(a);
    else pt_spec<false, true, true><<<gr, block, smem, c.stream>>>(a);
  } else if (node) {
    if (a.sched) pt_spec<true, true><<<gr, block, smem, c.stream>>>(a);
    else pt_spec<false, true><<<gr, block, smem, c.stream>>>(a);
  } else {
    if (a.sched) pt_spec<true, false><<<gr, block, smem, c.stream>>>(a);
    else pt_spec<false, false><<<gr, block, smem, c.stream>>>(a);
  }
  return cudaGetLastError();
}

cudaError_t launch_pt_query(cudaStream_t st, const void* scene, const float* rays, int64_t* hit,
                            float* t, uint64_t n) {
  PtHeader h;
  cudaError_t e = read_header(st, scene, h);
  if (e != cudaSuccess) return e;
  PtArgs a = base_args(scene);
  a.nodes = reinterpret_cast<const PtNode*>(a.scene + h.off_nodes);
  a.tris = reinterpret_cast<const PtTri*>(a.scene + h.off_tris);
  a.mats = reinterpret_cast<const PtMat*>(a.scene + h.off_mats);
  a.n = n;
#ifdef SR_BOUNDS_CHECK
  a.n_nodes = h.n_nodes;
  a.n_tris = h.n_tris;
  a.n_mats = h.n_mats;
#endif
  a.q_rays = rays;
  a.q_hit = hit;
  a.q_t = t;
  a.stack_cap = h.stack_need > 0 ? h.stack_need : 1u;
  const uint64_t grid = (n + 127) / 128;
  if (grid > 0x7fffffffull) {
    set_launch_note("too many rays for one launch");
    return cudaErrorInvalidValue;
  }
  const size_t smem = (size_t)a.stack_cap * 128 * sizeof(int32_t);
  if (smem > 48 * 1024) {
    e = cudaFuncSetAttribute(pt_query, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
  }
  record_launch((uint32_t)grid, 128, (uint32_t)smem);
  if (n) pt_query<<<(unsigned)grid, 128, smem, st>>>(a);
  return cudaGetLastError();
}

}  // namespace sr
