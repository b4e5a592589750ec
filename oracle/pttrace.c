/*
 * pttrace.c -- ORACLE part 2 for the path tracer (test / evaluation
 * infrastructure; see oracle.h).  Nothing here is used for parity: the path
 * tracer's parity oracle is pathtrace.c's brute-force renderer.
 *
 * (1) or_pt_trace replays configs[3]'s paths (reading R7, operation for
 *     operation as pathtrace.c) with the closest hit found by a BVH traversal
 *     over the scene image that sr_scene_build writes (the acceleration
 *     structure is input data here, its layout restated below), and records per
 *     lane the sequence of work items the kernels execute: node visits (with
 *     the leaf triangles they queue, push / pop / end of traversal), triangle
 *     tests (how far Moller-Trumbore gets), and each ray's shading outcome.  The
 *     traversal order is the kernels' (both children tested against the running
 *     t, leaves tested child 0 first, the nearer inner child first, the other
 *     pushed; empty next -> pop), so the closest hits -- and the image -- equal
 *     the brute force (tests/test_oracle_pttrace.py checks the image bit for bit).
 * (2) ws_pt replays those streams under the PDOM rule (the bounce loop and the
 *     traversal loop inside it, both reconverging at their latches) and under the split
 *     Loop Merge of pt_spec (two concurrent predictions: inner-node visits I vs leaf tests
 *     L, the larger group released when |G| >= T or no lane can refill, U work
 *     items per release; idle lanes shade, start the next sample and the next
 *     ray in advance rounds) -- each lane on its own pixel, or (WS_SPEC_LOOP_POOL)
 *     taking the next path of the warp's pool -- counting warp executions and active
 *     lanes per source region (WS_PT_*), as warpsim.c does for the other kernels.
 */
#include <math.h>
#include <string.h>
#include "oracle.h"

/* ---- the scene image (csrc/pt_scene.h's layout, restated) ---- */
typedef struct {
  uint32_t magic, n_nodes, n_tris, n_mats;
  uint64_t off_nodes, off_tris, off_mats, bytes;
  float cam[16];
  uint32_t stack_need, pad[3];
} img_hdr;
typedef struct {
  float lo[3][2], hi[3][2];   /* [axis][child] */
  int32_t ref0, cnt0, ref1, cnt1;
} img_node;
typedef struct {
  float v0[3], e1[3], e2[3];
  uint32_t id, mat, pad;
} img_tri;

typedef struct { float x, y, z; } v3;
static v3 mk(float x, float y, float z) { v3 r = {x, y, z}; return r; }
static v3 sub(v3 a, v3 b) { return mk(a.x - b.x, a.y - b.y, a.z - b.z); }
static v3 add(v3 a, v3 b) { return mk(a.x + b.x, a.y + b.y, a.z + b.z); }
static v3 scl(v3 a, float s) { return mk(a.x * s, a.y * s, a.z * s); }
static float dot(v3 a, v3 b) { return (a.x * b.x + a.y * b.y) + a.z * b.z; }
static v3 cross(v3 a, v3 b) {
  return mk(a.y * b.z - a.z * b.y, a.z * b.x - a.x * b.z, a.x * b.y - a.y * b.x);
}
static v3 normalize(v3 a) { return scl(a, 1.0f / sqrtf(dot(a, a))); }

/* conservative slab test of the padded child box (the kernels' expression) */
static int box_hit(const float* lo, const float* hi, v3 o, v3 inv, float tb, float* tnear) {
  float tx0 = (lo[0] - o.x) * inv.x, tx1 = (hi[0] - o.x) * inv.x;
  float ty0 = (lo[1] - o.y) * inv.y, ty1 = (hi[1] - o.y) * inv.y;
  float tz0 = (lo[2] - o.z) * inv.z, tz1 = (hi[2] - o.z) * inv.z;
  float tn = fmaxf(fmaxf(fminf(tx0, tx1), fminf(ty0, ty1)), fmaxf(fminf(tz0, tz1), 0.0f));
  float tf = fminf(fminf(fmaxf(tx0, tx1), fmaxf(ty0, ty1)), fmaxf(tz0, tz1));
  *tnear = tn;
  return tn * (1.0f - 1e-5f) <= tf * (1.0f + 1e-5f) && tn * (1.0f - 1e-5f) <= tb;
}

typedef struct {
  uint16_t* ops;
  uint64_t n, cap;
  int overflow;
} opbuf;
static void put(opbuf* b, uint16_t op) {
  if (b->n < b->cap) b->ops[b->n] = op;
  else b->overflow = 1;
  b->n++;
}

typedef struct {
  float tb;
  int32_t ib;
  uint32_t mb, slot;
} hitrec;

/* Moller-Trumbore on the image triangle `at` (edges precomputed as in the
 * kernels); returns how far the test got: 0 det, 1 u, 2 v, 3 t rejected,
 * 4 a hit that is not closer, 5 a closer hit (recorded) */
static uint32_t tri_test(const img_tri* T, int32_t at, v3 o, v3 d, hitrec* h) {
  v3 v0 = mk(T->v0[0], T->v0[1], T->v0[2]);
  v3 e1 = mk(T->e1[0], T->e1[1], T->e1[2]);
  v3 e2 = mk(T->e2[0], T->e2[1], T->e2[2]);
  v3 pv = cross(d, e2);
  float det = dot(e1, pv);
  if (fabsf(det) < 1.0e-12f) return 0;
  float inv = 1.0f / det;
  v3 tv = sub(o, v0);
  float u = dot(tv, pv) * inv;
  if (u < 0.0f || u > 1.0f) return 1;
  v3 qv = cross(tv, e1);
  float v = dot(d, qv) * inv;
  if (v < 0.0f || u + v > 1.0f) return 2;
  float t = dot(e2, qv) * inv;
  if (!(t > 1.0e-4f)) return 3;
  int32_t id = (int32_t)T->id;
  if (t < h->tb || (t == h->tb && id < h->ib)) {
    h->tb = t;
    h->ib = id;
    h->mb = T->mat;
    h->slot = (uint32_t)at;
    return 5;
  }
  return 4;
}

/* one ray's closest hit by BVH traversal, recording its work items */
static void closest(const unsigned char* img, const img_hdr* H, v3 o, v3 d, hitrec* h,
                    int32_t* stk, opbuf* b) {
  const img_node* nodes = (const img_node*)(img + H->off_nodes);
  const img_tri* tris = (const img_tri*)(img + H->off_tris);
  v3 inv = mk(1.0f / d.x, 1.0f / d.y, 1.0f / d.z);
  h->tb = INFINITY;
  h->ib = -1;
  h->mb = 0;
  h->slot = 0;
  int32_t node = 0, sp = 0;
  const int32_t cap = H->stack_need > 0 ? (int32_t)H->stack_need : 1;
  for (;;) {
    const img_node* N = &nodes[node];
    float tn0 = 0.0f, tn1 = 0.0f;
    const float lo0[3] = {N->lo[0][0], N->lo[1][0], N->lo[2][0]};
    const float hi0[3] = {N->hi[0][0], N->hi[1][0], N->hi[2][0]};
    const float lo1[3] = {N->lo[0][1], N->lo[1][1], N->lo[2][1]};
    const float hi1[3] = {N->hi[0][1], N->hi[1][1], N->hi[2][1]};
    int h0 = N->ref0 >= 0 && box_hit(lo0, hi0, o, inv, h->tb, &tn0);
    int h1 = N->ref1 >= 0 && box_hit(lo1, hi1, o, inv, h->tb, &tn1);
    uint32_t n0 = (h0 && N->cnt0 > 0) ? (uint32_t)N->cnt0 : 0u;
    uint32_t n1 = (h1 && N->cnt1 > 0) ? (uint32_t)N->cnt1 : 0u;
    int in0 = h0 && N->cnt0 == 0, in1 = h1 && N->cnt1 == 0;
    int32_t next = -1;
    uint32_t push = 0, pop = 0, end = 0;
    if (in0 && in1) {
      int first0 = tn0 <= tn1;
      next = first0 ? N->ref0 : N->ref1;
      if (sp < cap) stk[sp++] = first0 ? N->ref1 : N->ref0;
      push = 1;
    } else if (in0) {
      next = N->ref0;
    } else if (in1) {
      next = N->ref1;
    }
    if (next < 0) {
      if (sp == 0) end = 1;
      else { next = stk[--sp]; pop = 1; }
    }
    put(b, (uint16_t)(OR_PT_OP_NODE | n0 | (n1 << 4) | (push << 8) | (pop << 9) | (end << 10)));
    for (uint32_t k = 0; k < n0; ++k)
      put(b, (uint16_t)(OR_PT_OP_LEAF | tri_test(&tris[N->ref0 + (int32_t)k], N->ref0 + (int32_t)k,
                                                 o, d, h)));
    for (uint32_t k = 0; k < n1; ++k)
      put(b, (uint16_t)(OR_PT_OP_LEAF | tri_test(&tris[N->ref1 + (int32_t)k], N->ref1 + (int32_t)k,
                                                 o, d, h)));
    if (end) break;
    node = next;
  }
}

static void draw(uint32_t event, uint64_t q, uint64_t seed, uint32_t u[4]) {
  uint32_t ctr[4] = {event, (uint32_t)OR_TAG_PT << 16, (uint32_t)q, (uint32_t)(q >> 32)};
  uint32_t key[2] = {(uint32_t)seed, (uint32_t)(seed >> 32)};
  or_philox4x32_10(ctr, key, u);
}

uint64_t or_pt_trace(const unsigned char* img, uint64_t img_bytes, uint32_t width, uint32_t height,
                     uint32_t spp, uint32_t max_depth, uint64_t seed, const uint32_t* pixels,
                     uint32_t n_pixels, uint16_t* ops, uint64_t cap, uint64_t* off, float* rgb) {
  const img_hdr* H = (const img_hdr*)img;
  if (img_bytes < sizeof(img_hdr) || H->bytes > img_bytes) return UINT64_MAX - 1;
  const img_tri* tris = (const img_tri*)(img + H->off_tris);
  const float* mats = (const float*)(img + H->off_mats);
  int32_t stk[512];
  if (H->stack_need > 512) return UINT64_MAX - 1;
  opbuf b = {ops, 0, cap, 0};
  const float* cam = H->cam;
  v3 eye = mk(cam[0], cam[1], cam[2]), fwd = mk(cam[3], cam[4], cam[5]);
  v3 right = mk(cam[6], cam[7], cam[8]), up = mk(cam[9], cam[10], cam[11]);
  float tan_half = cam[12], aspect = cam[13];
  for (uint32_t k = 0; k < n_pixels; ++k) {
    uint32_t pix = pixels ? pixels[k] : k;
    uint32_t px = pix % width, py = pix / width;
    off[k] = b.n;
    v3 sum = mk(0.0f, 0.0f, 0.0f);
    for (uint32_t s = 0; s < spp; ++s) {
      uint64_t q = (uint64_t)pix * spp + s;
      uint32_t u[4];
      put(&b, OR_PT_OP_PATH);
      draw(0u, q, seed, u);
      float fx = ((float)px + or_u01(u[0])) / (float)width;
      float fy = ((float)py + or_u01(u[1])) / (float)height;
      float sx = (2.0f * fx - 1.0f) * tan_half * aspect;
      float sy = (1.0f - 2.0f * fy) * tan_half;
      v3 d = normalize(add(add(fwd, scl(right, sx)), scl(up, sy)));
      v3 o = eye;
      v3 thr = mk(1.0f, 1.0f, 1.0f), rad = mk(0.0f, 0.0f, 0.0f);
      for (uint32_t bnc = 0;; ++bnc) {
        hitrec h;
        closest(img, H, o, d, &h, stk, &b);
        uint32_t outcome, rr = 0, end = 0;
        if (h.ib < 0) {
          outcome = OR_PT_SH_MISS;
          end = 1;
        } else {
          const float* m = mats + 8u * h.mb;
          uint32_t kind = (uint32_t)m[0];
          rad = add(rad, mk(thr.x * m[4], thr.y * m[5], thr.z * m[6]));
          if (kind == 3u) {
            outcome = OR_PT_SH_LIGHT;
            end = 1;
          } else {
            outcome = kind == 0u ? OR_PT_SH_DIFFUSE : (kind == 1u ? OR_PT_SH_MIRROR : OR_PT_SH_GLASS);
            const img_tri* T = &tris[h.slot];
            v3 e1 = mk(T->e1[0], T->e1[1], T->e1[2]), e2 = mk(T->e2[0], T->e2[1], T->e2[2]);
            v3 ng = normalize(cross(e1, e2));
            v3 p = add(o, scl(d, h.tb));
            draw(bnc + 1u, q, seed, u);
            float di[3] = {d.x, d.y, d.z}, n3[3] = {ng.x, ng.y, ng.z}, dout[3];
            or_pt_scatter(kind, m[7], di, n3, u, dout);
            d = mk(dout[0], dout[1], dout[2]);
            thr = mk(thr.x * m[1], thr.y * m[2], thr.z * m[3]);
            o = p;
            if (bnc >= 3u) {
              rr = 1;
              float pm = fmaxf(thr.x, fmaxf(thr.y, thr.z));
              float prr = fminf(0.95f, pm);
              if (!(or_u01(u[3]) < prr)) end = 1;
              else thr = mk(thr.x / prr, thr.y / prr, thr.z / prr);
            }
          }
        }
        if (!end && bnc + 1u >= max_depth) end = 1;
        put(&b, (uint16_t)(OR_PT_OP_SHADE | outcome | (rr << 3) | (end << 4)));
        if (end) break;
      }
      sum = add(sum, rad);
    }
    if (rgb) {
      rgb[3u * k + 0] = sum.x;
      rgb[3u * k + 1] = sum.y;
      rgb[3u * k + 2] = sum.z;
    }
  }
  off[n_pixels] = b.n;
  return b.overflow ? UINT64_MAX : b.n;
}

/* ------------------------------------------------------------------ */
/* The schedules.                                                       */
static void hit(ws_counts* o, int r, uint32_t mask) {
  if (!mask) return;
  o->execs[r] += 1;
  o->lanes[r] += (uint64_t)__builtin_popcount(mask);
}
static int is_node(uint16_t op) { return (op & 0xE000u) == OR_PT_OP_NODE; }
static int is_leaf(uint16_t op) { return (op & OR_PT_OP_LEAF) != 0; }
static int is_shade(uint16_t op) { return (op & 0xC000u) == OR_PT_OP_SHADE; }

/* the triangle-test stages of the lanes in `m` whose current op is a LEAF */
static void tt_hits(ws_counts* o, const uint16_t* ops, const uint64_t* pc, uint32_t m) {
  uint32_t s[6] = {0};
  for (uint32_t l = 0; l < 32; ++l)
    if (m >> l & 1u) s[ops[pc[l]] & 7u] |= 1u << l;
  uint32_t ge1 = s[1] | s[2] | s[3] | s[4] | s[5], ge2 = s[2] | s[3] | s[4] | s[5];
  uint32_t ge3 = s[3] | s[4] | s[5], ge4 = s[4] | s[5];
  hit(o, WS_PT_TT, m);
  hit(o, WS_PT_TT_U, ge1);
  hit(o, WS_PT_TT_V, ge2);
  hit(o, WS_PT_TT_T, ge3);
  hit(o, WS_PT_TT_ID, ge4);
  hit(o, WS_PT_TT_UPD, s[5]);
}
static void node_hits(ws_counts* o, const uint16_t* ops, const uint64_t* pc, uint32_t m) {
  uint32_t push = 0, pop = 0, end = 0, nopush = 0;
  for (uint32_t l = 0; l < 32; ++l) {
    if (!(m >> l & 1u)) continue;
    uint16_t op = ops[pc[l]];
    if (op & 0x100u) push |= 1u << l;
    else nopush |= 1u << l;
    if (op & 0x200u) pop |= 1u << l;
    if (op & 0x400u) end |= 1u << l;
  }
  hit(o, WS_PT_NODE, m);
  hit(o, WS_PT_PUSH, push);
  hit(o, WS_PT_NOPUSH, nopush);
  hit(o, WS_PT_NEXTNONE, pop | end);
  hit(o, WS_PT_POP, pop);
}
static void shade_hits(ws_counts* o, const uint16_t* ops, const uint64_t* pc, uint32_t m) {
  uint32_t hitm = 0, surf = 0, k[5] = {0}, rr = 0, end = 0;
  for (uint32_t l = 0; l < 32; ++l) {
    if (!(m >> l & 1u)) continue;
    uint16_t op = ops[pc[l]];
    uint32_t oc = op & 7u;
    k[oc] |= 1u << l;
    if (oc != OR_PT_SH_MISS) hitm |= 1u << l;
    if (oc >= OR_PT_SH_DIFFUSE) surf |= 1u << l;
    if (op & 8u) rr |= 1u << l;
    if (op & 16u) end |= 1u << l;
  }
  hit(o, WS_PT_SH, m);
  hit(o, WS_PT_SH_HIT, hitm);
  hit(o, WS_PT_SH_SURF, surf);
  hit(o, WS_PT_SH_DIFF, k[OR_PT_SH_DIFFUSE]);
  hit(o, WS_PT_SH_MIRR, k[OR_PT_SH_MIRROR]);
  hit(o, WS_PT_SH_GLASS, k[OR_PT_SH_GLASS]);
  hit(o, WS_PT_SH_RR, rr);
  hit(o, WS_PT_SH_END, end);
}

/* ops / off: the streams of the warp's n_valid lanes (lane l: ops[off[l] .. off[l+1])) */
void ws_pt(const uint16_t* ops, const uint64_t* off, uint32_t n_valid, int mode, uint32_t T,
           uint32_t U, ws_counts* o) {
  memset(o, 0, sizeof *o);
  if (n_valid > 32) n_valid = 32;
  if (U == 0) U = 1;
  const uint32_t valid = n_valid >= 32 ? 0xffffffffu : ((1u << n_valid) - 1u);
  uint64_t pc[32] = {0}, endp[32] = {0};
  for (uint32_t l = 0; l < n_valid; ++l) { pc[l] = off[l]; endp[l] = off[l + 1]; }
  hit(o, WS_PT_ENTRY, 0xffffffffu);
  if (mode == WS_PDOM) {
    /* for s: (valid lanes) camera ray; do { bounce } while (alive) */
    for (;;) {
      uint32_t A = 0;   /* lanes starting a path */
      for (uint32_t l = 0; l < n_valid; ++l)
        if (pc[l] < endp[l]) { A |= 1u << l; pc[l]++; }   /* the PATH op */
      if (!A) break;
      hit(o, WS_PT_OUTER, 0xffffffffu);
      hit(o, WS_PT_LAUNCH, A);
      uint32_t alive = A;
      while (alive) {               /* one bounce of every live path */
        hit(o, WS_PT_BOUNCE, alive);
        hit(o, WS_PT_TBEGIN, alive);
        uint32_t tr = alive;        /* lanes still traversing */
        while (tr) {
          /* the loop's vote and latch run with every lane of the bounce (the
           * kernel reconverges them there); the visit with the traversing ones */
          hit(o, WS_PT_STEP, alive);
          node_hits(o, ops, pc, tr);
          /* the visit's inline leaf loop: child 0's tests, then child 1's */
          uint32_t nt[32] = {0}, mx = 0;
          uint32_t nxt = tr, hl = 0;
          for (uint32_t l = 0; l < 32; ++l) {
            if (!(tr >> l & 1u)) continue;
            uint16_t op = ops[pc[l]];
            nt[l] = (op & 15u) + ((op >> 4) & 15u);
            if (nt[l] > mx) mx = nt[l];
            if (nt[l]) hl |= 1u << l;
            if (op & 0x400u) nxt &= ~(1u << l);
            pc[l]++;
          }
          hit(o, WS_PT_LEAFIF, hl);
          for (uint32_t k = 0; k < mx; ++k) {
            uint32_t m = 0;
            for (uint32_t l = 0; l < 32; ++l) if (nt[l] > k) m |= 1u << l;
            hit(o, WS_PT_LEAF, m);
            tt_hits(o, ops, pc, m);
            for (uint32_t l = 0; l < 32; ++l) if (m >> l & 1u) pc[l]++;
          }
          tr = nxt;
        }
        shade_hits(o, ops, pc, alive);
        uint32_t still = 0;
        for (uint32_t l = 0; l < 32; ++l) {
          if (!(alive >> l & 1u)) continue;
          if (!(ops[pc[l]] & 16u)) still |= 1u << l;
          pc[l]++;
        }
        alive = still;
      }
    }
    return;
  }
  /* split Loop Merge (pt_spec<.., NODE, SPLIT>).  WS_SPEC_LOOP_POOL: the warp's
   * paths form one pool -- path q is sample q / n_valid of the warp's pixel
   * q % n_valid -- and a lane whose path has ended claims the next unclaimed one
   * in an advance round, idle lanes in lane order (pt_spec<.., POOL>) */
  const int pool = mode == WS_SPEC_LOOP_POOL;
  uint64_t pstart[32 * WS_PT_POOL_MAX_SPP], pend[32 * WS_PT_POOL_MAX_SPP];
  uint32_t npath = 0, qnext = 0;
  if (pool) {
    uint32_t spp = 0;
    for (uint32_t l = 0; l < n_valid; ++l) {   /* the paths of each lane's pixel */
      uint32_t k = 0;
      for (uint64_t i = off[l]; i < off[l + 1]; ++i)
        if ((ops[i] & 0xE000u) == OR_PT_OP_PATH) k++;
      if (k > spp) spp = k;
    }
    if (spp > WS_PT_POOL_MAX_SPP) spp = WS_PT_POOL_MAX_SPP;
    for (uint32_t sm = 0; sm < spp; ++sm)      /* pool order: sample-major */
      for (uint32_t l = 0; l < n_valid; ++l) {
        uint32_t k = 0;
        for (uint64_t i = off[l]; i < off[l + 1]; ++i) {
          if ((ops[i] & 0xE000u) != OR_PT_OP_PATH) continue;
          if (k++ != sm) continue;
          uint64_t e = i + 1;
          while (e < off[l + 1] && (ops[e] & 0xE000u) != OR_PT_OP_PATH) e++;
          pstart[npath] = i;
          pend[npath] = e;
          npath++;
          break;
        }
      }
    for (uint32_t l = 0; l < 32; ++l) pc[l] = endp[l] = 0;   /* no path held yet */
  }
  if (T == 0 || T > 32) T = 32;
  uint32_t trav = 0, alive = 0;
  uint32_t E = pool ? 0u : ~valid;   /* with a pool every lane of the warp takes paths */
  for (uint32_t l = 0; l < n_valid; ++l) if (!pool && pc[l] >= endp[l]) E |= 1u << l;
  for (;;) {
    uint32_t L = 0, I = 0;
    for (uint32_t l = 0; l < 32; ++l) {
      if (!(trav >> l & 1u)) continue;
      if (is_leaf(ops[pc[l]])) L |= 1u << l;
      else I |= 1u << l;
    }
    const uint32_t R = ~(I | L | E);
    if ((I | L | R) == 0u) break;
    o->rounds += 1;
    hit(o, WS_PT_ROUND, 0xffffffffu);
    const int leaf = __builtin_popcount(L) > __builtin_popcount(I);
    const uint32_t G = leaf ? L : I;
    if (G && ((uint32_t)__builtin_popcount(G) >= T || R == 0u)) {
      hit(o, WS_PT_REL, G);
      uint32_t S = G;
      if (leaf) {
        hit(o, WS_PT_LREL, G);
        for (uint32_t k = 0; k < U && S; ++k) {
          hit(o, WS_PT_LEAF, S);
          tt_hits(o, ops, pc, S);
          for (uint32_t l = 0; l < 32; ++l) {
            if (!(S >> l & 1u)) continue;
            pc[l]++;
            if (!is_leaf(ops[pc[l]])) S &= ~(1u << l);   /* queue empty */
          }
        }
      } else {
        hit(o, WS_PT_NREL, G);
        for (uint32_t k = 0; k < U && S; ++k) {
          hit(o, WS_PT_STEP, S);
          node_hits(o, ops, pc, S);
          for (uint32_t l = 0; l < 32; ++l) {
            if (!(S >> l & 1u)) continue;
            pc[l]++;
            if (!is_node(ops[pc[l]])) S &= ~(1u << l);   /* leaves queued, or done */
          }
        }
      }
      for (uint32_t l = 0; l < 32; ++l)   /* trav = leaf pending || node pending */
        if ((G >> l & 1u) && is_shade(ops[pc[l]])) trav &= ~(1u << l);
      continue;
    }
    hit(o, WS_PT_ADV, R);
    uint32_t sh = 0, launch = 0, begin = 0;
    for (uint32_t l = 0; l < 32; ++l) if ((R >> l & 1u) && (alive >> l & 1u)) sh |= 1u << l;
    shade_hits(o, ops, pc, sh);
    for (uint32_t l = 0; l < 32; ++l) {
      if (!(R >> l & 1u)) continue;
      if (alive >> l & 1u) {
        if (ops[pc[l]] & 16u) alive &= ~(1u << l);
        pc[l]++;
      }
      if (pool && !(alive >> l & 1u) && qnext < npath) {   /* claim the next path */
        pc[l] = pstart[qnext];
        endp[l] = pend[qnext];
        qnext++;
      }
      if (!(alive >> l & 1u) && pc[l] < endp[l]) {   /* next sample: camera ray */
        pc[l]++;                                     /* the PATH op */
        alive |= 1u << l;
        launch |= 1u << l;
      }
      if (alive >> l & 1u) {
        begin |= 1u << l;
        trav |= 1u << l;
      }
    }
    hit(o, WS_PT_LAUNCH, launch);
    hit(o, WS_PT_TBEGIN, begin);
    for (uint32_t l = 0; l < 32; ++l)
      if (!(alive >> l & 1u) && pc[l] >= endp[l] && (!pool || qnext >= npath)) E |= 1u << l;
  }
  /* with the pool: each valid lane then adds its pixel's samples in sample order */
  if (pool)
    for (uint32_t k = 0; k < npath / (n_valid ? n_valid : 1); ++k) hit(o, WS_PT_PSUM, valid);
}
