/*
 * oracle.h -- CPU ORACLE for the Speculative Reconvergence hot path.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and the
 * cpu_baseline / --impl reference legs of bench.py may load liboracle.so.
 * The product path (libsr.so, paper_conf_cgo_damanijskymg20_b200/) never
 * includes, links or calls anything in this directory, and nothing here
 * includes or links the CUDA path.  The two share no code.
 *
 * Paper: Damani et al., "Speculative Reconvergence for Improved SIMT
 * Efficiency", CGO'20.  Citations "P:N" are /root/reference/PAPER.md lines.
 *
 * Part 1 (divloop.c, commoncall.c, mcml.c, pathtrace.c): the unannotated
 *   program of Fig. 2 / Listing 1 executed one task
 *   at a time.  Convergence barriers "are not required for correctness of the
 *   program", so this is the expected output of EVERY mode,
 *   threshold, block size and GPU count.
 * Part 2 (warpsim.c): a lane-mask warp simulator that executes the PDOM
 *   rule and the Speculative Reconvergence rule with a
 *   soft-barrier threshold (Sec. 4.6) over per-lane event
 *   streams produced by part 1, and counts region executions / active lanes.
 *
 * Parity status per function is listed in DESIGN.md ("Oracle pins").
 * Built with: gcc -O2 -std=c11 -ffp-contract=off -fno-fast-math -fPIC -shared
 */
#ifndef SR_ORACLE_H
#define SR_ORACLE_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* ---- philox.c : Philox4x32-10 counter-based RNG (paper is silent on RNG;
 * DESIGN.md reading R1).  ctr = {event, (tag<<16)|sub, task_lo, task_hi},
 * key = {seed_lo, seed_hi}. */
enum { OR_TAG_DIV = 1, OR_TAG_CALL = 2, OR_TAG_MC = 3, OR_TAG_PT = 4 };
void or_philox4x32_10(const uint32_t ctr[4], const uint32_t key[2], uint32_t out[4]);
float or_u01(uint32_t u);   /* (u>>8) * 2^-24     in [0,1) */
float or_u01c(uint32_t u);  /* ((u>>8)+1) * 2^-24 in (0,1] */

/* ---- srmath.c : the two transcendental functions of the MC / PT steps,
 * defined op-by-op (reading R5) so CPU and GPU round identically. */
float or_sr_logf(float x);                             /* x in (0, 1]           */
void  or_sr_sincos2pif(float xi, float* s, float* c);  /* xi = k*2^-24, k<2^24  */
/* exhaustive accuracy sweeps (all 2^24 RNG-reachable inputs) vs double libm:
 * returns max |error| in units of the float ulp of the exact result. */
double or_sweep_logf_ulp(void);
double or_sweep_sincos2pif_ulp(void);
/* out[i] = fn(x[i]); fn: 0 log, 1 sin2pi, 2 cos2pi, 3 Expensive(1000 FMAs),
 * 4 Expensive(2000 FMAs) */
void or_eval_batch(int fn, const float* x, float* out, uint64_t n);

/* ---- divloop.c : config 1, divergent condition in a loop (Fig. 2(a)). */
typedef struct { uint32_t p_u32, fma_count; } or_divloop_params;
/* threads [t0, t0+n): acc[n], cnt[n] */
void or_divloop(const or_divloop_params* p, uint64_t t0, uint64_t n, uint32_t iters,
                uint64_t seed, float* acc, uint32_t* cnt);
/* event stream for the simulator: want[(t-t0)*iters + i] in {0,1} */
void or_divloop_wants(const or_divloop_params* p, uint64_t t0, uint64_t n, uint32_t iters,
                      uint64_t seed, uint8_t* want);
float or_expensive(float u, uint32_t fma_count);  /* the common code of c3/c4 */

/* ---- commoncall.c : config 2, common function call (Fig. 2(c)). */
typedef struct { uint32_t fma_count, split_u32; } or_commoncall_params;
void or_commoncall(const or_commoncall_params* p, uint64_t t0, uint64_t n, uint32_t iters,
                   uint64_t seed, float* y, uint8_t* arm /* may be NULL: arm of iter 0 */);

/* ---- mcml.c : configs 3/5, MCML photon transport in a layered slab. */
#define OR_MC_MAX_LAYERS 8
typedef struct { float n, mua, mus, g, d; } or_layer;  /* cm^-1, cm */
typedef struct {
  uint32_t n_layers;
  or_layer layer[OR_MC_MAX_LAYERS];
  float n_above, n_below;
  float dr, dz;
  uint32_t nr, nz;
  uint32_t step_cap;
} or_mcml_params;
/* counter slots (u64) */
enum { OR_MC_PHOTONS = 0, OR_MC_STEPS, OR_MC_RD_EXITS, OR_MC_TT_EXITS, OR_MC_RR_KILLS,
       OR_MC_RR_SURVIVE, OR_MC_CAPPED, OR_MC_ZERO_W, OR_MC_NCOUNTERS = 8 };
/* Adds into caller-zeroed tallies: A[nz*nr] (iz-major), Rd[nr], Tt[nr],
 * cnt[OR_MC_NCOUNTERS].  Photon ids [id0, id0+count).  steps_out (may be
 * NULL) receives the per-photon step count. */
void or_mcml(const or_mcml_params* p, uint64_t id0, uint64_t count, uint64_t seed,
             uint64_t* A, uint64_t* Rd, uint64_t* Tt, uint64_t* cnt, uint32_t* steps_out);
/* Per-photon event stream for the simulator (one byte per step) recording
 * which branches of the step ran (no effect on the arithmetic).  Returns
 * number of steps written (<= cap); stops at cap. */
typedef uint16_t or_event;
enum { OR_EV_BOUNDARY = 1, OR_EV_SLEFT = 2, OR_EV_REFLECT = 4, OR_EV_EXIT = 8,
       OR_EV_TRANSMIT = 16, OR_EV_ROULETTE = 32, OR_EV_SPIN_AXIS = 64,
       OR_EV_SPIN_GENERAL = 128, OR_EV_EXTERNAL = 256 /* boundary with the ambient */,
       OR_EV_MATCHED = 512 /* boundary with a layer of equal index: Fresnel r = 0 */ };
uint32_t or_mcml_events(const or_mcml_params* p, uint64_t id, uint64_t seed,
                        or_event* ev, uint32_t cap);
uint64_t or_mcml_events_batch(const or_mcml_params* p, uint64_t id0, uint64_t count,
                              uint64_t seed, or_event* ev, uint64_t cap, uint64_t* off,
                              uint32_t* nsteps);
/* MCML Fresnel reflectance (all-or-none decision uses it) */
float or_mcml_fresnel(float ni, float nt, float ca1, float* ca2);
/* Rsp as defined in mcml.c (specular reflectance at launch) */
float or_mcml_rsp(const or_mcml_params* p);
/* the step's building blocks, exactly as step() uses them (pins in tests/) */
float or_mcml_step_length(float mut, uint32_t u0);   /* -ln(U01c(u0)) / mu_t   */
float or_mcml_hg_cost(float g, float xi);            /* HG cos(theta)          */
void or_mcml_spin(float cost, float xi_psi, const float u_in[3], float u_out[3]);
void or_mcml_eval_batch(int fn, float p, const uint32_t* u, float* out, uint64_t n);

/* ---- pathtrace.c : config 4, path tracer with brute-force closest hit. */
typedef struct {
  const float* tris;     /* n_tris x 9 floats (v0, v1, v2)                  */
  const uint32_t* mat;   /* n_tris material ids                             */
  uint32_t n_tris;
  const float* mats;     /* n_mats x 8 {kind, r, g, b, er, eg, eb, ior}     */
  uint32_t n_mats;
  float cam[16];         /* eye, forward, right, up, tan(fov/2), aspect     */
} or_pt_scene;
/* closest hit over all triangles (t > 1e-4; ties -> smaller index); -1 = miss */
int64_t or_pt_closest(const float* tris, uint32_t n_tris, const float o[3], const float d[3],
                      float* t_best);
/* the direction half of one bounce (material kind 0/1/2; see pathtrace.c) */
void or_pt_scatter(uint32_t kind, float ior, const float d_in[3], const float ng_in[3],
                   const uint32_t u[4], float d_out[3]);
/* rgb[3k..3k+2] = sum over the spp samples of pixel pixels[k] (all pixels
 * 0..n_pixels-1 when pixels == NULL); counters[0] += paths, [1] += rays. */
void or_pt_render(const or_pt_scene* sc, uint32_t width, uint32_t height, uint32_t spp,
                  uint32_t max_depth, uint64_t seed, const uint32_t* pixels, uint32_t n_pixels,
                  float* rgb, uint64_t* counters);

/* ---- pttrace.c : the path tracer's work-item streams and schedules (oracle
 * part 2; see pttrace.c).  Op encoding (uint16): */
#define OR_PT_OP_NODE 0x0000u   /* node visit: n0 | n1 << 4 | push << 8 | pop << 9 | end << 10 */
#define OR_PT_OP_PATH 0x2000u   /* a path (sample) starts: camera ray                       */
#define OR_PT_OP_SHADE 0x4000u  /* a ray's shading: outcome | rr << 3 | path ends << 4      */
#define OR_PT_OP_LEAF 0x8000u   /* one triangle test: stage (0..5, see pttrace.c)           */
enum { OR_PT_SH_MISS = 0, OR_PT_SH_LIGHT, OR_PT_SH_DIFFUSE, OR_PT_SH_MIRROR, OR_PT_SH_GLASS };
/* rays / node visits / triangle tests of pixels[0..n_pixels) as per-lane op
 * streams (lane k: ops[off[k] .. off[k+1])) and, if rgb != NULL, their pixel
 * sums (must equal or_pt_render's).  Returns ops used, UINT64_MAX if cap is too
 * small, UINT64_MAX - 1 for a bad image. */
uint64_t or_pt_trace(const unsigned char* img, uint64_t img_bytes, uint32_t width, uint32_t height,
                     uint32_t spp, uint32_t max_depth, uint64_t seed, const uint32_t* pixels,
                     uint32_t n_pixels, uint16_t* ops, uint64_t cap, uint64_t* off, float* rgb);

/* ---- rsbench.c : NEXT-1, RSBench-shaped nested trip-count loop (Fig. 3). */
enum { OR_TAG_RS = 5 };
#define OR_RS_MATS 12
#define OR_RS_NUCLIDES 355
uint32_t or_rs_nuclides(uint32_t m);   /* nuclides of material m            */
uint32_t or_rs_threshold(uint32_t m);  /* cumulative 2^-32 selection bound   */
uint32_t or_rs_pick(uint32_t u);       /* material of a Philox word          */
float or_rs_body(float E, uint32_t nuc, uint32_t fma_count);
/* per thread: acc = sum over lookups of sum over nuclides of body(); nuc =
 * nuclides visited; trips[j*iters+k] (may be NULL) = inner trip count;
 * prolog_fma > 0: the prolog computes E = or_expensive(E, prolog_fma) */
void or_rsbench(uint32_t fma_count, uint32_t prolog_fma, uint64_t t0, uint64_t n,
                uint32_t iters, uint64_t seed, float* acc, uint32_t* nuc, uint32_t* trips);

/* ---- warpsim.c : lane-mask warp simulator (oracle part 2). */
enum { WS_PDOM = 0, WS_SPEC_LOOP = 1, WS_SPEC_CALL = 2, WS_SPEC_LOOP_POOL = 3 };
/* regions of the divloop program (Listing 1) */
enum { WS_DL_ENTRY = 0, WS_DL_PROLOG, WS_DL_EXPENSIVE, WS_DL_EPILOG, WS_DL_ROUND,
       WS_DL_RELEASE, WS_DL_ADVANCE, WS_DL_NREG };
/* regions of the commoncall program (Fig. 2(c)) */
enum { WS_CC_ENTRY = 0, WS_CC_THEN, WS_CC_ELSE_PRE, WS_CC_CALL, WS_CC_ELSE_POST,
       WS_CC_MERGE, WS_CC_NREG };
/* regions of the loop-merge program (Fig. 2(b), Fig. 3) */
enum { WS_LM_ENTRY = 0, WS_LM_LAUNCH, WS_LM_STEP, WS_LM_STEP_BOUNDARY,
       WS_LM_STEP_INTERACT, WS_LM_ROUND, WS_LM_RELEASE, WS_LM_ADVANCE,
       WS_LM_EV0 = 8,      /* .. WS_LM_EV0+15: step lanes whose event has bit b set   */
       WS_LM_NEV0 = 24,    /* .. WS_LM_NEV0+15: step lanes whose event has bit b clear */
       WS_LM_A_RR = 40,    /* roulette of interaction steps (part A)                  */
       WS_LM_B_RR = 41,    /* roulette of boundary steps (part B)                     */
       WS_LM_B_REL = 42,   /* part B of a boundary step; deferred mode: the release,
                              lanes = parked set                                      */
       WS_LM_BI = 43,      /* matched boundary finished inside part A (no part B)     */
       WS_LM_A_TAIL = 44,  /* end of part A: interaction + matched-boundary lanes     */
       WS_LM_CLAIM = 45,   /* dynamic claim: slow path entered (reservoir short)      */
       WS_LM_CLAIMIT = 46, /* dynamic claim: slow-path loop iterations                */
       WS_LM_CHUNK = 47,   /* dynamic claim: chunk fetches from the global counter   */
       WS_LM_NREG = 45 };
#define WS_MAX_REG 48
typedef struct {
  uint64_t rounds;                 /* SR scheduler rounds (0 under PDOM) */
  uint64_t execs[WS_MAX_REG];      /* warp-level executions of a region  */
  uint64_t lanes[WS_MAX_REG];      /* sum of popc(mask) over executions  */
} ws_counts;
/* One warp of W<=32 lanes, lane l valid iff l < n_valid.
 * want[l*L + i] = lane l takes the branch in iteration i. */
void ws_divloop_adv(const uint8_t* want, uint32_t W, uint32_t n_valid, uint32_t L, int mode,
                    uint32_t T, uint32_t V, ws_counts* o);
void ws_divloop(const uint8_t* want, uint32_t W, uint32_t n_valid, uint32_t L,
                int mode, uint32_t T, ws_counts* out);
/* arm[l] = 1 if lane l takes the then-arm (Fig. 2(c) line 8) */
void ws_commoncall(const uint8_t* arm, uint32_t W, uint32_t n_valid, int mode, ws_counts* out);
/* Loop merge: lane l owns tasks k < K; task (l,k) runs nsteps[l*K+k] >= 1 inner
 * iterations; ev (may be NULL) gives each step's bit0 = boundary, laid out
 * per task at ev_off[l*K+k]. */
/* Loop Merge with the merged inner loop partially unrolled by U (U = 1: plain) */
void ws_loopmerge_unrolled(const uint32_t* nsteps, const or_event* ev, const uint64_t* ev_off,
                           uint32_t W, uint32_t n_valid, uint32_t K, int mode, uint32_t T,
                           uint32_t U, ws_counts* out);
/* Loop Merge over a warp-shared task pool (Loop Merge's refill, with
 * the n_valid*K tasks of the warp's threads as one queue): task q is task
 * k = q / n_valid of thread q % n_valid (nsteps[l*K+k] as above); in an advance
 * round every one of the W lanes that is not in a task is in R, and the first
 * |R| unclaimed tasks go to R's lanes in lane order; the pool empty -> R = {}.
 * U = steps per release as in ws_loopmerge_unrolled.  SPEC rule only. */
void ws_loopmerge_pool(const uint32_t* nsteps, uint32_t W, uint32_t n_valid, uint32_t K,
                       uint32_t T, uint32_t U, ws_counts* out);
/* Loop Merge with the MC kernels' dynamic task claiming: the warp's W lanes
 * take tasks q = 0..Q-1 of one stream (nsteps[q] steps, events at ev_off[q]) in
 * claim order.  PDOM: each outer trip every lane claims one task (lane order);
 * the loop ends when no lane got one.  SPEC: an advance round hands the next
 * tasks to the idle lanes of R in lane order; a lane left without one is
 * exhausted (E) from then on.  U = steps per release. */
void ws_loopmerge_stream(const uint32_t* nsteps, const or_event* ev, const uint64_t* ev_off,
                         uint32_t W, uint64_t Q, int mode, uint32_t T, uint32_t U,
                         ws_counts* out);
/* Loop Merge + nested Iteration Delay of the boundary sub-step (warpsim.c) */
void ws_loopmerge_defer(const uint32_t* nsteps, const or_event* ev, const uint64_t* ev_off,
                        uint32_t W, uint32_t n_valid, uint32_t K, uint32_t T, uint32_t Tb,
                        ws_counts* out);
void ws_loopmerge(const uint32_t* nsteps, const or_event* ev, const uint64_t* ev_off,
                  uint32_t W, uint32_t n_valid, uint32_t K, int mode, uint32_t T,
                  ws_counts* out);
/* Exhaustive search (tiny warps) of the minimum number of Expensive
 * executions over ALL legal interleavings of the iteration-delay program
 * (any parked subset may be released, any free lane may advance). */
uint32_t ws_divloop_optimum(const uint8_t* want, uint32_t W, uint32_t L);
/* path tracer schedules (pttrace.c; ops from or_pt_trace) */
enum { WS_PT_ENTRY = 0, WS_PT_OUTER, WS_PT_LAUNCH, WS_PT_BOUNCE, WS_PT_TBEGIN, WS_PT_STEP,
       WS_PT_NODE, WS_PT_PUSH, WS_PT_NOPUSH, WS_PT_NEXTNONE, WS_PT_POP, WS_PT_LEAFIF,
       WS_PT_LEAF, WS_PT_TT, WS_PT_TT_U, WS_PT_TT_V, WS_PT_TT_T, WS_PT_TT_ID, WS_PT_TT_UPD,
       WS_PT_SH, WS_PT_SH_HIT, WS_PT_SH_SURF, WS_PT_SH_DIFF, WS_PT_SH_MIRR, WS_PT_SH_GLASS,
       WS_PT_SH_RR, WS_PT_SH_END, WS_PT_ROUND, WS_PT_REL, WS_PT_LREL, WS_PT_NREL, WS_PT_ADV,
       WS_PT_PSUM };
/* the PDOM (mode WS_PDOM) or split Loop Merge (WS_SPEC_LOOP, threshold T, U
 * work items per release) schedule of one warp of n_valid lanes; WS_SPEC_LOOP_POOL:
 * the split merge with the warp's n_valid x spp paths claimed from one pool
 * (spp <= WS_PT_POOL_MAX_SPP) */
#define WS_PT_POOL_MAX_SPP 64
void ws_pt(const uint16_t* ops, const uint64_t* off, uint32_t n_valid, int mode, uint32_t T,
           uint32_t U, ws_counts* out);

#ifdef __cplusplus
}
#endif
#endif
