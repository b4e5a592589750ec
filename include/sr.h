/*
 * sr.h -- C ABI of libsr, the B200-native (sm_100a) Speculative
 * Reconvergence hot path.
 *
 * Paper: Damani, Johnson, Stephenson, Keckler, Yan, McKeown, Giroux,
 * "Speculative Reconvergence for Improved SIMT Efficiency", CGO 2020.
 * "P:N" = line N of the paper text.
 *
 * The paper's user interface is a Predict(label) directive, a label marking
 * the reconvergence point, a function name for the common-call case and an
 * optional soft-barrier threshold (Sec. 4.1; Sec. 4.4
 * P:999-1002; Sec. 4.6).  Here the prediction region and label are
 * fixed per workload (the annotated loops of Fig. 2) and a call
 * selects the schedule with `mode` and the soft barrier with `threshold`.
 *
 * Conventions for every entry point:
 *   - returns SR_OK (0) or a negative sr_status; never throws, never aborts;
 *     sr_last_error() describes the last failure of the calling thread;
 *   - arguments are validated before any GPU work is enqueued;
 *   - all GPU work is enqueued on the stream given to sr_init (a cudaStream_t
 *     passed as void*; NULL = legacy default stream), in order;
 *   - device memory is owned by the caller; the library allocates none;
 *   - one process-global context per process (= per GPU); not re-entrant.
 */
#ifndef SR_H
#define SR_H
#include <stddef.h>
#include <stdint.h>

#if defined(__GNUC__)
#define SR_API __attribute__((visibility("default")))
#else
#define SR_API
#endif

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  SR_OK = 0,
  SR_E_INVALID = -1,  /* bad argument (see each call)                       */
  SR_E_STATE = -2,    /* call before sr_init / after sr_finalize / no run   */
  SR_E_NOMEM = -3,    /* workspace or destination buffer too small          */
  SR_E_CUDA = -4      /* CUDA runtime error; message carries the CUDA text  */
} sr_status;

/* Schedules.  SR_PDOM: plain structured code; the compiler reconverges at
 * the immediate post-dominator.  SR_SPEC_LOOP:
 * Iteration Delay / Loop Merge (Fig. 1(b)) with soft barrier
 * (Sec. 4.6).  SR_SPEC_CALL: reconvergence at the entry of the common
 * callee (Fig. 2(c), Sec. 4.4). */
typedef enum { SR_PDOM = 0, SR_SPEC_LOOP = 1, SR_SPEC_CALL = 2 } sr_mode;

typedef enum {
  SR_WL_DIVLOOP = 0,     /* Fig. 2(a): divergent condition in a loop (config 1) */
  SR_WL_COMMONCALL = 1,  /* Fig. 2(c): common function call          (config 2) */
  SR_WL_MCML = 2,        /* Fig. 2(b): MC photon transport, loop merge (3, 5)  */
  SR_WL_PATHTRACE = 3,   /* Fig. 2(b): path tracer, loop merge       (config 4) */
  SR_WL_RSBENCH = 4      /* Fig. 3: RSBench-shaped nested trip-count loop (NEXT-1) */
} sr_workload_kind;

/* sr_workload.flags */
#define SR_F_SCHED 1u   /* also write per-warp schedule counters (instrumented kernels) */
#define SR_F_STATIC 2u  /* MCML / PATHTRACE: static task->lane assignment (lane l owns tasks
                           l + k*n_threads) instead of the default dynamic per-warp claiming.
                           RSBENCH + SR_SPEC_LOOP: lane l runs thread l's lookups itself
                           instead of the default warp task pool (idle lanes claim the
                           warp's next lookup in lane order; per-lookup xs staged in shared
                           memory, (block/32)*(iters*32+32)*4 bytes per CTA, and summed per
                           thread in program order at the end; above 160 KB the static
                           assignment is used).  Results are identical; only the schedule
                           differs. */
#define SR_F_COARSE 4u  /* PATHTRACE + SR_SPEC_LOOP: merge at bounce granularity (one release =
                           traversal + shading of one bounce) instead of the default BVH-node
                           granularity (one release = one node visit). Results are identical. */
#define SR_F_NOSPLIT 8u /* PATHTRACE + SR_SPEC_LOOP at node granularity: one merged region per
                           node visit (its leaf triangle tests inline) instead of the default
                           two concurrent predictions, where inner-node visits
                           and leaf triangle tests are separate regions and each round runs the
                           larger waiting group (soft barrier T) while the other lanes wait.
                           Results and counters are identical (each lane's traversal order is
                           the same). */
#define SR_F_MATGROUP 16u /* PATHTRACE + SR_SPEC_LOOP, split node merge (the default): NEXT-3's
                           same-material grouping of the shading step -- in an
                           advance round the lanes that must shade a hit are grouped by material
                           kind (__match_any_sync); only the largest group shades, the others
                           wait for a later advance round.  Results and counters are identical. */
#define SR_F_POOL 32u   /* DIVLOOP + SR_SPEC_LOOP (needs prolog_batch = 64): Loop Merge of the
                           Expensive() calls over a warp task pool -- after each lane has run
                           ahead through a window's prologs, the warp's wanted (thread,
                           iteration) pairs are one queue and every release runs 32 of them,
                           any lane running any thread's call; results are added to each
                           thread's acc in iteration order.  `threshold` is not used.
                           Results are identical.
                           PATHTRACE + SR_SPEC_LOOP, split node merge (not with COARSE,
                           NOSPLIT or MATGROUP; needs pathtrace.pool_spp): the warp's
                           pixels x spp paths form one pool -- a lane whose path has ended
                           claims the next (sample-major) in an advance round, so no lane
                           idles while its warp has paths left; each path's radiance is
                           kept and the pixel sums are formed in sample order at the end.
                           Images and counters are identical. */

#define SR_MAX_LAYERS 8
typedef struct { float n, mua, mus, g, d; } sr_layer;  /* -, 1/cm, 1/cm, -, cm */

typedef struct {
  uint32_t p_u32;      /* P(condition) = p_u32 / 2^32 (1/8: 2^29)               */
  uint32_t fma_count;  /* FMAs in Expensive(); multiple of 8 (1000)             */
  uint32_t advance_unroll; /* SR_SPEC_LOOP: iterations a run-ahead lane may take in
                          one advance round before it parks (0 = 1, reading Q5).
                          Results are identical for every value.               */
  uint32_t prolog_batch; /* both modes: 0 or 1 = each iteration's Prolog (its one
                          Philox draw, reading R3) evaluated in program order,
                          one draw at a time, as Fig. 2(a) is written; 64 = a lane
                          evaluates the divergent conditions of up to 64 of its
                          iterations together (independent counters, ILP) into a
                          64-bit mask and keeps the Expensive() arguments of the
                          iterations that call it in shared memory (256 bytes per
                          thread; needs block_threads <= 512) (reading Q5').
                          Other values: SR_E_INVALID.  Results and schedule
                          counters are identical.                              */
  uint32_t pool_split;   /* with SR_F_POOL: warps per group of 32 threads, each
                          taking 64/pool_split iterations of every 64-iteration
                          window (0 or 1 = one warp; 2; 4 -- a CTA is one group
                          of pool_split warps, block_threads is not used).
                          Other values: SR_E_INVALID.  Results are identical. */
} sr_divloop_params;

typedef struct {
  uint32_t fma_count;  /* FMAs in the common callee foo(); multiple of 8 (2000)  */
  uint32_t split_u32;  /* P(then-arm) = split_u32 / 2^32 (1/2: 2^31)             */
} sr_commoncall_params;

typedef struct {
  uint32_t n_layers;   /* 1 .. SR_MAX_LAYERS                                     */
  sr_layer layers[SR_MAX_LAYERS];
  float n_above, n_below;  /* ambient refractive indices                         */
  float dr, dz;            /* tally grid spacing, cm                             */
  uint32_t nr, nz;         /* tally grid size (nr, nz >= 1)                      */
  uint32_t step_cap;       /* a photon dies after this many steps (>= 1)         */
  uint32_t defer_threshold;  /* SR_SPEC_LOOP only: 0 = off; T_b in [1,32] = nest an
                                Iteration Delay of the boundary sub-step (Fresnel /
                                transmit / exit) inside the Loop Merge: parked
                                boundary lanes run together once T_b have arrived
                                (two concurrent predictions).  Results
                                are identical for every value.                    */
  uint32_t merge_unroll;   /* SR_SPEC_LOOP: photon steps per release round, the
                              partial unroll of the merged loop;
                              0 = 1.  Results are identical for every value.    */
} sr_mcml_params;

typedef struct {
  const void* scene_dev;  /* device pointer to a scene built by sr_scene_build  */
  uint64_t scene_bytes;
  uint32_t width, height; /* image; n_threads must equal width*height           */
  uint32_t max_depth;     /* bounces per path (>= 1)                            */
  uint32_t merge_unroll;  /* SR_SPEC_LOOP node-granularity merge: BVH node visits
                             per release round, the partial unroll of P:1467-1474
                             (0 = 8). Results are identical for every value.   */
  uint32_t pool_spp;      /* with SR_F_POOL: the most samples per pixel (sr_run
                             iters) a run may ask for, in [1, 4096]; the workspace
                             then holds 12 * n_threads * pool_spp bytes of per-path
                             radiance (in SR_T_SCRATCH).  0 without SR_F_POOL.   */
} sr_pathtrace_params;

typedef struct {
  uint32_t fma_count;  /* FMAs of the per-nuclide body; multiple of 8 (64)       */
  uint32_t prolog_fma; /* FMAs of the lookup prolog (an expensive task fetch,
                          E = Expensive(E, prolog_fma)); multiple of 8, <= 65536;
                          0 = none (configs: 0; the Fig. 9 XSBench-like sweep: 2048) */
  uint32_t merge_unroll; /* SR_SPEC_LOOP: inner-loop iterations per release round,
                          the partial unroll of P:1467-1474 (0 = 1). Results are
                          identical for every value.                             */
} sr_rsbench_params;   /* materials / nuclide counts: DESIGN.md reading R8       */

typedef struct {
  int32_t kind;            /* sr_workload_kind                                   */
  uint32_t flags;          /* SR_F_*                                             */
  uint64_t task_offset;    /* global id of this caller's first task (sharding)  */
  uint32_t block_threads;  /* CTA size, multiple of 32 in [32, bound]; 0 = default.
                              bound: MCML 640, PATHTRACE 128, RSBENCH 256, else 1024
                              (the kernels' __launch_bounds__)                   */
  uint32_t grid_ctas;      /* dynamic-claiming kernels: CTAs; 0 = fill the GPU   */
  sr_divloop_params divloop;
  sr_commoncall_params commoncall;
  sr_mcml_params mcml;
  sr_pathtrace_params pathtrace;
  sr_rsbench_params rsbench;
} sr_workload;

/* Bind the context to a device, a stream and a caller-owned device
 * workspace.  May be called again to rebind (e.g. a bigger workspace).
 * SR_E_CUDA if the device cannot be selected (for instance, no GPU). */
SR_API int sr_init(int device, void* cuda_stream, void* workspace_dev, size_t workspace_bytes);

/* Workspace regions, each 256-byte aligned, in this order:
 *   SR_T_PERTHREAD  per-task outputs of the last run:
 *                   DIVLOOP    n_threads x {float acc; uint32 cnt}  (8 B, AoS)
 *                   COMMONCALL n_threads x float y
 *                   MCML       none (0 bytes)
 *                   PATHTRACE  n_threads x float[3] RGB sum over the spp, pixel-major
 *                              (row y, column x at y * width + x).  Lanes to
 *                              pixels: when width % 8 == 0 and height % 4 == 0,
 *                              warp w covers the w-th 8 x 4 tile (tiles
 *                              row-major, lanes row-major inside the tile),
 *                              else thread g has pixel g; the SR_T_SCHED record
 *                              of warp w describes that warp's pixels.
 *   SR_T_GRID       MCML: uint64 A[nz][nr], Rd[nr], Tt[nr]  (fixed point, 2^-32)
 *   SR_T_COUNTERS   uint64[16] workload counters (see sr_counter_names in DESIGN.md)
 *   SR_T_SCHED      per warp: uint32[8] schedule counters (only with SR_F_SCHED):
 *                   {rounds, release rounds, common-code lane-executions,
 *                    advance rounds, lanes taking part in advance rounds
 *                    (sum of popc(R); with DIVLOOP advance_unroll > 1 a lane
 *                    may run several prologs in one such round), 0, 0, 0};
 *                   one record per launched warp (warps past n_threads are
 *                   not written).  DIVLOOP with SR_F_POOL: one record per group
 *                   of 32 threads, {rounds, releases, Expensive() calls run,
 *                   windows x slices (the batched advances), that x valid
 *                   lanes, 0, 0, 0}.  PATHTRACE split merge: words 5, 6 =
 *                   leaf-test releases and their lanes (words 1, 2: node visits)
 *   SR_T_SCRATCH    internal (claim counters; PATHTRACE + SR_F_POOL: per-path radiance)
 * GRID and COUNTERS are contiguous so a multi-GPU caller can reduce them
 * in place as int64 (two's-complement addition = uint64 addition mod 2^64). */
enum { SR_T_PERTHREAD = 0, SR_T_GRID = 1, SR_T_COUNTERS = 2, SR_T_SCHED = 3, SR_T_SCRATCH = 4 };
SR_API size_t sr_workspace_bytes(const sr_workload* w, uint64_t n_threads);
SR_API int sr_workspace_region(const sr_workload* w, uint64_t n_threads, int what, size_t* offset,
                        size_t* bytes);

/* Run the hot path: n_threads logical threads, each executing `iters`
 * iterations of its outer loop (DIVLOOP: loop trips; COMMONCALL: repetitions;
 * MCML: photons per thread = thread coarsening P:336-359; PATHTRACE: samples
 * per pixel).  threshold: soft-barrier size T in [1,32], 0 = 32 ("wait for
 * all", Fig. 1(b)); ignored for SR_PDOM; must be 0 or 32 for SR_SPEC_CALL.
 * SR_SPEC_CALL is valid only for COMMONCALL; SR_SPEC_LOOP only for DIVLOOP,
 * MCML, PATHTRACE, RSBENCH.  Zeroes the output regions, then enqueues the
 * kernel(s); does not synchronize, so a run can be captured in a CUDA graph.
 * (PATHTRACE: the scene header is known on the host when sr_scene_build wrote
 * the image in this process; an image copied in by the caller is read once,
 * synchronously on the context stream -- SR_E_CUDA if that stream is
 * capturing -- and remembered afterwards.)  Every output bit is a function of (workload params,
 * seed, task ids) only -- never of mode, threshold, block size, grid size or
 * GPU count.
 * Errors: SR_E_STATE before sr_init; SR_E_INVALID (n_threads == 0,
 * n_threads*iters overflows 2^63, bad threshold/mode/params); SR_E_NOMEM
 * (workspace smaller than sr_workspace_bytes); SR_E_CUDA (launch failed). */
SR_API int sr_run(const sr_workload* w, uint64_t n_threads, uint32_t iters, uint64_t seed, int mode,
           uint32_t threshold);

/* Copy one region of the last run (what = SR_T_*) into dst, host or device
 * memory (UVA, cudaMemcpyDefault), on the context stream, then synchronize
 * that stream.  *written (may be NULL) receives the byte count.
 * SR_E_NOMEM if dst_bytes is smaller than the region. */
SR_API int sr_tally(int what, void* dst, size_t dst_bytes, size_t* written);

/* Release the context.  Idempotent. */
SR_API int sr_finalize(void);

/* Thread-local description of the last error; library-owned; valid until
 * the next call on this thread.  Empty string after success. */
SR_API const char* sr_last_error(void);

/* Library build identification: "sm_100a <nvcc version> <flags>". */
SR_API const char* sr_build_info(void);

/* Launch configuration of the last kernel sr_run enqueued:
 * out[0] = CTAs, out[1] = threads per CTA, out[2] = dynamic shared memory
 * bytes per CTA, out[3] = kernels launched by that sr_run.
 * SR_E_STATE if no run happened since sr_init. */
SR_API int sr_last_launch(uint32_t out[4]);

/* Diagnostics: evaluate one device building block of the hot path element
 * by element, out[i] = fn(x[i]), on the context stream (no synchronize).
 * x_dev, out_dev: device arrays of n floats, caller-owned.
 *   SR_FN_LOGF            sr_logf(x), x in (0,1]            (R5)
 *   SR_FN_SIN2PI/COS2PI   sin/cos(2 pi x), x = k 2^-24       (R5)
 *   SR_FN_EXPENSIVE_1000  Expensive() of config 1 started at x (R3)
 *   SR_FN_EXPENSIVE_2000  foo() of config 2 started at x     (R4)
 * Errors: SR_E_STATE before sr_init; SR_E_INVALID (unknown fn, NULL with
 * n > 0); SR_E_CUDA. */
enum { SR_FN_LOGF = 0, SR_FN_SIN2PI = 1, SR_FN_COS2PI = 2, SR_FN_EXPENSIVE_1000 = 3,
       SR_FN_EXPENSIVE_2000 = 4 };
SR_API int sr_math_eval(int fn, const float* x_dev, float* out_dev, uint64_t n);

/* Diagnostics: the MC step's IEEE divisions and square roots on their known
 * operand domains (nvcc's fast path without the FCHK range
 * check and slow-path branch), out[i] = fn(p, x[i]), on the context stream
 * (no synchronize).  x_dev, out_dev: device arrays of n floats, caller-owned.
 *   SR_FNP_DIV_XP    x / p             (div_dom)
 *   SR_FNP_DIV_PX    p / x             (div_dom)
 *   SR_FNP_SQRT      sqrt(x)           (sqrt_dom, p unused)
 *   SR_FNP_HG_COST   Henyey-Greenstein cos(theta) for g = p, xi = x (R6)
 *   SR_FNP_HG_SINT   sqrt(1 - cos(theta)^2) of the same
 *   SR_FNP_DIV2_XP   (x[2j], x[2j+1]) / p as one f32x2 pair (div2_dom, the
 *                    rotation's two quotients)
 *   SR_FNP_FRESNEL + v, v in [0, 8): MCML's Fresnel sub-step for cos(incidence)
 *                    = x at indices (ni, nt) = (p, 1) (v bit 2 clear) or (1, p)
 *                    (set); the reflectance (v bit 1 clear) or the transmitted
 *                    cosine ca2 (set); the FAST kernels' operations (v bit 0 set)
 *                    or the guarded IEEE ones (clear)
 * Each equals the IEEE binary32 result bit for bit on the domain its call
 * site guarantees; outside it the result is unspecified.
 * Errors: SR_E_STATE before sr_init; SR_E_INVALID (unknown fn, NULL with
 * n > 0); SR_E_CUDA. */
enum { SR_FNP_DIV_XP = 0, SR_FNP_DIV_PX = 1, SR_FNP_SQRT = 2, SR_FNP_HG_COST = 3,
       SR_FNP_HG_SINT = 4, SR_FNP_DIV2_XP = 5, SR_FNP_FRESNEL = 8 };
SR_API int sr_math_eval_p(int fn, float p, const float* x_dev, float* out_dev, uint64_t n);

/* Diagnostics: closest hit of n rays against a scene built by sr_scene_build,
 * with the BVH traversal the PATHTRACE kernels use (reading R7).
 *   rays_dev  device, n x 6 floats {origin xyz, direction xyz}
 *   hit_dev   device, n int64: original triangle index (ties -> smaller
 *             index), -1 = no hit with t > 1e-4
 *   t_dev     device, n floats: hit distance (+inf on a miss)
 * On the context stream; no synchronize.  Errors: SR_E_STATE before
 * sr_init; SR_E_INVALID (NULL arrays with n > 0, not a scene image). */
SR_API int sr_pt_closest(const void* scene_dev, const float* rays_dev, int64_t* hit_dev,
                         float* t_dev, uint64_t n);

/* PATHTRACE scene (config 4): build the BVH over a caller-provided triangle
 * soup on the host and write the device scene image.
 *   tris       host, n_tris x 9 floats (v0, v1, v2 xyz), caller-owned
 *   mat        host, n_tris x uint32 material ids (< n_mats)
 *   mats       host, n_mats x 8 floats {kind, r, g, b, er, eg, eb, ior}
 *              kind: 0 diffuse, 1 mirror, 2 dielectric, 3 emissive-only
 *   cam        host, 14 floats {eye xyz, forward xyz, right xyz, up xyz (an
 *              orthonormal basis), tan(fov/2), aspect = width/height}
 *   dst_dev    device buffer of dst_bytes; *needed receives the size.  If
 *              dst_dev is NULL only *needed is computed (an upper bound; after
 *              a build, the exact image size).
 * The image (pt_scene.h layout: header, two-wide BVH nodes, triangles in BVH
 * order, materials) is deterministic for a given input.  The header records
 * the deepest traversal stack a ray can need; the PATHTRACE kernels reject a
 * scene needing more than 256 entries.  Errors: SR_E_INVALID (NULL inputs,
 * n_tris = 0 or >= 2^31, material id >= n_mats, material kind not 0..3,
 * non-finite vertices),
 * SR_E_NOMEM (dst_bytes < *needed), SR_E_CUDA (the copy failed). */
SR_API int sr_scene_build(const float* tris, const uint32_t* mat, uint32_t n_tris, const float* mats,
                   uint32_t n_mats, const float* cam, void* dst_dev, size_t dst_bytes,
                   size_t* needed);

/* The same build into HOST memory (dst_host): no device, no context needed --
 * for inspecting / validating the BVH on the CPU. */
SR_API int sr_scene_build_host(const float* tris, const uint32_t* mat, uint32_t n_tris,
                               const float* mats, uint32_t n_mats, const float* cam,
                               void* dst_host, size_t dst_bytes, size_t* needed);

#ifdef __cplusplus
}
#endif
#endif
