// rsbench.cu -- NEXT-1: the RSBench-shaped nested trip-count loop that the
// paper uses to introduce Loop Merge (Fig. 3):
//
//   for (k = 0; k < lookups_per_thread; k++) {            // coarsened outer loop
//     Prolog: material m = pick(), energy E                // 12 materials
//     for (i = 0; i < nuclides(m); i++) L1: xs += body()  // 4 .. 321 trips
//     Epilog: acc += xs
//   }
//
//   rs_pdom  as written: the warp's inner loop runs until the lane with the
//            most nuclides is done ("threads that exit the inner loop early
//            wait for all threads").
//   rs_spec  Loop Merge + soft barrier: lanes whose inner loop ended run their
//            epilog and the next lookup's prolog while the others continue, as
//            in Fig. 3(b)(iii); the inner body runs with the lanes that have
//            nuclides left once popc >= T (or nobody can refill).
// Task sources of rs_spec:
//   static  (SR_F_STATIC) lane l of the warp is thread l of the problem and runs
//           its lookups k = 0..iters-1 itself, in program order;
//   pool    (default) the warp's 32 x iters lookups form one pool: an idle lane
//           claims the next lookup q (lookup k = q / nv of thread q % nv, nv =
//           valid threads of the warp) in lane order, so a lane whose lookups
//           were light keeps working while the heavy 321-nuclide ones finish --
//           no per-lane tail (the MC kernels' dynamic claiming, inside a warp).
//           Each lookup's xs lands in shared memory at [k][thread]; at the end
//           thread l sums its own xs in k order.
// Either way every lookup's nuclide order is program order and each thread's
// acc is the in-order sum of its lookups' xs, so the float results are
// schedule-free (reading R8).
#include <cmath>

#include "sr_device.cuh"
#include "sr_internal.h"

namespace sr {
namespace {

constexpr uint32_t kMats = 12, kNuclides = 355;
constexpr uint64_t kRsPoolSmemMax = 160 * 1024;  // pool smem per CTA; above it: static
__constant__ uint32_t c_nucs[kMats] = {321, 5, 4, 4, 27, 21, 21, 21, 21, 21, 9, 9};

struct RsArgs {
  uint64_t t0, n;
  RoundKeys keys;
  uint32_t thr[kMats];   // cumulative selection thresholds (host-computed)
  uint32_t iters, rounds, T;
  uint32_t prolog_rounds;  // expensive prolog (task fetch): 0 = none
  uint32_t unroll;         // inner iterations per release (partial unroll)
  uint2* out;            // {acc bits, nuclides}
  unsigned long long* counters;
  uint32_t* sched;
};

__device__ __forceinline__ uint32_t pick(const RsArgs& a, uint32_t u) {
  uint32_t m = kMats - 1;
#pragma unroll
  for (int i = kMats - 2; i >= 0; --i)
    if (u < a.thr[i]) m = (uint32_t)i;
  return m;
}

// Prolog energy: U01(u1), or Expensive() of it for an expensive task fetch.
// PROLOG > 0: compile-time rounds; 0: none; < 0: a.prolog_rounds at run time.
template <int PROLOG>
__device__ __forceinline__ float energy(const RsArgs& a, uint32_t u1) {
  const float E = u01(u1);
  if constexpr (PROLOG > 0) return expensive<PROLOG>(E, 0u);
  else if constexpr (PROLOG < 0) return a.prolog_rounds ? expensive<0>(E, a.prolog_rounds) : E;
  else return E;
}

// K: chains_round's addend pairs held in registers by the kernel (chain_addends;
// compile-time ROUNDS only)
template <int ROUNDS>
__device__ __forceinline__ float body(float E, uint32_t m, uint32_t i, uint32_t rounds,
                                      const ChainAdd& K) {
  const uint32_t nuc = (37u * m + 13u * i) % kNuclides;
  const float start = E + (float)nuc * 0x1p-9f;
  if constexpr (ROUNDS > 0) return expensive_k<ROUNDS>(start, K);
  else return expensive<0>(start, rounds);
}

__device__ __forceinline__ void finish(const RsArgs& a, uint64_t g, bool valid, float acc,
                                       uint32_t nucs, uint32_t rounds, uint32_t rel,
                                       uint32_t rel_lanes, uint32_t adv, uint32_t adv_lanes) {
  if (valid) a.out[g] = make_uint2(__float_as_uint(acc), nucs);
  const uint32_t tot = __reduce_add_sync(kFull, valid ? nucs : 0u);
  if (lane_id() == 0) {
    atomicAdd(a.counters, (unsigned long long)tot);
    if (a.sched && (g & ~31ull) < a.n) {
      uint4* p = reinterpret_cast<uint4*>(a.sched + (g >> 5) * kSchedWords);
      p[0] = make_uint4(rounds, rel, rel_lanes, adv);
      p[1] = make_uint4(adv_lanes, 0u, 0u, 0u);
    }
  }
}

template <int ROUNDS, int PROLOG, bool SCHED>
__global__ void __launch_bounds__(SR_RS_MAXT) rs_pdom(const RsArgs a) {
  const uint64_t g = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;  // @sr-region ENTRY:full
  const ChainAdd K = chain_addends(a.rounds - (uint32_t)ROUNDS);  // a.rounds == ROUNDS here
  const bool valid = g < a.n;
  const uint64_t t = a.t0 + g;
  float acc = 0.0f;
  uint32_t nucs = 0, rel = 0, rel_lanes = 0;
  for (uint32_t k = 0; k < a.iters; ++k) {  // @sr-region LAUNCH:full
    uint32_t N = 0, m = 0;
    float E = 0.0f;
    if (valid) {
      const uint4 u = draw(k, kTagRs, t, a.keys);  // @sr-region LAUNCH
      m = pick(a, u.x);
      E = energy<PROLOG>(a, u.y);
      N = c_nucs[m];
    }
    float xs = 0.0f;
#pragma unroll 1  // one body per trip, as written (an unrolled remainder would split trips)
    for (uint32_t i = 0; i < N; ++i) {  // @sr-region STEP
      if constexpr (SCHED) {
        const uint32_t mk = __activemask();
        if (lane_id() == (uint32_t)(__ffs(mk) - 1)) { ++rel; rel_lanes += __popc(mk); }
      }
      xs = xs + body<ROUNDS>(E, m, i, a.rounds, K);
    }
    acc = acc + xs;  // @sr-region LAUNCH:full
    nucs += N;
  }
  uint32_t r = 0, rl = 0;  // @sr-region ENTRY:full
  if constexpr (SCHED) { r = __reduce_add_sync(kFull, rel); rl = __reduce_add_sync(kFull, rel_lanes); }
  finish(a, g, valid, acc, nucs, a.iters, r, rl, a.iters, a.iters * (uint32_t)__popc(__ballot_sync(kFull, valid)));
}  // @sr-region END

template <int ROUNDS, int PROLOG, bool SCHED, bool POOL>
__global__ void __launch_bounds__(SR_RS_MAXT) rs_spec(const RsArgs a) {
  extern __shared__ float rs_xs[];  // POOL: per warp xs[iters][32], then nucs[32]
  const uint64_t g = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;  // @sr-region ENTRY:full
  const ChainAdd K = chain_addends(a.rounds - (uint32_t)ROUNDS);  // a.rounds == ROUNDS here
  const bool valid = g < a.n;
  uint64_t t = a.t0 + g;
  float acc = 0.0f, xs = 0.0f, E = 0.0f;
  uint32_t nucs = 0, k = 0, i = 0, N = 0, m = 0;
  bool busy = false;                       // inside a lookup's inner loop
  uint32_t rounds = 0, rel = 0, rel_lanes = 0, adv = 0, adv_lanes = 0;
  // POOL state (warp-uniform): valid threads, pool size, next unclaimed lookup
  const uint32_t nv = POOL ? (uint32_t)__popc(__ballot_sync(kFull, valid)) : 0u;
  const uint32_t pool = nv * a.iters;
  uint32_t qnext = 0, own = 0;             // own: thread (lane of the warp) of the lookup
  float* const xw = rs_xs + (threadIdx.x >> 5) * (a.iters * 32u + 32u);
  uint32_t* const nw = reinterpret_cast<uint32_t*>(xw + a.iters * 32u);
  if constexpr (POOL) {
    nw[lane_id()] = 0u;
    __syncwarp();
  }
  uint32_t E_mask = POOL ? (pool == 0u ? kFull : 0u)                 // nothing left (Cancel)
                         : __ballot_sync(kFull, !valid || a.iters == 0);
  uint32_t P = __ballot_sync(kFull, busy);  // round ballot, re-taken at the latch
  for (;;) {
    const uint32_t R = ~(P | E_mask);  // @sr-region ROUND:full
    if ((P | R) == 0u) break;
    if constexpr (SCHED) ++rounds;
    if ((uint32_t)__popc(P) >= a.T || R == 0u) {
      if constexpr (SCHED) { ++rel; rel_lanes += __popc(P); }  // @sr-region RELEASE:full
      if (busy) {
        __syncwarp(P);  // @sr-region STEP
        // up to `unroll` inner iterations per release; a lane whose lookup ends
        // inside the release idles for the rest of it
        for (uint32_t r = 0; r < a.unroll && busy; ++r) {
          xs = xs + body<ROUNDS>(E, m, i, a.rounds, K);
          i = i + 1u;
          if (i == N) {                    // inner loop done: Epilog
            if constexpr (POOL) {
              xw[(k - 1u) * 32u + own] = xs;  // k - 1: the lookup this lane holds
              atomicAdd(&nw[own], N);
            } else {
              acc = acc + xs;
              nucs += N;
            }
            busy = false;
          }
        }
      }
    } else {
      if constexpr (SCHED) { ++adv; adv_lanes += __popc(R); }  // @sr-region ADVANCE:full
      bool go = (R >> lane_id()) & 1u;
      if constexpr (POOL) {
        // claim in lane order: lookup q = qnext + rank among the idle lanes
        const uint32_t q = qnext + (uint32_t)__popc(R & lanemask_lt());
        go = go && q < pool;
        if (go) {
          own = nv == 32u ? (q & 31u) : q % nv;  // @sr-region LAUNCH
          k = nv == 32u ? (q >> 5) : q / nv;
          t = a.t0 + (g & ~31ull) + own;
        }
        qnext = min(pool, qnext + (uint32_t)__popc(R));  // @sr-region ADVANCE:full
      }
      if (go) {
        const uint4 u = draw(k, kTagRs, t, a.keys);  // @sr-region LAUNCH
        m = pick(a, u.x);
        E = energy<PROLOG>(a, u.y);
        N = c_nucs[m];
        i = 0;
        xs = 0.0f;
        busy = true;
        ++k;
      }
      if constexpr (POOL) E_mask = qnext >= pool ? kFull : 0u;  // @sr-region ADVANCE:full
      else E_mask = __ballot_sync(kFull, !valid || k >= a.iters);
    }
    P = __ballot_sync(kFull, busy);  // @sr-region ROUND:full
  }
  if constexpr (POOL) {  // @sr-region ENTRY:full
    __syncwarp();
    if (valid) {  // this thread's lookups in program order
#pragma unroll 1  // one trip per lookup (the simulator's PERK count)
      for (uint32_t kk = 0; kk < a.iters; ++kk) acc = acc + xw[kk * 32u + lane_id()];  // @sr-region PERK:full
      nucs = nw[lane_id()];  // @sr-region ENTRY:full
    }
  }
  finish(a, g, valid, acc, nucs, rounds, rel, rel_lanes, adv, adv_lanes);  // @sr-region ENTRY:full
}  // @sr-region END

template <bool SCHED>
cudaError_t set_rs_smem(const RsArgs& a, int smem) {
  cudaError_t e = cudaSuccess;
  auto set = [&](auto kern) {
    if (e == cudaSuccess)
      e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  };
  if (a.rounds == 8 && a.prolog_rounds == 0) set(rs_spec<8, 0, SCHED, true>);
  else if (a.rounds == 8 && a.prolog_rounds == 256) set(rs_spec<8, 256, SCHED, true>);
  else set(rs_spec<0, -1, SCHED, true>);
  return e;
}

template <bool SCHED>
cudaError_t launch_t(const LaunchCtx& c, const RsArgs& a, int mode, bool pool) {
  const uint32_t block = c.block;
  const uint64_t grid = (a.n + block - 1) / block;
  if (grid > 0x7fffffffull) return cudaErrorInvalidConfiguration;
  const bool spec = mode == SR_SPEC_LOOP;
  // the pool's shared memory: per warp iters x 32 xs + 32 nuclide counts
  const size_t smem = pool ? (size_t)(block / 32) * ((size_t)a.iters * 32 + 32) * 4 : 0;
  record_launch((uint32_t)grid, block, (uint32_t)smem);
  if (smem > 48 * 1024) {
    cudaError_t e = set_rs_smem<SCHED>(a, (int)smem);
    if (e != cudaSuccess) return e;
  }
#define SR_RS(R, PR)                                                                      \
  (spec ? (pool ? rs_spec<R, PR, SCHED, true><<<(unsigned)grid, block, smem, c.stream>>>(a) \
                : rs_spec<R, PR, SCHED, false><<<(unsigned)grid, block, 0, c.stream>>>(a)) \
        : rs_pdom<R, PR, SCHED><<<(unsigned)grid, block, 0, c.stream>>>(a))
  // compile-time shapes of the measured configurations (straight-line code,
  // static SASS costs for the simulator); anything else runs the generic one
  if (a.rounds == 8 && a.prolog_rounds == 0) SR_RS(8, 0);
  else if (a.rounds == 8 && a.prolog_rounds == 256) SR_RS(8, 256);
  else SR_RS(0, -1);
#undef SR_RS
  return cudaGetLastError();
}

}  // namespace

bool rs_pool_fits(uint32_t iters, uint32_t block) {
  return (uint64_t)(block / 32) * ((uint64_t)iters * 32 + 32) * 4 <= kRsPoolSmemMax;
}

cudaError_t launch_rsbench(const LaunchCtx& c, const sr_workload& w, uint64_t n, uint32_t iters,
                           uint64_t seed, int mode, uint32_t T) {
  // cumulative selection thresholds floor(2^32 * sum_{i<=m} p_i), last = 2^32-1
  static const double prob[kMats] = {0.140, 0.052, 0.275, 0.134, 0.154, 0.064,
                                     0.066, 0.055, 0.008, 0.015, 0.025, 0.013};
  RsArgs a;
  double cum = 0.0;
  for (uint32_t mm = 0; mm < kMats; ++mm) {
    cum += prob[mm];
    a.thr[mm] = mm + 1 == kMats ? 0xFFFFFFFFu : (uint32_t)std::floor(cum * 4294967296.0);
  }
  a.t0 = w.task_offset;
  a.n = n;
  a.keys = round_keys(seed);
  a.iters = iters;
  a.rounds = w.rsbench.fma_count / 8u;
  a.prolog_rounds = w.rsbench.prolog_fma / 8u;
  a.unroll = w.rsbench.merge_unroll ? w.rsbench.merge_unroll : 1u;
  a.T = T;
  a.out = reinterpret_cast<uint2*>(c.ws + c.lay.off[SR_T_PERTHREAD]);
  a.counters = reinterpret_cast<unsigned long long*>(c.ws + c.lay.off[SR_T_COUNTERS]);
  a.sched = (w.flags & SR_F_SCHED) ? reinterpret_cast<uint32_t*>(c.ws + c.lay.off[SR_T_SCHED])
                                   : nullptr;
  // the warp pool unless SR_F_STATIC, or its shared memory would not fit
  const uint32_t block = c.block;
  const bool pool = !(w.flags & SR_F_STATIC) && rs_pool_fits(iters, block);
  return a.sched ? launch_t<true>(c, a, mode, pool) : launch_t<false>(c, a, mode, pool);
}

}  // namespace sr
