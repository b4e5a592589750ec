// commoncall.cu -- config 2: "Common Function Call" (Fig. 2(c), P:443-463;
// Sec. 4.4).
//
//   foo() { Expensive(); }
//   if (divergent_condition()) { foo(); } else { ...; foo(); ...; }
//
//   commoncall_pdom  as written: foo is __noinline__ and called from both arms,
//                    so the warp runs foo twice, once per arm, each time with
//                    the lanes of that arm only; the arms reconverge at the
//                    post-dominator of the if/else.
//   commoncall_spec  call merge: the arms only compute foo's argument; all
//                    lanes reconverge (__syncwarp) at the entry of the single
//                    call -- "the function name ... indicate[s] the PC at which
//                    all threads must wait" -- and the divergent
//                    tail of the else arm runs after it.  No prolog/epilog
//                    serialization is added; the cost is the barrier
//                    (P:1004-1009).
#include "sr_device.cuh"
#include "sr_internal.h"

namespace sr {
namespace {

struct CallArgs {
  uint64_t t0, n, seed;
  RoundKeys keys;
  uint32_t iters, split_u32, rounds;
  float* y;
  unsigned long long* counters;
  uint32_t* sched;
};

template <int ROUNDS>
__device__ __noinline__ float foo(float v, uint32_t rounds) {
  return expensive<ROUNDS>(v, rounds);
}

template <bool SCHED>
__device__ __forceinline__ void count_call(uint32_t& execs, uint32_t& lanes) {
  if constexpr (SCHED) {
    const uint32_t m = __activemask();
    if (lane_id() == (uint32_t)(__ffs(m) - 1)) { ++execs; lanes += __popc(m); }
  }
}

template <int ROUNDS, bool SCHED>
__global__ void __launch_bounds__(1024) commoncall_pdom(const CallArgs a) {
  const uint64_t g = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;  // @sr-region ENTRY:full
  if (g >= a.n) return;
  const uint64_t t = a.t0 + g;
  float ysum = 0.0f;
  uint32_t then_cnt = 0, execs = 0, lanes = 0;
  for (uint32_t it = 0; it < a.iters; ++it) {  // @sr-region MERGE:full
    const uint4 u = draw(it, kTagCall, t, a.keys);
    const float x = u01(u.y);
    float y;
    if (u.x < a.split_u32) {                 // then-arm
      count_call<SCHED>(execs, lanes);  // @sr-region THEN
      y = foo<ROUNDS>(x, a.rounds);          // call site 1
      ++then_cnt;
    } else {                                 // else-arm
      float x1 = x * 0.5f;  // @sr-region ELSE_PRE
      x1 = x1 + 0.25f;
      count_call<SCHED>(execs, lanes);
      y = foo<ROUNDS>(x1, a.rounds);         // call site 2 (still ELSE_PRE's mask)
      y = y * y;  // @sr-region ELSE_POST
    }  // @sr-region MERGE:full
    ysum = ysum + y;
  }
  a.y[g] = ysum;  // @sr-region ENTRY:full
  const uint32_t vm = valid_mask(g & ~31ull, a.n);
  const uint32_t tot = __reduce_add_sync(vm, then_cnt);
  uint32_t e = 0, l = 0;
  if constexpr (SCHED) { e = __reduce_add_sync(vm, execs); l = __reduce_add_sync(vm, lanes); }
  if (lane_id() == 0) {
    atomicAdd(a.counters, (unsigned long long)tot);
    if constexpr (SCHED) {
      uint4* p = reinterpret_cast<uint4*>(a.sched + (g >> 5) * kSchedWords);
      p[0] = make_uint4(a.iters, e, l, 0u);
      p[1] = make_uint4(0u, 0u, 0u, 0u);
    }
  }
}  // @sr-region END

template <int ROUNDS, bool SCHED>
__global__ void __launch_bounds__(1024) commoncall_spec(const CallArgs a) {
  const uint64_t g = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;  // @sr-region ENTRY:full
  if (g >= a.n) return;
  const uint32_t vm = valid_mask(g & ~31ull, a.n);
  const uint64_t t = a.t0 + g;
  float ysum = 0.0f;
  uint32_t then_cnt = 0, execs = 0, lanes = 0;
  for (uint32_t it = 0; it < a.iters; ++it) {  // @sr-region MERGE:full
    const uint4 u = draw(it, kTagCall, t, a.keys);
    const float x = u01(u.y);
    const bool c = u.x < a.split_u32;
    float arg = x;                           // then-arm: argument only
    if (!c) {                                // else-arm prefix: argument only
      arg = x * 0.5f;
      arg = arg + 0.25f;
    }
    __syncwarp(vm);  // @sr-region CALL
    count_call<SCHED>(execs, lanes);
    float y = foo<ROUNDS>(arg, a.rounds);    // the one call, all lanes
    if (!c) y = y * y;  // @sr-region MERGE:full
    ysum = ysum + y;
    then_cnt += c ? 1u : 0u;
  }
  a.y[g] = ysum;  // @sr-region ENTRY:full
  const uint32_t tot = __reduce_add_sync(vm, then_cnt);
  uint32_t e = 0, l = 0;
  if constexpr (SCHED) { e = __reduce_add_sync(vm, execs); l = __reduce_add_sync(vm, lanes); }
  if (lane_id() == 0) {
    atomicAdd(a.counters, (unsigned long long)tot);
    if constexpr (SCHED) {
      uint4* p = reinterpret_cast<uint4*>(a.sched + (g >> 5) * kSchedWords);
      p[0] = make_uint4(a.iters, e, l, 0u);
      p[1] = make_uint4(0u, 0u, 0u, 0u);
    }
  }
}  // @sr-region END

template <bool SCHED>
cudaError_t launch_t(const LaunchCtx& c, const CallArgs& a, int mode) {
  const uint32_t block = c.block;
  const uint64_t grid = (a.n + block - 1) / block;
  if (grid > 0x7fffffffull) return cudaErrorInvalidConfiguration;
  const bool spec = mode == SR_SPEC_CALL;
  record_launch((uint32_t)grid, block, 0);
#define SR_CC(R)                                                                        \
  (spec ? commoncall_spec<R, SCHED><<<(unsigned)grid, block, 0, c.stream>>>(a)        \
        : commoncall_pdom<R, SCHED><<<(unsigned)grid, block, 0, c.stream>>>(a))
  if (a.rounds == 250) SR_CC(250);
  else if (a.rounds == 125) SR_CC(125);
  else SR_CC(0);
#undef SR_CC
  return cudaGetLastError();
}

}  // namespace

cudaError_t launch_commoncall(const LaunchCtx& c, const sr_workload& w, uint64_t n,
                              uint32_t iters, uint64_t seed, int mode) {
  CallArgs a;
  a.t0 = w.task_offset;
  a.n = n;
  a.seed = seed;
  a.keys = round_keys(seed);
  a.iters = iters;
  a.split_u32 = w.commoncall.split_u32;
  a.rounds = w.commoncall.fma_count / 8u;
  a.y = reinterpret_cast<float*>(c.ws + c.lay.off[SR_T_PERTHREAD]);
  a.counters = reinterpret_cast<unsigned long long*>(c.ws + c.lay.off[SR_T_COUNTERS]);
  a.sched = (w.flags & SR_F_SCHED) ? reinterpret_cast<uint32_t*>(c.ws + c.lay.off[SR_T_SCHED])
                                   : nullptr;
  return a.sched ? launch_t<true>(c, a, mode) : launch_t<false>(c, a, mode);
}

}  // namespace sr
