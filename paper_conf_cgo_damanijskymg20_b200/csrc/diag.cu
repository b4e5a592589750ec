// diag.cu -- sr_math_eval: evaluate one device building block of the hot path
// element-wise, so tests can compare the GPU's sr_logf / sr_sincos2pif /
// Expensive() with the CPU oracle bit for bit over every input the RNG can
// produce (readings R3, R5); sr_math_eval_p: the MC step's
// domain-restricted IEEE division / sqrt against IEEE arithmetic.
#include "sr_device.cuh"
#include "sr_internal.h"

namespace sr {
namespace {

__global__ void math_eval_kernel(int fn, const float* __restrict__ x, float* __restrict__ out,
                                 uint64_t n) {
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (uint64_t)gridDim.x * blockDim.x) {
    const float v = x[i];
    float r;
    switch (fn) {
      case SR_FN_LOGF: r = sr_logf(v); break;
      case SR_FN_SIN2PI: { float s, c; sr_sincos2pif(v, s, c); r = s; break; }
      case SR_FN_COS2PI: { float s, c; sr_sincos2pif(v, s, c); r = c; break; }
      case SR_FN_EXPENSIVE_1000: r = expensive<125>(v, 125); break;
      case SR_FN_EXPENSIVE_2000: r = expensive<250>(v, 250); break;
      default: r = 0.0f; break;
    }
    out[i] = r;
  }
}

// sr_math_eval_p: the MC step's division / square-root building blocks with
// one scalar parameter p: out[i] = fn(p, x[i]).
__global__ void math_eval_p_kernel(int fn, float p, const float* __restrict__ x,
                                   float* __restrict__ out, uint64_t n) {
  // layer constants of g = p, binary32, in the order of launch_mcml / the oracle
  const float g2 = p * p;
  const float one_m_g2 = 1.0f - g2, one_p_g2 = 1.0f + g2, one_m_g = 1.0f - p, two_g = 2.0f * p;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (uint64_t)gridDim.x * blockDim.x) {
    const float v = x[i];
    float r;
    switch (fn) {
      case SR_FNP_DIV_XP: r = div_dom(v, p); break;
      case SR_FNP_DIV_PX: r = div_dom(p, v); break;
      case SR_FNP_SQRT: r = sqrt_dom(v); break;
      case SR_FNP_HG_COST: r = hg_cost_dom(one_m_g2, one_p_g2, one_m_g, two_g, v); break;
      case SR_FNP_HG_SINT: {
        const float c = hg_cost_dom(one_m_g2, one_p_g2, one_m_g, two_g, v);
        r = sqrt_dom(1.0f - c * c);
        break;
      }
      case SR_FNP_DIV2_XP: {   // pairs (x[2j], x[2j+1]) / p through div2_dom
        if (i & 1u) continue;
        const uint64_t q = div2_dom(pack2(v, i + 1 < n ? x[i + 1] : 1.0f), p);
        float q0, q1;
        unpack2(q, q0, q1);
        out[i] = q0;
        if (i + 1 < n) out[i + 1] = q1;
        continue;
      }
      default: r = 0.0f; break;
    }
    out[i] = r;
  }
}

}  // namespace

cudaError_t launch_math_eval_p(cudaStream_t st, int sm_count, int fn, float p, const float* x,
                               float* out, uint64_t n) {
  const uint64_t want = (n + 255) / 256;
  const uint64_t cap = (uint64_t)sm_count * 16;
  const unsigned grid = (unsigned)(want < cap ? (want ? want : 1) : cap);
  record_launch(grid, 256, 0);
  math_eval_p_kernel<<<grid, 256, 0, st>>>(fn, p, x, out, n);
  return cudaGetLastError();
}

cudaError_t launch_math_eval(cudaStream_t st, int sm_count, int fn, const float* x, float* out,
                             uint64_t n) {
  const uint64_t want = (n + 255) / 256;
  const uint64_t cap = (uint64_t)sm_count * 16;
  const unsigned grid = (unsigned)(want < cap ? (want ? want : 1) : cap);
  record_launch(grid, 256, 0);
  math_eval_kernel<<<grid, 256, 0, st>>>(fn, x, out, n);
  return cudaGetLastError();
}

}  // namespace sr
