// Experiment (not part of the library): single-warp dependent-chain latencies on
// B200 of the operations the divergent-loop scheduler is built from -- a
// Philox4x32-10 draw (IMAD.WIDE form as the library compiles it, and with
// mul.hi / mul.lo split), IMAD.WIDE alone, FFMA2, VOTE.ANY (__ballot_sync) and
// WARPSYNC (__syncwarp with a computed mask).  clock64 around N dependent steps.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/lat tools/exp_latency.cu
#include <cstdint>
#include <cstdio>

__device__ __forceinline__ uint4 philox_wide(uint4 c, uint32_t k0, uint32_t k1) {
#pragma unroll
  for (int r = 0; r < 10; ++r) {
    const uint64_t p0 = (uint64_t)0xD2511F53u * c.x, p1 = (uint64_t)0xCD9E8D57u * c.z;
    c = make_uint4((uint32_t)(p1 >> 32) ^ c.y ^ k0, (uint32_t)p1, (uint32_t)(p0 >> 32) ^ c.w ^ k1,
                   (uint32_t)p0);
    k0 += 0x9E3779B9u;
    k1 += 0xBB67AE85u;
  }
  return c;
}
__device__ __forceinline__ uint4 philox_split(uint4 c, uint32_t k0, uint32_t k1) {
#pragma unroll
  for (int r = 0; r < 10; ++r) {
    uint32_t hi0, lo0, hi1, lo1;
    asm volatile("mul.hi.u32 %0, %1, 0xD2511F53;" : "=r"(hi0) : "r"(c.x));
    asm volatile("mul.lo.u32 %0, %1, 0xD2511F53;" : "=r"(lo0) : "r"(c.x));
    asm volatile("mul.hi.u32 %0, %1, 0xCD9E8D57;" : "=r"(hi1) : "r"(c.z));
    asm volatile("mul.lo.u32 %0, %1, 0xCD9E8D57;" : "=r"(lo1) : "r"(c.z));
    c = make_uint4(hi1 ^ c.y ^ k0, lo1, hi0 ^ c.w ^ k1, lo0);
    k0 += 0x9E3779B9u;
    k1 += 0xBB67AE85u;
  }
  return c;
}

__global__ void lat(int n, unsigned long long* out, uint32_t* sink) {
  uint4 c = make_uint4(threadIdx.x, 1, 2, 3);
  uint32_t acc = threadIdx.x;
  long long t0, t1;
  // 0: Philox draw (wide), dependent through c.x
  t0 = clock64();
  for (int i = 0; i < n; ++i) c = philox_wide(make_uint4(c.x, c.y, 7u, 9u), 11u, 13u);
  t1 = clock64();
  if (threadIdx.x == 0) out[0] = t1 - t0;
  // 1: Philox draw (split mul.hi / mul.lo)
  t0 = clock64();
  for (int i = 0; i < n; ++i) c = philox_split(make_uint4(c.x, c.y, 7u, 9u), 11u, 13u);
  t1 = clock64();
  if (threadIdx.x == 0) out[1] = t1 - t0;
  // 2: 64-bit product high word, dependent
  t0 = clock64();
  for (int i = 0; i < n; ++i) acc = (uint32_t)(((uint64_t)acc * 0xD2511F53u) >> 32) ^ (uint32_t)i;
  t1 = clock64();
  if (threadIdx.x == 0) out[2] = t1 - t0;
  // 3: FFMA2 chain
  float2 f = make_float2((float)threadIdx.x, 1.0f);
  t0 = clock64();
  for (int i = 0; i < n; ++i) {
    uint64_t v, m, a;
    asm("mov.b64 %0, {%1, %2};" : "=l"(v) : "f"(f.x), "f"(f.y));
    asm("mov.b64 %0, {%1, %1};" : "=l"(m) : "f"(0.999f));
    asm("mov.b64 %0, {%1, %1};" : "=l"(a) : "f"(0.5f));
    asm volatile("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(v) : "l"(v), "l"(m), "l"(a));
    asm("mov.b64 {%0, %1}, %2;" : "=f"(f.x), "=f"(f.y) : "l"(v));
  }
  t1 = clock64();
  if (threadIdx.x == 0) out[3] = t1 - t0;
  // 4: ballot chain (the vote's result feeds the next predicate)
  uint32_t b = threadIdx.x;
  t0 = clock64();
  for (int i = 0; i < n; ++i) b = __ballot_sync(0xffffffffu, ((b >> (threadIdx.x & 31)) & 1u) != 0u) + i;
  t1 = clock64();
  if (threadIdx.x == 0) out[4] = t1 - t0;
  // 5: syncwarp with a computed (full) mask, in a dependent loop
  uint32_t m = 0xffffffffu;
  t0 = clock64();
  for (int i = 0; i < n; ++i) { __syncwarp(m); m = (m ^ (uint32_t)i) | 0xffffffffu; }
  t1 = clock64();
  if (threadIdx.x == 0) out[5] = t1 - t0;
  sink[threadIdx.x] = c.x ^ c.y ^ acc ^ __float_as_uint(f.x) ^ b ^ m;
}

int main() {
  unsigned long long* d;
  uint32_t* s;
  cudaMalloc(&d, 8 * sizeof(unsigned long long));
  cudaMalloc(&s, 1024 * sizeof(uint32_t));
  const int n = 1000;
  lat<<<1, 32>>>(n, d, s);
  lat<<<1, 32>>>(n, d, s);
  unsigned long long h[8];
  cudaMemcpy(h, d, sizeof h, cudaMemcpyDeviceToHost);
  const char* names[] = {"philox draw (IMAD.WIDE)", "philox draw (mul.hi/lo)", "IMAD.WIDE hi + xor",
                         "FFMA2", "VOTE.ANY (ballot) + IADD", "WARPSYNC"};
  for (int i = 0; i < 6; ++i) printf("%-26s %8.1f cycles per step\n", names[i], (double)h[i] / n);
  return 0;
}
