/*
 * philox.c -- ORACLE (test infrastructure; see oracle.h).
 *
 * Philox4x32-10 (Salmon et al., "Parallel random numbers: as easy as 1, 2,
 * 3", SC'11).  The paper does not name its RNG (its Monte Carlo apps,
 * Table 2, each bring their own); reading R1 fixes
 * Philox4x32-10 keyed by (task, event) so that every random draw is a pure
 * function of its coordinates and the result cannot depend on the schedule
 * (reconvergence barriers must not change program results).
 *
 * Pinned by the Random123 known-answer vectors (tests/golden/philox_kat.txt).
 */
#include "oracle.h"

#define PHILOX_M0 0xD2511F53u
#define PHILOX_M1 0xCD9E8D57u
#define PHILOX_W0 0x9E3779B9u
#define PHILOX_W1 0xBB67AE85u

static void philox_round(uint32_t c[4], const uint32_t k[2]) {
  uint64_t p0 = (uint64_t)PHILOX_M0 * (uint64_t)c[0];
  uint64_t p1 = (uint64_t)PHILOX_M1 * (uint64_t)c[2];
  uint32_t hi0 = (uint32_t)(p0 >> 32), lo0 = (uint32_t)p0;
  uint32_t hi1 = (uint32_t)(p1 >> 32), lo1 = (uint32_t)p1;
  uint32_t n0 = hi1 ^ c[1] ^ k[0];
  uint32_t n1 = lo1;
  uint32_t n2 = hi0 ^ c[3] ^ k[1];
  uint32_t n3 = lo0;
  c[0] = n0; c[1] = n1; c[2] = n2; c[3] = n3;
}

void or_philox4x32_10(const uint32_t ctr[4], const uint32_t key[2], uint32_t out[4]) {
  uint32_t c[4] = {ctr[0], ctr[1], ctr[2], ctr[3]};
  uint32_t k[2] = {key[0], key[1]};
  for (int r = 0; r < 10; ++r) {
    if (r > 0) { k[0] += PHILOX_W0; k[1] += PHILOX_W1; }
    philox_round(c, k);
  }
  out[0] = c[0]; out[1] = c[1]; out[2] = c[2]; out[3] = c[3];
}

/* 24-bit uniforms: exact in binary32 (reading R2). */
float or_u01(uint32_t u) { return (float)(u >> 8) * 0x1p-24f; }
float or_u01c(uint32_t u) { return (float)((u >> 8) + 1u) * 0x1p-24f; }
