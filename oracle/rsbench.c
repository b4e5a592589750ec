/*
 * rsbench.c -- ORACLE (test infrastructure; see oracle.h).
 *
 * NEXT-1: the paper's central Loop Merge example,
 * RSBench (Fig. 3):
 *
 *     while (lookups left) {                       // coarsened outer loop
 *       Prolog: material = pick(); E = energy      // "get_random_material()"
 *       for (each nuclide in material)             // 4 .. 321 nuclides
 *         { L1: accumulate_cross_sections() }      // expensive common body
 *       Epilog: post_processing()
 *     }
 *
 * executed literally per thread.  DESIGN.md reading R8 fixes the synthetic
 * parts: the material table of the XSBench/RSBench "large" problem (12
 * materials, nuclide counts {321,5,4,4,27,21,21,21,21,21,9,9}, selection
 * probabilities {.140,.052,.275,.134,.154,.064,.066,.055,.008,.015,.025,.013}
 * as 2^-32 integer thresholds), nuclide ids n = (37 m + 13 j) mod 355, the
 * per-nuclide body = 8 FMA chains x (fma_count/8) rounds started from
 * (E + n/512), and the epilog acc = acc + xs.
 *
 * prolog_fma > 0: the lookup's prolog also does prolog_fma FMAs of work on the
 * energy, E = Expensive(U01(u1), prolog_fma) (reading R8'): an expensive task
 * fetch, XSBench's energy-grid search, the case where Fig. 9 finds the best
 * threshold far below full reconvergence.
 */
#include <math.h>
#include "oracle.h"

static const uint32_t kNucs[OR_RS_MATS] = {321, 5, 4, 4, 27, 21, 21, 21, 21, 21, 9, 9};
/* cumulative selection thresholds: floor(2^32 * cumsum(p)), last = 2^32-1 */
static const double kProb[OR_RS_MATS] = {0.140, 0.052, 0.275, 0.134, 0.154, 0.064,
                                         0.066, 0.055, 0.008, 0.015, 0.025, 0.013};

uint32_t or_rs_nuclides(uint32_t m) { return m < OR_RS_MATS ? kNucs[m] : 0; }

uint32_t or_rs_threshold(uint32_t m) {
  double c = 0.0;
  for (uint32_t i = 0; i <= m && i < OR_RS_MATS; ++i) c += kProb[i];
  if (m + 1 >= OR_RS_MATS) return 0xFFFFFFFFu;
  return (uint32_t)floor(c * 4294967296.0);
}

/* material of a draw: the first m with u < threshold(m) */
uint32_t or_rs_pick(uint32_t u) {
  for (uint32_t m = 0; m < OR_RS_MATS; ++m)
    if (u < or_rs_threshold(m)) return m;
  return OR_RS_MATS - 1;
}

/* the per-nuclide body: Expensive() of reading R3 started from E + n/512 */
float or_rs_body(float E, uint32_t nuc, uint32_t fma_count) {
  float start = E + (float)nuc * 0x1p-9f;
  return or_expensive(start, fma_count);
}

void or_rsbench(uint32_t fma_count, uint32_t prolog_fma, uint64_t t0, uint64_t n,
                uint32_t iters, uint64_t seed, float* acc_out, uint32_t* nuc_out,
                uint32_t* trips /* may be NULL */) {
  uint32_t key[2] = {(uint32_t)seed, (uint32_t)(seed >> 32)};
  for (uint64_t j = 0; j < n; ++j) {
    uint64_t t = t0 + j;
    float acc = 0.0f;
    uint32_t nucs = 0;
    for (uint32_t k = 0; k < iters; ++k) {
      uint32_t ctr[4] = {k, (uint32_t)OR_TAG_RS << 16, (uint32_t)t, (uint32_t)(t >> 32)};
      uint32_t u[4];
      or_philox4x32_10(ctr, key, u);                 /* Prolog */
      uint32_t m = or_rs_pick(u[0]);
      float E = or_u01(u[1]);
      if (prolog_fma) E = or_expensive(E, prolog_fma);
      float xs = 0.0f;
      uint32_t N = kNucs[m];
      for (uint32_t i = 0; i < N; ++i) {             /* inner loop, L1 */
        uint32_t nuc = (37u * m + 13u * i) % OR_RS_NUCLIDES;
        xs = xs + or_rs_body(E, nuc, fma_count);
      }
      acc = acc + xs;                                /* Epilog */
      nucs += N;
      if (trips) trips[j * iters + k] = N;
    }
    acc_out[j] = acc;
    nuc_out[j] = nucs;
  }
}
