/*
 * warpsim.c -- ORACLE part 2 (test infrastructure; see oracle.h).
 *
 * A lane-mask warp simulator.  It replays the per-lane event streams that
 * oracle part 1 produces (which iterations want Expensive(), which arm each
 * lane takes, how many inner steps each task runs) under two convergence
 * rules and counts, per source region, warp-level executions and active
 * lanes.  SIMT efficiency, "the average percentage of active threads per
 * warp", follows from these counts and a per-region instruction
 * cost table (tools/sass_regions.py reads it off the built cubin).
 *
 * PDOM rule (Fig. 1(a)): control follows the
 * program; a diverged warp reconverges at the immediate post-dominator, so a
 * region executes once per distinct arrival with mask = the lanes that
 * reached it.
 *
 * Speculative Reconvergence rule (Fig. 1(b), Iteration Delay
 * P:303-324, Loop Merge P:325-377, soft barrier Sec. 4.6 P:1108-1142,
 * Fig. 6), one scheduler round at a time:
 *   P = lanes waiting at the reconvergence point L1 ("Join"ed and arrived),
 *   R = lanes that can still make progress toward L1 without it.
 *   P = R = {}          -> exit.
 *   |P| >= T or R = {}  -> release: all of P run the common code together
 *                          (all waiting lanes, not T of them: P:1135-1137);
 *                          R = {} is the "threshold not satisfiable" exit of
 *                          P:1139-1141.
 *   otherwise           -> advance: R runs one step of the non-common code
 *                          (run-ahead of one iteration per round, reading Q5).
 * The GPU kernels implement the same rule with __ballot_sync; DESIGN.md
 * readings Q1-Q5, Q11.
 */
#include <stdlib.h>
#include <string.h>
#include "oracle.h"

static void hit(ws_counts* o, int r, uint32_t mask) {
  if (!mask) return;
  o->execs[r] += 1;
  o->lanes[r] += (uint64_t)__builtin_popcount(mask);
}

/* ------------------------------------------------------------------ */
/* Iteration Delay: Fig. 2(a) / Listing 1.                              */
void ws_divloop(const uint8_t* want, uint32_t W, uint32_t n_valid, uint32_t L, int mode,
                uint32_t T, ws_counts* o) {
  ws_divloop_adv(want, W, n_valid, L, mode, T, 1, o);
}

/* V > 1: in an advance round a run-ahead lane takes up to V iterations, stopping
 * at the first one that wants Expensive (it parks there). */
void ws_divloop_adv(const uint8_t* want, uint32_t W, uint32_t n_valid, uint32_t L, int mode,
                    uint32_t T, uint32_t V, ws_counts* o) {
  memset(o, 0, sizeof *o);
  if (V == 0) V = 1;
  if (n_valid > W) n_valid = W;
  uint32_t valid = n_valid >= 32 ? 0xffffffffu : ((1u << n_valid) - 1u);
  hit(o, WS_DL_ENTRY, valid);
  if (mode == WS_PDOM) {
    for (uint32_t i = 0; i < L; ++i) {
      hit(o, WS_DL_PROLOG, valid);
      uint32_t m = 0;
      for (uint32_t l = 0; l < n_valid; ++l)
        if (want[l * L + i]) m |= 1u << l;
      hit(o, WS_DL_EXPENSIVE, m);   /* then-block with the wanting lanes */
      hit(o, WS_DL_EPILOG, valid);  /* reconverged at the IPDOM */
    }
    return;
  }
  if (T == 0 || T > 32) T = 32;
  uint32_t it[32] = {0};
  uint32_t parked = 0;
  for (;;) {
    uint32_t P = parked, R = 0;
    for (uint32_t l = 0; l < n_valid; ++l)
      if (!(parked >> l & 1u) && it[l] < L) R |= 1u << l;
    if (!P && !R) break;
    o->rounds += 1;
    hit(o, WS_DL_ROUND, valid);
    if ((uint32_t)__builtin_popcount(P) >= T || !R) {
      hit(o, WS_DL_RELEASE, P);
      hit(o, WS_DL_EXPENSIVE, P);
      hit(o, WS_DL_EPILOG, P);
      for (uint32_t l = 0; l < n_valid; ++l)
        if (P >> l & 1u) it[l] += 1;
      parked = 0;
    } else {
      hit(o, WS_DL_ADVANCE, R);
      uint32_t S = R;   /* lanes still running ahead in this round */
      for (uint32_t v = 0; v < V && S; ++v) {
        hit(o, WS_DL_PROLOG, S);
        uint32_t E = 0;
        for (uint32_t l = 0; l < n_valid; ++l) {
          if (!(S >> l & 1u)) continue;
          if (want[l * L + it[l]]) { parked |= 1u << l; S &= ~(1u << l); } /* Join + Wait */
          else { E |= 1u << l; it[l] += 1; if (it[l] >= L) S &= ~(1u << l); } /* run ahead */
        }
        hit(o, WS_DL_EPILOG, E);
      }
    }
  }
}

/* ------------------------------------------------------------------ */
/* Common function call: Fig. 2(c), Sec. 4.4.                          */
void ws_commoncall(const uint8_t* arm, uint32_t W, uint32_t n_valid, int mode, ws_counts* o) {
  memset(o, 0, sizeof *o);
  if (n_valid > W) n_valid = W;
  uint32_t valid = n_valid >= 32 ? 0xffffffffu : ((1u << n_valid) - 1u);
  uint32_t then_m = 0;
  for (uint32_t l = 0; l < n_valid; ++l)
    if (arm[l]) then_m |= 1u << l;
  uint32_t else_m = valid & ~then_m;
  hit(o, WS_CC_ENTRY, valid);
  if (mode == WS_SPEC_CALL) {
    hit(o, WS_CC_THEN, then_m);
    hit(o, WS_CC_ELSE_PRE, else_m);
    hit(o, WS_CC_CALL, valid);       /* one call, all lanes: reconverged at foo entry */
    hit(o, WS_CC_ELSE_POST, else_m);
  } else {
    hit(o, WS_CC_THEN, then_m);
    hit(o, WS_CC_CALL, then_m);      /* call site 1 */
    hit(o, WS_CC_ELSE_PRE, else_m);
    hit(o, WS_CC_CALL, else_m);      /* call site 2 */
    hit(o, WS_CC_ELSE_POST, else_m);
  }
  hit(o, WS_CC_MERGE, valid);
}

/* ------------------------------------------------------------------ */
/* Loop Merge: Fig. 2(b), Fig. 3.                */
/* Split one step's mask by the branch outcomes recorded in the event bytes
 * (bit b set / clear), so every branch of the step body is costed with the
 * lanes that took it. */
static void step_split(ws_counts* o, const or_event* ev, const uint64_t* ev_off, uint32_t K,
                       const uint32_t* kk, const uint32_t* jj, uint32_t mask) {
  uint32_t set[16] = {0};
  for (uint32_t l = 0; l < 32; ++l) {
    if (!(mask >> l & 1u)) continue;
    or_event e = ev[ev_off[l * K + kk[l]] + jj[l]];
    for (int b = 0; b < 16; ++b)
      if (e >> b & 1u) set[b] |= 1u << l;
  }
  hit(o, WS_LM_STEP_BOUNDARY, set[0]);
  hit(o, WS_LM_STEP_INTERACT, mask & ~set[0]);
  /* the same step written as part A + part B with each part's roulette (the
   * regions ws_loopmerge_defer costs separately): a boundary with a layer of
   * equal index (bit 9) is finished inside part A; the other boundary lanes
   * run part B */
  const uint32_t b_lanes = set[0] & ~set[9];
  hit(o, WS_LM_BI, set[9]);
  hit(o, WS_LM_A_TAIL, mask & ~b_lanes);
  hit(o, WS_LM_A_RR, set[5] & ~b_lanes);
  hit(o, WS_LM_B_REL, b_lanes);
  hit(o, WS_LM_B_RR, set[5] & b_lanes);
  /* reflect / exit / transmit (bits 2-4) are branches of part B: a matched
   * boundary's reflect or transmit runs inside part A (BI) instead */
  set[2] &= b_lanes;
  set[3] &= b_lanes;
  set[4] &= b_lanes;
  for (int b = 0; b < 16; ++b) {
    hit(o, WS_LM_EV0 + b, set[b]);
    hit(o, WS_LM_NEV0 + b, mask & ~set[b]);
  }
}

void ws_loopmerge(const uint32_t* nsteps, const or_event* ev, const uint64_t* ev_off, uint32_t W,
                  uint32_t n_valid, uint32_t K, int mode, uint32_t T, ws_counts* o) {
  ws_loopmerge_unrolled(nsteps, ev, ev_off, W, n_valid, K, mode, T, 1, o);
}

/* U > 1: the merged inner loop partially unrolled by U: a
 * release runs up to U steps; a lane whose task ends inside the release idles
 * for the rest of it ("reconvergence is needed only once per N iterations"). */
void ws_loopmerge_unrolled(const uint32_t* nsteps, const or_event* ev, const uint64_t* ev_off,
                           uint32_t W, uint32_t n_valid, uint32_t K, int mode, uint32_t T,
                           uint32_t U, ws_counts* o) {
  if (U == 0) U = 1;
  memset(o, 0, sizeof *o);
  if (n_valid > W) n_valid = W;
  uint32_t valid = n_valid >= 32 ? 0xffffffffu : ((1u << n_valid) - 1u);
  uint32_t kk[32] = {0}, jj[32] = {0};
  hit(o, WS_LM_ENTRY, valid);
  if (mode == WS_PDOM) {
    for (uint32_t k = 0; k < K; ++k) {
      hit(o, WS_LM_LAUNCH, valid);
      for (uint32_t l = 0; l < n_valid; ++l) { kk[l] = k; jj[l] = 0; }
      for (;;) {
        uint32_t m = 0;
        for (uint32_t l = 0; l < n_valid; ++l)
          if (jj[l] < nsteps[l * K + k]) m |= 1u << l;
        if (!m) break;
        hit(o, WS_LM_STEP, m);
        if (ev) {
          step_split(o, ev, ev_off, K, kk, jj, m);
        }
        for (uint32_t l = 0; l < n_valid; ++l)
          if (m >> l & 1u) jj[l] += 1;
      }
    }
    return;
  }
  if (T == 0 || T > 32) T = 32;
  uint32_t alive = 0;
  uint32_t next[32] = {0};  /* next task index to launch */
  for (;;) {
    uint32_t P = alive, R = 0;
    for (uint32_t l = 0; l < n_valid; ++l)
      if (!(alive >> l & 1u) && next[l] < K) R |= 1u << l;
    if (!P && !R) break;
    o->rounds += 1;
    hit(o, WS_LM_ROUND, valid);
    if ((uint32_t)__builtin_popcount(P) >= T || !R) {
      hit(o, WS_LM_RELEASE, P);
      uint32_t S = P;
      for (uint32_t r = 0; r < U && S; ++r) {
        hit(o, WS_LM_STEP, S);
        if (ev) {
          step_split(o, ev, ev_off, K, kk, jj, S);
        }
        for (uint32_t l = 0; l < n_valid; ++l) {
          if (!(S >> l & 1u)) continue;
          jj[l] += 1;
          if (jj[l] == nsteps[l * K + kk[l]]) { alive &= ~(1u << l); S &= ~(1u << l); }
        }
      }
    } else {
      hit(o, WS_LM_ADVANCE, R);
      hit(o, WS_LM_LAUNCH, R);   /* epilog of the finished task + prolog of the next */
      for (uint32_t l = 0; l < n_valid; ++l) {
        if (!(R >> l & 1u)) continue;
        kk[l] = next[l]++;
        jj[l] = 0;
        alive |= 1u << l;
      }
    }
  }
}

/* Loop Merge over one stream of tasks claimed dynamically (see oracle.h).
 * step_split is called with K = 0 and kk[l] = the lane's task index q.
 * The claim itself is modelled as the kernels run it: a warp-level reservoir
 * [rv_next, rv_end) refilled CHUNK tasks at a time from the stream; a claim
 * for `need` lanes takes the fast path when the reservoir covers them, else a
 * loop that fetches chunks (CHUNK) and serves lanes in lane order (CLAIMIT),
 * stopping when the stream is empty. */
#define WS_CHUNK 32u
typedef struct { uint64_t next, end, fetch, Q; } ws_reservoir;

/* serve `want` lanes in lane order; returns the mask served (tasks in kk[]) */
static uint32_t ws_claim(ws_counts* o, ws_reservoir* rv, uint32_t want, uint32_t all,
                         uint32_t* kk) {
  const uint32_t need = (uint32_t)__builtin_popcount(want);
  uint32_t served = 0, got = 0;
  if (rv->end - rv->next < need) {
    hit(o, WS_LM_CLAIM, all);
    while (served < need) {
      hit(o, WS_LM_CLAIMIT, all);
      if (rv->next >= rv->end) {
        hit(o, WS_LM_CHUNK, all);
        if (rv->fetch >= rv->Q) break;
        rv->next = rv->fetch;
        rv->end = rv->fetch + WS_CHUNK < rv->Q ? rv->fetch + WS_CHUNK : rv->Q;
        rv->fetch += WS_CHUNK;
      }
      const uint64_t avail = rv->end - rv->next;
      const uint32_t take = (uint32_t)(avail < need - served ? avail : need - served);
      served += take;
      rv->next += take;
    }
  } else {
    served = need;
    rv->next += need;
  }
  /* the first `served` lanes of `want` (lane order) get consecutive tasks */
  uint64_t q = rv->next - served;
  uint32_t k = 0;
  for (uint32_t l = 0; l < 32 && k < served; ++l) {
    if (!(want >> l & 1u)) continue;
    kk[l] = (uint32_t)q++;
    got |= 1u << l;
    ++k;
  }
  return got;
}

void ws_loopmerge_stream(const uint32_t* nsteps, const or_event* ev, const uint64_t* ev_off,
                         uint32_t W, uint64_t Q, int mode, uint32_t T, uint32_t U,
                         ws_counts* o) {
  if (U == 0) U = 1;
  if (W > 32) W = 32;
  memset(o, 0, sizeof *o);
  const uint32_t all = W >= 32 ? 0xffffffffu : ((1u << W) - 1u);
  uint32_t kk[32] = {0}, jj[32] = {0};
  ws_reservoir rv = {0, 0, 0, Q};
  hit(o, WS_LM_ENTRY, all);
  if (mode == WS_PDOM) {
    for (;;) {
      const uint32_t H = ws_claim(o, &rv, all, all, kk);
      if (!H) break;
      for (uint32_t l = 0; l < W; ++l) jj[l] = 0;
      hit(o, WS_LM_LAUNCH, H);
      for (;;) {
        uint32_t m = 0;
        for (uint32_t l = 0; l < W; ++l)
          if ((H >> l & 1u) && jj[l] < nsteps[kk[l]]) m |= 1u << l;
        if (!m) break;
        hit(o, WS_LM_STEP, m);
        if (ev) step_split(o, ev, ev_off, 0, kk, jj, m);
        for (uint32_t l = 0; l < W; ++l)
          if (m >> l & 1u) jj[l] += 1;
      }
    }
    return;
  }
  if (T == 0 || T > 32) T = 32;
  uint32_t alive = 0, exhausted = 0;
  for (;;) {
    const uint32_t P = alive, R = all & ~alive & ~exhausted;
    if (!P && !R) break;
    o->rounds += 1;
    hit(o, WS_LM_ROUND, all);
    if ((uint32_t)__builtin_popcount(P) >= T || !R) {
      hit(o, WS_LM_RELEASE, P);
      uint32_t S = P;
      for (uint32_t r = 0; r < U && S; ++r) {
        hit(o, WS_LM_STEP, S);
        if (ev) step_split(o, ev, ev_off, 0, kk, jj, S);
        for (uint32_t l = 0; l < W; ++l) {
          if (!(S >> l & 1u)) continue;
          jj[l] += 1;
          if (jj[l] >= nsteps[kk[l]]) { alive &= ~(1u << l); S &= ~(1u << l); }
        }
      }
    } else {
      hit(o, WS_LM_ADVANCE, R);
      const uint32_t got = ws_claim(o, &rv, R, all, kk);
      exhausted |= R & ~got;
      for (uint32_t l = 0; l < W; ++l) {
        if (!(got >> l & 1u)) continue;
        jj[l] = 0;
        if (nsteps[kk[l]]) alive |= 1u << l;
      }
      hit(o, WS_LM_LAUNCH, got);
    }
  }
}

/* Loop Merge over a warp-shared pool of the warp's tasks (see oracle.h). */
void ws_loopmerge_pool(const uint32_t* nsteps, uint32_t W, uint32_t n_valid, uint32_t K,
                       uint32_t T, uint32_t U, ws_counts* o) {
  if (U == 0) U = 1;
  if (T == 0 || T > 32) T = 32;
  if (W > 32) W = 32;
  if (n_valid > W) n_valid = W;
  memset(o, 0, sizeof *o);
  const uint32_t valid = n_valid >= 32 ? 0xffffffffu : ((1u << n_valid) - 1u);
  const uint32_t all = W >= 32 ? 0xffffffffu : ((1u << W) - 1u);
  const uint64_t pool = (uint64_t)n_valid * K;
  uint64_t qnext = 0;
  uint32_t alive = 0, left[32] = {0};  /* steps left in the lane's task */
  hit(o, WS_LM_ENTRY, valid);
  for (;;) {
    const uint32_t P = alive;
    const uint32_t R = qnext < pool ? (all & ~alive) : 0u;
    if (!P && !R) break;
    o->rounds += 1;
    hit(o, WS_LM_ROUND, all);
    if ((uint32_t)__builtin_popcount(P) >= T || !R) {
      hit(o, WS_LM_RELEASE, P);
      uint32_t S = P;
      for (uint32_t r = 0; r < U && S; ++r) {
        hit(o, WS_LM_STEP, S);
        for (uint32_t l = 0; l < W; ++l) {
          if (!(S >> l & 1u)) continue;
          if (--left[l] == 0) { alive &= ~(1u << l); S &= ~(1u << l); }
        }
      }
    } else {
      hit(o, WS_LM_ADVANCE, R);
      uint32_t got = 0;
      for (uint32_t l = 0; l < W; ++l) {   /* lane order */
        if (!(R >> l & 1u) || qnext >= pool) continue;
        const uint64_t q = qnext++;
        const uint32_t owner = (uint32_t)(q % n_valid), k = (uint32_t)(q / n_valid);
        left[l] = nsteps[(uint64_t)owner * K + k];
        if (left[l]) alive |= 1u << l;
        got |= 1u << l;
      }
      hit(o, WS_LM_LAUNCH, got);
    }
  }
}

/* ------------------------------------------------------------------ */
/* Loop Merge with a second, nested prediction: Iteration Delay of the rare
 * boundary sub-step (two concurrent predictions).  A step is
 * split into part A (draw, path length, boundary distance; the interaction
 * branch runs to completion, a boundary hit only moves the photon to the
 * boundary and parks it) and part B (the boundary's Fresnel / transmit /
 * exit / roulette, run later for all parked lanes together).  Per round:
 *   B = parked, P = live and not parked, R = idle lanes with tasks left;
 *   |B| >= Tb -> boundary release; else |P| >= T -> step release;
 *   else R != {} -> advance; else P != {} -> step release; else B != {} ->
 *   boundary release; else exit.
 * Only the boundary bits (bit0, and bit9: a matched boundary finishes in part
 * A and does not park) of the events decide the schedule; the other
 * bits split each phase's mask for costing: phase A counts bits 1, 6, 7 and
 * the interaction roulette; phase B counts bits 2, 3, 4, 8 and its roulette. */
static or_event evt(const or_event* ev, const uint64_t* ev_off, uint32_t K, const uint32_t* kk,
                    const uint32_t* jj, uint32_t l) {
  return ev[ev_off[l * K + kk[l]] + jj[l]];
}

void ws_loopmerge_defer(const uint32_t* nsteps, const or_event* ev, const uint64_t* ev_off,
                        uint32_t W, uint32_t n_valid, uint32_t K, uint32_t T, uint32_t Tb,
                        ws_counts* o) {
  memset(o, 0, sizeof *o);
  if (n_valid > W) n_valid = W;
  if (T == 0 || T > 32) T = 32;
  if (Tb == 0 || Tb > 32) Tb = 32;
  uint32_t valid = n_valid >= 32 ? 0xffffffffu : ((1u << n_valid) - 1u);
  uint32_t kk[32] = {0}, jj[32] = {0}, next[32] = {0};
  uint32_t alive = 0, parked = 0;
  hit(o, WS_LM_ENTRY, valid);
  for (;;) {
    uint32_t Bm = parked, P = alive & ~parked, R = 0;
    for (uint32_t l = 0; l < n_valid; ++l)
      if (!(alive >> l & 1u) && next[l] < K) R |= 1u << l;
    if (!Bm && !P && !R) break;
    o->rounds += 1;
    hit(o, WS_LM_ROUND, valid);
    int phase;  /* 1 step release, 2 boundary release, 3 advance */
    if ((uint32_t)__builtin_popcount(Bm) >= Tb) phase = 2;
    else if ((uint32_t)__builtin_popcount(P) >= T) phase = 1;
    else if (R) phase = 3;
    else if (P) phase = 1;
    else phase = 2;
    if (phase == 1) {
      hit(o, WS_LM_RELEASE, P);
      hit(o, WS_LM_STEP, P);
      uint32_t bit[16] = {0};
      for (uint32_t l = 0; l < n_valid; ++l) {
        if (!(P >> l & 1u)) continue;
        or_event e = evt(ev, ev_off, K, kk, jj, l);
        for (int b = 0; b < 16; ++b)
          if (e >> b & 1u) bit[b] |= 1u << l;
      }
      hit(o, WS_LM_EV0, bit[0]);
      hit(o, WS_LM_NEV0, P & ~bit[0]);
      hit(o, WS_LM_EV0 + 1, bit[1]);
      hit(o, WS_LM_NEV0 + 1, P & ~bit[1]);
      hit(o, WS_LM_EV0 + 6, bit[6]);
      hit(o, WS_LM_EV0 + 7, bit[7]);
      const uint32_t b_lanes = bit[0] & ~bit[9];   /* matched boundaries finish in A */
      hit(o, WS_LM_BI, bit[9]);
      hit(o, WS_LM_A_TAIL, P & ~b_lanes);
      hit(o, WS_LM_A_RR, bit[5] & ~b_lanes);
      for (uint32_t l = 0; l < n_valid; ++l) {
        if (!(P >> l & 1u)) continue;
        if (b_lanes >> l & 1u) { parked |= 1u << l; continue; }   /* Join + Wait */
        jj[l] += 1;
        if (jj[l] == nsteps[l * K + kk[l]]) alive &= ~(1u << l);
      }
    } else if (phase == 2) {
      hit(o, WS_LM_B_REL, Bm);
      uint32_t bit[16] = {0};
      for (uint32_t l = 0; l < n_valid; ++l) {
        if (!(Bm >> l & 1u)) continue;
        or_event e = evt(ev, ev_off, K, kk, jj, l);
        for (int b = 0; b < 16; ++b)
          if (e >> b & 1u) bit[b] |= 1u << l;
      }
      hit(o, WS_LM_EV0 + 2, bit[2]);
      hit(o, WS_LM_EV0 + 3, bit[3]);
      hit(o, WS_LM_EV0 + 4, bit[4]);
      hit(o, WS_LM_EV0 + 8, bit[8]);
      hit(o, WS_LM_B_RR, bit[5]);
      for (uint32_t l = 0; l < n_valid; ++l) {
        if (!(Bm >> l & 1u)) continue;
        jj[l] += 1;
        if (jj[l] == nsteps[l * K + kk[l]]) alive &= ~(1u << l);
      }
      parked = 0;
    } else {
      hit(o, WS_LM_ADVANCE, R);
      hit(o, WS_LM_LAUNCH, R);
      for (uint32_t l = 0; l < n_valid; ++l) {
        if (!(R >> l & 1u)) continue;
        kk[l] = next[l]++;
        jj[l] = 0;
        alive |= 1u << l;
      }
    }
  }
}

/* ------------------------------------------------------------------ */
/* Exhaustive optimum of the iteration-delay program for W <= 4, L <= 4:
 * 0-1 BFS over (it[l], parked[l]); advancing one free lane costs 0,
 * releasing any non-empty subset of parked lanes costs 1 Expensive execution. */
uint32_t ws_divloop_optimum(const uint8_t* want, uint32_t W, uint32_t L) {
  if (W == 0 || W > 4 || L > 4) return 0xffffffffu;
  uint32_t base = L + 1u;
  uint32_t nstate = 1;
  for (uint32_t l = 0; l < W; ++l) nstate *= base * 2u;
  uint32_t* dist = (uint32_t*)malloc(sizeof(uint32_t) * nstate);
  /* 0-1 BFS deque: dist[] of a state improves at most L*W+1 times, so
   * front pushes <= nstate*32 and back pushes <= nstate*96 */
  uint32_t* dq = (uint32_t*)malloc(sizeof(uint32_t) * nstate * 128u);
  for (uint32_t s = 0; s < nstate; ++s) dist[s] = 0xffffffffu;
  /* state encoding: digit l = it[l]*2 + parked[l] in base 2(L+1) */
  uint32_t head = nstate * 32u, tail = head;
  dist[0] = 0;
  dq[tail++] = 0;
  uint32_t best = 0xffffffffu;
  while (head < tail) {
    uint32_t s = dq[head++];
    uint32_t d = dist[s];
    uint32_t it[4], pk[4], x = s;
    for (uint32_t l = 0; l < W; ++l) { uint32_t dg = x % (2u * base); x /= 2u * base; it[l] = dg / 2u; pk[l] = dg % 2u; }
    int done = 1;
    for (uint32_t l = 0; l < W; ++l) if (it[l] < L || pk[l]) done = 0;
    if (done) { if (d < best) best = d; continue; }
    /* cost-0 moves: advance one free lane */
    for (uint32_t l = 0; l < W; ++l) {
      if (pk[l] || it[l] >= L) continue;
      uint32_t nit[4], npk[4];
      memcpy(nit, it, sizeof nit); memcpy(npk, pk, sizeof npk);
      if (want[l * L + it[l]]) npk[l] = 1; else nit[l] += 1;
      uint32_t ns = 0, mul = 1;
      for (uint32_t q = 0; q < W; ++q) { ns += (nit[q] * 2u + npk[q]) * mul; mul *= 2u * base; }
      if (dist[ns] > d) { dist[ns] = d; dq[--head] = ns; }
    }
    /* cost-1 moves: release a non-empty subset of parked lanes */
    uint32_t pmask = 0;
    for (uint32_t l = 0; l < W; ++l) if (pk[l]) pmask |= 1u << l;
    for (uint32_t sub = pmask; sub; sub = (sub - 1u) & pmask) {
      uint32_t nit[4], npk[4];
      memcpy(nit, it, sizeof nit); memcpy(npk, pk, sizeof npk);
      for (uint32_t l = 0; l < W; ++l) if (sub >> l & 1u) { npk[l] = 0; nit[l] += 1; }
      uint32_t ns = 0, mul = 1;
      for (uint32_t q = 0; q < W; ++q) { ns += (nit[q] * 2u + npk[q]) * mul; mul *= 2u * base; }
      if (dist[ns] > d + 1u) { dist[ns] = d + 1u; dq[tail++] = ns; }
    }
  }
  free(dist);
  free(dq);
  return best;
}
