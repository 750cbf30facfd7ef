// ap_master.cuh -- the u32 fast path WITH the master stage (k = 1, p == P <= 16,
// P <= m <= 127): decision bits written during the offset-form sweep, and a walk of
// the critical path back from the sink (readings Q10, Q11).
//
// Shares nothing with oracle/.  Used by k_eval_fast (ap_eval_batch with master) and
// the heuristic's warp pool (k_heur_pool).  DESIGN.md §5.5.
//
// Decision bits of one simulation (row formulation of ap_device.cuh: F(x, j) sits in
// row j + x, B(x, y) in row y + P - 1):
//   F bit (x, r), 1 <= x <= P-1: "F(x) of row r takes its cross predecessor F(x-1)"
//          (cross > intra strictly: the intra-stage predecessor outranks on a tie, Q10).
//   B bit (x, t) of the cool-down row m-1+t, t = 0..P-1, stages x < t only: "B(x)
//          takes its cross predecessor B(x+1)" (cross >= intra: stage x+1 outranks on
//          a tie).
// Every other B bit is NOT stored: wherever stage x still runs a forward in row r+1,
// B(x, r) and F(x+1, r+1) compare the same pair (FF[x], b[x+1]) (the fused step of
// DESIGN.md §5.1), so B bit (x, r) = NOT F bit (x+1, r+1).
// Storage (MasterBits), per lane, lanes interleaved with `stride`:
//   cw  the F bits of the steady rows r = P..m-1 as COLUMN words: word (blk, x) holds
//       F bit (x, 32 blk + j) in bit j, at cw[(blk (P-1) + x - 1) stride]; rows < P
//       read as 0 (the warm-up and row P-1 record nothing: the walk ends there);
//   rw  the cool-down rows: F word of row m+i (bit x) at rw[i stride], i = 0..P-2,
//       then the B words, t = 0..P-1, at rw[(P-1+t) stride].
// The column layout lets the walk jump over the rows where the critical path stays on
// one stage (backtrack_master): one find-last-set per stage change instead of one
// step per row.
#pragma once
#include "ap_device.cuh"

namespace apdev {

struct MasterBits {
  uint32_t* cw;  // column words of the steady F bits
  uint16_t* rw;  // cool-down row words (F, then B)
  int stride;
};
// per-lane sizes: 32-bit column words, then 16-bit row words
__host__ __device__ inline int master_col_words(int m, int P) { return (((m - 1) >> 5) + 1) * (P - 1); }
__host__ __device__ inline int master_row_words(int P) { return 2 * P - 1; }
__host__ __device__ inline size_t master_bits_bytes(int m, int P, int lanes) {
  return ((size_t)master_col_words(m, P) * 4 + (size_t)master_row_words(P) * 2) * (size_t)lanes;
}

// n = max(a, t); word += BIT if a > t.  The compare and the max are ALU instructions,
// the bit goes in with a predicated IMAD (FMA pipe), so one decision costs two ALU
// slots instead of four (compare, max, select, or).
template <uint32_t BIT>
AP_DEV_INLINE uint32_t max_bit(uint32_t a, uint32_t t, uint32_t& word, uint32_t one) {
  uint32_t n;
  asm("{\n\t.reg .pred p;\n\t"
      "setp.gt.u32 p, %2, %3;\n\t"
      "max.u32 %0, %2, %3;\n\t"
      "@p mad.lo.u32 %1, %4, %5, %1;\n\t}"
      : "=r"(n), "+r"(word)
      : "r"(a), "r"(t), "r"(one), "n"(BIT));
  return n;
}

// Cool-down helpers (predicated IMADs for the bits, as max_bit):
// n = max(a, t); wf += BF if a > t; wb += BB if !(a > t)
template <uint32_t BF, uint32_t BB>
AP_DEV_INLINE uint32_t max_bit2(uint32_t a, uint32_t t, uint32_t& wf, uint32_t& wb, uint32_t one) {
  uint32_t n;
  asm("{\n\t.reg .pred p;\n\t"
      "setp.gt.u32 p, %3, %4;\n\t"
      "max.u32 %0, %3, %4;\n\t"
      "@p mad.lo.u32 %1, %5, %6, %1;\n\t"
      "@!p mad.lo.u32 %2, %5, %7, %2;\n\t}"
      : "=r"(n), "+r"(wf), "+r"(wb)
      : "r"(a), "r"(t), "r"(one), "n"(BF), "n"(BB));
  return n;
}
// n = max(a, t); wb += BB if a >= t
template <uint32_t BB>
AP_DEV_INLINE uint32_t max_bit_ge(uint32_t a, uint32_t t, uint32_t& wb, uint32_t one) {
  uint32_t n;
  asm("{\n\t.reg .pred p;\n\t"
      "setp.ge.u32 p, %2, %3;\n\t"
      "max.u32 %0, %2, %3;\n\t"
      "@p mad.lo.u32 %1, %4, %5, %1;\n\t}"
      : "=r"(n), "+r"(wb)
      : "r"(a), "r"(t), "r"(one), "n"(BB));
  return n;
}
AP_DEV_INLINE uint32_t madd(uint32_t a, uint32_t b, uint32_t one) {  // a + b on the FMA pipe
  uint32_t d;
  asm("mad.lo.u32 %0, %1, %2, %3;" : "=r"(d) : "r"(a), "r"(one), "r"(b));
  return d;
}

template <int P, int T, int X>
AP_DEV_INLINE void cool_row_x(uint32_t (&FF)[P], uint32_t (&L)[P], const uint32_t (&wF)[P],
                              const uint32_t (&wB)[P], uint32_t& b, uint32_t& wordF,
                              uint32_t& wordB, uint32_t one) {
  if constexpr (X >= 0) {
    if constexpr (X >= T) {
      // B(X) and (T < P-1) F(X+1) of the next row share max(FF[X], b[X+1]); B(X)'s bit
      // is the complement of F(X+1)'s, so only the F bit is recorded
      const uint32_t M = max_bit<(1u << (X + 1))>(FF[X], b, wordF, one);
      if constexpr (T < P - 1) FF[X + 1] = madd(M, wF[X + 1], one);
      b = madd(M, wB[X], one);
      if constexpr (X == T) L[X] = b;
    } else {
      // stage X already ran its last forward: B(X) = max(B(X+1), L[X]) + wB
      b = madd(max_bit_ge<(1u << X)>(b, L[X], wordB, one), wB[X], one);
      L[X] = b;
    }
    cool_row_x<P, T, X - 1>(FF, L, wF, wB, b, wordF, wordB, one);
  }
}

template <int P, int T>
AP_DEV_INLINE void cool_rows(uint32_t (&FF)[P], uint32_t (&L)[P], const uint32_t (&wF)[P],
                             const uint32_t (&wB)[P], uint32_t& b, MasterBits br, uint32_t one) {
  if constexpr (T < P) {
    uint32_t wordB = 0, wordF = 0;
    b = madd(FF[P - 1], wB[P - 1], one);
    cool_row_x<P, T, P - 2>(FF, L, wF, wB, b, wordF, wordB, one);
    br.rw[(size_t)(P - 1 + T) * br.stride] = (uint16_t)wordB;
    if constexpr (T < P - 1) br.rw[(size_t)T * br.stride] = (uint16_t)wordF;
    cool_rows<P, T + 1>(FF, L, wF, wB, b, br, one);
  }
}

// n = max(a, t); col += rb if a > t (rb: the row's bit in its column word, a register;
// the add is a predicated IMAD on the FMA pipe, as max_bit)
AP_DEV_INLINE uint32_t max_bitr(uint32_t a, uint32_t t, uint32_t& col, uint32_t rb, uint32_t one) {
  uint32_t n;
  asm("{\n\t.reg .pred p;\n\t"
      "setp.gt.u32 p, %2, %3;\n\t"
      "max.u32 %0, %2, %3;\n\t"
      "@p mad.lo.u32 %1, %4, %5, %1;\n\t}"
      : "=r"(n), "+r"(col)
      : "r"(a), "r"(t), "r"(rb), "r"(one));
  return n;
}

// Column words of the steady rows: bit rb of col[x] = F bit x of the current row;
// advance() moves to the next row and stores the P-1 words when a 32-row block is full.
template <int P>
struct ColAcc {
  uint32_t col[P];  // col[x], x = 1..P-1 (col[0] unused)
  uint32_t rb;
  uint32_t* cw;
  int stride;
  AP_DEV_INLINE void flush() {
#pragma unroll
    for (int x = 1; x < P; ++x) {
      cw[(size_t)(x - 1) * stride] = col[x];
      col[x] = 0;
    }
    cw += (size_t)(P - 1) * stride;
  }
  AP_DEV_INLINE void advance() {
    rb <<= 1;
    if (rb == 0u) {  // warp-uniform: every lane is on the same row
      flush();
      rb = 1u;
    }
  }
};

// One fused steady step in the offset form that also records the F
// bits of the next row: n'[x] = max(n'[x+1] + s[x+1], N[x-1]), bit x+1 = N[x-1] >
// n'[x+1] + s[x+1] (= FF[x] > b[x+1]); at x = 0 the intra operand is N[0] + s[0].
template <int P, int X>
AP_DEV_INLINE void nstep_cols_x(uint32_t (&n)[P], const uint32_t (&N)[P], const uint32_t (&sw)[P],
                                ColAcc<P>& ca, uint32_t one) {
  if constexpr (X >= 1) {
    uint32_t t;
    asm("mad.lo.u32 %0, %1, %2, %3;" : "=r"(t) : "r"(n[X + 1]), "r"(one), "r"(sw[X + 1]));
    n[X] = max_bitr(N[X - 1], t, ca.col[X + 1], ca.rb, one);
    nstep_cols_x<P, X - 1>(n, N, sw, ca, one);
  } else {
    uint32_t t, u;
    asm("mad.lo.u32 %0, %1, %2, %3;" : "=r"(t) : "r"(n[1]), "r"(one), "r"(sw[1]));
    asm("mad.lo.u32 %0, %1, %2, %3;" : "=r"(u) : "r"(N[0]), "r"(one), "r"(sw[0]));
    n[0] = max_bitr(u, t, ca.col[1], ca.rb, one);
  }
}

template <int P>
AP_DEV_INLINE void nstep_cols(uint32_t (&N)[P], const uint32_t (&sw)[P], ColAcc<P>& ca, uint32_t one) {
  static_assert(P >= 3, "");
  uint32_t n[P], t;
  asm("mad.lo.u32 %0, %1, %2, %3;" : "=r"(t) : "r"(N[P - 2]), "r"(one), "r"(sw[P - 1]));
  n[P - 2] = max_bitr(N[P - 3], t, ca.col[P - 1], ca.rb, one);
  nstep_cols_x<P, P - 3>(n, N, sw, ca, one);
#pragma unroll
  for (int x = 0; x <= P - 2; ++x) N[x] = n[x];
}

// Aligned 8-row chunks of the steady rows (AP_MASTER_CHUNK, default on).  Row j of a
// chunk that starts at a row r with r % 8 == 0 puts its bits at rbase << j, rbase = the
// bit of row r in its column word, so every bit is a predicated IMAD with an immediate
// multiplier and the 8 rows are one straight-line block: ptxas can overlap the rows
// (row r+1's first decision needs only row r's second), where the one-row loop with its
// block-full test after every row ran each row's 15-decision chain alone.  The value
// itself is one fused add+max (VIADDMNMX) on the chain; the compare that sets the bit
// uses its own add (t, an IMAD with the runtime `one`, so it is not merged into the
// chain) and sits beside it.
#ifndef AP_MASTER_CHUNK
#define AP_MASTER_CHUNK 1
#endif
// rbj = the row's bit (rbase << J, a register); the bit goes in as rbj * one with the
// runtime `one`, which keeps it ONE predicated IMAD (with an immediate multiplier ptxas
// folded rbase * 2^J into a hoisted register and emitted add + SEL, an ALU instruction)
AP_DEV_INLINE uint32_t dec_chunk(uint32_t nx1, uint32_t s, uint32_t a, uint32_t& col,
                                 uint32_t rbj, uint32_t one) {
  uint32_t t;
  asm("mad.lo.u32 %0, %1, %2, %3;" : "=r"(t) : "r"(nx1), "r"(one), "r"(s));
  const uint32_t n = max(nx1 + s, a);
  asm("{\n\t.reg .pred p;\n\t"
      "setp.gt.u32 p, %1, %2;\n\t"
      "@p mad.lo.u32 %0, %3, %4, %0;\n\t}"
      : "+r"(col)
      : "r"(a), "r"(t), "r"(rbj), "r"(one));
  return n;
}

template <int P, int J, int X>
AP_DEV_INLINE void chunk_row_x(uint32_t (&n)[P], const uint32_t (&N)[P], const uint32_t (&sw)[P],
                               uint32_t (&col)[P], uint32_t rbj, uint32_t one) {
  if constexpr (X >= 1) {
    n[X] = dec_chunk(n[X + 1], sw[X + 1], N[X - 1], col[X + 1], rbj, one);
    chunk_row_x<P, J, X - 1>(n, N, sw, col, rbj, one);
  } else {
    uint32_t u;
    asm("mad.lo.u32 %0, %1, %2, %3;" : "=r"(u) : "r"(N[0]), "r"(one), "r"(sw[0]));
    n[0] = dec_chunk(n[1], sw[1], u, col[1], rbj, one);
  }
}

template <int P, int J>
AP_DEV_INLINE void chunk_rows(uint32_t (&N)[P], const uint32_t (&sw)[P], uint32_t (&col)[P],
                              uint32_t rbase, uint32_t one) {
  if constexpr (J < 8) {
    uint32_t n[P], rbj;
    asm("mad.lo.u32 %0, %1, %2, 0;" : "=r"(rbj) : "r"(rbase), "n"(1u << J));
    n[P - 2] = dec_chunk(N[P - 2], sw[P - 1], N[P - 3], col[P - 1], rbj, one);
    chunk_row_x<P, J, P - 3>(n, N, sw, col, rbj, one);
#pragma unroll
    for (int x = 0; x <= P - 2; ++x) N[x] = n[x];
    chunk_rows<P, J + 1>(N, sw, col, rbase, one);
  }
}

// Every CR rows the steady state is either clamped to S (RENORM = false: a candidate
// whose T reaches S is not exact and is recomputed by the caller) or RENORMALISED
// (RENORM = true): the least running value is subtracted from all of them and added to
// a 64-bit base.  The row recurrence only adds weights to state values and takes
// maxima of them, so shifting the whole state by a constant shifts every later value by
// it and leaves every comparison -- every decision bit -- unchanged; T = base + the
// returned value.  The state stays within S of its minimum except in pathological
// cases, which clear `exact` (the caller recomputes those).  Offset form: N >= 0 holds
// after a shift by min N.
struct Renorm {
  unsigned long long base = 0;
  bool exact = true;
};
template <int P, bool RENORM, int CNT>
AP_DEV_INLINE void fix_state(uint32_t (&V)[P], uint32_t S, Renorm& rn) {
  if constexpr (RENORM) {
    uint32_t mn = V[0], mx = V[0];
#pragma unroll
    for (int x = 1; x < CNT; ++x) {
      mn = min(mn, V[x]);
      mx = max(mx, V[x]);
    }
#pragma unroll
    for (int x = 0; x < CNT; ++x) V[x] -= mn;
    rn.base += mn;
    rn.exact = rn.exact && (mx - mn < S);
  } else {
#pragma unroll
    for (int x = 0; x < CNT; ++x) V[x] = min(V[x], S);
  }
}

// T (u32; >= S means "not exact, recompute") of one candidate, k = 1, p == P, m >= P,
// with the decision bits above.  wF/wB: stage weights incl. the receiver-side Comm.
// Values are clamped to S (or renormalised, see Renorm) every CR rows of the steady
// part; the caller's S leaves room for max(CR, P) + 1 rows of growth
// (heur_fast_bound).
template <int P, bool RENORM = false>
AP_DEV_INLINE uint32_t sim_master(int m, const uint32_t (&wF)[P], const uint32_t (&wB)[P],
                                  uint32_t S, int CR, MasterBits br, uint32_t one,
                                  Renorm* rnp = nullptr) {
  Renorm rn;
  static_assert(P >= 2 && P <= 16, "16-bit cool-down words");
  uint32_t FF[P], L[P];
  // micro-batch 0 (k = 1): F(x, 0) in row x, cross predecessor only (no bit)
  FF[0] = wF[0];
#pragma unroll
  for (int x = 1; x < P; ++x) FF[x] = FF[x - 1] + wF[x];
  // warm-up rows r = 1..P-2 (stage x <= r-1 runs F(x, r-x)) and the forward part of
  // row P-1: no bits, the backtrack stops before them
#pragma unroll
  for (int r = 1; r <= P - 2; ++r) {
#pragma unroll
    for (int x = r - 1; x >= 1; --x) FF[x] = max(FF[x - 1], FF[x]) + wF[x];
    FF[0] = FF[0] + wF[0];
  }
#pragma unroll
  for (int x = 0; x < P; ++x) L[x] = FF[x];
#pragma unroll
  for (int x = P - 2; x >= 1; --x) FF[x] = max(FF[x - 1], L[x]) + wF[x];
  if (P >= 2) FF[0] = L[0] + wF[0];
  if constexpr (!RENORM) {  // (RENORM: the warm-up values are small, and a shift here
                            // would break the offset form's N >= 0)
#pragma unroll
    for (int x = 0; x < P; ++x) FF[x] = min(FF[x], S);
  }
  int rem = m - P;
  // the steady rows' F bits, rows P..m-1, as column words (bits of rows < P stay 0)
  ColAcc<P> ca;
#pragma unroll
  for (int x = 0; x < P; ++x) ca.col[x] = 0;
  ca.rb = 1u << P;
  ca.cw = br.cw;
  ca.stride = br.stride;
  if constexpr (P >= 3) {
    if (rem > 0) {
      uint32_t c[P], sw[P], N[P];
      c[0] = wF[0];
#pragma unroll
      for (int x = 1; x < P; ++x) c[x] = c[x - 1] + wF[x];
#pragma unroll
      for (int x = 0; x < P; ++x) sw[x] = wF[x] + wB[x];
      {  // first fused step in the M-form, kept as N = M - c (F bits of row P)
        uint32_t b = FF[P - 1] + wB[P - 1];
#pragma unroll
        for (int x = P - 2; x >= 0; --x) {
          const uint32_t M = max_bitr(FF[x], b, ca.col[x + 1], ca.rb, one);
          N[x] = M - c[x];
          b = M + wB[x];
        }
        ca.advance();
      }
#if AP_MASTER_CHUNK
      // rows P+1 .. m-1: single rows up to an 8-aligned row, aligned 8-row chunks, single
      // rows for the rest; a clamp whenever the next piece would take the rows since the
      // last one past CR (the caller's S leaves room for CR + 1 rows of growth)
      int r = P + 1, since = 1;
      const int mrow = P + rem;  // = m
      while (r < mrow) {
        const bool chunk = CR >= 8 && (r & 7) == 0 && r + 8 <= mrow;
        const int len = chunk ? 8 : 1;
        if (since + len > CR) {
          fix_state<P, RENORM, P - 1>(N, S, rn);
          since = 0;
        }
        if (chunk) {
          chunk_rows<P, 0>(N, sw, ca.col, ca.rb, one);
          ca.rb <<= 8;
          if (ca.rb == 0u) {
            ca.flush();
            ca.rb = 1u;
          }
        } else {
          nstep_cols<P>(N, sw, ca, one);
          ca.advance();
        }
        r += len;
        since += len;
      }
      fix_state<P, RENORM, P - 1>(N, S, rn);
#else
      int blk = (rem < CR ? rem : CR) - 1;
      rem -= blk + 1;
      for (;;) {
        for (; blk > 0; --blk) {
          nstep_cols<P>(N, sw, ca, one);
          ca.advance();
        }
        fix_state<P, RENORM, P - 1>(N, S, rn);
        if (rem <= 0) break;
        blk = rem < CR ? rem : CR;
        rem -= blk;
      }
#endif
#pragma unroll
      for (int x = 0; x <= P - 2; ++x) FF[x + 1] = N[x] + c[x + 1];
      FF[0] = N[0] + c[0] + sw[0];
    }
  } else {
    // P = 2: one decision per row, M-form
    while (rem > 0) {
      int blk = rem < CR ? rem : CR;
      rem -= blk;
      for (; blk > 0; --blk) {
        const uint32_t b = FF[1] + wB[1];
        const uint32_t M = max_bitr(FF[0], b, ca.col[1], ca.rb, one);
        FF[1] = M + wF[1];
        FF[0] = M + wB[0] + wF[0];
        ca.advance();
      }
      fix_state<P, RENORM, P>(FF, S, rn);
    }
  }
  // the last, partial block (rb == 1: the previous row filled a block, already stored)
  if (m > P && ca.rb != 1u) ca.flush();
  // cool-down t = 0..P-1 (row m-1+t): B of the row, F of the next row for x >= t+1.
  // Stages x < t ran their last forward already: their B reads L[x].
  uint32_t b = 0;
  cool_rows<P, 0>(FF, L, wF, wB, b, br, one);
  if (rnp) *rnp = rn;
  return b;
}

// Master stage of the simulation recorded by sim_master (same P, m): walk the unique
// critical path back from the sink B(0, m-1) (row m+P-2) to the source with the tie
// rule of Q10, and count per stage its ops in the 1F1B phase (rows [P-1, m-1+x] of
// stage x, for F and B alike); master = most ops, ties -> higher stage, P-1 if none
// (Q11).  Every edge of the path stays in its row (B(x) -> B(x+1) cross, B(x) -> F(x)
// intra) or goes one row up (F(x) -> F(x-1) cross, F(x) -> B(x) intra, cool-down
// B(x) -> B(x)).  Per-stage counts are CB-bit fields of NW registers, flushed when the
// path changes stage.  CB = 8 needs 2m <= 255.
//  1. Cool-down rows m+P-2 .. m-1, one row per step, as the row words dictate.
//  2. Steady rows m-2 .. P-1: on B(x, r) the path stays on stage x (B(x, r) -> F(x, r)
//     -> B(x, r-1), two ops per row) until the first row r' <= r with
//       B bit (x, r') = NOT F bit (x+1, r'+1)   (B takes B(x+1)), or  F bit (x, r'),
//     the highest set bit of (col[x] | ~(col[x+1] >> 1)) below r: one find-last-set
//     per stage change (or per 32-row block), not one step per row.
template <int P, int CB>
AP_DEV_INLINE int backtrack_master(int m, MasterBits br) {
  constexpr unsigned PER = 32 / CB;
  constexpr int NW = (P + PER - 1) / PER;
  constexpr uint32_t maskB = (1u << (P - 1)) - 1u;  // B bits of stages 0..P-2
  const uint16_t* fw = br.rw;                        // F words of rows m .. m+P-2
  const uint16_t* bw = br.rw + (size_t)(P - 1) * br.stride;
  const uint32_t* cw = br.cw;
  const int st = br.stride;
  uint32_t cnt[NW];
#pragma unroll
  for (int w = 0; w < NW; ++w) cnt[w] = 0;
  auto flush = [&](unsigned x, uint32_t run) {
    AP_CHECK(x < (unsigned)P && run <= 2u * (uint32_t)m + 2u);
    const uint32_t inc = run << (CB * (x % PER));
#pragma unroll
    for (int w = 0; w < NW; ++w) cnt[w] += (w == (int)(x / PER)) ? inc : 0u;
  };
  // F bit (x, r) of a steady row r <= m-1 (stage 0 has none)
  auto fbit = [&](unsigned x, int r) -> uint32_t {
    return x >= 1 ? (cw[(size_t)((r >> 5) * (P - 1) + (int)x - 1) * st] >> (r & 31)) & 1u : 0u;
  };
  unsigned x = 0;
  bool onB = true;
  uint32_t run = 0, wn = 0;  // wn: F word of row r+1
  // 1. the cool-down rows (t = r - (m-1) = P-1 .. 0)
  for (int r = m + P - 2; r >= m - 1; --r) {
    const int t = r - (m - 1);
    // F word of row r (row m-1 is a steady row: its bits are in the columns, and
    // only the one of the stage the walk is on after its B chain is read)
    const uint32_t wr = (t > 0) ? (uint32_t)fw[(size_t)(t - 1) * st] : 0u;
    if (onB) {
      // B bits of row r: NOT the F bits of row r+1 where stage x+1 forwards in row r+1
      // (x >= t), the stored ones for x < t
      uint32_t bB = ~(wn >> 1) & maskB;
      if (t > 0) bB = (bB & ~((1u << t) - 1u)) | (uint32_t)bw[(size_t)t * st];
      uint32_t tt = bB >> x;  // bit j: B(x+j, r) takes its cross predecessor B(x+j+1, r)
      if (tt & 1u) {
        run += ((int)x >= t) ? 1u : 0u;
        flush(x, run);
        run = 0;
        ++x;
        tt >>= 1;
        while (tt & 1u) {  // one more cross B, on stage x
          flush(x, ((int)x >= t) ? 1u : 0u);
          ++x;
          tt >>= 1;
        }
      }
      // B(x, r) takes its intra predecessor; it is in the 1F1B phase iff r <= m-1+x
      const bool fhere = (int)x >= t;
      run += fhere ? 1u : 0u;
      if (!fhere) {  // cool-down, stage x ran no F in this row: B(x, r-1) next
        wn = wr;
        continue;
      }
      // F(x, r) next, same row
    }
    // F(x, r), micro-batch r - x, in the 1F1B phase
    ++run;
    if ((t > 0 ? (wr >> x) & 1u : fbit(x, r)) != 0u) {  // cross: F(x-1, r-1)
      flush(x, run);
      run = 0;
      --x;
      onB = false;
    } else {
      onB = true;  // B(x, r-1)
    }
    wn = wr;
  }
  // 2. the steady rows, by column words (rows < P-1 are warm-up forwards: not counted)
  const int lastb = (m - 1) >> 5;
  int r = m - 2;
  while (r >= P - 1) {
    const int b = r >> 5, rl = r & 31;
    AP_CHECK(b <= ((m - 1) >> 5) && x < (unsigned)P);
    const uint32_t* cb = cw + (size_t)(b * (P - 1)) * st;
    if (onB) {
      const uint32_t cx = x >= 1 ? cb[(size_t)(x - 1) * st] : 0u;
      // bit j of nx: F bit (x+1, 32b + j + 1); row 32b+32 is block b+1's bit 0 (it
      // exists whenever it can be read: j <= rl and 32b + rl + 1 <= m-1)
      uint32_t nx = 0xffffffffu;  // stage P-1 has no cross B predecessor
      if ((int)x <= P - 2) {
        const uint32_t lo = cb[(size_t)x * st] >> 1;
        const uint32_t hi = b < lastb ? cb[(size_t)((P - 1) + x) * st] << 31 : 0u;
        nx = lo | hi;
      }
      const int lo_row = b == 0 ? P - 1 : 0;  // rows < P-1 are not walked
      uint32_t E = (cx | ~nx) & ((2u << rl) - 1u) & ~((1u << lo_row) - 1u);
      if (E == 0u) {  // stays on stage x down to the block's first walked row
        run += 2u * (uint32_t)(rl - lo_row + 1);
        r = 32 * b + lo_row - 1;
        continue;
      }
      const int j = 31 - __clz(E);
      run += 2u * (uint32_t)(rl - j);
      r = 32 * b + j;
      if ((~nx >> j) & 1u) {  // B(x, r) takes B(x+1, r)
        flush(x, run + 1u);
        run = 0;
        ++x;
      } else {  // B(x, r) -> F(x, r) -> F(x-1, r-1)
        flush(x, run + 2u);
        run = 0;
        --x;
        --r;
        onB = false;
      }
    } else {  // F(x, r)
      ++run;
      if (x >= 1 && ((cb[(size_t)(x - 1) * st] >> rl) & 1u)) {
        flush(x, run);
        run = 0;
        --x;
      } else {
        onB = true;
      }
      --r;
    }
  }
  flush(x, run);
  constexpr uint32_t MASK = (CB == 8) ? 0xffu : 0xffffu;
  int best = P - 1;
  uint32_t bc = (cnt[(P - 1) / PER] >> (CB * ((P - 1) % PER))) & MASK;
#pragma unroll
  for (int xx = P - 2; xx >= 0; --xx) {
    const uint32_t c = (cnt[xx / PER] >> (CB * (xx % PER))) & MASK;
    if (c > bc) {
      best = xx;
      bc = c;
    }
  }
  return best;
}


}  // namespace apdev
