// ap_master.cuh -- the u32 fast path WITH the master stage (k = 1, p == P <= 16,
// P <= m <= 127): decision words written during the offset-form sweep, and a
// run-length backtrack of the critical path (readings Q10, Q11).
//
// Shares nothing with oracle/.  Used by k_eval_fast (ap_eval_batch with master) and
// the heuristic's warp pool (k_heur_wpool).  DESIGN.md §5.5.
//
// Decision words, one simulation (rows r = 0 .. m+P-2 of the row formulation,
// ap_device.cuh: F(x, j) sits in row j + x, B(x, y) in row y + P - 1):
//   fw[r]  (uint16) F bits: bit x (1 <= x <= P-1) = "F(x) of row r takes its cross
//          predecessor F(x-1)" (cross > intra strictly: the intra-stage predecessor
//          outranks on a tie, Q10).  Bit 0 and bits >= P are 0.
//   bw[t]  (uint16) B bits of the cool-down row m-1+t, t = 0..P-1, for the stages x < t
//          only: bit x = "B(x) takes its cross predecessor B(x+1)" (cross >= intra:
//          the cross one, stage x+1, outranks on a tie).
// Every other B bit is NOT stored: wherever stage x still runs a forward in row r+1,
// B(x, r) and F(x+1, r+1) compare the same pair (FF[x], b[x+1]) (the fused step of
// DESIGN.md §5.1), so B bit x of row r = NOT F bit x+1 of row r+1.
// Only the rows the backtrack reads are written: the warm-up rows 0..P-2 hold no op of
// the 1F1B phase, so the walk stops when it reaches them (backtrack_rows) and the sweep
// records no bits there.
// Layout: word i of the simulation at base[i * stride] (the lanes of a warp/CTA are
// interleaved, so 32 lanes store 64 contiguous bytes).
#pragma once
#include "ap_device.cuh"

namespace apdev {

struct Bits16 {
  uint16_t* base;  // fw[0 .. m+P-2], then bw[0 .. P-1]
  int stride;
};

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
AP_DEV_INLINE void cool_rows(int m, uint32_t (&FF)[P], uint32_t (&L)[P], const uint32_t (&wF)[P],
                             const uint32_t (&wB)[P], uint32_t& b, Bits16 br, uint16_t* bw,
                             uint32_t one) {
  if constexpr (T < P) {
    uint32_t wordB = 0, wordF = 0;
    b = madd(FF[P - 1], wB[P - 1], one);
    cool_row_x<P, T, P - 2>(FF, L, wF, wB, b, wordF, wordB, one);
    bw[(size_t)T * br.stride] = (uint16_t)wordB;
    if constexpr (T < P - 1) br.base[(size_t)(m + T) * br.stride] = (uint16_t)wordF;
    cool_rows<P, T + 1>(m, FF, L, wF, wB, b, br, bw, one);
  }
}

// One fused steady step in the offset form that also records the F
// bits of the next row: n'[x] = max(n'[x+1] + s[x+1], N[x-1]), bit x+1 = N[x-1] >
// n'[x+1] + s[x+1] (= FF[x] > b[x+1]); at x = 0 the intra operand is N[0] + s[0].
template <int P, int X>
AP_DEV_INLINE void nstep_bits_x(uint32_t (&n)[P], const uint32_t (&N)[P], const uint32_t (&sw)[P],
                                uint32_t& word, uint32_t one) {
  if constexpr (X >= 1) {
    uint32_t t;
    asm("mad.lo.u32 %0, %1, %2, %3;" : "=r"(t) : "r"(n[X + 1]), "r"(one), "r"(sw[X + 1]));
    n[X] = max_bit<(1u << (X + 1))>(N[X - 1], t, word, one);
    nstep_bits_x<P, X - 1>(n, N, sw, word, one);
  } else {
    uint32_t t, u;
    asm("mad.lo.u32 %0, %1, %2, %3;" : "=r"(t) : "r"(n[1]), "r"(one), "r"(sw[1]));
    asm("mad.lo.u32 %0, %1, %2, %3;" : "=r"(u) : "r"(N[0]), "r"(one), "r"(sw[0]));
    n[0] = max_bit<2u>(u, t, word, one);
  }
}

template <int P>
AP_DEV_INLINE uint32_t nstep_bits(uint32_t (&N)[P], const uint32_t (&sw)[P], uint32_t one) {
  static_assert(P >= 3, "");
  uint32_t n[P], word = 0, t;
  asm("mad.lo.u32 %0, %1, %2, %3;" : "=r"(t) : "r"(N[P - 2]), "r"(one), "r"(sw[P - 1]));
  n[P - 2] = max_bit<(1u << (P - 1))>(N[P - 3], t, word, one);
  nstep_bits_x<P, P - 3>(n, N, sw, word, one);
#pragma unroll
  for (int x = 0; x <= P - 2; ++x) N[x] = n[x];
  return word;
}

// T (u32; >= S means "not exact, recompute") of one candidate, k = 1, p == P, m >= P,
// with the decision words above.  wF/wB: stage weights incl. the receiver-side Comm.
// Values are clamped to S every CR rows of the steady part; the caller's S leaves room
// for max(CR, P) + 1 rows of growth (heur_fast_bound).
template <int P>
AP_DEV_INLINE uint32_t sim_bits16(int m, const uint32_t (&wF)[P], const uint32_t (&wB)[P],
                                  uint32_t S, int CR, Bits16 br, uint32_t one) {
  static_assert(P >= 2 && P <= 16, "16-bit decision words");
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
#pragma unroll
  for (int x = 0; x < P; ++x) FF[x] = min(FF[x], S);
  int r = P - 1;  // the row whose B part the next step computes
  int rem = m - P;
  if constexpr (P >= 3) {
    if (rem > 0) {
      uint32_t c[P], sw[P], N[P];
      c[0] = wF[0];
#pragma unroll
      for (int x = 1; x < P; ++x) c[x] = c[x - 1] + wF[x];
#pragma unroll
      for (int x = 0; x < P; ++x) sw[x] = wF[x] + wB[x];
      {  // first fused step in the M-form, kept as N = M - c
        uint32_t word = 0;
        uint32_t b = FF[P - 1] + wB[P - 1];
#pragma unroll
        for (int x = P - 2; x >= 0; --x) {
          word |= (FF[x] > b ? 1u : 0u) << (x + 1);
          const uint32_t M = max(FF[x], b);
          N[x] = M - c[x];
          b = M + wB[x];
        }
        br.base[(size_t)(r + 1) * br.stride] = (uint16_t)word;
        ++r;
      }
      int blk = (rem < CR ? rem : CR) - 1;
      rem -= blk + 1;
      for (;;) {
        for (; blk > 0; --blk) {
          const uint32_t word = nstep_bits<P>(N, sw, one);
          br.base[(size_t)(r + 1) * br.stride] = (uint16_t)word;
          ++r;
        }
#pragma unroll
        for (int x = 0; x <= P - 2; ++x) N[x] = min(N[x], S);
        if (rem <= 0) break;
        blk = rem < CR ? rem : CR;
        rem -= blk;
      }
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
        const uint32_t word = (FF[0] > b ? 1u : 0u) << 1;
        const uint32_t M = max(FF[0], b);
        FF[1] = M + wF[1];
        FF[0] = M + wB[0] + wF[0];
        br.base[(size_t)(r + 1) * br.stride] = (uint16_t)word;
        ++r;
      }
#pragma unroll
      for (int x = 0; x < P; ++x) FF[x] = min(FF[x], S);
    }
  }
  // cool-down t = 0..P-1 (row m-1+t): B of the row, F of the next row for x >= t+1.
  // Stages x < t ran their last forward already: their B reads L[x].
  uint16_t* bw = br.base + (size_t)(m + P - 1) * br.stride;
  uint32_t b = 0;
  cool_rows<P, 0>(m, FF, L, wF, wB, b, br, bw, one);
  return b;
}

// Master stage of the simulation recorded by sim_bits16 (same P, m): walk the unique
// critical path back from the sink B(0, m-1) (row m+P-2) to the source F(0, 0) with
// the tie rule of Q10, and count per stage its ops in the 1F1B phase (rows [P-1,
// m-1+x] of stage x, for F and B alike); master = most ops, ties -> higher stage, P-1
// if none (Q11).
// Every edge of the path stays in its row (B(x) -> B(x+1) cross, B(x) -> F(x) intra)
// or goes one row up (F(x) -> F(x-1) cross, F(x) -> B(x) / F(x) intra, cool-down
// B(x) -> B(x)), so the walk runs row by row, r = m+P-2 .. 0, the same loop in every
// lane of a warp: per row one B-chain (almost always empty), at most one B and one F
// op.  Per-stage counts are CB-bit fields of NW registers, flushed when the path
// changes stage.  CB = 8 needs 2m <= 255.
template <int P, int CB>
AP_DEV_INLINE int backtrack_rows(int m, Bits16 br) {
  constexpr unsigned PER = 32 / CB;
  constexpr int NW = (P + PER - 1) / PER;
  constexpr uint32_t maskB = (1u << (P - 1)) - 1u;  // B bits of stages 0..P-2
  const uint16_t* fw = br.base;
  const uint16_t* bw = br.base + (size_t)(m + P - 1) * br.stride;
  const int st = br.stride;
  uint32_t cw[NW];
#pragma unroll
  for (int w = 0; w < NW; ++w) cw[w] = 0;
  auto flush = [&](unsigned x, uint32_t run) {
    const uint32_t inc = run << (CB * (x % PER));
#pragma unroll
    for (int w = 0; w < NW; ++w) cw[w] += (w == (int)(x / PER)) ? inc : 0u;
  };
  unsigned x = 0;
  bool onB = true;
  uint32_t run = 0, wn = 0;  // wn: F word of row r+1
  // rows r < P-1 hold no 1F1B-phase op (warm-up forwards only): the counts are final
  // once the walk leaves row P-1
  for (int r = m + P - 2; r >= P - 1; --r) {
    const uint32_t wr = fw[(size_t)r * st];
    if (onB) {
      // B bits of row r: NOT the F bits of row r+1 where stage x+1 forwards in row r+1
      // (x >= t = r-(m-1) in the cool-down), the stored ones for x < t
      const int t = r - (m - 1);
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
    // F(x, r), micro-batch r - x, in the 1F1B phase (r >= P-1)
    ++run;
    if ((wr >> x) & 1u) {  // cross: F(x-1, r-1) (x >= 1; r > x here)
      flush(x, run);
      run = 0;
      --x;
      onB = false;
    } else {
      onB = true;  // B(x, r-1), or for r = P-1 the warm-up (the loop ends)
    }
    wn = wr;
  }
  flush(x, run);
  constexpr uint32_t MASK = (CB == 8) ? 0xffu : 0xffffu;
  int best = P - 1;
  uint32_t bc = (cw[(P - 1) / PER] >> (CB * ((P - 1) % PER))) & MASK;
#pragma unroll
  for (int xx = P - 2; xx >= 0; --xx) {
    const uint32_t c = (cw[xx / PER] >> (CB * (xx % PER))) & MASK;
    if (c > bc) {
      best = xx;
      bc = c;
    }
  }
  return best;
}

__host__ __device__ inline int bits16_words(int m, int P) { return m + 2 * P - 1; }

}  // namespace apdev
