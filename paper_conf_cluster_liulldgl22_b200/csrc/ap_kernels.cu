// ap_kernels.cu -- sm_100a kernels of the AutoPipe planner/slicer hot path.
//
//   k_sweep_exact<P,V>  K1 exhaustive sweep, p == P, m >= P.  V = uint32_t is the
//                       exact saturating fast path, V = uint64_t
//                       the plain int64 one.  Per thread: unrank once, lex
//                       successor, row sweep per (rank, k), register argmin,
//                       warp-shuffle -> block -> atomicMin (K5).
//   k_sweep_generic<P>  K1 for any p <= P and any m (exact int64, runtime p).
//   k_eval<P>           K2 thread-per-candidate T (+ master via bits/backtrack).
//   k_heur<P>           K3 heuristic restarts, one lane per restart, refilled from
//                       an atomic restart counter.
//   k_alg1              Algorithm 1 DP, one CTA.
//   k_cpath<P>          critical path with op times for one candidate.
//   k_unrank, k_init    decode / key init.
// Every kernel starts with the K4 prologue (TMA bulk copy of the tables into
// shared memory + warp-shuffle prefix sums), see ap_device.cuh.
#include <atomic>
#include <climits>
#include <cstdlib>
#include <cstdio>

#include "ap_device.cuh"
#include "ap_launch.h"
#include "ap_master.cuh"

namespace apk {
using namespace apdev;

// Every kernel launch of the library bumps this counter (ap_kernel_launches), so a
// bench can state how many of its own kernels ran in a timed region.
static std::atomic<unsigned long long> g_kernel_launches{0};
static inline void count_launch() { g_kernel_launches.fetch_add(1, std::memory_order_relaxed); }
unsigned long long kernel_launches() { return g_kernel_launches.load(std::memory_order_relaxed); }

// ===========================================================================
// K1 fast sweep.
template <typename V>
AP_DEV_INLINE V vmax(V a, V b) {
  return a > b ? a : b;
}
template <typename V>
AP_DEV_INLINE V vmin(V a, V b) {
  return a < b ? a : b;
}

// floor(v / k) for the u32 path: one umulhi with M_k = floor(2^32/k) (k=1:
// 2^32-1) under-estimates by at most 1, fixed by one compare.
AP_DEV_INLINE uint32_t divk(uint32_t v, uint32_t k, uint32_t M) {
  uint32_t q = __umulhi(v, M);
  const uint32_t r = v - q * k;
  return q + (r >= k ? 1u : 0u);
}
AP_DEV_INLINE uint64_t divk(uint64_t v, uint32_t k, uint32_t) { return v / k; }
// floor(v / k) as ONE umulhi with M = ceil(2^32/k), k >= 2: with e = M*k - 2^32 <= k-1,
// umulhi(v, M) = floor(v/k + v*e/(k*2^32)), exact whenever v*e < 2^32, i.e. for every
// v < 2^28 (k <= 16).  The host enables it (SweepArgs.div1) only if every stage
// compute total and every comm is below 2^28; the table then holds the ceil magic,
// for which divk's correction step is a no-op.
AP_DEV_INLINE uint32_t divk(uint32_t v, uint32_t k, uint32_t M, bool div1) {
  return div1 ? __umulhi(v, M) : divk(v, k, M);
}
AP_DEV_INLINE uint64_t divk(uint64_t v, uint32_t k, uint32_t, bool) { return v / k; }


// Integer ops of the sweep, as plain operators: ptxas fuses the add of the backward
// chain into the max (VIADDMNMX, ALU pipe) and puts most other adds on IMAD.IADD (FMA
// pipe).  The steady step forces its remaining adds onto IMAD (fma_add below); doing
// that everywhere, or a signed offset form without adds, measured slower on C4
// (profiles/r01_sweep_variants.md).
template <typename V>
struct XOps {
  static AP_DEV_INLINE V mx(V a, V b) { return a > b ? a : b; }
  static AP_DEV_INLINE V ad(V a, V b, uint32_t) { return a + b; }
  static AP_DEV_INLINE V amx(V a, V b, V c) {  // max(a + b, c)
    const V t = a + b;
    return t > c ? t : c;
  }
};

// One fused steady step: the backward pass of row r and the
// forward pass of row r+1 share their maxima.  With b_r[x] = max(b_r[x+1], FF_r[x]) +
// wB[x] and FF_{r+1}[x+1] = max(FF_r[x], b_r[x+1]) + wF[x+1], both are
// M[x] = max(FF_r[x], b_r[x+1]) plus a weight, and M[x] = max(M[x+1] + wB[x+1],
// FF_r[x]) is one fused add+max (VIADDMNMX, ALU pipe).  A step is P-1 ALU
// instructions plus P IMAD adds (FMA pipe): 2P-1 instructions for the 2P max-plus
// ops of a row.  State between steps: FF[0..P-1] only.
// a + b issued on the FMA pipe (IMAD with a multiplier the compiler cannot fold).
// AP_MSTEP_IMAD = 2 puts every add of the fused steady step there, so a step is P-1
// VIADDMNMX (ALU) + P IMAD (FMA): C4 258.5 -> 252.1 ms (profiles/r01_sweep_variants.md);
// 1 = only FF'[0], 0 = let ptxas choose (it moves some adds to ALU IADD3).
#ifndef AP_MSTEP_IMAD
#define AP_MSTEP_IMAD 2
#endif
template <typename V>
AP_DEV_INLINE V fma_add(V a, V b, uint32_t one) {
  if constexpr (sizeof(V) == 4) {
    uint32_t d;
    asm("mad.lo.u32 %0, %1, %2, %3;" : "=r"(d) : "r"(a), "r"(one), "r"(b));
    return d;
  } else {
    return a + b;
  }
}

template <int P, typename V>
AP_DEV_INLINE void mstep(V (&FF)[P], const V (&wF)[P], const V (&wB)[P], V wBF0, uint32_t one) {
  using O = XOps<V>;
  if constexpr (P == 1) {
    FF[0] = O::ad(FF[0], wBF0, one);
  } else {
    V nF[P];
    V M = O::amx(FF[P - 1], wB[P - 1], FF[P - 2]);
    nF[P - 1] = (AP_MSTEP_IMAD >= 2) ? fma_add(M, wF[P - 1], one) : O::ad(M, wF[P - 1], one);
#pragma unroll
    for (int x = P - 3; x >= 0; --x) {
      M = O::amx(M, wB[x + 1], FF[x]);
      nF[x + 1] = (AP_MSTEP_IMAD >= 2) ? fma_add(M, wF[x + 1], one) : O::ad(M, wF[x + 1], one);
    }
    nF[0] = (AP_MSTEP_IMAD >= 1) ? fma_add(M, wBF0, one) : O::ad(M, wBF0, one);
#pragma unroll
    for (int x = 0; x < P; ++x) FF[x] = nF[x];
  }
}

// Offset form of the fused steady step.  With the per-stage constants
// c_x = wF[0] + .. + wF[x] and s_x = wF[x] + wB[x], store N_x = M_x - c_x (M_x of the
// M-form step).  Then FF'[x] = M_{x-1} + wF[x] = N_{x-1} + c_x for x >= 1 and
// FF'[0] = M_0 + s_0, so the next step is
//   N'_{P-2} = max(N_{P-2} + s_{P-1}, N_{P-3}),
//   N'_x     = max(N'_{x+1} + s_{x+1}, N_{x-1})       x = P-3 .. 1,
//   N'_0     = max(N'_1 + s_1, N_0 + s_0):
// P-1 fused add+max (VIADDMNMX) + 1 add per row instead of 2P-1 instructions.  N >= 0:
// M_x >= FF[x] >= c_x, because every steady-row forward is an unsliced micro-batch whose
// forward chain alone takes c_x.  P >= 3; state N[0..P-2].
template <int P, typename V>
AP_DEV_INLINE void nstep(V (&N)[P], const V (&sw)[P], uint32_t one) {
  using O = XOps<V>;
  static_assert(P >= 3, "");
  V n[P];
  n[P - 2] = O::amx(N[P - 2], sw[P - 1], N[P - 3]);
#pragma unroll
  for (int x = P - 3; x >= 1; --x) n[x] = O::amx(n[x + 1], sw[x + 1], N[x - 1]);
  n[0] = O::amx(n[1], sw[1], fma_add(N[0], sw[0], one));
#pragma unroll
  for (int x = 0; x <= P - 2; ++x) N[x] = n[x];
}

template <int P, typename V>
AP_DEV_INLINE void clamp_n(V (&N)[P], V S) {
  if constexpr (sizeof(V) == 4) {
#pragma unroll
    for (int x = 0; x <= P - 2; ++x) N[x] = min(N[x], S);
  }
}

#ifndef AP_NFORM
#define AP_NFORM 1
#endif
#ifndef AP_EVAL_RENORM
#define AP_EVAL_RENORM 1
#endif

template <int P, typename V>
AP_DEV_INLINE void clamp_ff(V (&FF)[P], V S) {
  if constexpr (sizeof(V) == 4) {
#pragma unroll
    for (int x = 0; x < P; ++x) FF[x] = min(FF[x], S);
  }
}

// Micro-batch 0's forward, sliced into k pieces (reading Q6): FF[x] = finish of the
// last piece F(x, 0, k-1).  The raw stage compute/comm are re-read from shared
// memory only on the k > 1 path.
template <int P, typename V>
AP_DEV_INLINE void pieces(int k, const V (&wF)[P], const int (&c)[P + 1], const V* sPf,
                          const V* sC, uint32_t Mk, bool div1, uint32_t one, V (&FF)[P]) {
  using O = XOps<V>;
  if (k == 1) {
    FF[0] = wF[0];
#pragma unroll
    for (int x = 1; x < P; ++x) FF[x] = fma_add(FF[x - 1], wF[x], one);  // FMA pipe: ALU-bound
  } else {
    V a[P];
#pragma unroll
    for (int x = 0; x < P; ++x) {
      const V Fx = sPf[c[x + 1]] - sPf[c[x]];
      const V Cin = (x > 0) ? sC[c[x] - 1] : V(0);
      a[x] = divk(Fx, (uint32_t)k, Mk, div1) + ((x > 0) ? divk(Cin, (uint32_t)k, Mk, div1) : V(0));
    }
    // Offset form: piece q's finish FF_q[x] = max(FF_q[x-1],
    // FF_{q-1}[x]) + a_x.  With s_x = a_0 + .. + a_x (= FF_0[x]) and E_q = FF_q - s,
    //   E_q[x] = max(E_{q-1}[x] + a_x, E_q[x-1]),  E_q[0] = q a_0,  E_0 = 0,
    // one fused add+max per op; E >= 0 because FF_q >= FF_0.  The last piece (weights
    // al_x = wF_x - (k-1) a_x) reads FF_{k-2}[x] = E[x] + s_x.
    V E[P];
#pragma unroll
    for (int x = 0; x < P; ++x) E[x] = 0;
    for (int q = 1; q < k - 1; ++q) {
      E[0] = fma_add(E[0], a[0], one);
#pragma unroll
      for (int x = 1; x < P; ++x) E[x] = O::amx(E[x], a[x], E[x - 1]);
    }
    const V km1 = V(k - 1);
    V sxr = a[0];
    FF[0] = fma_add(fma_add(E[0], sxr, one), wF[0] - km1 * a[0], one);
#pragma unroll
    for (int x = 1; x < P; ++x) {
      sxr = fma_add(sxr, a[x], one);
      const V t = fma_add(E[x], sxr, one);  // FF_{k-2}[x]
      FF[x] = fma_add(O::mx(FF[x - 1], t), wF[x] - km1 * a[x], one);
    }
  }
}

// Saturating-clamp schedule of the u32 sweep, computed by the host:
// `first` steady rows before the first clamp (0 = clamp right after the warm-up), then
// a clamp every `every` steady rows, and `fin` = clamp once more at the end of the
// steady rows.  Ignored for 64-bit V.
struct ClampSched {
  int first_, every_, fin_;
  AP_DEV_INLINE int first() const { return first_; }
  AP_DEV_INLINE int every() const { return every_; }
  AP_DEV_INLINE int fin() const { return fin_; }
};

// Everything after the pieces, for p == P, m >= P: warm-up rows, the first 1F1B row,
// the fused steady steps and the fused cool-down.
//  REV = false: input FF = finishes of F(x, 0, k-1); returns T = end of B(0, m-1).
//  REV = true : the same sweep on the REVERSED task DAG (weights wF/wB swapped by the
//      caller), which is again a 1F1B schedule: its op B'(x, y) is the original
//      F(x, m-1-y) and F'(x, j) the original B(x, m-1-j), and its "finish" times are
//      the original longest paths to the sink.  It stops before the last backward
//      row (the original micro-batch-0 forwards) and writes
//        G[x] = B'(x, m-2) for x <= P-2 (longest path from the end of F(x,0) via
//               F(x,1)),   G[P-1] = F'(P-1, m-1) (via B(P-1,0)),
//      so that T(k) = max_x (FF_x(k) + G[x]) for every k.
// RENORM (u32, ap_eval_batch T only): the saturating clamps become renormalisations
// (Renorm, ap_master.cuh): the least running value moves into rn->base, so a
// candidate past the u32 bound stays exact; the clamp right after the warm-up is
// skipped (a shift there would break the offset form's N >= 0; those values are small).
template <int P, typename V, bool REV, typename CS, bool RENORM = false>
AP_DEV_INLINE V sweep_tail(int m, V (&FF)[P], const V (&wF)[P], const V (&wB)[P], V S,
                           CS cs, uint32_t one, V (&G)[P], Renorm* rn = nullptr) {
  using O = XOps<V>;
  V L[P];
  // warm-up rows r = 1..P-2: stage x <= r-1 does F(x, r-x); L == FF here
#pragma unroll
  for (int r = 1; r <= P - 2; ++r) {
#pragma unroll
    for (int x = r - 1; x >= 1; --x) FF[x] = O::ad(O::mx(FF[x - 1], FF[x]), wF[x], one);
    FF[0] = O::ad(FF[0], wF[0], one);
  }
#pragma unroll
  for (int x = 0; x < P; ++x) L[x] = FF[x];
  // row P-1, forward part: stages 0..P-2 do F(x, P-1-x); F(P-1, 0) was a piece
#pragma unroll
  for (int x = P - 2; x >= 1; --x) FF[x] = O::ad(O::mx(FF[x - 1], L[x]), wF[x], one);
  if (P >= 2) FF[0] = O::ad(L[0], wF[0], one);
  // fused steps r = P-1..m-2: backward pass of row r + forward pass of row r+1,
  // u32: clamped on the host's schedule `cs` (no-wrap bounds)
  {
    constexpr int U = (P <= 8) ? 8 : 4;
    const V wBF0 = wB[0] + wF[0];
    int rem = m - P;
    if (sizeof(V) == 4 && cs.first() == 0 && !RENORM) clamp_ff<P, V>(FF, S);
    int seg = (sizeof(V) == 4 && cs.first() > 0) ? cs.first() : cs.every();
    if (sizeof(V) != 4) seg = rem;
    if constexpr (P >= 3 && AP_NFORM) {
      if (rem > 0) {
        // (adds outside the max chain go to the FMA pipe: the kernel is ALU-bound)
        V c[P], sw[P], N[P];
        c[0] = wF[0];
#pragma unroll
        for (int x = 1; x < P; ++x) c[x] = fma_add(c[x - 1], wF[x], one);
#pragma unroll
        for (int x = 0; x < P; ++x) sw[x] = fma_add(wF[x], wB[x], one);
        {  // the first step in the M-form, kept as N_x = M_x - c_x
          V M = O::amx(FF[P - 1], wB[P - 1], FF[P - 2]);
          N[P - 2] = M - c[P - 2];
#pragma unroll
          for (int x = P - 3; x >= 0; --x) {
            M = O::amx(M, wB[x + 1], FF[x]);
            N[x] = M - c[x];
          }
        }
        int blk = (rem < seg ? rem : seg) - 1;
        rem -= blk + 1;
        for (;;) {
          for (; blk >= U; blk -= U) {
#pragma unroll
            for (int u = 0; u < U; ++u) nstep<P, V>(N, sw, one);
          }
          // the remaining blk < U rows: one computed jump instead of a counted loop
          switch (blk) {
            case 7: if constexpr (U > 7) nstep<P, V>(N, sw, one); [[fallthrough]];
            case 6: if constexpr (U > 6) nstep<P, V>(N, sw, one); [[fallthrough]];
            case 5: if constexpr (U > 5) nstep<P, V>(N, sw, one); [[fallthrough]];
            case 4: if constexpr (U > 4) nstep<P, V>(N, sw, one); [[fallthrough]];
            case 3: nstep<P, V>(N, sw, one); [[fallthrough]];
            case 2: nstep<P, V>(N, sw, one); [[fallthrough]];
            case 1: nstep<P, V>(N, sw, one); [[fallthrough]];
            default: break;
          }
          if (rem <= 0) break;
          if constexpr (RENORM) fix_state<P, true, P - 1>(N, S, *rn);
          else clamp_n<P, V>(N, S);
          blk = rem < cs.every() ? rem : cs.every();
          rem -= blk;
        }
        // back to finishes (u32: FF = N + c sits up to one row's growth above N, which
        // the host's clamp_final test allows for: last segment + 1 + p rows)
        if (cs.fin()) {
          if constexpr (RENORM) fix_state<P, true, P - 1>(N, S, *rn);
          else clamp_n<P, V>(N, S);
        }
#pragma unroll
        for (int x = 0; x <= P - 2; ++x) FF[x + 1] = fma_add(N[x], c[x + 1], one);
        FF[0] = fma_add(N[0], fma_add(c[0], sw[0], one), one);
      }
      rem = 0;
    }
    while (rem > 0) {
      int blk = rem < seg ? rem : seg;
      rem -= blk;
      for (; blk >= U; blk -= U) {
#pragma unroll
        for (int u = 0; u < U; ++u) mstep<P, V>(FF, wF, wB, wBF0, one);
      }
      for (; blk > 0; --blk) mstep<P, V>(FF, wF, wB, wBF0, one);
      if (rem > 0 || cs.fin()) {
        if constexpr (RENORM) fix_state<P, true, P>(FF, S, *rn);  // M-form: no offsets
        else clamp_ff<P, V>(FF, S);
      }
      seg = cs.every();
    }
    if (m == P && cs.fin() && cs.first() != 0 && !RENORM) clamp_ff<P, V>(FF, S);
  }
  // cool-down, fused the same way: step t = 0..P-1 is the backward pass of row
  // r = m-1+t plus the forward pass of row r+1, which only stages x >= t+1 still
  // do.  Stages x < t did no forward in row r: their backward reads L[x] (their
  // last op) instead of a shared maximum.  M carries max(FF[x], b[x+1]) with
  // b[x+1] = M + wB[x+1] folded into the next fused add+max.
  V b = 0;
  constexpr int TEND = REV ? P - 1 : P;
  // Every backward of the step carries the pending weight of the one above it:
  // b[x+1] = M + wpend, so each op is one fused add+max (VIADDMNMX) on the ALU pipe
  // plus the adds that materialise finishes, which go to the FMA pipe.
#pragma unroll
  for (int t = 0; t < TEND; ++t) {
    if constexpr (P == 1) {
      b = O::ad(FF[0], wB[0], one);
    } else {
      V M = FF[P - 1];
      V wpend = wB[P - 1];  // b[P-1] = M + wpend
#pragma unroll
      for (int x = P - 2; x >= 0; --x) {
        if (x >= t) {
          M = O::amx(M, wpend, FF[x]);  // max(b[x+1], FF[x])
          if (t < P - 1) FF[x + 1] = fma_add(M, wF[x + 1], one);
          if (x == t) L[x] = fma_add(M, wB[x], one);
        } else {
          M = O::amx(M, wpend, L[x]);  // max(b[x+1], L[x]): stage x forwards no more
          L[x] = fma_add(M, wB[x], one);
        }
        wpend = wB[x];
      }
      b = fma_add(M, wpend, one);  // B(0) of the row
    }
  }
  if constexpr (REV) {
#pragma unroll
    for (int x = 0; x < P - 1; ++x) G[x] = L[x];
    G[P - 1] = FF[P - 1];
  }
  return b;
}

// ap_eval_batch T only: the same with renormalisation instead of the clamps (u32);
// T = rn.base + the returned value when rn.exact.
template <int P>
AP_DEV_INLINE uint32_t sim_fast_rn(int m, int k, const uint32_t (&wF)[P], const uint32_t (&wB)[P],
                                   const int (&c)[P + 1], const uint32_t* sPf, const uint32_t* sC,
                                   uint32_t Mk, bool div1, uint32_t S, int CR, uint32_t one,
                                   Renorm& rn) {
  uint32_t FF[P], G[P];
  pieces<P, uint32_t>(k, wF, c, sPf, sC, Mk, div1, one, FF);
  const ClampSched cs{0, CR, 1};
  return sweep_tail<P, uint32_t, false, ClampSched, true>(m, FF, wF, wB, S, cs, one, G, &rn);
}

// Simulate one (candidate, k) for p == P, m >= P.  Returns T (u32: saturated at S).
template <int P, typename V, typename CS>
AP_DEV_INLINE V sim_fast(int m, int k, const V (&wF)[P], const V (&wB)[P], const int (&c)[P + 1],
                         const V* sPf, const V* sC, uint32_t Mk, bool div1, V S,
                         CS cs, uint32_t one) {
  V FF[P], G[P];
  pieces<P, V>(k, wF, c, sPf, sC, Mk, div1, one, FF);
  return sweep_tail<P, V, false>(m, FF, wF, wB, S, cs, one, G);
}

struct SweepArgs {
  DevTables t;
  int p, m, k_lo, k_hi;
  uint64_t rank_lo, rank_hi, chunk;
  uint64_t S;
  int rb;
  unsigned long long* key;
  int clamp_rows;  // u32 path: steady rows between saturating clamps (>= 1)
  int clamp_first; // u32 path: steady rows before the first clamp (0: right after warm-up)
  int clamp_final; // u32 path: clamp at the end of the steady rows
  uint32_t one;    // = 1 (adds are plain operators; kept for the XOps interface)
  int mode;        // 0 full, 1 k-factored, 2 k-factored + lower-bound skipping
  unsigned long long* rec;  // two-phase: per-CTA (T, index) records instead of `key`
  const int64_t* mem;       // memory filter (generic kernel): [2][n+1] prefix sums
  int64_t mem_cap;
  unsigned long long* ctr;  // non-null: warp-dynamic work cursor (zeroed), chunk = ranks/lane/unit
  int div1;                 // u32: all stage computes / comms < 2^28, one-umulhi floor(v/k)
  const SweepDev* dp;       // S and the clamp schedule (k_sweep_prep, stream-ordered)
  int is_u32;               // this launch is the u32 variant
};

// k_sweep_prep: T_ref -> S, u32 choice and clamp schedule, on the device.
// Same arithmetic as the host had: T_ref = min_k T(Alg.-1 partition, k) (or the memory
// mode's fallback), capped by the caller's bound; S = T_ref + 1; with W = wrow the
// growth per row, A0 = floor((2^32-1)/W) rows from 0 and R = floor((2^32-1-S)/W) rows
// from a clamp at S; u32 iff R >= p + 1.
__global__ void k_sweep_prep(PrepArgs a, SweepDev* out) {
  long long tref = a.trefs[0];
  for (int i = 1; i < a.nk; ++i) tref = a.trefs[i] < tref ? a.trefs[i] : tref;
  if (a.mem) {
    // reading R-N4: the Alg.-1 partition must fit, else every candidate stays
    bool fits = true;
    const int n = a.n, p = a.p;
    int lo = 0;
    for (int x = 0; x < p; ++x) {
      const int hi = (x < p - 1) ? a.a1[x] : n;
      const long long inflight = (p - x < a.m) ? p - x : a.m;
      const long long need = (a.mem[hi] - a.mem[lo]) + inflight * (a.mem[n + 1 + hi] - a.mem[n + 1 + lo]);
      fits = fits && need <= a.mem_cap;
      lo = hi;
    }
    if (!fits) tref = a.mem_tot;
  }
  if (a.t_bound < tref) tref = a.t_bound;
  SweepDev d{};
  d.tref = tref;
  d.S = (unsigned long long)tref + 1;
  d.skip = 0;
  if (a.key && (a.rb >= 63 || (unsigned long long)tref >= ((1ull << (63 - a.rb)) - 1))) {
    *a.key = 0x8000000000000000ull;  // AP_KEY_RANGE (INT64_MIN): the packed key does not fit
    d.skip = 1;
  }
  const unsigned long long lim = 0xffffffffull, W = a.wrow;
  const long long a0 = (long long)(lim / W);
  const long long r_allow = (d.S >= lim) ? -1 : (long long)((lim - d.S) / W);
  const int p = a.p, m = a.m;
  int u32 = a.try_u32 && r_allow >= (long long)p + 1;
  int clamp_first = 0, clamp_rows = 1, clamp_final = 1;
  if (u32) {
    auto whole = [](long long r) { return r >= 8 ? (r & ~7ll) : (r >= 4 ? (r & ~3ll) : r); };
    const long long steady = m - p;
    if (steady + 2 * (long long)p <= a0) {
      clamp_first = (int)steady + 1;  // no clamp at all
      clamp_rows = m;
      clamp_final = 0;
    } else {
      long long s1 = a0 - p;
      if (s1 >= 1) s1 = whole(s1 < steady ? s1 : steady);
      else s1 = 0;  // clamp right after the warm-up
      clamp_first = (int)s1;
      const long long L = steady - s1;
      long long every = L < r_allow ? L : r_allow;
      every = every >= 1 ? whole(every) : 1;
      clamp_rows = (int)every;
      if (L == 0) {
        clamp_final = 1;
      } else {
        const long long last = L - every * ((L - 1) / every);
        // + 1: the offset-form sweep converts N back to finishes (FF = N + c) before the
        // p cool-down rows, one more row of growth
        clamp_final = (last + p + 1 > r_allow) ? 1 : 0;
      }
    }
  }
  d.u32 = u32;
  d.clamp_first = clamp_first;
  d.clamp_rows = clamp_rows < 1 ? 1 : clamp_rows;
  d.clamp_final = clamp_final;
  *out = d;
}

cudaError_t launch_sweep_prep(const PrepArgs& a, SweepDev* out, cudaStream_t s) {
  count_launch();
  k_sweep_prep<<<1, 1, 0, s>>>(a, out);
  return cudaGetLastError();
}

AP_DEV_INLINE uint64_t binom_at(const uint64_t* binom, int a, int b) {
  return (a < 0 || b < 0 || b > a) ? 0ull : binom[a * 33 + b];
}

// Block-level min of a u64 key, one atomicMin per CTA.
AP_DEV_INLINE void block_min_atomic(unsigned long long v, unsigned long long* out) {
  __shared__ unsigned long long s_warp[32];
#pragma unroll
  for (int o = 16; o >= 1; o >>= 1) v = min(v, __shfl_xor_sync(0xffffffffu, v, o));
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (lane == 0) s_warp[warp] = v;
  __syncthreads();
  if (warp == 0) {
    const int nw = (blockDim.x + 31) >> 5;
    v = (lane < nw) ? s_warp[lane] : 0x7fffffffffffffffull;
#pragma unroll
    for (int o = 16; o >= 1; o >>= 1) v = min(v, __shfl_xor_sync(0xffffffffu, v, o));
    if (lane == 0 && v != 0x7fffffffffffffffull) atomicMin(out, v);
  }
}

// Two-phase reduction (NEXT N3): the CTA's lexicographic min of (T, index) stored
// as record rec[2*blockIdx.x .. +1]; k_reduce2 then reduces the records.
AP_DEV_INLINE void block_lexmin_store(unsigned long long t, unsigned long long i,
                                      unsigned long long* rec) {
  __shared__ unsigned long long s_t[32], s_i[32];
#pragma unroll
  for (int o = 16; o >= 1; o >>= 1) {
    const unsigned long long ot = __shfl_xor_sync(0xffffffffu, t, o);
    const unsigned long long oi = __shfl_xor_sync(0xffffffffu, i, o);
    if (ot < t || (ot == t && oi < i)) {
      t = ot;
      i = oi;
    }
  }
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (lane == 0) {
    s_t[warp] = t;
    s_i[warp] = i;
  }
  __syncthreads();
  if (warp == 0) {
    const int nw = (blockDim.x + 31) >> 5;
    t = (lane < nw) ? s_t[lane] : 0x7fffffffffffffffull;
    i = (lane < nw) ? s_i[lane] : 0x7fffffffffffffffull;
#pragma unroll
    for (int o = 16; o >= 1; o >>= 1) {
      const unsigned long long ot = __shfl_xor_sync(0xffffffffu, t, o);
      const unsigned long long oi = __shfl_xor_sync(0xffffffffu, i, o);
      if (ot < t || (ot == t && oi < i)) {
        t = ot;
        i = oi;
      }
    }
    if (lane == 0) {
      rec[2 * (size_t)blockIdx.x] = t;
      rec[2 * (size_t)blockIdx.x + 1] = i;
    }
  }
}

// Sweep epilogue: one packed key (T << rb | index) or, two-phase, a (T, index) record.
AP_DEV_INLINE void sweep_result(const SweepArgs& A, bool found, uint64_t T, uint64_t idx) {
  if (A.rec) {
    block_lexmin_store(found ? T : 0x7fffffffffffffffull, found ? idx : 0x7fffffffffffffffull,
                       A.rec);
  } else {
    block_min_atomic(found ? ((T << A.rb) | idx) : 0x7fffffffffffffffull, A.key);
  }
}

// out[0] = min T over the records, out[1] = least index among the records with that T.
__global__ void __launch_bounds__(256) k_reduce2(const unsigned long long* rec, int nrec,
                                                 long long* out) {
  unsigned long long t = 0x7fffffffffffffffull, i = 0x7fffffffffffffffull;
  for (int r = threadIdx.x; r < nrec; r += blockDim.x) {
    const unsigned long long rt = rec[2 * (size_t)r], ri = rec[2 * (size_t)r + 1];
    if (rt < t || (rt == t && ri < i)) {
      t = rt;
      i = ri;
    }
  }
  __shared__ unsigned long long s_t[32], s_i[32];
#pragma unroll
  for (int o = 16; o >= 1; o >>= 1) {
    const unsigned long long ot = __shfl_xor_sync(0xffffffffu, t, o);
    const unsigned long long oi = __shfl_xor_sync(0xffffffffu, i, o);
    if (ot < t || (ot == t && oi < i)) {
      t = ot;
      i = oi;
    }
  }
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (lane == 0) {
    s_t[warp] = t;
    s_i[warp] = i;
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    for (int w = 1; w < (int)(blockDim.x >> 5); ++w)
      if (s_t[w] < t || (s_t[w] == t && s_i[w] < i)) {
        t = s_t[w];
        i = s_i[w];
      }
    out[0] = (long long)t;
    out[1] = (long long)i;
  }
}

// Phase 2 of the multi-GPU two-phase reduction: this GPU's index if its T is T*.
__global__ void k_key2_select(const long long* local, const long long* t_star, long long* idx) {
  *idx = (local[0] == *t_star && local[0] != 0x7fffffffffffffffll) ? local[1]
                                                                    : 0x7fffffffffffffffll;
}

template <int P, typename V, bool FACT>
__device__ __forceinline__ void sweep_range(const SweepArgs& A, uint64_t r0, uint64_t r1, V S,
                                            ClampSched cs, const V* sPf, const V* sPb,
                                            const V* sC, const uint32_t* s_mk, V& bestT,
                                            uint64_t& bestIdx);

// FACT = false: the FULL mode (every (partition, k) pair swept); FACT = true: the
// k-factored and pruned modes.  Separate instances, so the full sweep's register
// allocation does not carry the pruned mode's bound and re-rank code.
template <int P, typename V, bool FACT>
#ifndef AP_SWEEP_MINB
#define AP_SWEEP_MINB (P <= 8 ? 3 : 2)
#endif
__global__ void __launch_bounds__(256, AP_SWEEP_MINB) k_sweep_exact(SweepArgs A) {
  // S and the clamp schedule come from k_sweep_prep; the variant it did not pick (and
  // every launch after a key-packing overflow) returns at once
  const int d_u32 = A.dp->u32, d_skip = A.dp->skip;
  if (d_skip || d_u32 != A.is_u32) return;
  const uint64_t dS = A.dp->S;
  // (held in registers: re-reading it through memory at each use cost 26% on C4,
  // profiles/r02_split_compile.md)
  const ClampSched dcs{A.dp->clamp_first, A.dp->clamp_rows, A.dp->clamp_final};
  extern __shared__ __align__(16) unsigned char smem[];
  size_t used;
  const Tables T = stage_and_scan(A.t.tab, A.t.n, A.t.npad, smem, &used);
  const int n = A.t.n;
  // V-typed copies of the prefix sums / comm (u32 path: exact by the host's bound)
  V* sPf = reinterpret_cast<V*>(smem + used);
  V* sPb = sPf + (n + 1);
  V* sC = sPb + (n + 1);
  __shared__ uint32_t s_mk[kMaxK + 1];  // floor(2^32 / k) (k = 1: 2^32 - 1), see divk
  for (int i = threadIdx.x; i <= n; i += blockDim.x) {
    sPf[i] = (V)T.Pf[i];
    sPb[i] = (V)T.Pb[i];
    if (i < n) sC[i] = (V)T.comm[i];
  }
  if (threadIdx.x <= kMaxK)
    s_mk[threadIdx.x] = (threadIdx.x <= 1) ? 0xffffffffu
                        : A.div1 ? (uint32_t)(((1ull << 32) + threadIdx.x - 1) / threadIdx.x)
                                 : (uint32_t)((1ull << 32) / threadIdx.x);
  __syncthreads();

  const V S = (V)dS;
  V bestT = S;
  uint64_t bestIdx = 0;
  if (A.ctr) {
    // persistent, warp-dynamic: a warp claims unit u = 32 lanes x `chunk` consecutive
    // ranks from the global cursor, so warps the scheduler favoured do not leave the
    // SM under-occupied at the end
    const int lane = threadIdx.x & 31;
    for (;;) {
      unsigned long long u = 0;
      if (lane == 0) u = atomicAdd(A.ctr, 1ull);
      u = __shfl_sync(0xffffffffu, u, 0);
      const uint64_t span = A.rank_hi - A.rank_lo;
      if (u * 32ull >= (span + A.chunk - 1) / A.chunk) break;
      const uint64_t r0 = A.rank_lo + (u * 32ull + (uint64_t)lane) * A.chunk;
      if (r0 < A.rank_hi)
        sweep_range<P, V, FACT>(A, r0, min(r0 + A.chunk, A.rank_hi), S, dcs, sPf, sPb, sC, s_mk, bestT, bestIdx);
    }
  } else {
    const uint64_t tid = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const uint64_t r0 = A.rank_lo + tid * A.chunk;
    if (r0 < A.rank_hi)
      sweep_range<P, V, FACT>(A, r0, min(r0 + A.chunk, A.rank_hi), S, dcs, sPf, sPb, sC, s_mk, bestT, bestIdx);
  }
  sweep_result(A, bestT < S, (uint64_t)bestT, bestIdx);
}

// Ranks [r0, r1) x k of one thread: unrank r0, then lex successors (a2-a7).
template <int P, typename V, bool FACT>
__device__ __forceinline__ void sweep_range(const SweepArgs& A, uint64_t r0, uint64_t r1, V S,
                                            ClampSched cs, const V* sPf, const V* sPb,
                                            const V* sC, const uint32_t* s_mk, V& bestT,
                                            uint64_t& bestIdx) {
  const int n = A.t.n;
  const int m = A.m, k_lo = A.k_lo, k_hi = A.k_hi;
  const uint64_t K = (uint64_t)(k_hi - k_lo + 1);
  {
    // unrank r0 (reading O7 lex order)
    int c[P + 1];
    c[0] = 0;
    c[P] = n;
    {
      uint64_t rr = r0;
      int prev = 0;
#pragma unroll
      for (int x = 1; x <= P - 1; ++x) {
        int v = prev + 1;
        for (;;) {
          const uint64_t cnt = binom_at(A.t.binom, n - 1 - v, P - 1 - x);
          if (rr >= cnt) {
            rr -= cnt;
            ++v;
          } else {
            break;
          }
        }
        c[x] = v;
        prev = v;
      }
    }
    for (uint64_t r = r0; r < r1; ++r) {
#if AP_DEBUG_CHECKS
      AP_CHECK(c[0] == 0 && c[P] == n);
      for (int x = 0; x < P; ++x) AP_CHECK(c[x] < c[x + 1]);
#endif
      // stage weights (a3): compute + receiver-side comm
      V wF[P], wB[P];
#pragma unroll
      for (int x = 0; x < P; ++x) {
        const V Fx = sPf[c[x + 1]] - sPf[c[x]];
        const V Bx = sPb[c[x + 1]] - sPb[c[x]];
        const V Cin = (x > 0) ? sC[c[x] - 1] : V(0);
        const V Cout = (x < P - 1) ? sC[c[x + 1] - 1] : V(0);
        wF[x] = Fx + Cin;
        wB[x] = Bx + Cout;
      }
      const uint64_t base = r * K;
      bool live = true;
      if (FACT && A.mode == 2) {
        // SURVEY O11 lower bound for every k <= k_hi (pinned by the oracle's P6):
        // LB_x = fill_x + m*(F_x+B_x+C_in+C_out) + sum_{i<x}(B_i+C_i), fill_x =
        // sum_{i<x} floor(F_i/K) + sum_{i<x-1} floor(C_i/K).  A partition with LB >= S
        // cannot hold a candidate with T < S = T_ref + 1.
        // (64-bit: m * load can exceed 2^32 for the heavy partitions it prunes)
        const uint32_t Kh = (uint32_t)k_hi, MK = s_mk[k_hi];
        uint64_t fill = 0, tail = 0;
        int xf = P;        // first stage whose bound reaches S
        bool mono = false;  // ... and does so without its comm terms
        uint64_t alast = 0;  // the last stage's bound terms that do not depend on c_{P-1}
#pragma unroll
        for (int x = 0; x < P; ++x) {
          const V Fx = sPf[c[x + 1]] - sPf[c[x]];
          const V Cin = (x > 0) ? sC[c[x] - 1] : V(0);
          if (x == P - 2) alast = fill + (uint64_t)divk(Cin, Kh, MK) + tail;
          uint64_t v = fill + (uint64_t)m * ((uint64_t)wF[x] + (uint64_t)wB[x]) + tail;
          if (x < P - 1) {
            // 1F1B bubble: B(x, 0) waits for micro-batch 0's round trip
            // through the later stages, R = sum_{i>x} (split(F_i,k,k-1) + B_i) >=
            // floor(sum_{i>x} F_i / K) - (P-1-x) + sum_{i>x} B_i (comms dropped, so R
            // depends on c_{x+1} only), while the stage itself has only w_x = P-1-x
            // forwards to run before it: T >= LB_x + max(0, R - w_x * wF_x).
            const V Rf = sPf[n] - sPf[c[x + 1]], Rb = sPb[n] - sPb[c[x + 1]];
            const uint64_t q = (uint64_t)divk(Rf, Kh, MK), w = (uint64_t)(P - 1 - x);
            const uint64_t R = (Kh == 1 ? q : (q > w ? q - w : 0)) + (uint64_t)Rb;
            const uint64_t own = w * (uint64_t)wF[x];
            if (R > own) v += R - own;
          }
          if (v >= (uint64_t)S && xf == P) {
            xf = x;
            const V Bx = sPb[c[x + 1]] - sPb[c[x]];
            mono = fill + (uint64_t)m * ((uint64_t)Fx + (uint64_t)Bx) + tail >= (uint64_t)S;
          }
          fill += (uint64_t)divk(Fx, Kh, MK) + (uint64_t)divk(Cin, Kh, MK);
          tail += (uint64_t)wB[x];
        }
        live = xf == P;
        // (P >= 2: the P = 1 instance never runs this block; its indices are clamped so
        // it does not even name c[-1])
        if (P >= 2 && xf == P - 1) {
          // Only the last stage fails.  Its bound without the comm terms C_{P-2},
          // L(c) = alast + floor((Pf[c]-Pf[c_{P-2}])/K) + Pb[c]-Pb[c_{P-2}]
          //        + m*(Pf[n]-Pf[c] + Pb[n]-Pb[c]),  c = c_{P-1},
          // is <= LB_{P-1} and non-increasing in c (one more sub-layer (f,b) adds at most
          // f + b and removes m*(f+b)), so the failing c form a prefix of [c_{P-2}+1, n-1]:
          // step c_{P-1} past it in shared memory instead of one rank at a time.
          const int cl = c[P >= 2 ? P - 2 : 0];
          auto L = [&](int cc) -> uint64_t {
            return alast + (uint64_t)divk(V(sPf[cc] - sPf[cl]), Kh, MK) + (uint64_t)(sPb[cc] - sPb[cl]) +
                   (uint64_t)m * ((uint64_t)(sPf[n] - sPf[cc]) + (uint64_t)(sPb[n] - sPb[cc]));
          };
          int cc = c[P - 1];
          if (L(cc) >= (uint64_t)S) {
            do ++cc; while (cc <= n - 1 && L(cc) >= (uint64_t)S);
            if (cc <= n - 1) {
              c[P - 1] = cc;
              uint64_t nr = 0;
#pragma unroll
              for (int x = 1; x <= P - 1; ++x)
                nr += binom_at(A.t.binom, n - 1 - c[x - 1], P - x) - binom_at(A.t.binom, n - c[x], P - x);
              r = nr - 1;
              continue;
            }
            // every c_{P-1} left fails: the prefix c_1..c_{P-2} is done
            xf = P - 2;
            mono = true;
          }
        }
        if (!live && (xf < P - 1 || mono)) {
          // LB_xf depends only on the prefix c_1..c_{xf+1}, so every partition with
          // that prefix is pruned too.  If the bound holds on the stage's compute alone
          // (fill and tail depend on c_1..c_xf; F_xf + B_xf grows with c_{xf+1}), every
          // larger c_{xf+1} fails as well, and the prefix c_1..c_xf is done.  Jump to
          // the first lex partition after the pruned block (the lex successor restricted
          // to positions <= j) and re-rank it,
          // rank = sum_x C(n-1-c_{x-1}, P-x) - C(n-c_x, P-x) (hockey-stick form of O7)
          const int j = mono ? xf : xf + 1;
          if (j == 0) break;  // stage 0 fails for this c_1 and every larger one
          int pos = 0;
#pragma unroll
          for (int x = P - 1; x >= 1; --x)
            if (x <= j && pos == 0 && c[x] < n - (P - x)) pos = x;
          if (pos == 0) break;  // no partition left in the whole space
#pragma unroll
          for (int x = 1; x <= P - 1; ++x) {
            if (x == pos) c[x] = c[x] + 1;
            else if (x > pos) c[x] = c[x - 1] + 1;
          }
          uint64_t nr = 0;
#pragma unroll
          for (int x = 1; x <= P - 1; ++x)
            nr += binom_at(A.t.binom, n - 1 - c[x - 1], P - x) - binom_at(A.t.binom, n - c[x], P - x);
          r = nr - 1;  // the loop's ++r lands on it
          continue;
        }
      }
      if (!FACT) {
        for (int k = k_lo; k <= k_hi; ++k) {
          const uint32_t Mk = s_mk[k];
          const V Tc = sim_fast<P, V>(m, k, wF, wB, c, sPf, sC, Mk, A.div1 != 0, S, cs, A.one);
          if (Tc < bestT) {
            bestT = Tc;
            bestIdx = base + (uint64_t)(k - k_lo);
          }
        }
      } else if (live) {  // FACT
        // k-factored: one reversed sweep gives G, then T(k) = max_x FF_x(k) + G_x
        V G[P];
        if constexpr (P >= 2) {
          V rF[P], rB[P], FF0[P];
#pragma unroll
          for (int x = 0; x < P; ++x) {
            rF[x] = wB[x];
            rB[x] = wF[x];
          }
          FF0[0] = rF[0];
#pragma unroll
          for (int x = 1; x < P; ++x) FF0[x] = FF0[x - 1] + rF[x];
          sweep_tail<P, V, true>(m, FF0, rF, rB, S, cs, A.one, G);
        }
        for (int k = k_lo; k <= k_hi; ++k) {
          V Tc;
          if constexpr (P >= 2) {
            V FF[P];
            pieces<P, V>(k, wF, c, sPf, sC, s_mk[k], A.div1 != 0, A.one, FF);
            Tc = FF[0] + G[0];
#pragma unroll
            for (int x = 1; x < P; ++x) {
              const V v = FF[x] + G[x];
              Tc = v > Tc ? v : Tc;
            }
          } else {
            Tc = sim_fast<P, V>(m, k, wF, wB, c, sPf, sC, s_mk[k], A.div1 != 0, S, cs, A.one);
          }
          if (Tc < bestT) {
            bestT = Tc;
            bestIdx = base + (uint64_t)(k - k_lo);
          }
        }
      }
      // lexicographic successor (a2)
      int pos = 0;
#pragma unroll
      for (int x = P - 1; x >= 1; --x)
        if (pos == 0 && c[x] < n - (P - x)) pos = x;
#pragma unroll
      for (int x = 1; x <= P - 1; ++x) {
        if (x == pos) c[x] = c[x] + 1;
        else if (x > pos && pos > 0) c[x] = c[x - 1] + 1;
      }
    }
  }
}

// Generic exhaustive sweep: runtime p <= P, any m, exact int64.
template <int P>
__global__ void __launch_bounds__(128) k_sweep_generic(SweepArgs A) {
  if (A.dp->skip) return;
  const uint64_t dS = A.dp->S;
  extern __shared__ __align__(16) unsigned char smem[];
  size_t used;
  const Tables T = stage_and_scan(A.t.tab, A.t.n, A.t.npad, smem, &used);
  const int n = A.t.n, p = A.p, m = A.m;
  const int64_t* s_mem = nullptr;
  if (A.mem) {
    int64_t* sm = reinterpret_cast<int64_t*>(smem + ((used + 15) & ~size_t(15)));
    for (int i = threadIdx.x; i < 2 * (n + 1); i += blockDim.x) sm[i] = A.mem[i];
    __syncthreads();
    s_mem = sm;
  }
  const uint64_t K = (uint64_t)(A.k_hi - A.k_lo + 1);
  int64_t bestT = (int64_t)dS;
  uint64_t bestIdx = 0;
  const uint64_t tid = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const uint64_t r0 = A.rank_lo + tid * A.chunk;
  if (r0 < A.rank_hi) {
    const uint64_t r1 = min(r0 + A.chunk, A.rank_hi);
    int c[P + 1];
#pragma unroll
    for (int x = 0; x <= P; ++x) c[x] = n;
    c[0] = 0;
    {
      uint64_t rr = r0;
      int prev = 0;
#pragma unroll
      for (int x = 1; x <= P - 1; ++x) {
        if (x <= p - 1) {
          int v = prev + 1;
          for (;;) {
            const uint64_t cnt = binom_at(A.t.binom, n - 1 - v, p - 1 - x);
            if (rr >= cnt) {
              rr -= cnt;
              ++v;
            } else {
              break;
            }
          }
          c[x] = v;
          prev = v;
        }
      }
    }
    BitsRef nob{nullptr, 0};
    TimesRef not_{nullptr, nullptr, nullptr};
    uint32_t pb[P];
    for (uint64_t r = r0; r < r1; ++r) {
      int64_t F[P], B[P], C[P];
      stage_costs<P>(T, p, c, F, B, C);
      bool fits = true;
      if (s_mem) {
        // reading R-N4: static bytes + min(p-x, m) stashed micro-batches per stage
#pragma unroll
        for (int x = 0; x < P; ++x) {
          if (x < p) {
            const int64_t inflight = (p - x < m) ? p - x : m;
            const int64_t need = (s_mem[c[x + 1]] - s_mem[c[x]]) +
                                 inflight * (s_mem[n + 1 + c[x + 1]] - s_mem[n + 1 + c[x]]);
            fits = fits && need <= A.mem_cap;
          }
        }
      }
      for (int k = A.k_lo; fits && k <= A.k_hi; ++k) {
        const int64_t Tc = sim_exact<P, 0>(p, m, k, F, B, C, nob, pb, not_);
        if (Tc < bestT) {
          bestT = Tc;
          bestIdx = r * K + (uint64_t)(k - A.k_lo);
        }
      }
      int pos = 0;
#pragma unroll
      for (int x = P - 1; x >= 1; --x)
        if (x <= p - 1 && pos == 0 && c[x] < n - (p - x)) pos = x;
#pragma unroll
      for (int x = 1; x <= P - 1; ++x) {
        if (x <= p - 1) {
          if (x == pos) c[x] = c[x] + 1;
          else if (x > pos && pos > 0) c[x] = c[x - 1] + 1;
        }
      }
    }
  }
  sweep_result(A, bestT < (int64_t)dS, (uint64_t)bestT, bestIdx);
}

__global__ void k_init_key(unsigned long long* key) { *key = 0x7fffffffffffffffull; }

// ===========================================================================
// K2 eval.
// u32 saturating p-specialised simulation (k = 1, p == P, m >= P) that also writes
// the decision bits the backtrack reads, in exactly the layout of sim_exact (rows
// y + W0 = r; F bit x, B bit 16+x).  It is the M-form sweep of sweep_tail: B(x, y) and
// F(x+1, .) of the next row compare the same pair (FF[x], b[x+1]), so the FP bit is
// FF[x] > b[x+1] and the BP bit its complement (reading Q10's tie rule).  Values are
// clamped to S every CR rows; a result >= S means "recompute exactly" (the caller
// falls back to the int64 sim_exact).  P <= 16 (one bit word per row).
template <int P>
AP_DEV_INLINE uint32_t sim_fast_bits(int m, const uint32_t (&wF)[P], const uint32_t (&wB)[P],
                                     uint32_t S, int CR, BitsRef br) {
  static_assert(P >= 2 && P <= 16, "one bit word per row");
  uint32_t FF[P], L[P];
  FF[0] = wF[0];
#pragma unroll
  for (int x = 1; x < P; ++x) FF[x] = FF[x - 1] + wF[x];
  br.base[0] = 0;
  // warm-up rows r = 1..P-2
#pragma unroll
  for (int r = 1; r <= P - 2; ++r) {
    uint32_t word = 0;
#pragma unroll
    for (int x = r - 1; x >= 1; --x) {
      word |= (FF[x - 1] > FF[x] ? 1u : 0u) << x;
      FF[x] = max(FF[x - 1], FF[x]) + wF[x];
    }
    FF[0] = FF[0] + wF[0];
    br.base[(size_t)r * br.stride] = word;
  }
#pragma unroll
  for (int x = 0; x < P; ++x) L[x] = FF[x];
  uint32_t nxt = 0;  // F bits of the current r-row (its B bits come with the next step)
#pragma unroll
  for (int x = P - 2; x >= 1; --x) {
    nxt |= (FF[x - 1] > L[x] ? 1u : 0u) << x;
    FF[x] = max(FF[x - 1], L[x]) + wF[x];
  }
  FF[0] = L[0] + wF[0];
#pragma unroll
  for (int x = 0; x < P; ++x) FF[x] = min(FF[x], S);
  int r = P - 1;
  int rem = m - P;
#if AP_NFORM
  if constexpr (P >= 3) {
    // offset form with the same decision bits: the first step in the
    // M-form below keeps N = M - c; then per stage t = N'[x+1] + s[x+1],
    // gt_x = N[x-1] > t (i.e. FF[x] > b[x+1]), N'[x] = max(t, N[x-1]), and at x = 0 the
    // intra operand is N[0] + s[0].  Clamps apply to N; the conversion back sits at
    // most one row's growth above S, inside heur_fast_bound's margin.
    if (rem > 0) {
      uint32_t c[P], sw[P], N[P];
      c[0] = wF[0];
#pragma unroll
      for (int x = 1; x < P; ++x) c[x] = c[x - 1] + wF[x];
#pragma unroll
      for (int x = 0; x < P; ++x) sw[x] = wF[x] + wB[x];
      {  // first step, M-form
        uint32_t wordF = 0;
        uint32_t b = FF[P - 1] + wB[P - 1];
#pragma unroll
        for (int x = P - 2; x >= 0; --x) {
          const bool gt = FF[x] > b;
          if (gt) wordF |= 1u << (x + 1);
          const uint32_t M = max(FF[x], b);
          N[x] = M - c[x];
          b = M + wB[x];
        }
        const uint32_t wordB = ((~wordF >> 1) & ((1u << (P - 1)) - 1u)) << 16;
        br.base[(size_t)r * br.stride] = nxt | wordB;
        nxt = wordF;
        ++r;
      }
      int blk = (rem < CR ? rem : CR) - 1;
      rem -= blk + 1;
      for (;;) {
        for (; blk > 0; --blk) {
          uint32_t wordF = 0, n[P];
          uint32_t t = N[P - 2] + sw[P - 1];
          bool gt = N[P - 3 >= 0 ? P - 3 : 0] > t;
          if (P >= 3) {
            if (gt) wordF |= 1u << (P - 1);
            n[P - 2] = max(N[P - 3], t);
          }
#pragma unroll
          for (int x = P - 3; x >= 1; --x) {
            t = n[x + 1] + sw[x + 1];
            gt = N[x - 1] > t;
            if (gt) wordF |= 1u << (x + 1);
            n[x] = max(N[x - 1], t);
          }
          t = n[1] + sw[1];
          const uint32_t u = N[0] + sw[0];
          gt = u > t;
          if (gt) wordF |= 1u << 1;
          n[0] = max(u, t);
#pragma unroll
          for (int x = 0; x <= P - 2; ++x) N[x] = n[x];
          const uint32_t wordB = ((~wordF >> 1) & ((1u << (P - 1)) - 1u)) << 16;
          br.base[(size_t)r * br.stride] = nxt | wordB;
          nxt = wordF;
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
    rem = 0;
  }
#endif
  while (rem > 0) {
    int blk = rem < CR ? rem : CR;
    rem -= blk;
    for (; blk > 0; --blk) {
      // one compare per stage: the F bit x+1 is gt_x, the B bit 16+x its complement,
      // formed once per row from wordF
      uint32_t wordF = 0, nF[P];
      uint32_t b = FF[P - 1] + wB[P - 1];
#pragma unroll
      for (int x = P - 2; x >= 0; --x) {
        const bool gt = FF[x] > b;
        if (gt) wordF |= 1u << (x + 1);
        const uint32_t M = max(FF[x], b);
        nF[x + 1] = M + wF[x + 1];
        b = M + wB[x];
      }
      nF[0] = b + wF[0];
      const uint32_t wordB = ((~wordF >> 1) & ((1u << (P - 1)) - 1u)) << 16;
      br.base[(size_t)r * br.stride] = nxt | wordB;
      nxt = wordF;
      ++r;
#pragma unroll
      for (int x = 0; x < P; ++x) FF[x] = nF[x];
    }
#pragma unroll
    for (int x = 0; x < P; ++x) FF[x] = min(FF[x], S);
  }
  // cool-down t = 0..P-1: B of r-row m-1+t, F of the next row for x >= t+1
  uint32_t b = 0;
#pragma unroll
  for (int t = 0; t < P; ++t) {
    uint32_t wordB = 0, wordF = 0;
    b = FF[P - 1] + wB[P - 1];
#pragma unroll
    for (int x = P - 2; x >= 0; --x) {
      if (x >= t) {
        const bool gt = FF[x] > b;
        wordB |= (gt ? 0u : 1u) << (x + 16);
        const uint32_t M = gt ? FF[x] : b;
        if (t < P - 1) {
          wordF |= (gt ? 1u : 0u) << (x + 1);
          FF[x + 1] = M + wF[x + 1];
        }
        b = M + wB[x];
        if (x == t) L[x] = b;
      } else {
        wordB |= (b >= L[x] ? 1u : 0u) << (x + 16);
        b = max(b, L[x]) + wB[x];
        L[x] = b;
      }
    }
    br.base[(size_t)r * br.stride] = nxt | wordB;
    nxt = wordF;
    ++r;
  }
  return b;
}

// backtrack_master (ap_device.cuh) specialised to the fast path (p == P, k == 1,
// m >= P, so w_x = P-1-x, W0 = P-1; m <= 32767) and written without divergent
// branches: each op's move is computed with selects, so the lanes of a warp only part
// at the loop exit (C5 pool kernel 1.68 -> 1.19 ms).  Same walk and reading (O5 tie rule, O6 master; the 1F1B phase of stage x is
// rows [P-1, m-1+x] for both F and B).  Per-stage counts are CB-bit fields of NW
// registers (CB = 8 needs 2m <= 255), flushed when the path changes stage.
template <int P, int CB>
AP_DEV_INLINE int backtrack_master_bl(int m, BitsRef br) {
  constexpr int PER = 32 / CB;
  constexpr int NW = (P + PER - 1) / PER;
  uint32_t cw[NW];
#pragma unroll
  for (int w = 0; w < NW; ++w) cw[w] = 0;
  int x = 0, row = m + P - 2;  // the sink B(0, m-1)
  bool onB = true;
  uint32_t run = 0;
  for (;;) {
    const uint32_t word = br.base[(size_t)row * br.stride];
    run += (row >= P - 1 && row <= m - 1 + x) ? 1u : 0u;
    if (!onB && row == 0) break;  // the source F(0, 0)
    const bool cB = onB && x < P - 1 && ((word >> (x + 16)) & 1u);
    const bool cF = !onB && x > 0 && (row == x || ((word >> x) & 1u));
    if (cB || cF) {
      const uint32_t inc = run << (CB * (x % PER));
#pragma unroll
      for (int w = 0; w < NW; ++w) cw[w] += (w == x / PER) ? inc : 0u;
      run = 0;
    }
    const bool Fhere = row <= m - 1 + x;  // F(x) exists in this row
    const int r0 = row;
    row = onB ? ((cB || Fhere) ? r0 : r0 - 1) : r0 - 1;
    const bool nB = onB ? (cB || !Fhere) : (!cF && r0 > P - 1);
    x += (cB ? 1 : 0) - (cF ? 1 : 0);
    onB = nB;
  }
  {
    const uint32_t inc = run << (CB * (x % PER));
#pragma unroll
    for (int w = 0; w < NW; ++w) cw[w] += (w == x / PER) ? inc : 0u;
  }
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

struct EvalArgs {
  DevTables t;
  int p, m;
  const int32_t* cuts;
  int cuts_stride;
  const int32_t* kptr;
  int k_const, k_iota;
  int64_t count;
  int64_t* time_ns;
  int32_t* master;
  uint32_t* gbits;  // global bit scratch when shared memory is too small (or null)
  int s_const;      // sliced leading micro-batches (1 = micro-batch 0 only, the default)
  int s_iota;       // 1: row i uses s = i (paper-form slice sweep), k = k_const
  uint32_t fastS;   // > 0: u32 fast path (p == P <= 16, m >= P, s = 1) exact below fastS,
                    // clamped every CR rows; a result >= fastS is recomputed in int64
  int CR, div1;     // clamp interval; one-umulhi pieces (see divk)
  // fast pass: a candidate whose u32 result reaches fastS is appended to redo (count at
  // redo[0], indices at redo[1..]) instead of diverging its warp into the int64 path;
  // redo pass (fastS = 0, redo_in set): evaluates exactly the listed candidates
  unsigned int* redo;
  const unsigned int* redo_in;
  uint32_t one;     // = 1, opaque to the compiler (keeps the adds on IMAD)
  unsigned long long* n_invalid;  // optional: + 1 per invalid row (zeroed by launch_eval)
};
// u32 copies of the prefix sums Pf, Pb, the comm and the floor(v/k) magics (fast path)
__host__ __device__ inline size_t eval_fast_smem(int n) {
  return ((size_t)(3 * n + 2 + kMaxK + 1) * 4 + 15) & ~size_t(15);
}

template <int P>
AP_DEV_INLINE bool load_cuts(const int32_t* row, int p, int n, int (&c)[P + 1]) {
  bool ok = true;
#pragma unroll
  for (int x = 0; x <= P; ++x) c[x] = n;
  c[0] = 0;
  int prev = 0;
#pragma unroll
  for (int x = 1; x <= P - 1; ++x) {
    if (x <= p - 1) {
      const int v = row[x - 1];
      ok = ok && (v > prev) && (v <= n - 1);
      c[x] = v;
      prev = v;
    }
  }
  return ok;
}

// SLICED = true: the paper's Slicer form (s != 1 leading micro-batches sliced, T only),
// in a kernel of its own so its per-piece arrays do not weigh on the common one.
template <int P, bool SLICED>
__global__ void __launch_bounds__(128) k_eval(EvalArgs A) {
  // the generic exact int64 evaluation (any p <= P, m, k, s); with A.redo_in set it
  // evaluates exactly the candidates k_eval_fast listed (usually none: return at once)
  if (A.redo_in && A.redo_in[0] == 0u) return;
  extern __shared__ __align__(16) unsigned char smem[];
  size_t used;
  const Tables T = stage_and_scan(A.t.tab, A.t.n, A.t.npad, smem, &used);
  const size_t off = (used + 15) & ~size_t(15);
  const int p = A.p, m = A.m, n = A.t.n;
  // grid-stride (persistent) loop: the table prologue above runs once per CTA
  const int64_t cnt = A.redo_in ? (int64_t)A.redo_in[0] : A.count;
  for (int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; j < cnt;
       j += (int64_t)gridDim.x * blockDim.x) {
    const int64_t i = A.redo_in ? (int64_t)A.redo_in[1 + j] : j;

    int c[P + 1];
    const bool okc = load_cuts<P>(A.cuts + (size_t)i * A.cuts_stride, p, n, c);
    const int k = A.kptr ? A.kptr[i] : (A.k_iota ? (int)(i + 1) : A.k_const);
    const int sl = A.s_iota ? (int)i : A.s_const;
    if (!okc || k < 1 || k > kMaxK || sl < 0 || sl > A.m) {
      A.time_ns[i] = -1;
      if (A.master) A.master[i] = -1;
      if (A.n_invalid) atomicAdd(A.n_invalid, 1ull);
      continue;
    }
    int64_t F[P], B[P], C[P];
    stage_costs<P>(T, p, c, F, B, C);
    if constexpr (SLICED) {  // paper Slicer form: T only
      A.time_ns[i] = sim_sliced<P>(p, m, sl, k, F, B, C);
      if (A.master) A.master[i] = -1;
      continue;
    }
    uint32_t pb[P];
    TimesRef not_{nullptr, nullptr, nullptr};
    if (A.master == nullptr) {
      BitsRef nob{nullptr, 0};
      A.time_ns[i] = sim_exact<P, 0>(p, m, k, F, B, C, nob, pb, not_);
      continue;
    }
    BitsRef br{nullptr, 0};
    if (A.gbits) {
      br.base = A.gbits + i;
      br.stride = (int)A.count;
    } else {
      uint32_t* sbits = reinterpret_cast<uint32_t*>(smem + off);
      br.base = sbits + threadIdx.x;
      br.stride = blockDim.x;
    }
    A.time_ns[i] = sim_exact<P, 1>(p, m, k, F, B, C, br, pb, not_);
    int len;
    A.master[i] = backtrack_master<P>(p, m, k, br, pb, &len, NoEmit{});
  }
}

// K2 fast path (p == P <= 16, m >= P, micro-batch 0 sliced, u32 exact below fastS):
// T for any k with the N-form sweep (sim_fast), T + master for k = 1, m <= 127 with
// the recorded decision words and the run-length backtrack (ap_master.cuh).  Every
// candidate it cannot finish exactly -- saturated at fastS, or T + master with k > 1
// or m > 127 -- goes to A.redo for the generic k_eval.  A kernel of its own, so its
// register allocation is not the generic path's.
// MASTER: T + master (A.master != nullptr) and T only are separate instances, so the
// register allocation of one does not move with changes to the other.
template <int P, bool MASTER>
__global__ void __launch_bounds__(128) k_eval_fast(EvalArgs A) {
  extern __shared__ __align__(16) unsigned char smem[];
  size_t used;
  const Tables T = stage_and_scan(A.t.tab, A.t.n, A.t.npad, smem, &used);
  size_t off = (used + 15) & ~size_t(15);
  const int m = A.m, n = A.t.n;
  uint32_t* s32Pf = reinterpret_cast<uint32_t*>(smem + off);
  uint32_t* s32Pb = s32Pf + (n + 1);
  uint32_t* s32C = s32Pb + (n + 1);
  uint32_t* s32mk = s32C + n;
  for (int e = threadIdx.x; e <= n; e += blockDim.x) {
    s32Pf[e] = (uint32_t)T.Pf[e];
    s32Pb[e] = (uint32_t)T.Pb[e];
    if (e < n) s32C[e] = (uint32_t)T.comm[e];
  }
  if (threadIdx.x <= kMaxK)
    s32mk[threadIdx.x] = (threadIdx.x <= 1) ? 0xffffffffu
                         : A.div1 ? (uint32_t)(((1ull << 32) + threadIdx.x - 1) / threadIdx.x)
                                  : (uint32_t)((1ull << 32) / threadIdx.x);
  off += eval_fast_smem(n);
  __syncthreads();
  off = (off + 15) & ~size_t(15);
  uint32_t* s_cw = reinterpret_cast<uint32_t*>(smem + off);
  const MasterBits br{s_cw + threadIdx.x,
                      reinterpret_cast<uint16_t*>(s_cw + (size_t)master_col_words(m, P) * blockDim.x) +
                          threadIdx.x,
                      (int)blockDim.x};
  const uint32_t S = A.fastS, one = A.one;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < A.count;
       i += (int64_t)gridDim.x * blockDim.x) {
    int c[P + 1];
    const bool okc = load_cuts<P>(A.cuts + (size_t)i * A.cuts_stride, P, n, c);
    const int k = A.kptr ? A.kptr[i] : (A.k_iota ? (int)(i + 1) : A.k_const);
    if (!okc || k < 1 || k > kMaxK) {
      A.time_ns[i] = -1;
      if (A.master) A.master[i] = -1;
      if (A.n_invalid) atomicAdd(A.n_invalid, 1ull);
      continue;
    }
    uint32_t wF[P], wB[P];
#pragma unroll
    for (int x = 0; x < P; ++x) {
      wF[x] = (s32Pf[c[x + 1]] - s32Pf[c[x]]) + ((x > 0) ? s32C[c[x] - 1] : 0u);
      wB[x] = (s32Pb[c[x + 1]] - s32Pb[c[x]]) + ((x < P - 1) ? s32C[c[x + 1] - 1] : 0u);
    }
    bool done = false;
    if constexpr (!MASTER) {
#if AP_EVAL_RENORM
      Renorm rn;
      const uint32_t t32 = sim_fast_rn<P>(m, k, wF, wB, c, s32Pf, s32C, s32mk[k], A.div1 != 0, S,
                                          A.CR, one, rn);
      if (rn.exact) {
        A.time_ns[i] = (int64_t)(rn.base + t32);
        done = true;
      }
#else
      const ClampSched cs{0, A.CR, 1};
      const uint32_t t32 = sim_fast<P, uint32_t>(m, k, wF, wB, c, s32Pf, s32C, s32mk[k],
                                                 A.div1 != 0, S, cs, one);
      if (t32 < S) {
        A.time_ns[i] = (int64_t)t32;
        done = true;
      }
#endif
    } else if (k == 1 && m <= 127) {
      // renormalised instead of clamped (Renorm, ap_master.cuh): exact for every
      // candidate whose state spread stays below S, however large T is, so the
      // saturated ones need no generic int64 pass
      (void)c;
      Renorm rn;
      const uint32_t t32 = sim_master<P, true>(m, wF, wB, S, A.CR, br, one, &rn);
      if (rn.exact) {
        A.time_ns[i] = (int64_t)(rn.base + t32);
        A.master[i] = backtrack_master<P, 8>(m, br);
        done = true;
      }
    }
    if (!done) A.redo[1 + atomicAdd(&A.redo[0], 1u)] = (unsigned int)i;
  }
}

// Exact pass over the candidates k_eval_fast listed as saturated (T >= its u32 bound),
// T only, p == P, m >= P, s = 1: the same offset-form sweep in 64-bit (sim_fast<P, u64>,
// the sweep kernels' exact variant) instead of the generic event-order kernel.  The list
// is short (C4 random partitions: ~2 %), so the pass is one simulation per thread and
// its length is one simulation's latency: C4 2^22 candidates, 98 us with the generic
// kernel (profiles/r02_eval_redo.md).
static cudaError_t set_smem(const void* fn, size_t bytes);
int num_sms(int device);

template <int P>
__global__ void __launch_bounds__(128) k_eval_redo64(EvalArgs A) {
  if (A.redo_in[0] == 0u) return;
  extern __shared__ __align__(16) unsigned char smem[];
  size_t used;
  const Tables T = stage_and_scan(A.t.tab, A.t.n, A.t.npad, smem, &used);
  const int n = A.t.n, m = A.m;
  const uint64_t* sPf = reinterpret_cast<const uint64_t*>(T.Pf);
  const uint64_t* sPb = reinterpret_cast<const uint64_t*>(T.Pb);
  const uint64_t* sC = reinterpret_cast<const uint64_t*>(T.comm);
  const int64_t cnt = (int64_t)A.redo_in[0];
  const ClampSched cs{0, 1, 0};  // ignored by the 64-bit sweep
  for (int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; j < cnt;
       j += (int64_t)gridDim.x * blockDim.x) {
    const int64_t i = (int64_t)A.redo_in[1 + j];
    int c[P + 1];
    load_cuts<P>(A.cuts + (size_t)i * A.cuts_stride, P, n, c);  // valid: checked by the fast pass
    const int k = A.kptr ? A.kptr[i] : (A.k_iota ? (int)(i + 1) : A.k_const);
    uint64_t wF[P], wB[P];
#pragma unroll
    for (int x = 0; x < P; ++x) {
      wF[x] = (sPf[c[x + 1]] - sPf[c[x]]) + ((x > 0) ? sC[c[x] - 1] : 0ull);
      wB[x] = (sPb[c[x + 1]] - sPb[c[x]]) + ((x < P - 1) ? sC[c[x + 1] - 1] : 0ull);
    }
    A.time_ns[i] = (int64_t)sim_fast<P, uint64_t>(m, k, wF, wB, c, sPf, sC, 0u, false, 0ull, cs, 1u);
  }
}

template <int P>
static cudaError_t eval_redo64_P(const EvalArgs& A, cudaStream_t s, int* launches) {
  const int threads = 128;
  const size_t smem = (tables_smem_bytes(A.t.npad, A.t.n) + 15) & ~size_t(15);
  cudaError_t e = set_smem((const void*)k_eval_redo64<P>, smem);
  if (e != cudaSuccess) return e;
  int occ = 0, dev = 0;
  cudaGetDevice(&dev);
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_eval_redo64<P>, threads, smem);
  if (e != cudaSuccess) return e;
  occ = occ < 1 ? 1 : occ;
  int64_t blocks = (A.count + threads - 1) / threads;
  const int64_t wave = (int64_t)num_sms(dev) * occ;
  if (blocks > wave) blocks = wave;
  if (blocks > 0) {
    count_launch();
    k_eval_redo64<P><<<(unsigned)blocks, threads, smem, s>>>(A);
    if (launches) ++*launches;
  }
  return cudaGetLastError();
}

// ===========================================================================
// Algorithm 1, one CTA.  time[0][0] = 0, others +inf;
// time[i][j] = min_k max(time[k][j-1], P[i]-P[k]) over k ascending, strict '<'
// (smallest k wins ties); the arg table drives line 15's reconstruction.
__global__ void __launch_bounds__(1024) k_alg1(DevTables t, int p, int16_t* arg, int32_t* cuts,
                                               int64_t* value) {
  extern __shared__ __align__(16) unsigned char smem[];
  size_t used;
  const Tables T = stage_and_scan(t.tab, t.n, t.npad, smem, &used);
  const int n = t.n, P1 = p + 1;
  int64_t* tt = reinterpret_cast<int64_t*>(smem + ((used + 15) & ~size_t(15)));
  // prefix_sum of f+b (line 6): Pf + Pb
  for (int e = threadIdx.x; e < (n + 1) * P1; e += blockDim.x) {
    tt[e] = (e == 0) ? 0 : INT64_MAX;
    arg[e] = -1;
  }
  __syncthreads();
  // time[i][j] reads only column j-1, so the columns go one after another and every i of
  // a column in parallel (a warp per i, lanes over k): p dependent steps instead of n.
  // Same values and the same argmin as the paper's i-outer loop (smallest k on ties).
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, nw = blockDim.x >> 5;
  for (int j = 1; j <= p; ++j) {
    for (int i = j + warp; i <= n; i += nw) {
      const int64_t Pi = T.Pf[i] + T.Pb[i];
      int64_t bv = INT64_MAX;
      int bk = INT32_MAX;
      for (int kk = j - 1 + lane; kk <= i - 1; kk += 32) {
        const int64_t prev = tt[kk * P1 + (j - 1)];
        const int64_t seg = Pi - (T.Pf[kk] + T.Pb[kk]);
        const int64_t v = prev > seg ? prev : seg;
        if (v < bv) {  // kk ascending within the lane: first wins
          bv = v;
          bk = kk;
        }
      }
#pragma unroll
      for (int o = 16; o >= 1; o >>= 1) {
        const int64_t ov = __shfl_xor_sync(0xffffffffu, bv, o);
        const int ok = __shfl_xor_sync(0xffffffffu, bk, o);
        if (ov < bv || (ov == bv && ok < bk)) {
          bv = ov;
          bk = ok;
        }
      }
      if (lane == 0 && bv != INT64_MAX) {
        tt[i * P1 + j] = bv;
        arg[i * P1 + j] = (int16_t)bk;
      }
    }
    __syncthreads();
  }
  if (threadIdx.x == 0) {
    *value = tt[n * P1 + p];
    int e = n;
    for (int jj = p; jj >= 2; --jj) {
      const int st = arg[e * P1 + jj];
      cuts[jj - 2] = st;
      e = st;
    }
  }
}

// ===========================================================================
// Certified minLB (reading R-LB), one CTA.  Per-stage
// relaxation of the O11 bound, g(x, a, b) for stage x = [a, b):
//   ceil+((Pf[a] - x(K-1)) / K) + (x-1) floor(cmin/K)              (fill)
//   + m (F + B + [x>0] comm[a-1] + [x<p-1] comm[b-1])              (busy)
//   + Pb[a] + [x>0] (comm[a-1] + (x-1) cmin)                       (tail)
// bottleneck DP D[x+1][b] = min_a max(D[x][a], g), a ascending, strict '<'.
AP_DEV_INLINE int64_t minlb_term(const Tables& T, int p, int m, int K, int64_t cmin, int x,
                                 int a, int b) {
  int64_t fill = T.Pf[a] - (int64_t)x * (K - 1);
  fill = fill <= 0 ? 0 : (fill + K - 1) / K;
  const int64_t cin = x > 0 ? T.comm[a - 1] : 0;
  const int64_t cout = x < p - 1 ? T.comm[b - 1] : 0;
  if (x > 0) fill += (int64_t)(x - 1) * (cmin / K);
  const int64_t busy = (int64_t)m * (T.Pf[b] - T.Pf[a] + T.Pb[b] - T.Pb[a] + cin + cout);
  const int64_t tail = T.Pb[a] + (x > 0 ? cin + (int64_t)(x - 1) * cmin : 0);
  return fill + busy + tail;
}

__global__ void __launch_bounds__(256) k_minlb(DevTables t, int p, int m, int K, int16_t* arg,
                                               int32_t* cuts, int64_t* value) {
  extern __shared__ __align__(16) unsigned char smem[];
  size_t used;
  const Tables T = stage_and_scan(t.tab, t.n, t.npad, smem, &used);
  const int n = t.n, N1 = n + 1;
  int64_t* D = reinterpret_cast<int64_t*>(smem + ((used + 15) & ~size_t(15)));
  __shared__ int64_t s_cmin;
  for (int e = threadIdx.x; e < (p + 1) * N1; e += blockDim.x) {
    D[e] = (e == 0) ? 0 : INT64_MAX;
    arg[e] = -1;
  }
  if (threadIdx.x == 0) {
    int64_t c = 0;
    for (int i = 0; i + 1 < n; ++i) c = (i == 0 || T.comm[i] < c) ? T.comm[i] : c;
    s_cmin = c;
  }
  __syncthreads();
  const int64_t cmin = s_cmin;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, nw = blockDim.x >> 5;
  for (int x = 0; x < p; ++x) {
    const int b_lo = (x == p - 1) ? n : x + 1, b_hi = n - (p - 1 - x);
    for (int b = b_lo + warp; b <= b_hi; b += nw) {
      int64_t bv = INT64_MAX;
      int ba = INT32_MAX;
      for (int a = x + lane; a < b; a += 32) {
        const int64_t prev = D[x * N1 + a];
        if (prev == INT64_MAX) continue;
        const int64_t g = minlb_term(T, p, m, K, cmin, x, a, b);
        const int64_t v = prev > g ? prev : g;
        if (v < bv) {  // a ascending within the lane: first wins
          bv = v;
          ba = a;
        }
      }
#pragma unroll
      for (int o = 16; o >= 1; o >>= 1) {
        const int64_t ov = __shfl_xor_sync(0xffffffffu, bv, o);
        const int oa = __shfl_xor_sync(0xffffffffu, ba, o);
        if (ov < bv || (ov == bv && oa < ba)) {
          bv = ov;
          ba = oa;
        }
      }
      if (lane == 0 && bv != INT64_MAX) {
        D[(x + 1) * N1 + b] = bv;
        arg[(x + 1) * N1 + b] = (int16_t)ba;
      }
    }
    __syncthreads();
  }
  if (threadIdx.x == 0) {
    *value = D[p * N1 + n];
    int e = n;
    for (int x = p; x >= 2; --x) {
      e = arg[x * N1 + e];
      cuts[x - 2] = e;
    }
  }
}

// ===========================================================================
// K3 heuristic restarts (adjust_mode none; reading O9).  The u32
// simulation with decision bits (sim_fast_bits) and the branch-free master backtrack
// (backtrack_master_bl) are defined above, next to K2, which shares them.
struct HeurArgs {
  DevTables t;
  int p, m;
  uint64_t seed;
  int radius;
  uint32_t r_lo, r_hi;
  const int16_t* arg;
  const int32_t* alg1;
  unsigned int* counter;
  unsigned long long* key;
  int32_t* replay;
  unsigned long long* sims;  // optional: total simulations run (atomicAdd per warp)
  int16_t* best_out;         // optional: [r - r_lo][p-1] best cut vector of each restart
  uint32_t S;                // fast path: u32 saturation bound (see sim_fast_bits)
  int CR;                    // fast path: rows between clamps
  unsigned int* redo;        // FAST: [0] = count, [1..] restarts abandoned on saturation;
                             // generic: if non-null, run exactly the listed restarts
  int adjust_mode;           // 0 none, 1 Eq. (1) step 2
};

// Algorithm 1 on the prefix [0, c) with j stages: writes c_1..c_{j-1} (line 15).
AP_DEV_INLINE void alg1_prefix(const int16_t* s_arg, int P1, int c, int j, int* cut) {
  int e = c;
  for (int jj = j; jj >= 2; --jj) {
    const int st = s_arg[e * P1 + jj];
    cut[jj - 1] = st;
    e = st;
  }
}

// FAST = true: u32 sim_fast_bits only (p == P, m >= P); a restart whose simulation
// saturates is abandoned and its id appended to A.redo.  FAST = false: the exact int64
// sim_exact (runtime p <= P), over [r_lo, r_hi) or over the ids listed in A.redo.
template <int P, bool FAST>
__global__ void __launch_bounds__(128) k_heur(HeurArgs A) {
  // the exact redo pass over the restarts the u32 pass abandoned (usually none)
  if (!FAST && A.redo && A.redo[0] == 0u) return;
  extern __shared__ __align__(16) unsigned char smem[];
  size_t used;
  const Tables T = stage_and_scan(A.t.tab, A.t.n, A.t.npad, smem, &used);
  const int n = A.t.n, p = A.p, m = A.m, P1 = p + 1;
  int16_t* s_arg = reinterpret_cast<int16_t*>(smem + ((used + 15) & ~size_t(15)));
  const int narg = (n + 1) * P1;
  int32_t* s_a1 = reinterpret_cast<int32_t*>(s_arg + ((narg + 7) & ~7));
  uint32_t* s_bits = reinterpret_cast<uint32_t*>(s_a1 + 32);
  for (int e = threadIdx.x; e < narg; e += blockDim.x) s_arg[e] = A.arg[e];
  for (int e = threadIdx.x; e < p - 1; e += blockDim.x) s_a1[e] = A.alg1[e];
  __syncthreads();
  BitsRef br{s_bits + threadIdx.x, (int)blockDim.x};
  TimesRef not_{nullptr, nullptr, nullptr};

  int cur[P + 1] = {0}, cand[P + 1] = {0}, best[P + 1] = {0}, sel[P + 1] = {0};
  unsigned long long lane_key = 0x7fffffffffffffffull;
  unsigned int nsims = 0;
  const int smax = n * p;
  int phase = 0;  // 0 need restart, 1 start evaluated next, 2 child evaluated next
  uint32_t r = 0;
  int64_t bestT = 0, selT = 0;
  int curM = 0, selM = 0, steps = 0, chIdx = 0;

  // child generator: idx 0 a, 1 a', 2 b, 3 b' (reading Q17)
  auto gen_child = [&](int idx, int i) -> bool {
    const int size_i = cur[i + 1] - cur[i];
    if (size_i < 2) return false;
#pragma unroll
    for (int x = 0; x <= P; ++x) cand[x] = cur[x];
    if (idx <= 1) {
      cand[i] += 1;  // first block of stage i -> stage i-1
      if (idx == 0) return true;
      if (i - 1 < 1) return false;
      alg1_prefix(s_arg, P1, cand[i - 1], i - 1, cand);
      bool diff = false;
      for (int x = 1; x < i - 1; ++x) diff = diff || (cand[x] != cur[x]);
      return diff;
    }
    if (i > p - 2) return false;
    cand[i + 1] -= 1;  // last block of stage i -> stage i+1
    if (idx == 2) return true;
    alg1_prefix(s_arg, P1, cand[i], i, cand);
    bool diff = false;
    for (int x = 1; x < i; ++x) diff = diff || (cand[x] != cur[x]);
    return diff;
  };

  // ---- paper step 2 (adjust_mode 1): Eq. (1), reading Q19/Q20, DESIGN.md §2
  int adj_i = 0, adj_s = 0, nring = 0;
  uint64_t ring[32];
  // first s >= adj_s (<= p-2) where Eq. (1) is violated for master adj_i and stage s
  // still has >= 2 blocks; on success cand = cur with stage s's last block moved to s+1
  auto adj_find = [&]() -> bool {
    for (; adj_s <= p - 2; ++adj_s) {
      const int i = adj_i;
      const int64_t lhs = (T.Pf[cur[adj_s + 1]] + T.Pb[cur[adj_s + 1]]) -
                          (T.Pf[cur[i + 1]] + T.Pb[cur[i + 1]]);
      const int64_t Bi = T.Pb[cur[i + 1]] - T.Pb[cur[i]];
      if (lhs > (int64_t)(adj_s - i) * Bi && cur[adj_s + 1] - cur[adj_s] >= 2) {
#pragma unroll
        for (int x = 0; x <= P; ++x) cand[x] = cur[x];
        cand[adj_s + 1] -= 1;
        phase = 3;
        return true;
      }
    }
    return false;
  };
  auto start_children = [&]() -> bool {
    ++steps;
    selT = INT64_MAX;
    for (int idx = 0; idx <= 3; ++idx)
      if (gen_child(idx, curM)) {
        chIdx = idx;
        phase = 2;
        return true;
      }
    return false;
  };
  // after the adjustment: stop on a repeated scheme (mode 1), stop at master 0,
  // otherwise generate the children of step 3
  auto post_adjust = [&]() -> bool {
    if (A.adjust_mode == 1) {
      uint64_t h = 0;
      for (int x = 1; x <= p - 1; ++x) h = splitmix64(h ^ (uint64_t)(uint32_t)cur[x]);
      bool seen = false;
      for (int q = 0; q < nring && q < 32; ++q) seen = seen || (ring[q] == h);
      if (seen) return false;
      ring[nring % 32] = h;
      ++nring;
    }
    if (curM == 0) return false;
    return start_children();
  };
  // top of a walk step: the step cap, then (mode 1) the Eq. (1) adjustment
  auto begin_step = [&]() -> bool {
    if (steps >= smax) return false;
    if (A.adjust_mode == 1 && p >= 3) {
      adj_i = curM;
      adj_s = curM + 1;
      if (adj_find()) return true;
    }
    return post_adjust();
  };

  unsigned int rsims = 0;  // simulations of the current restart
  for (;;) {
    if (phase == 0) {
      if (!FAST && A.redo) {
        const unsigned int i = atomicAdd(A.counter, 1u);
        if (i >= A.redo[0]) break;
        r = A.redo[1 + i];
      } else {
        r = atomicAdd(A.counter, 1u) + A.r_lo;
        if (r >= A.r_hi) break;
      }
      rsims = 0;
      // restart start: Alg. 1 (r = 0) or the seeded perturbation (reading Q21)
      cand[0] = 0;
#pragma unroll
      for (int x = 1; x <= P; ++x) cand[x] = n;
      int prev = 0;
      for (int x = 1; x <= p - 1; ++x) {
        int64_t v = s_a1[x - 1];
        if (r != 0) {
          const uint64_t u = splitmix64(A.seed ^ ((uint64_t)r << 32) ^ (uint64_t)x);
          v += (int64_t)(u % (uint64_t)(2 * A.radius + 1)) - A.radius;
          v = v < prev + 1 ? prev + 1 : v;
          v = v > n - (p - x) ? n - (p - x) : v;
        }
        cand[x] = (int)v;
        prev = (int)v;
      }
      phase = 1;
    }
    // ---- simulate cand (k = 1) with its master stage
    int cc[P + 1];
#pragma unroll
    for (int x = 0; x <= P; ++x) cc[x] = cand[x];
    int64_t F[P], B[P], C[P];
    stage_costs<P>(T, p, cc, F, B, C);
    uint32_t pb[P];
#pragma unroll
    for (int x = 0; x < P; ++x) pb[x] = 0;
    int64_t Tc;
    if constexpr (FAST) {
      uint32_t wF[P], wB[P];
#pragma unroll
      for (int x = 0; x < P; ++x) {
        wF[x] = (uint32_t)(F[x] + ((x > 0) ? C[x - 1] : 0));
        wB[x] = (uint32_t)(B[x] + C[x]);
      }
      const uint32_t t32 = sim_fast_bits<P>(m, wF, wB, A.S, A.CR, br);
      if (t32 >= A.S) {  // not exact: hand the whole restart to the int64 pass
        const unsigned int slot = atomicAdd(&A.redo[0], 1u);
        A.redo[1 + slot] = r;
        phase = 0;
        continue;
      }
      Tc = (int64_t)t32;
    } else {
      Tc = sim_exact<P, 1>(p, m, 1, F, B, C, br, pb, not_);
    }
    int Mc;
    if constexpr (FAST) {
      Mc = m <= 127 ? backtrack_master_bl<P, 8>(m, br) : backtrack_master_bl<P, 16>(m, br);
    } else {
      int len;
      Mc = backtrack_master<P>(p, m, 1, br, pb, &len, NoEmit{});
    }
    ++rsims;
    bool ready;  // true: the next candidate is in cand; false: the restart is finished
    if (phase == 1) {
      curM = Mc;
      bestT = Tc;
      for (int x = 0; x <= p; ++x) {
        cur[x] = cand[x];
        best[x] = cand[x];
      }
      steps = 0;
      nring = 0;
      ready = begin_step();
    } else if (phase == 2) {
      if (Tc < bestT) {
        bestT = Tc;
        for (int x = 0; x <= p; ++x) best[x] = cand[x];
      }
      if (Mc <= curM && Tc < selT) {
        selT = Tc;
        selM = Mc;
        for (int x = 0; x <= p; ++x) sel[x] = cand[x];
      }
      bool found = false;
      for (int idx = chIdx + 1; idx <= 3 && !found; ++idx)
        if (gen_child(idx, curM)) {
          chIdx = idx;
          found = true;
        }
      if (found) {
        ready = true;
      } else if (selT == INT64_MAX) {
        ready = false;  // no child qualifies
      } else {
        for (int x = 0; x <= p; ++x) cur[x] = sel[x];
        curM = selM;
        ready = begin_step();
      }
    } else {  // phase 3: an Eq. (1) adjustment was simulated
      if (Tc < bestT) {
        bestT = Tc;
        for (int x = 0; x <= p; ++x) best[x] = cand[x];
      }
      for (int x = 0; x <= p; ++x) cur[x] = cand[x];
      if (Mc != adj_i) {
        curM = Mc;  // "if the master stage changes ..., stop the adjustment"
        ready = post_adjust();
      } else if (adj_find()) {
        ready = true;
      } else {
        ready = post_adjust();
      }
    }
    const bool finish = !ready;
    if (finish) {
      nsims += rsims;
      if (bestT < (1ll << 43)) lane_key = min(lane_key, ((unsigned long long)bestT << 20) | r);
      if (A.replay)
        for (int x = 1; x <= p - 1; ++x) A.replay[x - 1] = best[x];
      if (A.best_out)
        for (int x = 1; x <= p - 1; ++x)
          A.best_out[(size_t)(r - A.r_lo) * (p - 1) + (x - 1)] = (int16_t)best[x];
      phase = 0;
    }
  }
  if (A.sims) {
    unsigned long long s = nsims;
#pragma unroll
    for (int o = 16; o >= 1; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
    if ((threadIdx.x & 31) == 0) atomicAdd(A.sims, s);
  }
  block_min_atomic(lane_key, A.key);
}

// ===========================================================================
// K3p heuristic restarts as WARP-OWNED simulation pools (adjust_mode 0, u32 fast path,
// p == P <= 16, P <= m <= 127).  With one lane per restart (k_heur) a
// warp runs as long as its longest walk and its lanes simulate out of step.  Here each
// warp owns NSW restart slots: lane l < NSW advances slot l's walk (reading O9, in
// exactly k_heur's order) and queues its simulation jobs -- the start, or the up to
// four children a, a', b, b' of a step -- in the warp's ring; then each of the 32
// lanes simulates one queued job (sim_master + backtrack_master, ap_master.cuh), all in
// step.  A slot whose jobs are all done advances at the next pass; free slots refill
// from the global restart cursor.  Only __syncwarp: the warps of a CTA never wait for
// each other.
namespace hpool {
constexpr int NT = 128;   // threads per CTA (4 independent warp pools)
constexpr int NW = NT / 32;
// 32 slots per warp (every lane owns a walk): with speculation filling idle lanes,
// measured 0.96-0.99 ms against 1.06-1.08 ms at 24 and 28 (profiles/r02_heur_pool_variants.md)
#ifndef AP_HEUR_NSW
#define AP_HEUR_NSW 32
#endif
constexpr int NSW = AP_HEUR_NSW;  // restart slots per warp (lanes 0..NSW-1 own them)
constexpr int RING = 128;         // job ring per warp, >= 4 * NSW
}  // namespace hpool
// Speculation in the lanes a pass leaves idle: for a walk waiting on
// its step's children, simulate the children of child a under a guessed master of child
// a (lower after a same-master move, same after a lower one: C5 walks alternate, 82 %
// of steps); if the walk then moves to child a with that master, the next step's
// results are already there and the walk takes two steps in one pass.  The walk, its
// simulation count and its result are exactly those without speculation.
#ifndef AP_HEUR_SPEC
#define AP_HEUR_SPEC 1
#endif

// Child idx (0 a, 1 a', 2 b, 3 b') of `cur` with master i (
// reading Q17), as k_heur's gen_child, built in place in shared memory (no local
// arrays); false if invalid or a duplicate (a' == a, b' == b).
// Cut vectors of the warp pools are CP-padded int16 rows, 16-byte aligned, copied as
// CP/8 16-byte words (CP = 0: element by element, p + 1 entries).
template <int CP>
AP_DEV_INLINE void copy_cuts(int16_t* dst, const int16_t* src, int p) {
  if constexpr (CP > 0) {
    static_assert(CP % 8 == 0, "");
#pragma unroll
    for (int q = 0; q < CP / 8; ++q)
      reinterpret_cast<uint4*>(dst)[q] = reinterpret_cast<const uint4*>(src)[q];
  } else {
    for (int x = 0; x <= p; ++x) dst[x] = src[x];
  }
}

template <int CP = 0>
AP_DEV_INLINE bool pool_child(const int16_t* cur, int idx, int i, int p, int P1,
                              const int16_t* s_arg, int16_t* cand) {
  AP_CHECK(i >= 0 && i < p && idx >= 0 && idx <= 3);
  if (cur[i + 1] - cur[i] < 2) return false;
  copy_cuts<CP>(cand, cur, p);
  int j, e;
  if (idx <= 1) {
    cand[i] += 1;  // first block of stage i -> stage i-1
    if (idx == 0) return true;
    if (i - 1 < 1) return false;
    j = i - 1;  // Alg. 1 on [0, c_{i-1}) with i-1 stages
  } else {
    if (i > p - 2) return false;
    cand[i + 1] -= 1;  // last block of stage i -> stage i+1
    if (idx == 2) return true;
    j = i;  // Alg. 1 on [0, c_i) with i stages
  }
  e = cand[j];
  bool diff = false;
  for (int jj = j; jj >= 2; --jj) {  // Algorithm 1 line 15 (alg1_prefix)
    AP_CHECK(e >= 0 && e <= cand[p]);
    const int st = s_arg[e * P1 + jj];
    // compare before the write: cand may be cur itself (in-place, the pool's
    // speculative grandchildren); the prefix indices jj-1 <= j-1 are below the moved cut
    diff = diff || (st != cur[jj - 1]);
    cand[jj - 1] = (int16_t)st;
    e = st;
  }
  return diff;
}

// pool_child's answer without building the child: the same size test, and for a'/b'
// the Algorithm-1 prefix compared with cur until the first difference (cand[j] = cur[j]
// there: the moved cut is i for a', i+1 for b').
AP_DEV_INLINE bool pool_child_valid(const int16_t* cur, int idx, int i, int p, int P1,
                                    const int16_t* s_arg) {
  if (cur[i + 1] - cur[i] < 2) return false;
  int j;
  if (idx <= 1) {
    if (idx == 0) return true;
    if (i - 1 < 1) return false;
    j = i - 1;
  } else {
    if (i > p - 2) return false;
    if (idx == 2) return true;
    j = i;
  }
  int e = cur[j];
  for (int jj = j; jj >= 2; --jj) {
    const int st = s_arg[e * P1 + jj];
    if (st != cur[jj - 1]) return true;
    e = st;
  }
  return false;
}

#ifndef AP_HEUR_MINB
#define AP_HEUR_MINB 4
#endif
// One pool job: stage weights of the cut row `src`, sim_master and the master walk.
// Returns T in the low word (>= S: saturated, no master) and the master in the high
// word.  AP_HEUR_NOINLINE=1 makes it a real call (its own register allocation); A/B on
// one box (profiles/r02_heur_pool_variants.md): inline 1.06-1.08 ms, call 1.07-1.53 ms
// depending on the surrounding code, so it is inlined.
#ifndef AP_HEUR_NOINLINE
#define AP_HEUR_NOINLINE 0
#endif
// Everything is addressed through the dynamic shared-memory window (byte offsets), so
// the callee knows its loads and stores are shared ones.
template <int P>
#if AP_HEUR_NOINLINE
__device__ __noinline__
#else
AP_DEV_INLINE
#endif
unsigned long long pool_sim(uint32_t src_sh, uint32_t off32, int n, int m, uint32_t S, int CR,
                            uint32_t off_cw, int tid, uint32_t one) {
  extern __shared__ __align__(16) unsigned char smem[];
  const uint32_t* s32Pf = reinterpret_cast<const uint32_t*>(smem + off32);
  const uint32_t* s32Pb = s32Pf + (n + 1);
  const uint32_t* s32C = s32Pb + (n + 1);
  uint32_t* s_cw = reinterpret_cast<uint32_t*>(smem + off_cw);
  const MasterBits br{s_cw + tid,
                      reinterpret_cast<uint16_t*>(s_cw + (size_t)master_col_words(m, P) * hpool::NT) + tid,
                      hpool::NT};
  int c[P + 1];
#pragma unroll
  for (int x = 0; x <= P; ++x) {
    short v;
    asm volatile("ld.shared.s16 %0, [%1];" : "=h"(v) : "r"(src_sh + 2u * x));
    c[x] = v;
  }
  uint32_t wF[P], wB[P];
#pragma unroll
  for (int x = 0; x < P; ++x) {
    wF[x] = (s32Pf[c[x + 1]] - s32Pf[c[x]]) + ((x > 0) ? s32C[c[x] - 1] : 0u);
    wB[x] = (s32Pb[c[x + 1]] - s32Pb[c[x]]) + ((x < P - 1) ? s32C[c[x + 1] - 1] : 0u);
  }
  const uint32_t t32 = sim_master<P>(m, wF, wB, S, CR, br, one);
  const uint32_t M = t32 < S ? (uint32_t)backtrack_master<P, 8>(m, br) : 0u;
  return (unsigned long long)t32 | ((unsigned long long)M << 32);
}
template <int P>
__global__ void __launch_bounds__(hpool::NT, AP_HEUR_MINB) k_heur_pool(HeurArgs A) {
  using namespace hpool;
  extern __shared__ __align__(16) unsigned char smem[];
  size_t used;
  const Tables T = stage_and_scan(A.t.tab, A.t.n, A.t.npad, smem, &used);
  const int n = A.t.n, p = P, m = A.m, P1 = P + 1;
  int16_t* s_arg = reinterpret_cast<int16_t*>(smem + ((used + 15) & ~size_t(15)));
  const int narg = (n + 1) * P1;
  int32_t* s_a1 = reinterpret_cast<int32_t*>(s_arg + ((narg + 7) & ~7));
  uint32_t* s32Pf = reinterpret_cast<uint32_t*>(s_a1 + 32);
  uint32_t* s32Pb = s32Pf + (n + 1);
  uint32_t* s32C = s32Pb + (n + 1);
  uint32_t* s_cw = s32C + ((n + 3) & ~3);  // the master bits (MasterBits)
  // per-warp slot state: cut vectors [slot][0 cur | 1 best][P+1]; a job is a slot and a
  // code (0-3: child a, a', b, b' of cur, 4: cur itself), and the lane that simulates it
  // rebuilds the child in its own scratch vector (s_scr) from cur
  constexpr int CP = ((P + 1 + 7) / 8) * 8;  // padded cut row (copy_cuts)
  __shared__ __align__(16) int16_t s_cuts[NW][NSW][2][CP];
  static_assert(NSW <= 32 && 4 * NSW <= RING, "");
  __shared__ __align__(16) int16_t s_scr[NW][32][CP];
  __shared__ uint32_t s_chT[NW][NSW][4];
  __shared__ int8_t s_chM[NW][NSW][4];
  __shared__ int8_t s_curM[NW][NSW];
  __shared__ int s_pend[NW][NSW];
  __shared__ int8_t s_aband[NW][NSW];
  __shared__ uint16_t s_ring[NW][2][RING];  // [0] walks past HOT steps, [1] the rest
#if AP_HEUR_SPEC
  // speculative grandchildren (lanes a pass leaves idle): the children of child a under
  // a guessed master g of child a; M = -1 invalid child, -2 saturated (unusable)
  __shared__ uint32_t s_spT[NW][NSW][4];
  __shared__ int8_t s_spM[NW][NSW][4];
  __shared__ int8_t s_spG[NW][NSW];
#endif
  const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
  for (int e = tid; e < narg; e += NT) s_arg[e] = A.arg[e];
  for (int e = tid; e < p - 1; e += NT) s_a1[e] = A.alg1[e];
  for (int e = tid; e <= n; e += NT) {
    s32Pf[e] = (uint32_t)T.Pf[e];
    s32Pb[e] = (uint32_t)T.Pb[e];
    if (e < n) s32C[e] = (uint32_t)T.comm[e];
  }
  __syncthreads();
  const MasterBits br{s_cw + tid, reinterpret_cast<uint16_t*>(s_cw + (size_t)master_col_words(m, P) * NT) + tid,
                      NT};
  int16_t* scr = s_scr[w][lane];
  const int smax = n * p;
  const uint32_t one = A.CR > 0 ? 1u : 0u;  // = 1, not a compile-time constant
  unsigned long long my_key = 0x7fffffffffffffffull;
  unsigned int my_sims = 0;
  // state of the slot owned by this lane (NSW = 32: one slot per lane), in registers
  int st = 0, curM = 0, steps = 0, nsims = 0, valid = 0;
  uint32_t r = 0, bestT = 0;
  bool stop = false;
  int head[2] = {0, 0}, tail[2] = {0, 0};  // warp-uniform ring cursors
  // Walks are bimodal (C5: 80 % end within 8 steps, the rest take 21-29), and the last
  // long walks set the kernel's length: the jobs of walks past HOT steps go first.
#ifndef AP_HEUR_HOT
#define AP_HEUR_HOT 6
#endif
  constexpr int HOT = AP_HEUR_HOT;
  const bool owner = lane < NSW;  // lanes 0..NSW-1 own one restart slot each
  int16_t* cur = s_cuts[w][owner ? lane : 0][0];
  int16_t* best = s_cuts[w][owner ? lane : 0][1];

  for (;;) {
    // ---- phase A: advance this lane's walk if its jobs are all done, refill if free
    int nj = 0;
    if (owner && st != 0 && s_pend[w][lane] == 0) {
      if (s_aband[w][lane]) {
        // a simulation saturated: the exact int64 pass redoes the whole restart
        const unsigned int slot = atomicAdd(&A.redo[0], 1u);
        A.redo[1 + slot] = r;
        st = 0;
      } else {
        bool walk = true, again = true;
        while (again) {
        again = false;
#if AP_HEUR_SPEC
        // the speculation issued for this step is usable if child a is the move and its
        // master is the guessed one (every grandchild simulated, none saturated)
        bool su = false;
#endif
        if (st == 1) {  // the start was simulated
          curM = s_chM[w][lane][0];
          bestT = s_chT[w][lane][0];
          copy_cuts<CP>(best, cur, P);
          steps = 0;
          nsims = 1;
          valid = 1 << 6;  // no move yet: guess a lower master first
        } else {  // the children of a step were simulated: visit them in child order
          uint32_t selT = 0xffffffffu;
          int sel = -1, selM = 0, bidx = -1;
          for (int idx = 0; idx < 4; ++idx) {
            if (!((valid >> idx) & 1)) continue;
            ++nsims;
            const uint32_t Tc = s_chT[w][lane][idx];
            const int Mc = s_chM[w][lane][idx];
            if (Tc < bestT) {  // first visited minimum; built once, below
              bestT = Tc;
              bidx = idx;
            }
            if (Mc <= curM && Tc < selT) {
              selT = Tc;
              selM = Mc;
              sel = idx;
            }
          }
          if (bidx >= 0 && bidx != sel) {  // from the scheme before the move
            pool_child<CP>(cur, bidx, curM, p, P1, s_arg, scr);
            copy_cuts<CP>(best, scr, P);
          }
          if (sel < 0) {
            walk = false;  // no child qualifies
          } else {
#if AP_HEUR_SPEC
            if (sel == 0 && ((valid >> 5) & 1) && selM == s_spG[w][lane]) {
              su = true;
#pragma unroll
              for (int idx = 0; idx < 4; ++idx) su = su && s_spM[w][lane][idx] != -2;
            }
#endif
            pool_child<CP>(cur, sel, curM, p, P1, s_arg, cur);  // in place
            if (bidx == sel) copy_cuts<CP>(best, cur, P);
            valid = (selM == curM) ? (1 << 6) : 0;  // after a same-master move guess lower
            curM = selM;
          }
        }
        // next step (k_heur's begin_step with adjust_mode 0): the step cap, stop at
        // master 0, else the children of step 3
        valid &= 1 << 6;
        if (walk && steps < smax && curM != 0) {
          ++steps;
#if AP_HEUR_SPEC
          if (su) {  // this step's children were simulated speculatively: visit them now
            for (int idx = 0; idx < 4; ++idx) {
              const int Mi = s_spM[w][lane][idx];
              if (Mi >= 0) {
                valid |= 1 << idx;
                s_chT[w][lane][idx] = s_spT[w][lane][idx];
                s_chM[w][lane][idx] = (int8_t)Mi;
              }
            }
            if (valid & 15) {
              st = 2;
              again = true;
              continue;
            }
          } else
#endif
          for (int idx = 0; idx < 4; ++idx)
            if (pool_child_valid(cur, idx, curM, p, P1, s_arg)) {
              valid |= 1 << idx;
              ++nj;
            }
        }
        }  // while (again)
        if (nj > 0) {
          s_curM[w][lane] = (int8_t)curM;
          st = 2;
        } else {  // the restart is finished
          my_sims += (unsigned int)nsims;
          my_key = min(my_key, ((unsigned long long)bestT << 20) | r);
          if (A.best_out) {
            AP_CHECK(r >= A.r_lo && r < A.r_hi);
            for (int x = 1; x <= p - 1; ++x)
              A.best_out[(size_t)(r - A.r_lo) * (p - 1) + (x - 1)] = best[x];
          }
          st = 0;
        }
      }
    }
    // refill: one global atomic per warp for all its free slots
    const bool want = owner && st == 0 && !stop;
    const unsigned int wmask = __ballot_sync(0xffffffffu, want);
    if (wmask) {
      unsigned int base = 0;
      if (lane == __ffs(wmask) - 1) base = atomicAdd(A.counter, (unsigned int)__popc(wmask));
      base = __shfl_sync(0xffffffffu, base, __ffs(wmask) - 1);
      if (want) {
        r = base + (unsigned int)__popc(wmask & ((1u << lane) - 1u)) + A.r_lo;
        if (r >= A.r_hi) {
          stop = true;
        } else {
          // restart start: Alg. 1 (r = 0) or the seeded perturbation (reading Q21)
          int prev = 0;
          cur[0] = 0;
          cur[P] = (int16_t)n;
          for (int x = 1; x <= p - 1; ++x) {
            int64_t v = s_a1[x - 1];
            if (r != 0) {
              const uint64_t u = splitmix64(A.seed ^ ((uint64_t)r << 32) ^ (uint64_t)x);
              v += (int64_t)(u % (uint64_t)(2 * A.radius + 1)) - A.radius;
              v = v < prev + 1 ? prev + 1 : v;
              v = v > n - (p - x) ? n - (p - x) : v;
            }
            cur[x] = (int16_t)v;
            prev = (int)v;
          }
          s_aband[w][lane] = 0;
          valid = 16;  // job code 4: cur itself
          nj = 1;
          st = 1;
        }
      }
    }
    // stop: the cursor ran out for one lane, so it has for every later refill too
    stop = __any_sync(0xffffffffu, stop);
    // queue the jobs: warp prefix sums of nj per ring (no atomics)
    const int hot = (st == 2 && steps >= HOT) ? 0 : 1;
    int off0 = hot == 0 ? nj : 0, off1 = hot == 1 ? nj : 0;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const int v0 = __shfl_up_sync(0xffffffffu, off0, o);
      const int v1 = __shfl_up_sync(0xffffffffu, off1, o);
      if (lane >= o) {
        off0 += v0;
        off1 += v1;
      }
    }
    const int tot0 = __shfl_sync(0xffffffffu, off0, 31);
    const int tot1 = __shfl_sync(0xffffffffu, off1, 31);
    if (nj > 0) {
      int q = tail[hot] + (hot == 0 ? off0 : off1) - nj;
      for (int code = 0; code < 5; ++code)
        if ((valid >> code) & 1) s_ring[w][hot][(q++) & (RING - 1)] = (uint16_t)(lane * 8 + code);
      s_pend[w][lane] = nj;
    }
    tail[0] += tot0;
    tail[1] += tot1;
    AP_CHECK(tail[0] - head[0] <= RING && tail[1] - head[1] <= RING);
    if (!__any_sync(0xffffffffu, owner && st != 0)) break;
    const int nj0 = min(tail[0] - head[0], 32);
    const int nj1 = min(tail[1] - head[1], 32 - nj0);
    const int nreal = nj0 + nj1;
#if AP_HEUR_SPEC
    // speculation: 4 idle lanes per walk waiting on a step whose child a is valid and
    // has not been speculated on yet; walks past HOT steps first
    const int gs = curM - ((valid >> 6) & 1);
    const bool spc = owner && st == 2 && !((valid >> 5) & 1) && (valid & 1) && gs >= 1;
    const unsigned hm = __ballot_sync(0xffffffffu, spc && steps >= HOT);
    const unsigned cm = __ballot_sync(0xffffffffu, spc && steps < HOT);
    const int nh = __popc(hm);
    const int ncand = min((32 - nreal) >> 2, nh + __popc(cm));
    if (spc) {
      const unsigned lt = (1u << lane) - 1u;
      const int rank = (steps >= HOT) ? __popc(hm & lt) : nh + __popc(cm & lt);
      if (rank < ncand) {
        valid |= 1 << 5;
        s_spG[w][lane] = (int8_t)gs;
      }
    }
#else
    const int ncand = 0;
    (void)ncand;
#endif
    __syncwarp();
    // ---- phase B: one queued job per lane, all simulated in step
    bool has = false, spec = false;
    int sl = 0, ri = 0;
    const int16_t* src = scr;
    if (lane < nreal) {
      const int job = lane < nj0 ? s_ring[w][0][(head[0] + lane) & (RING - 1)]
                                 : s_ring[w][1][(head[1] + lane - nj0) & (RING - 1)];
      const int code = job & 7;
      sl = job >> 3;
      AP_CHECK(sl < NSW && code <= 4);
      ri = code & 3;  // the start's result goes to index 0
      src = s_cuts[w][sl][0];
      if (code < 4) {
        pool_child<CP>(src, code, s_curM[w][sl], p, P1, s_arg, scr);
        src = scr;
      }
      has = true;
    }
#if AP_HEUR_SPEC
    else if (lane < nreal + 4 * ncand) {
      int k = (lane - nreal) >> 2;
      ri = (lane - nreal) & 3;
      unsigned msk = k < nh ? hm : cm;
      for (k = k < nh ? k : k - nh; k > 0; --k) msk &= msk - 1u;
      sl = __ffs(msk) - 1;
      spec = true;
      copy_cuts<CP>(scr, s_cuts[w][sl][0], P);
      pool_child<CP>(scr, 0, s_curM[w][sl], p, P1, s_arg, scr);  // child a (checked on issue)
      has = pool_child<CP>(scr, ri, s_spG[w][sl], p, P1, s_arg, scr);
      if (!has) s_spM[w][sl][ri] = -1;
    }
    // real and speculative lanes must simulate together: without the explicit
    // reconvergence the two groups ran sim_master one after the other (ncu: 1.77x the
    // warp-level executions of the row blocks)
    __syncwarp();
#endif
    // the ring cursors move before the simulation (fewer registers live across it)
    const bool real = lane < nreal;
    head[0] += nj0;
    head[1] += nj1;
    if (has) {
      const unsigned long long res =
          pool_sim<P>((uint32_t)__cvta_generic_to_shared(src),
                      (uint32_t)(reinterpret_cast<unsigned char*>(s32Pf) - smem), n, m, A.S, A.CR,
                      (uint32_t)(reinterpret_cast<unsigned char*>(s_cw) - smem), tid, one);
      const uint32_t t32 = (uint32_t)res;
      const int8_t Mc = (int8_t)(res >> 32);
      if (spec) {
#if AP_HEUR_SPEC
        if (t32 >= A.S) {
          s_spM[w][sl][ri] = -2;  // unusable: the real job will abandon the restart
        } else {
          s_spT[w][sl][ri] = t32;
          s_spM[w][sl][ri] = Mc;
        }
#endif
      } else if (t32 >= A.S) {
        s_aband[w][sl] = 1;
      } else {
        s_chT[w][sl][ri] = t32;
        s_chM[w][sl][ri] = Mc;
      }
    }
    if (real) atomicSub(&s_pend[w][sl], 1);
    __syncwarp();
  }
  if (A.sims) {
    unsigned long long sm = my_sims;
#pragma unroll
    for (int o = 16; o >= 1; o >>= 1) sm += __shfl_xor_sync(0xffffffffu, sm, o);
    if (lane == 0 && sm) atomicAdd(A.sims, sm);
  }
  block_min_atomic(my_key, A.key);
}

// ===========================================================================
// K3r reachable-set search (NEXT N1; reading R-N1): the literal reading of
// PAPER.md:196, every qualifying child is processed.  One QUAD (4 lanes) per restart,
// breadth-first: the quad pops the next queued scheme with master i > 0, lane q
// builds child q (a, a', b, b' -- the order of k_heur's gen_child), drops it if it
// is invalid or already evaluated (a 32-bit hash scan of the quad's evaluated list,
// then a full compare), and the new children are simulated together.  They join the
// evaluated list in child order; those with master <= i join the queue.  The outer
// loop is warp-uniform, so the simulations of all quads of a warp in one iteration
// run converged.  At most vmax schemes per restart are evaluated (exactly the
// oracle's cut-off).  Per-quad lists live in global scratch (L1/L2-resident).
struct ReachArgs {
  DevTables t;
  int p, m;
  uint64_t seed;
  int radius;
  uint32_t r_lo, r_hi;
  const int16_t* arg;
  const int32_t* alg1;
  unsigned int* counter;
  unsigned long long* key;
  int vmax;
  int16_t* g_cuts;            // [quads][vmax][P]
  uint32_t* g_hash;           // [quads][vmax]
  uint32_t* g_queue;          // [quads][vmax]: node | master << 24
  unsigned long long* stats;  // optional: [0] simulations, [1] truncated restarts
  int32_t* replay;            // optional: best cuts of the (single) restart
  uint32_t S;                 // > 0: u32 fast simulation below S (as k_heur_pool), int64
                              // sim_exact for a simulation that reaches S
  uint32_t* g_tab;            // pool: per-list open-addressing table [lists][tab_size] of
  int tab_size;               //   (restart tag << 11 | node), zeroed per search
};

AP_DEV_INLINE uint32_t cut_hash(const int (&c)[33], int p) {
  uint32_t h = 0x811c9dc5u;
  for (int x = 1; x <= p - 1; ++x) h = (h ^ (uint32_t)c[x]) * 0x01000193u;
  return h;
}

template <int P>
__global__ void __launch_bounds__(128) k_reach(ReachArgs A) {
  extern __shared__ __align__(16) unsigned char smem[];
  size_t used;
  const Tables T = stage_and_scan(A.t.tab, A.t.n, A.t.npad, smem, &used);
  const int n = A.t.n, p = A.p, m = A.m, P1 = p + 1, vmax = A.vmax;
  int16_t* s_arg = reinterpret_cast<int16_t*>(smem + ((used + 15) & ~size_t(15)));
  const int narg = (n + 1) * P1;
  int32_t* s_a1 = reinterpret_cast<int32_t*>(s_arg + ((narg + 7) & ~7));
  uint32_t* s_bits = reinterpret_cast<uint32_t*>(s_a1 + 32);
  for (int e = threadIdx.x; e < narg; e += blockDim.x) s_arg[e] = A.arg[e];
  for (int e = threadIdx.x; e < p - 1; e += blockDim.x) s_a1[e] = A.alg1[e];
  __syncthreads();
  BitsRef br{s_bits + threadIdx.x, (int)blockDim.x};
  TimesRef not_{nullptr, nullptr, nullptr};

  const int lane = threadIdx.x & 31, q = lane & 3, qb = lane & ~3;
  const unsigned qmask = 0xFu << qb;
  const size_t quad = ((size_t)blockIdx.x * blockDim.x + threadIdx.x) >> 2;
  int16_t* Qc = A.g_cuts + quad * (size_t)vmax * P;
  uint32_t* Qh = A.g_hash + quad * (size_t)vmax;
  uint32_t* Qq = A.g_queue + quad * (size_t)vmax;

  int phase = 0;  // 0 need a restart, 1 simulate the start, 2 expand, 3 no work left
  uint32_t r = 0;
  int nv = 0, qh = 0, qt = 0;
  bool trunc = false;
  int64_t bestT = INT64_MAX;
  int bestNode = 0;
  unsigned long long lane_key = 0x7fffffffffffffffull, nsims = 0, ntrunc = 0;
  for (;;) {
    if (phase == 0) {
      unsigned int v = 0;
      if (q == 0) v = atomicAdd(A.counter, 1u);
      v = __shfl_sync(qmask, v, qb);
      r = v + A.r_lo;
      if (r >= A.r_hi || v >= A.r_hi - A.r_lo) {
        phase = 3;
      } else {
        phase = 1;
        nv = qh = qt = 0;
        trunc = false;
        bestT = INT64_MAX;
        bestNode = 0;
      }
    }
    if (__all_sync(0xffffffffu, phase == 3)) break;

    // ---- this iteration's candidate of this lane
    int cand[33];
    cand[0] = 0;
#pragma unroll
    for (int x = 1; x <= 32; ++x) cand[x] = n;
    bool want = false;
    int slot = 0, parentM = 0;
    if (phase == 1) {
      // restart start: Alg. 1 (r = 0) or the seeded perturbation (reading Q21)
      int prev = 0;
      for (int x = 1; x <= p - 1; ++x) {
        int64_t v = s_a1[x - 1];
        if (r != 0) {
          const uint64_t u = splitmix64(A.seed ^ ((uint64_t)r << 32) ^ (uint64_t)x);
          v += (int64_t)(u % (uint64_t)(2 * A.radius + 1)) - A.radius;
          v = v < prev + 1 ? prev + 1 : v;
          v = v > n - (p - x) ? n - (p - x) : v;
        }
        cand[x] = (int)v;
        prev = (int)v;
      }
      want = (q == 0);
      slot = 0;
    } else if (phase == 2) {
      // pop the next queued scheme with master > 0 (master-0 schemes are not expanded)
      while (qh < qt && (Qq[qh] >> 24) == 0) ++qh;
      if (qh == qt) {
        phase = 4;  // queue exhausted: finish below
      } else {
        const uint32_t e = Qq[qh++];
        const int u = (int)(e & 0xffffffu), i = (int)(e >> 24);
        parentM = i;
        for (int x = 1; x <= p - 1; ++x) cand[x] = Qc[(size_t)u * P + (x - 1)];
        // child q of u (reading Q17)
        bool valid = cand[i + 1] - cand[i] >= 2;
        if (valid) {
          if (q <= 1) {
            cand[i] += 1;  // first block of stage i -> stage i-1
            if (q == 1) {
              if (i - 1 < 1) {
                valid = false;
              } else {
                int before[33];
                for (int x = 1; x < i - 1; ++x) before[x] = cand[x];
                alg1_prefix(s_arg, P1, cand[i - 1], i - 1, cand);
                bool diff = false;
                for (int x = 1; x < i - 1; ++x) diff = diff || (cand[x] != before[x]);
                valid = diff;
              }
            }
          } else if (i > p - 2) {
            valid = false;
          } else {
            cand[i + 1] -= 1;  // last block of stage i -> stage i+1
            if (q == 3) {
              int before[33];
              for (int x = 1; x < i; ++x) before[x] = cand[x];
              alg1_prefix(s_arg, P1, cand[i], i, cand);
              bool diff = false;
              for (int x = 1; x < i; ++x) diff = diff || (cand[x] != before[x]);
              valid = diff;
            }
          }
        }
        // already evaluated?
        bool dup = false;
        if (valid) {
          const uint32_t h = cut_hash(cand, p);
          for (int j = 0; j < nv && !dup; ++j) {
            if (Qh[j] != h) continue;
            bool same = true;
            for (int x = 1; x <= p - 1; ++x) same = same && (Qc[(size_t)j * P + (x - 1)] == cand[x]);
            dup = same;
          }
        }
        const bool isnew = valid && !dup;
        const unsigned bal = (__ballot_sync(qmask, isnew) >> qb) & 0xFu;
        const int cnt = __popc(bal), pre = __popc(bal & ((1u << q) - 1u));
        const int room = vmax - nv;
        if (cnt > room) trunc = true;
        want = isnew && pre < room;
        slot = nv + pre;
      }
    }

    // ---- simulate (converged across the quads of the warp)
    int64_t Tc = INT64_MAX;
    int Mc = 0;
    if (want) {
      int cc[P + 1];
#pragma unroll
      for (int x = 0; x <= P; ++x) cc[x] = (x <= p) ? cand[x] : n;
      int64_t F[P], B[P], C[P];
      stage_costs<P>(T, p, cc, F, B, C);
      bool exact = true;
      if constexpr (P >= 2 && P <= 16) {
        // u32 fast path (p == P, m >= P): T below S is exact; at S recompute in int64
        if (A.S > 0 && p == P && m >= P && m <= 32767) {
          uint32_t wF[P], wB[P];
#pragma unroll
          for (int x = 0; x < P; ++x) {
            wF[x] = (uint32_t)(F[x] + ((x > 0) ? C[x - 1] : 0));
            wB[x] = (uint32_t)(B[x] + C[x]);
          }
          const uint32_t t32 = sim_fast_bits<P>(m, wF, wB, A.S, 32, br);
          if (t32 < A.S) {
            Tc = (int64_t)t32;
            Mc = m <= 127 ? backtrack_master_bl<P, 8>(m, br) : backtrack_master_bl<P, 16>(m, br);
            exact = false;
          }
        }
      }
      if (exact) {
        uint32_t pb[P];
#pragma unroll
        for (int x = 0; x < P; ++x) pb[x] = 0;
        Tc = sim_exact<P, 1>(p, m, 1, F, B, C, br, pb, not_);
        int len;
        Mc = backtrack_master<P>(p, m, 1, br, pb, &len, NoEmit{});
      }
      for (int x = 1; x <= p - 1; ++x) Qc[(size_t)slot * P + (x - 1)] = (int16_t)cand[x];
      Qh[slot] = cut_hash(cand, p);
    }

    // ---- bookkeeping (quad-uniform)
    if (phase == 1) {
      Tc = __shfl_sync(qmask, Tc, qb);
      Mc = __shfl_sync(qmask, Mc, qb);
      if (q == 0) Qq[0] = (uint32_t)Mc << 24;
      bestT = Tc;
      bestNode = 0;
      nv = 1;
      qh = 0;
      qt = 1;
      nsims += (q == 0);
      phase = 2;
    } else if (phase == 2) {
      const bool qual = want && Mc <= parentM;
      const unsigned bq = (__ballot_sync(qmask, qual) >> qb) & 0xFu;
      if (qual) Qq[qt + __popc(bq & ((1u << q) - 1u))] = (uint32_t)slot | ((uint32_t)Mc << 24);
      // least (T, evaluation order) of this round, then against the restart's best
      int64_t bt = Tc;
      int bn = want ? slot : INT32_MAX;
#pragma unroll
      for (int o = 1; o <= 2; o <<= 1) {
        const int64_t ot = __shfl_xor_sync(qmask, bt, o);
        const int on = __shfl_xor_sync(qmask, bn, o);
        if (ot < bt || (ot == bt && on < bn)) {
          bt = ot;
          bn = on;
        }
      }
      if (bt < bestT) {
        bestT = bt;
        bestNode = bn;
      }
      const int kept = __popc((__ballot_sync(qmask, want) >> qb) & 0xFu);
      nsims += (q == 0) ? (unsigned long long)kept : 0ull;
      nv += kept;
      qt += __popc(bq);
      if (trunc) phase = 4;
    }
    if (phase == 4) {  // restart finished: queue exhausted or vmax reached
      if (q == 0) {
        if (bestT < (1ll << 43)) lane_key = min(lane_key, ((unsigned long long)bestT << 20) | r);
        ntrunc += trunc ? 1 : 0;
        if (A.replay)
          for (int x = 1; x <= p - 1; ++x) A.replay[x - 1] = Qc[(size_t)bestNode * P + (x - 1)];
      }
      phase = 0;
    }
    __syncwarp();
  }
  if (A.stats) {
    unsigned long long s = nsims, t = ntrunc;
#pragma unroll
    for (int o = 16; o >= 1; o >>= 1) {
      s += __shfl_xor_sync(0xffffffffu, s, o);
      t += __shfl_xor_sync(0xffffffffu, t, o);
    }
    if (lane == 0) {
      atomicAdd(&A.stats[0], s);
      if (t) atomicAdd(&A.stats[1], t);
    }
  }
  block_min_atomic(lane_key, A.key);
}

// ===========================================================================
// Critical path with times (single candidate; thread 0).
struct CpathArgs {
  DevTables t;
  int p, m, k;
  const int32_t* cuts;
  OpRec* ops;
  int cap;
  int32_t* len_master;  // [0] = len, [1] = master
  int64_t* T;
  uint32_t* bits;
  int64_t* finF;
  int64_t* finB;
  int64_t* finP;
  int* order;  // path scratch: encoded ops sink -> source
};

// ---------------------------------------------------------------------------
// K3r as a simulation pool (DESIGN.md R-N1, §5.5): the reachable-set search of k_reach,
// restructured like k_heur_pool.  A CTA owns NS restart slots; each slot's evaluated
// list (cuts, hash) and FIFO queue live in global scratch (per-slot, L1/L2-resident).
//   phase A, one thread per slot: fold the finished children of the node it expanded
//     into the evaluated list in child order (new ones only, up to vmax: the
//     truncation point of k_reach and the oracle), queue those with master <= i,
//     then pop the next queued scheme with master > 0 and emit its children as jobs;
//   phase B, one job per thread: drop the child if it is already evaluated (hash scan
//     + compare over the slot's list), else simulate it (u32 fast path with an
//     in-lane int64 fallback at the bound, as k_reach).
// Siblings a, a', b, b' are pairwise distinct, so deduplicating each child against the
// list as it stood before the expansion is the serial order's result.
constexpr int RP_NT = 256, RP_NS = 96, RP_RING = 512;

AP_DEV_INLINE uint32_t cut_hash16(const int16_t* c, int p) {
  uint32_t h = 0x811c9dc5u;
  for (int x = 1; x <= p - 1; ++x) h = (h ^ (uint32_t)(int)c[x]) * 0x01000193u;
  return h;
}

template <int P>
__global__ void __launch_bounds__(RP_NT, 2) k_reach_pool(ReachArgs A) {
  constexpr int NT = RP_NT, NS = RP_NS, RING = RP_RING;
  extern __shared__ __align__(16) unsigned char smem[];
  size_t used;
  const Tables T = stage_and_scan(A.t.tab, A.t.n, A.t.npad, smem, &used);
  const int n = A.t.n, p = A.p, m = A.m, P1 = p + 1, vmax = A.vmax;
  int16_t* s_arg = reinterpret_cast<int16_t*>(smem + ((used + 15) & ~size_t(15)));
  const int narg = (n + 1) * P1;
  int32_t* s_a1 = reinterpret_cast<int32_t*>(s_arg + ((narg + 7) & ~7));
  uint32_t* s_bits = reinterpret_cast<uint32_t*>(s_a1 + 32);
  __shared__ int16_t s_cuts[NS][5][P + 1];  // [0] node being expanded, [1+idx] child idx
  __shared__ int64_t s_chT[NS][4], s_bestT[NS];
  __shared__ int8_t s_chM[NS][4], s_chDup[NS][4];
  __shared__ uint32_t s_r[NS];
  __shared__ int s_pend[NS], s_nv[NS], s_qh[NS], s_qt[NS], s_best[NS], s_nsims[NS];
  __shared__ int8_t s_state[NS], s_parM[NS], s_valid[NS];
  __shared__ uint16_t s_ring[RING];
  __shared__ int s_head, s_tail, s_stop;
  const int tid = threadIdx.x;
  for (int e = tid; e < narg; e += NT) s_arg[e] = A.arg[e];
  for (int e = tid; e < p - 1; e += NT) s_a1[e] = A.alg1[e];
  for (int q = tid; q < NS; q += NT) s_state[q] = 0;
  if (tid == 0) {
    s_head = 0;
    s_tail = 0;
    s_stop = 0;
  }
  __syncthreads();
  const BitsRef br{s_bits + tid, NT};
  TimesRef not_{nullptr, nullptr, nullptr};
  unsigned long long my_key = 0x7fffffffffffffffull, my_sims = 0, my_trunc = 0;

  for (;;) {
    // ---- phase A: fold results, expand the next queued scheme, refill free slots
    if (tid < NS) {
      const int s = tid;
      const size_t L = (size_t)blockIdx.x * NS + s;  // this slot's global lists
      int16_t* Qc = A.g_cuts + L * (size_t)vmax * P;
      uint32_t* Qh = A.g_hash + L * (size_t)vmax;
      uint32_t* Qq = A.g_queue + L * (size_t)vmax;
      int st = s_state[s];
      if (st != 0 && s_pend[s] == 0) {
        int nv = s_nv[s], qh = s_qh[s], qt = s_qt[s], best = s_best[s], nsims = s_nsims[s];
        int64_t bestT = s_bestT[s];
        bool trunc = false;
        uint32_t* Tb = A.g_tab + L * (size_t)A.tab_size;
        const uint32_t tag = (s_r[s] + 1u) & 0x1fffffu;
        auto insert = [&](uint32_t h, int node) {  // linear probing; other tags = empty
          uint32_t pos = h & (uint32_t)(A.tab_size - 1);
          while ((Tb[pos] >> 11) == tag) pos = (pos + 1) & (uint32_t)(A.tab_size - 1);
          Tb[pos] = (tag << 11) | (uint32_t)node;
        };
        if (st == 1) {  // the start was simulated: it is node 0
          for (int x = 1; x <= p - 1; ++x) Qc[x - 1] = s_cuts[s][1][x];
          Qh[0] = cut_hash16(s_cuts[s][1], p);
          insert(Qh[0], 0);
          Qq[0] = (uint32_t)s_chM[s][0] << 24;
          nv = 1;
          qh = 0;
          qt = 1;
          best = 0;
          bestT = s_chT[s][0];
          nsims = 1;
        } else {  // children of the expanded node, in child order
          const int valid = s_valid[s], i = s_parM[s];
          for (int idx = 0; idx < 4 && !trunc; ++idx) {
            if (!((valid >> idx) & 1) || s_chDup[s][idx]) continue;
            if (nv >= vmax) {
              trunc = true;
              break;
            }
            for (int x = 1; x <= p - 1; ++x) Qc[(size_t)nv * P + (x - 1)] = s_cuts[s][1 + idx][x];
            Qh[nv] = cut_hash16(s_cuts[s][1 + idx], p);
            insert(Qh[nv], nv);
            ++nsims;
            const int64_t Tc = s_chT[s][idx];
            const int Mc = s_chM[s][idx];
            if (Tc < bestT) {
              bestT = Tc;
              best = nv;
            }
            if (Mc <= i) Qq[qt++] = (uint32_t)nv | ((uint32_t)Mc << 24);
            ++nv;
          }
        }
        // pop queued schemes (master-0 ones are not expanded) until one has children
        int valid = 0, nj = 0;
        while (!trunc && nj == 0 && qh < qt) {
          const uint32_t e = Qq[qh++];
          const int i = (int)(e >> 24);
          if (i == 0) continue;
          const int u = (int)(e & 0xffffffu);
          int16_t* cur = s_cuts[s][0];
          cur[0] = 0;
          cur[p] = (int16_t)n;
          for (int x = 1; x <= p - 1; ++x) cur[x] = Qc[(size_t)u * P + (x - 1)];
          for (int idx = 0; idx < 4; ++idx)
            if (pool_child(cur, idx, i, p, P1, s_arg, s_cuts[s][1 + idx])) {
              valid |= 1 << idx;
              ++nj;
            }
          s_parM[s] = (int8_t)i;
        }
        if (nj > 0) {
          const int at = atomicAdd(&s_tail, nj);
          int q = 0;
          for (int idx = 0; idx < 4; ++idx)
            if ((valid >> idx) & 1) s_ring[(at + q++) & (RING - 1)] = (uint16_t)(s * 4 + idx);
          s_pend[s] = nj;
          s_valid[s] = (int8_t)valid;
          s_nv[s] = nv;
          s_qh[s] = qh;
          s_qt[s] = qt;
          s_best[s] = best;
          s_bestT[s] = bestT;
          s_nsims[s] = nsims;
          st = 2;
        } else {  // queue exhausted or vmax reached: the restart is finished
          my_sims += (unsigned long long)nsims;
          my_trunc += trunc ? 1 : 0;
          if (bestT < (1ll << 43))
            my_key = min(my_key, ((unsigned long long)bestT << 20) | s_r[s]);
          st = 0;
        }
      }
      if (st == 0 && atomicAdd(&s_stop, 0) == 0) {
        const uint32_t r = atomicAdd(A.counter, 1u) + A.r_lo;
        if (r >= A.r_hi) {
          atomicOr(&s_stop, 1);
        } else {
          // restart start: Alg. 1 (r = 0) or the seeded perturbation (reading Q21)
          int prev = 0;
          int16_t* c = s_cuts[s][1];
          c[0] = 0;
          c[p] = (int16_t)n;
          for (int x = 1; x <= p - 1; ++x) {
            int64_t v = s_a1[x - 1];
            if (r != 0) {
              const uint64_t u = splitmix64(A.seed ^ ((uint64_t)r << 32) ^ (uint64_t)x);
              v += (int64_t)(u % (uint64_t)(2 * A.radius + 1)) - A.radius;
              v = v < prev + 1 ? prev + 1 : v;
              v = v > n - (p - x) ? n - (p - x) : v;
            }
            c[x] = (int16_t)v;
            prev = (int)v;
          }
          s_r[s] = r;
          s_nv[s] = 0;  // the start is simulated without a duplicate check
          s_pend[s] = 1;
          const int at = atomicAdd(&s_tail, 1);
          s_ring[at & (RING - 1)] = (uint16_t)(s * 4);
          st = 1;
        }
      }
      s_state[s] = (int8_t)st;
    }
    if (!__syncthreads_or(tid < NS && s_state[tid] != 0)) break;
    // ---- phase B: one queued child per thread
    const int head = s_head;
    const int nj = min(s_tail - head, NT);
    if (tid < nj) {
      const int job = s_ring[(head + tid) & (RING - 1)];
      const int s = job >> 2, idx = job & 3;
      const int16_t* cr = s_cuts[s][1 + idx];
      // already evaluated?  (the list as it stood before this expansion)
      bool dup = false;
      const int nv = s_nv[s];
      if (nv > 0) {
        const size_t L = (size_t)blockIdx.x * NS + s;
        const int16_t* Qc = A.g_cuts + L * (size_t)vmax * P;
        const uint32_t* Qh = A.g_hash + L * (size_t)vmax;
        const uint32_t* Tb = A.g_tab + L * (size_t)A.tab_size;
        const uint32_t tag = (s_r[s] + 1u) & 0x1fffffu;
        const uint32_t h = cut_hash16(cr, p);
        for (uint32_t pos = h & (uint32_t)(A.tab_size - 1);; pos = (pos + 1) & (uint32_t)(A.tab_size - 1)) {
          const uint32_t e = Tb[pos];
          if ((e >> 11) != tag) break;  // empty for this restart: not evaluated
          const int j = (int)(e & 0x7ffu);
          if (Qh[j] != h) continue;
          bool same = true;
          for (int x = 1; x <= p - 1; ++x) same = same && (Qc[(size_t)j * P + (x - 1)] == cr[x]);
          if (same) {
            dup = true;
            break;
          }
        }
      }
      s_chDup[s][idx] = dup ? 1 : 0;
      if (!dup) {
        int cc[P + 1];
#pragma unroll
        for (int x = 0; x <= P; ++x) cc[x] = (x <= p) ? (int)cr[x] : n;
        int64_t F[P], B[P], C[P];
        stage_costs<P>(T, p, cc, F, B, C);
        int64_t Tc = 0;
        int Mc = 0;
        bool exact = true;
        if constexpr (P >= 2 && P <= 16) {
          if (A.S > 0 && p == P && m >= P && m <= 32767) {
            uint32_t wF[P], wB[P];
#pragma unroll
            for (int x = 0; x < P; ++x) {
              wF[x] = (uint32_t)(F[x] + ((x > 0) ? C[x - 1] : 0));
              wB[x] = (uint32_t)(B[x] + C[x]);
            }
            const uint32_t t32 = sim_fast_bits<P>(m, wF, wB, A.S, 32, br);
            if (t32 < A.S) {
              Tc = (int64_t)t32;
              Mc = m <= 127 ? backtrack_master_bl<P, 8>(m, br) : backtrack_master_bl<P, 16>(m, br);
              exact = false;
            }
          }
        }
        if (exact) {
          uint32_t pb[P];
#pragma unroll
          for (int x = 0; x < P; ++x) pb[x] = 0;
          Tc = sim_exact<P, 1>(p, m, 1, F, B, C, br, pb, not_);
          int len;
          Mc = backtrack_master<P>(p, m, 1, br, pb, &len, NoEmit{});
        }
        s_chT[s][idx] = Tc;
        s_chM[s][idx] = (int8_t)Mc;
      }
      atomicSub(&s_pend[s], 1);
    }
    __syncthreads();
    if (tid == 0) s_head = head + nj;
  }
  if (A.stats) {
    unsigned long long sm = my_sims, tr = my_trunc;
#pragma unroll
    for (int o = 16; o >= 1; o >>= 1) {
      sm += __shfl_xor_sync(0xffffffffu, sm, o);
      tr += __shfl_xor_sync(0xffffffffu, tr, o);
    }
    if ((tid & 31) == 0) {
      if (sm) atomicAdd(&A.stats[0], sm);
      if (tr) atomicAdd(&A.stats[1], tr);
    }
  }
  block_min_atomic(my_key, A.key);
}

template <int P>
__global__ void k_cpath(CpathArgs A) {
  extern __shared__ __align__(16) unsigned char smem[];
  size_t used;
  const Tables T = stage_and_scan(A.t.tab, A.t.n, A.t.npad, smem, &used);
  if (threadIdx.x != 0) return;
  const int p = A.p, m = A.m, k = A.k, n = A.t.n;
  int c[P + 1];
  if (!load_cuts<P>(A.cuts, p, n, c)) {
    A.len_master[0] = -1;
    return;
  }
  int64_t F[P], B[P], C[P];
  stage_costs<P>(T, p, c, F, B, C);
  uint32_t pb[P];
  BitsRef br{A.bits, 1};
  TimesRef tr{A.finF, A.finB, A.finP};
  const int64_t Tc = sim_exact<P, 2>(p, m, k, F, B, C, br, pb, tr);
  int len = 0;
  int* order = A.order;
  int cnt = 0;
  const int master = backtrack_master<P>(p, m, k, br, pb, &len, [&](int kind, int x, int j, int q) {
    // kind:1 | x:5 | q:5 | j:20 bits (m <= 2^20, p <= 32, k <= 16)
    order[cnt++] = (int)((((uint32_t)kind << 10 | (uint32_t)x << 5 | (uint32_t)q) << 20) | (uint32_t)j);
  });
  A.len_master[0] = len;
  A.len_master[1] = master;
  *A.T = Tc;
  if (len > A.cap) return;
  const int W0 = min(p - 1, m);
  for (int e = 0; e < len; ++e) {
    const uint32_t code = (uint32_t)order[len - 1 - e];
    const int j = (int)(code & ((1u << 20) - 1));
    const int q = (int)((code >> 20) & 31u);
    const int x = (int)((code >> 25) & 31u);
    const int kind = (int)(code >> 30);
    int64_t fin = 0, cost = 0;
    int xx = 0;
#pragma unroll
    for (int s = 0; s < P; ++s) xx = (s == x) ? s : xx;
    int64_t Fx = 0, Bx = 0;
#pragma unroll
    for (int s = 0; s < P; ++s)
      if (s == x) {
        Fx = F[s];
        Bx = B[s];
      }
    const int wx = min(p - 1 - x, m);
    if (kind == 1) {
      fin = A.finB[(j + W0) * P + x];
      cost = Bx;
    } else if (j == 0) {
      fin = A.finP[x * kMaxK + q];
      cost = (q < k - 1) ? Fx / k : Fx - (int64_t)(k - 1) * (Fx / k);
    } else {
      fin = A.finF[(j - wx + W0) * P + x];
      cost = Fx;
    }
    (void)xx;
    OpRec o;
    o.stage = x;
    o.kind = kind;
    o.microbatch = j;
    o.piece = q;
    o.start_ns = fin - cost;
    o.end_ns = fin;
    A.ops[e] = o;
  }
}

// Algorithm 2: the Slicer's analytic number mb of leading
// micro-batches to slice in halves.  One thread, after the K4 prologue.  Readings
// (Q22-Q24): x/2 = floor; Comm per boundary (forward hop i->i+1: C_i,
// gradient hop i->i-1: C_{i-1}); line 21 as printed; endt row p stays 0; stop test
// reading 0 = pseudocode "tempt <= endt[0][1]", 1 = text "start of the unbroken
// micro-batch >= end of the second half"; mb stops at p.
__global__ void k_alg2(DevTables t, int p, const int32_t* cuts, int reading, int32_t* mb_out) {
  extern __shared__ __align__(16) unsigned char smem[];
  size_t used;
  const Tables T = stage_and_scan(t.tab, t.n, t.npad, smem, &used);
  if (threadIdx.x != 0) return;
  const int n = t.n;
  int64_t F[kMaxP], Bv[kMaxP], Cv[kMaxP], startt[kMaxP], endt[kMaxP + 1][2];
  int prev = 0;
  for (int x = 0; x < p; ++x) {
    const int hi = (x == p - 1) ? n : cuts[x];
    if (hi <= prev || hi > n) {
      *mb_out = -1;
      return;
    }
    F[x] = T.Pf[hi] - T.Pf[prev];
    Bv[x] = T.Pb[hi] - T.Pb[prev];
    Cv[x] = (x < p - 1) ? T.comm[hi - 1] : 0;
    prev = hi;
  }
  for (int x = 0; x <= p; ++x) {
    if (x < p) startt[x] = 0;
    endt[x][0] = endt[x][1] = 0;
  }
  int64_t tempt = 0;
  int mb = 1;
  for (int i = 0; i <= p - 2; ++i) tempt += F[i] / 2 + Cv[i] / 2;  // forward fill, halves
  tempt += F[p - 1] / 2;
  for (int i = p - 1; i >= 1; --i) {  // backward chain of micro-batch 0
    tempt += Bv[i] + Cv[i - 1];
    startt[p - 1 - i] = tempt;
  }
  tempt += Bv[0];
  startt[p - 1] = tempt;
  for (;;) {
    for (int i = 0; i <= p - mb; ++i)
      for (int j = 0; j <= 1; ++j) {
        int64_t e = endt[i][(j + 1) % 2] + F[i] / 2;
        if (i > 0) e = max(e, endt[i - 1][j] + F[i - 1] / 2);
        if (i != p - 1) e += Cv[i] / 2;
        e = max(e, endt[i + 1][(j + 1) % 2]);
        endt[i][j] = e;
      }
    tempt = startt[mb - 1];
    for (int i = p - 1 - mb; i >= 1; --i) tempt -= F[i] + Cv[i - 1];
    tempt -= F[0];
    const bool stop = (reading == 0) ? (tempt <= endt[0][1]) : (tempt >= endt[0][1]);
    if (stop || mb >= p) break;
    ++mb;
  }
  *mb_out = mb;
}

cudaError_t launch_alg2(const DevTables& t, int p, const int32_t* cuts, int reading, int32_t* mb,
                        cudaStream_t s) {
  const size_t smem = tables_smem_bytes(t.npad, t.n);
  count_launch();
  k_alg2<<<1, 32, smem, s>>>(t, p, cuts, reading, mb);
  return cudaGetLastError();
}

__global__ void k_unrank(DevTables t, int p, uint64_t rank, int32_t* cuts) {
  // one warp: c_x = the least v > c_{x-1} with rank < sum_{u=c_{x-1}+1}^{v} C(n-1-u, p-1-x)
  // (reading O7), 32 candidate v per step with a warp prefix sum
  if (blockIdx.x != 0 || threadIdx.x >= 32) return;
  const int n = t.n, lane = threadIdx.x;
  uint64_t rr = rank;
  int prev = 0;
  for (int x = 1; x <= p - 1; ++x) {
    int base = prev + 1;
    for (;;) {
      const int v = base + lane;
      uint64_t c = (v <= n - 1) ? binom_at(t.binom, n - 1 - v, p - 1 - x) : 0ull;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {  // inclusive prefix sum over the 32 candidates
        const uint64_t u = __shfl_up_sync(0xffffffffu, c, o);
        if (lane >= o) c += u;
      }
      // the first lane whose running sum exceeds rr holds c_x
      const unsigned int hit = __ballot_sync(0xffffffffu, c > rr);
      if (hit) {
        const int l = __ffs(hit) - 1;
        const uint64_t below = __shfl_sync(0xffffffffu, c, l > 0 ? l - 1 : 0);
        if (l > 0) rr -= below;
        prev = base + l;
        break;
      }
      rr -= __shfl_sync(0xffffffffu, c, 31);
      base += 32;
      if (base > n) {  // rank beyond C(n-1, p-1): the caller validated it, cannot happen
        prev = n;
        break;
      }
    }
    if (lane == 0) cuts[x - 1] = prev;
  }
}

// ===========================================================================
// Launchers.
static int pick_P(int p) { return p <= 2 ? 2 : p <= 4 ? 4 : p <= 8 ? 8 : p <= 16 ? 16 : 32; }

int num_sms(int device) {
  int v = 0;
  cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, device);
  return v;
}

static cudaError_t set_smem(const void* fn, size_t bytes) {
  if (bytes > 48 * 1024)
    return cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)bytes);
  return cudaSuccess;
}

cudaError_t launch_alg1(const DevTables& t, int p, int16_t* arg, int32_t* cuts, int64_t* value,
                        cudaStream_t s) {
  const size_t smem = ((tables_smem_bytes(t.npad, t.n) + 15) & ~size_t(15)) +
                      (size_t)(t.n + 1) * (p + 1) * 8;
  cudaError_t e = set_smem((const void*)k_alg1, smem);
  if (e != cudaSuccess) return e;
  count_launch();
  k_alg1<<<1, 1024, smem, s>>>(t, p, arg, cuts, value);
  return cudaGetLastError();
}

cudaError_t launch_minlb(const DevTables& t, int p, int m, int K, int16_t* arg, int32_t* cuts,
                         int64_t* value, cudaStream_t s) {
  const size_t smem = ((tables_smem_bytes(t.npad, t.n) + 15) & ~size_t(15)) +
                      (size_t)(t.n + 1) * (p + 1) * 8;
  cudaError_t e = set_smem((const void*)k_minlb, smem);
  if (e != cudaSuccess) return e;
  count_launch();
  k_minlb<<<1, 256, smem, s>>>(t, p, m, K, arg, cuts, value);
  return cudaGetLastError();
}

template <int P>
static cudaError_t eval_P(const EvalArgs& A0, cudaStream_t s, int* launches) {
  EvalArgs A = A0;
  const size_t base = (tables_smem_bytes(A.t.npad, A.t.n) + 15) & ~size_t(15);
  int threads = 128;
  size_t smem = base;
  if (A.master) {
    const int rows = A.m + min(A.p - 1, A.m);
    const size_t per = (size_t)rows * BitsLayout<P>::WPR * 4;
    const size_t budget = 200 * 1024 - base;
    if (per * 32 > budget) {
      // bits in global scratch: caller provided A.gbits
      if (!A.gbits) return cudaErrorInvalidValue;
    } else {
      A.gbits = nullptr;
      { const size_t cap = (budget / per) / 32 * 32; threads = (int)(cap < 128 ? cap : 128); }
      smem = base + per * threads;
    }
  }
  const bool sliced = A.s_iota || A.s_const != 1;
  const void* fn = sliced ? (const void*)k_eval<P, true> : (const void*)k_eval<P, false>;
  cudaError_t e = set_smem(fn, smem);
  if (e != cudaSuccess) return e;
  // persistent grid: at most one wave (the kernel strides over the candidates)
  int occ = 0, dev = 0;
  cudaGetDevice(&dev);
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, fn, threads, smem);
  if (e != cudaSuccess) return e;
  occ = occ < 1 ? 1 : occ;
  int64_t blocks = (A.count + threads - 1) / threads;
  const int64_t wave = (int64_t)num_sms(dev) * occ;
  if (blocks > wave) blocks = wave;  // (redo pass: the listed count is <= A.count)
  if (blocks > 0) {
    count_launch();
    if (sliced)
      k_eval<P, true><<<(unsigned)blocks, threads, smem, s>>>(A);
    else
      k_eval<P, false><<<(unsigned)blocks, threads, smem, s>>>(A);
    if (launches) ++*launches;
  }
  return cudaGetLastError();
}

template <int P>
static cudaError_t eval_fast_P(const EvalArgs& A, cudaStream_t s, int* launches) {
  const int threads = 128;
  const size_t smem = ((tables_smem_bytes(A.t.npad, A.t.n) + 15) & ~size_t(15)) +
                      ((eval_fast_smem(A.t.n) + 15) & ~size_t(15)) +
                      (A.master ? master_bits_bytes(A.m, P, threads) : 0);
  const void* fn = A.master ? (const void*)k_eval_fast<P, true> : (const void*)k_eval_fast<P, false>;
  cudaError_t e = set_smem(fn, smem);
  if (e != cudaSuccess) return e;
  int occ = 0, dev = 0;
  cudaGetDevice(&dev);
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, fn, threads, smem);
  if (e != cudaSuccess) return e;
  occ = occ < 1 ? 1 : occ;
  int64_t blocks = (A.count + threads - 1) / threads;
  const int64_t wave = (int64_t)num_sms(dev) * occ;
  if (blocks > wave) blocks = wave;
  if (blocks > 0) {
    count_launch();
    if (A.master)
      k_eval_fast<P, true><<<(unsigned)blocks, threads, smem, s>>>(A);
    else
      k_eval_fast<P, false><<<(unsigned)blocks, threads, smem, s>>>(A);
    if (launches) ++*launches;
  }
  return cudaGetLastError();
}

cudaError_t launch_eval(const DevTables& t, cudaMemPool_t pool, int p, int m, const int32_t* cuts,
                        int cuts_stride,
                        const int32_t* kptr, int k_const, int k_iota, int64_t count,
                        int64_t* time_ns, int32_t* master, cudaStream_t s, int* launches,
                        int s_const, int s_iota, uint32_t fastS, int fastCR, int div1,
                        unsigned long long* n_invalid) {
  EvalArgs A{t, p, m, cuts, cuts_stride, kptr, k_const, k_iota, count, time_ns, master, nullptr,
             s_const, s_iota, fastS, fastCR < 1 ? 1 : fastCR, div1, nullptr, nullptr, 1u,
             n_invalid};
  if (n_invalid) {
    cudaError_t e = cudaMemsetAsync(n_invalid, 0, sizeof(*n_invalid), s);
    if (e != cudaSuccess) return e;
  }
  uint32_t* gbits = nullptr;
  unsigned int* redo = nullptr;
  if (fastS && count >= (1ll << 32)) fastS = A.fastS = 0;  // redo indices are 32-bit
  // the fast kernel covers p == P in {2, 4, 8, 16} (exact-P templates), m >= p, and the
  // north-star slicing form (s = 1); everything else is the generic kernel's
  if (!(pick_P(p) == p && p >= 2 && p <= 16 && m >= p && s_const == 1 && !s_iota))
    fastS = A.fastS = 0;
  if (fastS) {
    cudaError_t e = cudaMallocFromPoolAsync((void**)&redo, 4 * ((size_t)count + 1), pool, s);
    if (e != cudaSuccess) return e;
    e = cudaMemsetAsync(redo, 0, 4, s);
    if (e != cudaSuccess) return e;
    A.redo = redo;
  }
  if (master) {
    const int rows = m + min(p - 1, m);
    const int P = pick_P(p);
    const size_t per = (size_t)rows * (P <= 16 ? 1 : 2) * 4;
    const size_t base = (tables_smem_bytes(t.npad, t.n) + 15) & ~size_t(15);
    if (per * 32 > 200 * 1024 - base) {
      cudaError_t e = cudaMallocFromPoolAsync((void**)&gbits, per * (size_t)count + 16, pool, s);
      if (e != cudaSuccess) return e;
      A.gbits = gbits;
    }
  }
  cudaError_t e;
  auto run = [&](const EvalArgs& X) {
    switch (pick_P(p)) {
      case 2: return eval_P<2>(X, s, launches);
      case 4: return eval_P<4>(X, s, launches);
      case 8: return eval_P<8>(X, s, launches);
      case 16: return eval_P<16>(X, s, launches);
      default: return eval_P<32>(X, s, launches);
    }
  };
  if (redo) {
    switch (p) {
      case 2: e = eval_fast_P<2>(A, s, launches); break;
      case 4: e = eval_fast_P<4>(A, s, launches); break;
      case 8: e = eval_fast_P<8>(A, s, launches); break;
      default: e = eval_fast_P<16>(A, s, launches); break;
    }
  } else {
    e = run(A);
  }
  if (e == cudaSuccess && redo) {
    // exact int64 pass over the candidates the fast kernel listed (saturated ones, and
    // T + master at k > 1); one wave, it reads the count on the device and exits at
    // once when the list is empty
    EvalArgs X = A;
    X.fastS = 0;
    X.redo = nullptr;
    X.redo_in = redo;
#ifndef AP_EVAL_REDO64
#define AP_EVAL_REDO64 1
#endif
    if (AP_EVAL_REDO64 && !master) {  // T only: the 64-bit offset-form sweep
      switch (p) {
        case 2: e = eval_redo64_P<2>(X, s, launches); break;
        case 4: e = eval_redo64_P<4>(X, s, launches); break;
        case 8: e = eval_redo64_P<8>(X, s, launches); break;
        default: e = eval_redo64_P<16>(X, s, launches); break;
      }
    } else {
      e = run(X);
    }
  }
  if (gbits) cudaFreeAsync(gbits, s);
  if (redo) cudaFreeAsync(redo, s);
  return e;
}

int sweep_max_blocks(int dev);

template <int P, typename V>
static cudaError_t sweep_exact_P(SweepArgs A, cudaStream_t s, SweepPlan* sp, int dev) {
  const size_t smem = tables_smem_bytes(A.t.npad, A.t.n) + (size_t)(3 * (A.t.n + 1) + 4) * sizeof(V);
  const bool fact = A.mode != 0;
  const void* fn = fact ? (const void*)k_sweep_exact<P, V, true> : (const void*)k_sweep_exact<P, V, false>;
  cudaError_t e = set_smem(fn, smem);
  if (e != cudaSuccess) return e;
  const int threads = 256;
  int occ = 0;
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, fn, threads, smem);
  if (e != cudaSuccess) return e;
  occ = occ < 1 ? 1 : occ;
  const uint64_t nr = A.rank_hi - A.rank_lo;
  const uint64_t target = (uint64_t)num_sms(dev) * occ * threads;
  uint64_t blocks;
  if (A.ctr) {
    // persistent warp-dynamic grid (one wave): units of 32 lanes x chunk ranks, about
    // kUnitsPerWarp units per warp so the end-of-kernel imbalance is ~1/kUnitsPerWarp
    // of a warp's work, while the per-unit unrank stays negligible
    uint64_t kUnitsPerWarp = 128, kMinSims = 128;
    // pruned mode skips whole prefix blocks inside a lane's range: longer ranges
    if (A.mode == 2) kUnitsPerWarp = 16;  // A/B: profiles/r01_pruned_upw.txt
    if (const char* e = getenv("AP_SWEEP_UPW")) kUnitsPerWarp = strtoull(e, nullptr, 10);
    if (const char* e = getenv("AP_SWEEP_MINSIMS")) kMinSims = strtoull(e, nullptr, 10);
    const uint64_t K = (uint64_t)(A.k_hi - A.k_lo + 1);
    A.chunk = (nr + target * kUnitsPerWarp - 1) / (target * kUnitsPerWarp);
    const uint64_t cmin = (kMinSims + K - 1) / K;  // amortise the per-unit unrank
    if (A.chunk < cmin) A.chunk = cmin;
    if (A.chunk == 0) A.chunk = 1;
    const uint64_t units = (nr + 32 * A.chunk - 1) / (32 * A.chunk);
    const uint64_t need = (units * 32 + threads - 1) / threads;
    blocks = (uint64_t)num_sms(dev) * occ;
    if (blocks > need) blocks = need;
    if (blocks < 1) blocks = 1;
    cudaError_t em = cudaMemsetAsync(A.ctr, 0, sizeof(unsigned long long), s);
    if (em != cudaSuccess) return em;
  } else {
    A.chunk = (nr + target - 1) / target;
    if (A.chunk == 0) A.chunk = 1;
    const uint64_t nthreads = (nr + A.chunk - 1) / A.chunk;
    blocks = (nthreads + threads - 1) / threads;
  }
  if (A.rec && blocks > (uint64_t)sweep_max_blocks(dev)) return cudaErrorInvalidValue;
  count_launch();
  if (fact)
    k_sweep_exact<P, V, true><<<(unsigned)blocks, threads, smem, s>>>(A);
  else
    k_sweep_exact<P, V, false><<<(unsigned)blocks, threads, smem, s>>>(A);
  sp->blocks = (int)blocks;
  sp->threads = threads;
  sp->chunk = A.chunk;
  return cudaGetLastError();
}

template <int P>
static cudaError_t sweep_generic_P(SweepArgs A, cudaStream_t s, SweepPlan* sp, int dev) {
  const size_t smem = ((tables_smem_bytes(A.t.npad, A.t.n) + 15) & ~size_t(15)) +
                      (A.mem ? 2 * (size_t)(A.t.n + 1) * 8 : 0);
  const void* fn = (const void*)k_sweep_generic<P>;
  cudaError_t e = set_smem(fn, smem);
  if (e != cudaSuccess) return e;
  const int threads = 128;
  int occ = 0;
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_sweep_generic<P>, threads, smem);
  if (e != cudaSuccess) return e;
  occ = occ < 1 ? 1 : occ;
  const uint64_t nr = A.rank_hi - A.rank_lo;
  const uint64_t target = (uint64_t)num_sms(dev) * occ * threads;
  A.chunk = (nr + target - 1) / target;
  if (A.chunk == 0) A.chunk = 1;
  const uint64_t nthreads = (nr + A.chunk - 1) / A.chunk;
  const uint64_t blocks = (nthreads + threads - 1) / threads;
  if (A.rec && blocks > (uint64_t)sweep_max_blocks(dev)) return cudaErrorInvalidValue;
  count_launch();
  k_sweep_generic<P><<<(unsigned)blocks, threads, smem, s>>>(A);
  sp->blocks = (int)blocks;
  sp->threads = threads;
  sp->chunk = A.chunk;
  return cudaGetLastError();
}

#define AP_EXACT_CASE(PP)                                                   \
  case PP:                                                                  \
    return want_u32 ? sweep_exact_P<PP, uint32_t>(A, s, sp, dev)            \
                    : sweep_exact_P<PP, uint64_t>(A, s, sp, dev);

static cudaError_t sweep_exact_dispatch(int p, int want_u32, const SweepArgs& A, cudaStream_t s,
                                        SweepPlan* sp, int dev) {
  switch (p) {
    AP_EXACT_CASE(1)
    AP_EXACT_CASE(2)
    AP_EXACT_CASE(3)
    AP_EXACT_CASE(4)
    AP_EXACT_CASE(5)
    AP_EXACT_CASE(6)
    AP_EXACT_CASE(7)
    AP_EXACT_CASE(8)
    AP_EXACT_CASE(10)
    AP_EXACT_CASE(12)
    AP_EXACT_CASE(16)
    default: return cudaErrorNotSupported;
  }
}

cudaError_t launch_reduce2(const unsigned long long* rec, int nrec, long long* out,
                           cudaStream_t s) {
  count_launch();
  k_reduce2<<<1, 256, 0, s>>>(rec, nrec, out);
  return cudaGetLastError();
}

cudaError_t launch_key2_select(const long long* local, const long long* t_star, long long* idx,
                               cudaStream_t s) {
  count_launch();
  k_key2_select<<<1, 1, 0, s>>>(local, t_star, idx);
  return cudaGetLastError();
}

int sweep_max_blocks(int dev) { return num_sms(dev) * 32; }

bool has_exact(int p) {
  return (p >= 1 && p <= 8) || p == 10 || p == 12 || p == 16;
}

bool sweep_has_exact(int p, int m, int mode, int force_generic, bool mem) {
  return !mem && has_exact(p) && m >= p && (!force_generic || mode != 0);
}

cudaError_t launch_sweep(const DevTables& t, int p, int m, int k_lo, int k_hi, uint64_t rank_lo,
                         uint64_t rank_hi, const SweepDev* dp, int rb, int try_u32,
                         int force_generic, int mode, unsigned long long* key, cudaStream_t s,
                         SweepPlan* sp, unsigned long long* rec, const int64_t* mem,
                         int64_t mem_cap, unsigned long long* ctr, int div1) {
  int dev = 0;
  cudaGetDevice(&dev);
  SweepArgs A{t, p, m, k_lo, k_hi, rank_lo, rank_hi, 1, 0, rb, key, 1, 0, 1, 1u, mode, rec,
              mem, mem_cap, ctr, div1, dp, 0};
  const bool exact = sweep_has_exact(p, m, mode, force_generic, mem != nullptr);
  sp->exact_p = exact ? 1 : 0;
  sp->fast_u32 = (exact && try_u32) ? 1 : 0;  // the device picks; see SweepDev::u32
  if (rec) {
    // records of the variant that does not run stay "empty" (all ones > any real record)
    cudaError_t e = cudaMemsetAsync(rec, 0xff, 16 * (size_t)sweep_max_blocks(dev), s);
    if (e != cudaSuccess) return e;
  }
  if (exact) {
    int blocks = 0;
    cudaError_t e = cudaSuccess;
    if (try_u32) {
      A.is_u32 = 1;
      e = sweep_exact_dispatch(p, 1, A, s, sp, dev);
      if (e != cudaSuccess) return e;
      blocks = sp->blocks;
    }
    A.is_u32 = 0;
    A.div1 = 0;
    SweepPlan sp64 = *sp;
    e = sweep_exact_dispatch(p, 0, A, s, &sp64, dev);
    if (e != cudaSuccess) return e;
    if (!try_u32) *sp = sp64;
    sp->blocks = blocks > sp64.blocks ? blocks : sp64.blocks;
    sp->fast_u32 = try_u32 ? 1 : 0;
    sp->exact_p = 1;
    return cudaSuccess;
  }
  A.div1 = 0;
  switch (pick_P(p)) {
    case 2: return sweep_generic_P<2>(A, s, sp, dev);
    case 4: return sweep_generic_P<4>(A, s, sp, dev);
    case 8: return sweep_generic_P<8>(A, s, sp, dev);
    case 16: return sweep_generic_P<16>(A, s, sp, dev);
    default: return sweep_generic_P<32>(A, s, sp, dev);
  }
}

template <int P, bool FAST>
static cudaError_t heur_P(const HeurArgs& A, cudaStream_t s, int dev, uint64_t nwork) {
  const int threads = A.replay ? 32 : 128;
  const int rows = A.m + min(A.p - 1, A.m);
  const size_t narg = (size_t)(A.t.n + 1) * (A.p + 1);
  const size_t base = ((tables_smem_bytes(A.t.npad, A.t.n) + 15) & ~size_t(15)) +
                      ((narg + 7) & ~size_t(7)) * 2 + 32 * 4;
  const size_t smem = base + (size_t)rows * BitsLayout<P>::WPR * 4 * threads;
  if (smem > 227 * 1024) return cudaErrorInvalidValue;
  cudaError_t e = set_smem((const void*)k_heur<P, FAST>, smem);
  if (e != cudaSuccess) return e;
  int occ = 0;
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_heur<P, FAST>, threads, smem);
  if (e != cudaSuccess) return e;
  occ = occ < 1 ? 1 : occ;
  uint64_t blocks = (uint64_t)num_sms(dev) * occ;
  const uint64_t need = (nwork + threads - 1) / threads;
  if (blocks > need) blocks = need;
  if (blocks < 1) blocks = 1;
  count_launch();
  k_heur<P, FAST><<<(unsigned)blocks, threads, smem, s>>>(A);
  return cudaGetLastError();
}

template <int P>
static cudaError_t heur_pool_P(const HeurArgs& A, cudaStream_t s, int dev, uint64_t nwork) {
  const int threads = hpool::NT;
  const size_t narg = (size_t)(A.t.n + 1) * (A.p + 1);
  const size_t base = ((tables_smem_bytes(A.t.npad, A.t.n) + 15) & ~size_t(15)) +
                      ((narg + 7) & ~size_t(7)) * 2 + 32 * 4 +
                      (size_t)(2 * (A.t.n + 1) + ((A.t.n + 3) & ~3)) * 4;
  const size_t smem = base + master_bits_bytes(A.m, P, threads);
  // the static slot state plus the dynamic part can pass 48 KB while the dynamic part
  // alone does not, so the attribute is always set
  cudaError_t e = cudaFuncSetAttribute((const void*)k_heur_pool<P>,
                                       cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  int occ = 0;
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_heur_pool<P>, threads, smem);
  if (e != cudaSuccess) return e;
  occ = occ < 1 ? 1 : occ;
  if (const char* ov = getenv("AP_HEUR_OCC")) {  // A/B: CTAs per SM
    const int v = atoi(ov);
    if (v >= 1 && v < occ) occ = v;
  }
  uint64_t blocks = (uint64_t)num_sms(dev) * occ;
  const uint64_t need = (nwork + hpool::NSW * hpool::NW - 1) / (hpool::NSW * hpool::NW);
  if (blocks > need) blocks = need;
  if (blocks < 1) blocks = 1;
  count_launch();
  k_heur_pool<P><<<(unsigned)blocks, threads, smem, s>>>(A);
  return cudaGetLastError();
}

cudaError_t launch_heuristic(const DevTables& t, int p, int m, uint64_t seed, int radius,
                             uint32_t r_lo, uint32_t r_hi, const int16_t* arg,
                             const int32_t* alg1_cuts, unsigned int* counter,
                             unsigned long long* key, int32_t* replay_cuts,
                             unsigned long long* sims, int16_t* best_out, uint32_t fastS,
                             int fastCR, int adjust_mode, cudaStream_t s) {
  int dev = 0;
  cudaGetDevice(&dev);
  // counter[0]: restart cursor of the first pass; counter[1]: cursor of the redo
  // pass; counter[2]: redo count; counter[3..]: redo ids (caller zeroes [0..2])
  const bool fast = fastS > 0 && pick_P(p) == p && p >= 2 && p <= 16 && m >= p && m <= 32767 &&
                    !replay_cuts;
  // the warp pool's 8-bit master counters need 2m <= 255 (ap_master.cuh)
  const bool pool_ok = m <= 127;
  HeurArgs A{t, p, m, seed, radius, r_lo, r_hi, arg, alg1_cuts, counter, key, replay_cuts, sims,
             best_out, fastS, fastCR < 1 ? 1 : fastCR, nullptr, adjust_mode};
  const uint64_t R = r_hi - r_lo;
  if (!fast) {
    switch (pick_P(p)) {
      case 2: return heur_P<2, false>(A, s, dev, R);
      case 4: return heur_P<4, false>(A, s, dev, R);
      case 8: return heur_P<8, false>(A, s, dev, R);
      case 16: return heur_P<16, false>(A, s, dev, R);
      default: return heur_P<32, false>(A, s, dev, R);
    }
  }
  A.redo = counter + 2;
  cudaError_t e;
  const char* pv = getenv("AP_HEUR_POOL");  // A/B: AP_HEUR_POOL=0 runs k_heur<P, true>
  if (adjust_mode == 0 && pool_ok && !(pv && pv[0] == '0')) {
    switch (p) {
      case 2: e = heur_pool_P<2>(A, s, dev, R); break;
      case 4: e = heur_pool_P<4>(A, s, dev, R); break;
      case 8: e = heur_pool_P<8>(A, s, dev, R); break;
      default: e = heur_pool_P<16>(A, s, dev, R); break;
    }
  } else {
    switch (p) {
      case 2: e = heur_P<2, true>(A, s, dev, R); break;
      case 4: e = heur_P<4, true>(A, s, dev, R); break;
      case 8: e = heur_P<8, true>(A, s, dev, R); break;
      default: e = heur_P<16, true>(A, s, dev, R); break;
    }
  }
  if (e != cudaSuccess) return e;
  // exact pass over the abandoned restarts (exits at once when the list is empty)
  HeurArgs B = A;
  B.counter = counter + 1;
  switch (p) {
    case 2: return heur_P<2, false>(B, s, dev, 128);
    case 4: return heur_P<4, false>(B, s, dev, 128);
    case 8: return heur_P<8, false>(B, s, dev, 128);
    default: return heur_P<16, false>(B, s, dev, 128);
  }
}

// Pool form of the reachable-set search (k_reach_pool, P <= 16, not the single-restart
// decode replay); AP_REACH_POOL=0 keeps k_reach.  *lists_out = per-restart lists the
// launch uses (scratch: lists x vmax entries).
template <int P>
static cudaError_t reach_pool_P(ReachArgs* A, cudaStream_t s, int dev, uint64_t R, bool launch,
                                int* lists_out) {
  const size_t narg = (size_t)(A->t.n + 1) * (A->p + 1);
  const int rows = A->m + min(A->p - 1, A->m);
  const size_t base = ((tables_smem_bytes(A->t.npad, A->t.n) + 15) & ~size_t(15)) +
                      ((narg + 7) & ~size_t(7)) * 2 + 32 * 4;
  const size_t smem = base + (size_t)rows * 4 * RP_NT;
  if (smem > 160 * 1024) return cudaErrorInvalidValue;
  cudaError_t e = cudaFuncSetAttribute((const void*)k_reach_pool<P>,
                                       cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  int occ = 0;
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_reach_pool<P>, RP_NT, smem);
  if (e != cudaSuccess) return e;
  occ = occ < 1 ? 1 : occ;
  uint64_t blocks = (uint64_t)num_sms(dev) * occ;
  const uint64_t need = (R + RP_NS - 1) / RP_NS;
  if (blocks > need) blocks = need;
  if (blocks < 1) blocks = 1;
  *lists_out = (int)blocks * RP_NS;
  if (!launch) return cudaSuccess;
  count_launch();
  k_reach_pool<P><<<(unsigned)blocks, RP_NT, smem, s>>>(*A);
  return cudaGetLastError();
}

static bool reach_use_pool(const ReachArgs* A) {
  const char* v = getenv("AP_REACH_POOL");
  return !A->replay && pick_P(A->p) <= 16 && A->m + min(A->p - 1, A->m) <= 128 &&
         A->vmax <= 2048 && !(v && v[0] == '0');
}

template <int P>
static cudaError_t reach_P(ReachArgs* A, cudaStream_t s, int dev, uint64_t R, bool launch,
                           int* blocks_out) {
  if constexpr (P <= 16) {
    if (reach_use_pool(A)) return reach_pool_P<P>(A, s, dev, R, launch, blocks_out);
  }
  const int threads = 128;
  const int rows = A->m + min(A->p - 1, A->m);
  const size_t narg = (size_t)(A->t.n + 1) * (A->p + 1);
  const size_t base = ((tables_smem_bytes(A->t.npad, A->t.n) + 15) & ~size_t(15)) +
                      ((narg + 7) & ~size_t(7)) * 2 + 32 * 4;
  const size_t smem = base + (size_t)rows * BitsLayout<P>::WPR * 4 * threads;
  if (smem > 227 * 1024) return cudaErrorInvalidValue;
  cudaError_t e = set_smem((const void*)k_reach<P>, smem);
  if (e != cudaSuccess) return e;
  int occ = 0;
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_reach<P>, threads, smem);
  if (e != cudaSuccess) return e;
  occ = occ < 1 ? 1 : occ;
  uint64_t blocks = (uint64_t)num_sms(dev) * occ;
  const uint64_t need = (R * 4 + threads - 1) / threads;
  if (blocks > need) blocks = need;
  if (blocks < 1) blocks = 1;
  *blocks_out = (int)blocks * 32;  // one list per quad
  if (!launch) return cudaSuccess;
  count_launch();
  k_reach<P><<<(unsigned)blocks, threads, smem, s>>>(*A);
  return cudaGetLastError();
}

static cudaError_t reach_dispatch(ReachArgs* A, cudaStream_t s, int dev, uint64_t R, bool launch,
                                  int* blocks) {
  switch (pick_P(A->p)) {
    case 2: return reach_P<2>(A, s, dev, R, launch, blocks);
    case 4: return reach_P<4>(A, s, dev, R, launch, blocks);
    case 8: return reach_P<8>(A, s, dev, R, launch, blocks);
    case 16: return reach_P<16>(A, s, dev, R, launch, blocks);
    default: return reach_P<32>(A, s, dev, R, launch, blocks);
  }
}

// pool dedupe table entries per list: a power of two >= 2 * vmax (load <= 1/2)
static size_t reach_tab_size(int vmax) {
  size_t t = 64;
  while (t < 2 * (size_t)vmax) t <<= 1;
  return t;
}

cudaError_t reach_scratch_bytes(const DevTables& t, int p, int m, uint32_t R, int vmax,
                                size_t* bytes) {
  int dev = 0;
  cudaGetDevice(&dev);
  ReachArgs A{};
  A.t = t;
  A.p = p;
  A.m = m;
  A.vmax = vmax;
  // the larger of the two kernels' list counts (the decode replay uses k_reach)
  int lists = 0, lists_q = 0;
  cudaError_t e = reach_dispatch(&A, nullptr, dev, R, false, &lists);
  if (e != cudaSuccess) return e;
  int32_t dummy = 0;
  A.replay = &dummy;
  e = reach_dispatch(&A, nullptr, dev, R, false, &lists_q);
  if (e != cudaSuccess) return e;
  const size_t nl = (size_t)(lists > lists_q ? lists : lists_q);
  const size_t P = (size_t)pick_P(p);
  A.replay = nullptr;
  const size_t tab = reach_use_pool(&A) ? (size_t)lists * reach_tab_size(vmax) * 4 : 0;
  *bytes = nl * (size_t)vmax * (P * 2 + 8) + tab + 512;
  return cudaSuccess;
}

cudaError_t launch_reach(const DevTables& t, int p, int m, uint64_t seed, int radius,
                         uint32_t r_lo, uint32_t r_hi, int vmax, const int16_t* arg,
                         const int32_t* alg1_cuts, unsigned int* counter,
                         unsigned long long* key, unsigned long long* stats, int32_t* replay,
                         void* scratch, cudaStream_t s, uint32_t fastS) {
  int dev = 0;
  cudaGetDevice(&dev);
  ReachArgs A{};
  A.S = fastS;
  A.t = t;
  A.p = p;
  A.m = m;
  A.seed = seed;
  A.radius = radius;
  A.r_lo = r_lo;
  A.r_hi = r_hi;
  A.arg = arg;
  A.alg1 = alg1_cuts;
  A.counter = counter;
  A.key = key;
  A.vmax = vmax;
  A.stats = stats;
  A.replay = replay;
  int lists = 0;
  cudaError_t e = reach_dispatch(&A, s, dev, r_hi - r_lo, false, &lists);
  if (e != cudaSuccess) return e;
  const size_t nl = (size_t)lists;
  const size_t P = (size_t)pick_P(p);
  unsigned char* b = reinterpret_cast<unsigned char*>(scratch);
  A.g_cuts = reinterpret_cast<int16_t*>(b);
  b += nl * (size_t)vmax * P * 2;
  A.g_hash = reinterpret_cast<uint32_t*>(b);
  b += nl * (size_t)vmax * 4;
  A.g_queue = reinterpret_cast<uint32_t*>(b);
  b += nl * (size_t)vmax * 4;
  if (reach_use_pool(&A)) {
    b = reinterpret_cast<unsigned char*>(((uintptr_t)b + 255) & ~(uintptr_t)255);
    A.g_tab = reinterpret_cast<uint32_t*>(b);
    A.tab_size = (int)reach_tab_size(vmax);
    e = cudaMemsetAsync(A.g_tab, 0, nl * (size_t)A.tab_size * 4, s);
    if (e != cudaSuccess) return e;
  }
  return reach_dispatch(&A, s, dev, r_hi - r_lo, true, &lists);
}

size_t cpath_scratch_bytes(int p, int m) {
  const int rows = m + min(p - 1, m);
  const int P = pick_P(p);
  const size_t ops = (size_t)p * (2 * m + kMaxK);
  return 256 + (size_t)rows * 2 * 4 + 2 * (size_t)rows * P * 8 + (size_t)P * kMaxK * 8 +
         ops * 4 + 64;
}

template <int P>
static cudaError_t cpath_P(CpathArgs A, cudaStream_t s) {
  const size_t smem = tables_smem_bytes(A.t.npad, A.t.n);
  cudaError_t e = set_smem((const void*)k_cpath<P>, smem);
  if (e != cudaSuccess) return e;
  count_launch();
  k_cpath<P><<<1, 32, smem, s>>>(A);
  return cudaGetLastError();
}

cudaError_t launch_cpath(const DevTables& t, int p, int m, int k, const int32_t* cuts, OpRec* ops,
                         int cap, int32_t* len_master, int64_t* T, void* scratch,
                         cudaStream_t s) {
  const int rows = m + min(p - 1, m);
  const int P = pick_P(p);
  unsigned char* b = reinterpret_cast<unsigned char*>(scratch);
  CpathArgs A;
  A.t = t;
  A.p = p;
  A.m = m;
  A.k = k;
  A.cuts = cuts;
  A.ops = ops;
  A.cap = cap;
  A.len_master = len_master;
  A.T = T;
  size_t off = 0;
  auto take = [&](size_t bytes) {
    void* r = b + off;
    off += (bytes + 255) & ~size_t(255);
    return r;
  };
  A.bits = reinterpret_cast<uint32_t*>(take((size_t)rows * 2 * 4));
  A.finF = reinterpret_cast<int64_t*>(take((size_t)rows * P * 8));
  A.finB = reinterpret_cast<int64_t*>(take((size_t)rows * P * 8));
  A.finP = reinterpret_cast<int64_t*>(take((size_t)P * kMaxK * 8));
  A.order = reinterpret_cast<int*>(take((size_t)p * (2 * m + kMaxK) * 4));
  switch (P) {
    case 2: return cpath_P<2>(A, s);
    case 4: return cpath_P<4>(A, s);
    case 8: return cpath_P<8>(A, s);
    case 16: return cpath_P<16>(A, s);
    default: return cpath_P<32>(A, s);
  }
}

__global__ void k_widen16(const int16_t* src, int32_t* dst, int n) {
  for (int i = threadIdx.x; i < n; i += blockDim.x) dst[i] = src[i];
}
cudaError_t launch_widen16(const int16_t* src, int32_t* dst, int n, cudaStream_t s) {
  count_launch();
  k_widen16<<<1, 32, 0, s>>>(src, dst, n);
  return cudaGetLastError();
}

cudaError_t launch_init_key(unsigned long long* key, unsigned int* counter, cudaStream_t s) {
  count_launch();
  k_init_key<<<1, 1, 0, s>>>(key);
  if (counter) {
    cudaError_t e = cudaMemsetAsync(counter, 0, 3 * sizeof(unsigned int), s);  // cursors + redo count
    if (e != cudaSuccess) return e;
  }
  return cudaGetLastError();
}

cudaError_t launch_unrank(const DevTables& t, int p, uint64_t rank, int32_t* cuts,
                          cudaStream_t s) {
  count_launch();
  k_unrank<<<1, 32, 0, s>>>(t, p, rank, cuts);
  return cudaGetLastError();
}

}  // namespace apk
