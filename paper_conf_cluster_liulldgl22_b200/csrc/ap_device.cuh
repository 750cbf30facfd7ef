// ap_device.cuh -- device building blocks of the AutoPipe hot path (sm_100a).
//
// Shares nothing with oracle/.  Semantics follow DESIGN.md §2 (the readings of
// PAPER.md:103-125); see include/ap.h for the public contract.
//
// Row formulation of the 1F1B DAG.  With w_x = min(p-1-x, m) warm-up
// forwards on stage x (stage x owns max(0, m-p+x+1) 1F1B blocks), put
// F(x, j) in row y = j - w_x and B(x, y) in row y.  Inside a row every dependency
// points to an earlier row or to an op already visited by a forward pass over x
// ascending followed by a backward pass over x descending:
//   F(x,j): intra pred = last op of stage x (row y-1), cross pred F(x-1,j) in row
//           y-1 (w_{x-1} = w_x+1) or row y (both clamped to m);
//   B(x,y): intra pred = F(x, y+w_x) in this row, or the stage's last op;
//           cross pred B(x+1, y) in this row.
// So the whole simulation keeps 2p running values: FF[x] (finish of stage x's last
// forward) and L[x] (finish of stage x's last op).  Micro-batch 0's sliced forward
// F(x,0,q) only depends on other F(.,0,.) pieces, so it is computed first.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

#define AP_DEV_INLINE __device__ __forceinline__

// Device-side bounds checks (AP_DEBUG_CHECKS=1 builds only; the product build compiles
// them out).  The GPU pool refuses compute-sanitizer, so tests/test_gpu_debug_checks.py
// builds this variant and drives every kernel family with it: a failed check prints
// its location and traps, which fails the call.
#ifndef AP_DEBUG_CHECKS
#define AP_DEBUG_CHECKS 0
#endif
#if AP_DEBUG_CHECKS
#include <cstdio>
#define AP_CHECK(cond)                                                                   \
  do {                                                                                   \
    if (!(cond)) {                                                                       \
      printf("AP_CHECK failed %s:%d: %s (block %d thread %d)\n", __FILE__, __LINE__,     \
             #cond, (int)blockIdx.x, (int)threadIdx.x);                                  \
      __trap();                                                                          \
    }                                                                                    \
  } while (0)
#else
#define AP_CHECK(cond) ((void)0)
#endif

namespace apdev {

constexpr int kMaxP = 32;
constexpr int kMaxK = 16;
constexpr int kMaxN = 512;  // AP_MAX_N

AP_DEV_INLINE uint32_t smem_addr(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

// ---------------------------------------------------------------------------
// K4 prologue: one TMA bulk copy (cp.async.bulk + mbarrier complete_tx) of the
// plan's [f | b | comm] int64 table (3*npad entries, npad even => 16-B multiple)
// into shared memory, then warp-shuffle inclusive scans -> Pf[0..n], Pb[0..n].
AP_DEV_INLINE void tma_stage_tables(const int64_t* g_tab, int npad, int64_t* s_raw,
                                    uint64_t* s_mbar) {
  const uint32_t bytes = 3u * static_cast<uint32_t>(npad) * 8u;
  const uint32_t mbar = smem_addr(s_mbar);
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(mbar) : "memory");
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(mbar),
                 "r"(bytes)
                 : "memory");
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, "
        "[%3];" ::"r"(smem_addr(s_raw)),
        "l"(g_tab), "r"(bytes), "r"(mbar)
        : "memory");
  }
  asm volatile(
      "{\n"
      ".reg .pred P1;\n"
      "AP_WAIT_%=:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], 0;\n"
      "@!P1 bra AP_WAIT_%=;\n"
      "}\n" ::"r"(mbar)
      : "memory");
}

// Warp 0 scans f and b (chunks of 32 with a carried offset).  Caller syncs after.
AP_DEV_INLINE void warp_prefix(const int64_t* s_f, const int64_t* s_b, int n, int64_t* s_Pf,
                               int64_t* s_Pb) {
  if (threadIdx.x >= 32) return;
  const int lane = threadIdx.x;
  int64_t cf = 0, cb = 0;
  if (lane == 0) {
    s_Pf[0] = 0;
    s_Pb[0] = 0;
  }
  for (int base = 0; base < n; base += 32) {
    const int i = base + lane;
    int64_t vf = (i < n) ? s_f[i] : 0;
    int64_t vb = (i < n) ? s_b[i] : 0;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const int64_t tf = __shfl_up_sync(0xffffffffu, vf, o);
      const int64_t tb = __shfl_up_sync(0xffffffffu, vb, o);
      if (lane >= o) {
        vf += tf;
        vb += tb;
      }
    }
    if (i < n) {
      s_Pf[i + 1] = cf + vf;
      s_Pb[i + 1] = cb + vb;
    }
    cf += __shfl_sync(0xffffffffu, vf, 31);
    cb += __shfl_sync(0xffffffffu, vb, 31);
  }
}

// Shared-memory footprint of the staged tables (bytes), and their carving.
struct Tables {
  const int64_t* f;
  const int64_t* b;
  const int64_t* comm;
  const int64_t* Pf;
  const int64_t* Pb;
};
__host__ __device__ inline size_t tables_smem_bytes(int npad, int n) {
  return 16 /*mbarrier*/ + 3ull * npad * 8 + 2ull * (n + 2) * 8;
}
// Stage + scan.  Returns pointers into `smem` and the first free byte offset.
AP_DEV_INLINE Tables stage_and_scan(const int64_t* g_tab, int n, int npad, unsigned char* smem,
                                    size_t* used) {
  uint64_t* s_mbar = reinterpret_cast<uint64_t*>(smem);
  int64_t* s_raw = reinterpret_cast<int64_t*>(smem + 16);
  int64_t* s_Pf = s_raw + 3 * npad;
  int64_t* s_Pb = s_Pf + (n + 2);
  tma_stage_tables(g_tab, npad, s_raw, s_mbar);
  warp_prefix(s_raw, s_raw + npad, n, s_Pf, s_Pb);
  __syncthreads();
  *used = tables_smem_bytes(npad, n);
  return Tables{s_raw, s_raw + npad, s_raw + 2 * npad, s_Pf, s_Pb};
}

// ---------------------------------------------------------------------------
// Stage totals for a cut vector (PAPER.md:113 f_x, b_x; reading Q4 for C_x).
// c[0..p] with c[0]=0, c[p]=n.  C[x] = comm leaving stage x (0 for x = p-1).
template <int P>
AP_DEV_INLINE void stage_costs(const Tables& t, int p, const int (&c)[P + 1], int64_t (&F)[P],
                               int64_t (&B)[P], int64_t (&C)[P]) {
#pragma unroll
  for (int x = 0; x < P; ++x) {
    if (x < p) {
      F[x] = t.Pf[c[x + 1]] - t.Pf[c[x]];
      B[x] = t.Pb[c[x + 1]] - t.Pb[c[x]];
      C[x] = (x < p - 1) ? t.comm[c[x + 1] - 1] : 0;
    } else {
      F[x] = 0;
      B[x] = 0;
      C[x] = 0;
    }
  }
}

// ---------------------------------------------------------------------------
// Decision-bit storage: per simulated candidate, one row word per row of the
// sweep (P <= 16: F bits [0,16), B bits [16,32); P = 32: two words).  `base` +
// (row*WPR + w)*stride addresses one lane's word; the lanes of a block (shared
// memory) or grid (global scratch) are interleaved so stores coalesce.
template <int P>
struct BitsLayout {
  static constexpr int WPR = (P <= 16) ? 1 : 2;
  static constexpr int BSHIFT = (P <= 16) ? 16 : 0;
  static constexpr int BWORD = (P <= 16) ? 0 : 1;
};
struct BitsRef {
  uint32_t* base;
  int stride;
};

// Optional per-op finish-time capture (critical-path kernel only).
struct TimesRef {
  int64_t* fin_F;  // [rows][P]  finish of F(x, j) at row j - w_x + W0
  int64_t* fin_B;  // [rows][P]  finish of B(x, y) at row y + W0
  int64_t* fin_P;  // [P][kMaxK] finish of piece q of F(x, 0)
};

// ---------------------------------------------------------------------------
// Exact int64 simulation of one candidate with runtime p <= P, any m >= 1,
// k in [1, kMaxK].  MODE 0: T only.  MODE 1: + decision bits.  MODE 2: + times.
// Decision bit of an op with two predecessors = "the cross-stage predecessor is
// the binding one" under the tie rule of PAPER.md:101 / reading Q10: for FP the
// intra-stage predecessor (stage x) outranks the cross one (x-1), so bit = cross >
// intra; for BP the cross one (x+1) outranks, so bit = cross >= intra.
template <int P, int MODE>
AP_DEV_INLINE int64_t sim_exact(int p, int m, int k, const int64_t (&F)[P],
                                const int64_t (&B)[P], const int64_t (&C)[P], BitsRef br,
                                uint32_t (&pbits)[P], TimesRef tr) {
  using BL = BitsLayout<P>;
  int64_t wF[P], wB[P], FF[P], L[P];
  int w[P];
#pragma unroll
  for (int x = 0; x < P; ++x) {
    wF[x] = F[x] + ((x > 0) ? C[x - 1] : 0);         // Comm charged on receiver (Q2)
    wB[x] = B[x] + ((x < p - 1) ? C[x] : 0);
    w[x] = min(p - 1 - x, m);
    pbits[x] = 0;
  }
  // ---- micro-batch 0's forward: k pieces per stage (reading Q6)
  if (k == 1) {
#pragma unroll
    for (int x = 0; x < P; ++x) {
      if (x < p) {
        FF[x] = ((x > 0) ? FF[x - 1] : 0) + wF[x];
        if (MODE == 2) tr.fin_P[x * kMaxK + 0] = FF[x];
      }
    }
  } else {
    int64_t a[P], al[P];
#pragma unroll
    for (int x = 0; x < P; ++x) {
      a[x] = F[x] / k + ((x > 0) ? C[x - 1] / k : 0);
      al[x] = wF[x] - (int64_t)(k - 1) * a[x];
      FF[x] = 0;
    }
    for (int q = 0; q < k; ++q) {
#pragma unroll
      for (int x = 0; x < P; ++x) {
        if (x < p) {
          const int64_t wq = (q < k - 1) ? a[x] : al[x];
          if (x == 0) {
            FF[0] = FF[0] + wq;
          } else if (q == 0) {
            FF[x] = FF[x - 1] + wq;
          } else {
            const int64_t cr = FF[x - 1], in = FF[x];
            if (MODE >= 1) pbits[x] |= (cr > in ? 1u : 0u) << q;
            FF[x] = max(cr, in) + wq;
          }
          if (MODE == 2) tr.fin_P[x * kMaxK + q] = FF[x];
        }
      }
    }
  }
#pragma unroll
  for (int x = 0; x < P; ++x) L[x] = FF[x];
  // ---- rows
  const int W0 = min(p - 1, m);
  for (int y = -W0; y < m; ++y) {
    uint32_t fbits = 0, bbits = 0;
    int64_t prev_old = 0;
#pragma unroll
    for (int x = 0; x < P; ++x) {
      if (x < p) {
        const int j = y + w[x];
        const int64_t old = FF[x];
        if (j >= 1 && j < m) {
          const int64_t in = L[x];
          int64_t v;
          if (x == 0) {
            v = in + wF[0];
          } else {
            const int64_t cr = (w[x - 1] == w[x] + 1) ? prev_old : FF[x - 1];
            if (MODE >= 1) fbits |= (cr > in ? 1u : 0u) << x;
            v = max(cr, in) + wF[x];
          }
          FF[x] = v;
          L[x] = v;
          if (MODE == 2) tr.fin_F[(y + W0) * P + x] = v;
        }
        prev_old = old;
      }
    }
    if (y >= 0) {
      int64_t bprev = 0;
#pragma unroll
      for (int x = P - 1; x >= 0; --x) {
        if (x < p) {
          const int64_t in = L[x];
          int64_t v;
          if (x == p - 1) {
            v = in + wB[x];
          } else {
            if (MODE >= 1) bbits |= (bprev >= in ? 1u : 0u) << (x + BL::BSHIFT);
            v = max(bprev, in) + wB[x];
          }
          L[x] = v;
          bprev = v;
          if (MODE == 2) tr.fin_B[(y + W0) * P + x] = v;
        }
      }
    }
    if (MODE >= 1) {
      const int row = y + W0;
      if (BL::WPR == 1) {
        br.base[(size_t)row * br.stride] = fbits | bbits;
      } else {
        br.base[(size_t)(row * 2) * br.stride] = fbits;
        br.base[(size_t)(row * 2 + 1) * br.stride] = bbits;
      }
    }
  }
  return L[0];
}

// The paper's Slicer form: micro-batches 0..s-1 have their
// forward split into k pieces (s = 0: none).  Same row sweep as sim_exact (MODE 0,
// T only).  A sliced F(x, j, q) depends on F(x-1, j, q) and on the stage's previous
// op (piece q-1, or for q = 0 the stage's last op L[x]).  PV[x][.] holds the pieces
// of stage x's latest sliced forward; because the forward pass runs x ascending and
// stage x-1 may already have sliced F(x-1, j+1) in this row (w_{x-1} = w_x + 1),
// the cross pieces are taken from a copy saved before that overwrite.
template <int P>
AP_DEV_INLINE int64_t sim_sliced(int p, int m, int s, int k, const int64_t (&F)[P],
                                 const int64_t (&B)[P], const int64_t (&C)[P]) {
  if (s <= 0) k = 1;
  if (k <= 1) s = 0;
  int64_t wF[P], wB[P], FF[P], L[P];
  int w[P];
  int64_t PV[P][kMaxK];
#pragma unroll
  for (int x = 0; x < P; ++x) {
    wF[x] = F[x] + ((x > 0) ? C[x - 1] : 0);
    wB[x] = B[x] + ((x < p - 1) ? C[x] : 0);
    w[x] = min(p - 1 - x, m);
  }
  auto piece_w = [&](int x, int q) -> int64_t {  // split(F_x,k,q) + split(C_{x-1},k,q)
    const int64_t f0 = F[x] / k, c0 = (x > 0) ? C[x - 1] / k : 0;
    return (q < k - 1) ? f0 + c0 : (F[x] - (int64_t)(k - 1) * f0) + ((x > 0) ? C[x - 1] - (int64_t)(k - 1) * c0 : 0);
  };
  // micro-batch 0's forwards (all pieces; they only depend on each other)
  if (s == 0) {
#pragma unroll
    for (int x = 0; x < P; ++x)
      if (x < p) FF[x] = ((x > 0) ? FF[x - 1] : 0) + wF[x];
  } else {
#pragma unroll
    for (int x = 0; x < P; ++x) FF[x] = 0;
    for (int q = 0; q < k; ++q) {
#pragma unroll
      for (int x = 0; x < P; ++x) {
        if (x < p) {
          const int64_t wq = piece_w(x, q);
          if (x == 0) FF[0] = FF[0] + wq;
          else if (q == 0) FF[x] = FF[x - 1] + wq;
          else FF[x] = max(FF[x - 1], FF[x]) + wq;
          PV[x][q] = FF[x];
        }
      }
    }
  }
#pragma unroll
  for (int x = 0; x < P; ++x) L[x] = FF[x];
  const int W0 = min(p - 1, m);
  for (int y = -W0; y < m; ++y) {
    int64_t prev_old = 0;
    int64_t prevPV[kMaxK];
#pragma unroll
    for (int x = 0; x < P; ++x) {
      if (x < p) {
        const int j = y + w[x];
        const int64_t old = FF[x];
        const bool sliced = (j >= 1 && j < m && j < s);
        int64_t savePV[kMaxK];
        if (sliced)
          for (int q = 0; q < k; ++q) savePV[q] = PV[x][q];
        if (j >= 1 && j < m) {
          const bool use_old = (x > 0) && (w[x - 1] == w[x] + 1);
          if (sliced) {
            int64_t run = L[x];
            for (int q = 0; q < k; ++q) {
              int64_t in = run;
              if (x > 0) {
                const int64_t cr = use_old ? prevPV[q] : PV[x - 1][q];
                in = max(cr, in);
              }
              run = in + piece_w(x, q);
              PV[x][q] = run;
            }
            FF[x] = run;
            L[x] = run;
          } else {
            const int64_t in = L[x];
            int64_t v;
            if (x == 0) {
              v = in + wF[0];
            } else {
              const int64_t cr = use_old ? prev_old : FF[x - 1];
              v = max(cr, in) + wF[x];
            }
            FF[x] = v;
            L[x] = v;
          }
        }
        prev_old = old;
        if (sliced) {
          for (int q = 0; q < k; ++q) prevPV[q] = savePV[q];
        } else {
          for (int q = 0; q < k; ++q) prevPV[q] = PV[x][q];
        }
      }
    }
    if (y >= 0) {
      int64_t bprev = 0;
#pragma unroll
      for (int x = P - 1; x >= 0; --x) {
        if (x < p) {
          const int64_t in = L[x];
          const int64_t v = (x == p - 1) ? in + wB[x] : max(bprev, in) + wB[x];
          L[x] = v;
          bprev = v;
        }
      }
    }
  }
  return L[0];
}

// Backtrack the unique critical path from B(0, m-1) using the decision bits and
// return the master stage: most path ops in the 1F1B phase (F(x,j) with j >= w_x,
// B(x,y) with y < m - w_x; slice pieces count individually), ties -> higher stage,
// p-1 if none (readings Q10, Q11).  `emit(kind, x, j, q)` is called sink -> source.
template <int P, typename Emit>
AP_DEV_INLINE int backtrack_master(int p, int m, int k, BitsRef br, const uint32_t (&pbits)[P],
                                   int* path_len, Emit emit) {
  using BL = BitsLayout<P>;
  int cnt[P];
#pragma unroll
  for (int x = 0; x < P; ++x) cnt[x] = 0;
  const int W0 = min(p - 1, m);
  int kind = 1, x = 0, j = m - 1, q = 0, len = 0;
  for (;;) {
    ++len;
    const int wx = min(p - 1 - x, m);
    emit(kind, x, j, q);
    if (kind == 1) {
      if (j < m - wx) cnt[x]++;
      const int y = j;
      bool cross = false;
      if (x < p - 1) {
        const uint32_t word = br.base[(size_t)((y + W0) * BL::WPR + BL::BWORD) * br.stride];
        cross = (word >> (x + BL::BSHIFT)) & 1u;
      }
      if (cross) {
        ++x;
        continue;
      }
      const int jf = y + wx;
      if (jf <= m - 1) {  // F(x, y + w_x) just before it in the same row
        kind = 0;
        j = jf;
        q = (jf == 0) ? k - 1 : 0;
      } else if (y >= 1) {  // previous BP of the stage
        j = y - 1;
      } else {  // w_x = m: the stage's last forward F(x, m-1)
        kind = 0;
        j = m - 1;
        q = (j == 0) ? k - 1 : 0;
      }
    } else {
      if (j >= wx) cnt[x]++;
      if (j == 0) {  // slice pieces of micro-batch 0
        if (x == 0) {
          if (q == 0) break;  // the source F(0, 0, 0)
          --q;
        } else if (q == 0) {
          --x;
        } else {
          if ((pbits[x] >> q) & 1u) --x;
          else --q;
        }
        continue;
      }
      bool cross = false;
      if (x > 0) {
        const uint32_t word = br.base[(size_t)((j - wx + W0) * BL::WPR) * br.stride];
        cross = (word >> x) & 1u;
      }
      if (cross) {
        --x;
        q = 0;
        continue;
      }
      if (j > wx) {  // 1F1B: the previous op is B(x, j - w_x - 1)
        kind = 1;
        j = j - wx - 1;
      } else {  // warm-up: F(x, j-1)
        j = j - 1;
        q = (j == 0) ? k - 1 : 0;
      }
    }
  }
  int best = p - 1;
#pragma unroll
  for (int xx = P - 1; xx >= 0; --xx)
    if (xx < p && cnt[xx] > cnt[best]) best = xx;
  *path_len = len;
  return best;
}

struct NoEmit {
  AP_DEV_INLINE void operator()(int, int, int, int) const {}
};

// splitmix64 (Steele, Lea, Flood 2014) -- the restart seed mixer of reading Q21.
AP_DEV_INLINE uint64_t splitmix64(uint64_t s) {
  uint64_t z = s + 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

}  // namespace apdev
