// ap_launch.h -- internal interface between the C-ABI host layer (ap_host.cu) and
// the kernels (ap_kernels.cu).  Not part of the public ABI.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace apk {

struct DevTables {
  const int64_t* tab;     // [f | b | comm], 3*npad int64, 16-B aligned (TMA source)
  const uint64_t* binom;  // C(a, b) for a in [0, n], b in [0, 32], saturating
  int n;
  int npad;
};

// Algorithm 1 on the device: arg table int16[(n+1)*(p+1)],
// the Alg.-1 cut vector int32[p-1] and its value.
cudaError_t launch_alg1(const DevTables& t, int p, int16_t* arg, int32_t* cuts, int64_t* value,
                        cudaStream_t s);

// Certified minLB: arg scratch int16[(n+1)*(p+1)], argmin cuts int32[p-1].
cudaError_t launch_minlb(const DevTables& t, int p, int m, int K, int16_t* arg, int32_t* cuts,
                         int64_t* value, cudaStream_t s);

// Generic exact evaluation of `count` candidates.  cuts_stride = p-1 (batch) or 0
// (all rows share one cut vector).  k source: kptr if non-null, else k_iota ? row+1
// : k_const.  master may be null.  Invalid rows -> time -1, master -1, and +1 on
// *n_invalid if given (zeroed first, stream-ordered).
cudaError_t launch_eval(const DevTables& t, cudaMemPool_t pool, int p, int m, const int32_t* cuts,
                        int cuts_stride,
                        const int32_t* kptr, int k_const, int k_iota, int64_t count,
                        int64_t* time_ns, int32_t* master, cudaStream_t s, int* launches,
                        int s_const = 1, int s_iota = 0, uint32_t fastS = 0, int fastCR = 16,
                        int div1 = 0, unsigned long long* n_invalid = nullptr);

// Sweep parameters that depend on T_ref, computed on the device by k_sweep_prep right
// after the T_ref evaluation and read by the sweep kernels at their start, so a search
// never waits for the host.
struct SweepDev {
  unsigned long long S;  // T_ref + 1 (a candidate with T >= S cannot win)
  long long tref;
  int u32;               // 1: the u32 saturating kernel runs, 0: the int64 one
  int clamp_first, clamp_rows, clamp_final;  // u32 clamp schedule
  int skip;              // 1: the packed key does not fit; *key = AP_KEY_RANGE, no sweep
  int pad;
};
// Host-known inputs of k_sweep_prep.
struct PrepArgs {
  const long long* trefs;     // T(Alg.-1 partition, k), nk entries
  int nk;
  int p, m, rb;
  int try_u32;                // the u32 kernel exists for this search (exact p, no override)
  unsigned long long wrow;    // max growth of a running value per row (< 2^62)
  long long t_bound;          // caller's attained bound (INT64_MAX: none)
  unsigned long long* key;    // packed-key searches: written with AP_KEY_RANGE on overflow
  // memory mode: the Alg.-1 partition must fit, else T_ref = mem_tot
  const int32_t* a1;          // Alg.-1 cut vector (device)
  const int64_t* mem;         // [2][n+1] static / stash prefix sums, or null
  int64_t mem_cap;
  long long mem_tot;
  int n;
};
cudaError_t launch_sweep_prep(const PrepArgs& a, SweepDev* out, cudaStream_t s);

struct SweepPlan {
  int fast_u32;   // exact u32 saturating sweep
  int exact_p;    // kernel specialised to this p
  int blocks, threads;
  uint64_t chunk;
  int clamp_rows;
};
// Exhaustive sweep of ranks [rank_lo, rank_hi) x k in [k_lo, k_hi].  S = T_ref + 1:
// a candidate with T >= S can never win.  atomicMin into *key (init it first).
// ctr (8 B, device): the p-specialised kernel then runs persistent with warp-dynamic
// work units (zeroed here, stream-ordered); null = static per-thread chunks.
// u32 clamp schedule: clamp_first steady rows before the first clamp (-1: legacy =
// clamp after the warm-up and at the end), then every clamp_rows, clamp_final = one
// more clamp at the end of the steady rows.
// The sweep reads S and the clamp schedule from `dp` (k_sweep_prep).  With try_u32 the
// u32 and the int64 kernels are both launched and each returns at once unless dp->u32
// selects it; plan_out->blocks is the larger grid (records of two-phase searches are
// preset to "empty" so the idle variant's slots are neutral).
cudaError_t launch_sweep(const DevTables& t, int p, int m, int k_lo, int k_hi, uint64_t rank_lo,
                         uint64_t rank_hi, const SweepDev* dp, int rb, int try_u32,
                         int force_generic, int mode, unsigned long long* key, cudaStream_t s,
                         SweepPlan* plan_out, unsigned long long* rec = nullptr,
                         const int64_t* mem = nullptr, int64_t mem_cap = 0,
                         unsigned long long* ctr = nullptr, int div1 = 0);
// The host-side test whether the p-specialised kernel serves this (p, m, mode).
bool sweep_has_exact(int p, int m, int mode, int force_generic, bool mem);

// Two-phase reduction (NEXT N3).  With `rec` (u64[2 * sweep_max_blocks(dev)]) passed
// to launch_sweep, each CTA stores its lexicographic min (T, index) there instead of
// packing a key; launch_reduce2 reduces plan_out->blocks records into out[0] = T,
// out[1] = index.  launch_key2_select: *idx = local[1] if local[0] == *t_star else
// INT64_MAX (the second all-reduce's operand).
int sweep_max_blocks(int dev);
cudaError_t launch_reduce2(const unsigned long long* rec, int nrec, long long* out,
                           cudaStream_t s);
cudaError_t launch_key2_select(const long long* local, const long long* t_star, long long* idx,
                               cudaStream_t s);

// Heuristic restarts [r_lo, r_hi); key = min (T << 20 | r).  replay_cuts (int32[p-1])
// non-null: single-restart replay writing that restart's best cut vector.  counter
// must hold 3 + (r_hi - r_lo) words (cursors, redo count, redo ids).  fastS > 0 enables
// the u32 pass (restarts that saturate are redone by an exact int64 pass).
cudaError_t launch_heuristic(const DevTables& t, int p, int m, uint64_t seed, int radius,
                             uint32_t r_lo, uint32_t r_hi, const int16_t* arg,
                             const int32_t* alg1_cuts, unsigned int* counter,
                             unsigned long long* key, int32_t* replay_cuts,
                             unsigned long long* sims, int16_t* best_out, uint32_t fastS,
                             int fastCR, int adjust_mode, cudaStream_t s);

struct OpRec {
  int32_t stage, kind, microbatch, piece;
  int64_t start_ns, end_ns;
};
// Critical path of one candidate: ops (source -> sink) into `ops` (cap entries),
// len, master, T.  scratch: device bytes >= cpath_scratch_bytes(p, m).
size_t cpath_scratch_bytes(int p, int m);
cudaError_t launch_cpath(const DevTables& t, int p, int m, int k, const int32_t* cuts, OpRec* ops,
                         int cap, int32_t* len_master, int64_t* T, void* scratch,
                         cudaStream_t s);

// key = INT64_MAX (and counter[0..2] = 0 if non-null); precedes launch_sweep/heuristic.
cudaError_t launch_init_key(unsigned long long* key, unsigned int* counter, cudaStream_t s);
// dst[i] = src[i] for i < n (int16 -> int32), one warp
cudaError_t launch_widen16(const int16_t* src, int32_t* dst, int n, cudaStream_t s);

// Reachable-set search (NEXT N1): restarts [r_lo, r_hi), key = min (T << 20 | r).
// scratch: reach_scratch_bytes() for the same (p, m, R = r_hi - r_lo, vmax); counter[0]
// zeroed (launch_init_key); stats (u64[2]: sims, truncated restarts) zeroed or NULL;
// replay (int32[p-1]) non-null: the single restart r_lo's best cut vector.
cudaError_t reach_scratch_bytes(const DevTables& t, int p, int m, uint32_t R, int vmax,
                                size_t* bytes);
cudaError_t launch_reach(const DevTables& t, int p, int m, uint64_t seed, int radius,
                         uint32_t r_lo, uint32_t r_hi, int vmax, const int16_t* arg,
                         const int32_t* alg1_cuts, unsigned int* counter,
                         unsigned long long* key, unsigned long long* stats, int32_t* replay,
                         void* scratch, cudaStream_t s, uint32_t fastS = 0);

// Decode helper: unrank lex rank -> cut vector int32[p-1].
cudaError_t launch_unrank(const DevTables& t, int p, uint64_t rank, int32_t* cuts,
                          cudaStream_t s);

// Algorithm 2 on the device: mb (int32) for one cut vector.
cudaError_t launch_alg2(const DevTables& t, int p, const int32_t* cuts, int reading, int32_t* mb,
                        cudaStream_t s);

int num_sms(int device);

// Kernels launched by the library since load (all threads, all devices).
unsigned long long kernel_launches();

}  // namespace apk
