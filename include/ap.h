/*
 * ap.h -- C ABI of the B200-native AutoPipe planner/slicer hot path.
 *
 * The library (paper_conf_cluster_liulldgl22_b200/libap.so, sm_100a) simulates
 * candidate pipeline partitions under the 1F1B schedule and searches them.  Every
 * step of the path runs in CUDA kernels; the host code only validates, allocates
 * and launches.  No exceptions and no torch types cross this boundary.
 *
 * Citations: "PAPER.md:N" is line N of the AutoPipe paper text (Liu et al., IEEE
 * CLUSTER 2022) with the section/equation/algorithm it belongs to; DESIGN.md
 * readings Q1..Q26 fix what the paper leaves open.
 *
 * Conventions for every call:
 *  - Times are int64 nanoseconds.  Results are bit-exact with the CPU oracle.
 *  - Sub-layer i in [0,n) is one block of the model (Fig. 3: embedding,
 *    ResidualAttentionBlock / ResidualFFNBlock halves of each layer, head).
 *  - A partition of n sub-layers into p stages is its cut vector
 *    cuts[0..p-2] = (c_1 < ... < c_{p-1}), every c in [1, n-1]; stage x owns
 *    sub-layers [c_x, c_{x+1}) with c_0 = 0, c_p = n.
 *    Partitions are ranked in lexicographic order of their cut vectors.
 *  - Ownership: the plan owns its device tables.  The caller owns every buffer it
 *    passes.  Device pointers must be on the plan's device.
 *  - Synchronisation: calls that write device outputs are asynchronous and
 *    stream-ordered on `stream` (ap_eval_batch, ap_search_*): nothing in them waits
 *    for the device (the reference time T_ref and everything derived from it are
 *    computed and consumed on the device), so they can be captured in a CUDA graph.
 *    Calls with host outputs block until they are ready.
 *  - Errors: every call returns an ap_status.  The message of the most recent
 *    failure on the calling thread is available from ap_last_error().  On error
 *    the outputs are unspecified.  A missing/unsupported GPU is AP_ERR_CUDA: there
 *    is no CPU fallback.
 *  - Thread safety: a plan is immutable after creation; concurrent calls on
 *    different streams are safe.
 */
#ifndef AP_H_
#define AP_H_

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct CUstream_st* ap_stream_t; /* == cudaStream_t; NULL = legacy default */

#define AP_MAX_P 32   /* pipeline stages  */
#define AP_MAX_K 16   /* slice pieces of micro-batch 0 */
#define AP_MAX_N 512  /* sub-layers       */

/* Packed exhaustive key written when T_ref << rb | index does not fit in 63 bits (the
 * test needs T_ref, known only on the device, so it cannot be a return status of the
 * asynchronous call).  It is the least int64, so all_reduce(MIN) over ranks keeps it
 * and every rank switches to ap_search_exhaustive2 together; ap_decode returns
 * AP_ERR_RANGE for it. */
#define AP_KEY_RANGE ((int64_t)(-9223372036854775807LL - 1))

typedef enum {
  AP_OK = 0,
  AP_ERR_INVALID = 1,  /* argument out of its documented domain          */
  AP_ERR_RANGE = 2,    /* int64 overflow guard or 63-bit key packing      */
  AP_ERR_CUDA = 3,     /* CUDA runtime error / no sm_100 device           */
  AP_ERR_NOMEM = 4,    /* device or host allocation failed                */
  AP_ERR_CAPACITY = 5  /* caller buffer too small                         */
} ap_status;

/* Message describing the last failure on this thread ("" if none). */
const char* ap_last_error(void);

/* Library version string and the compute capability it was built for. */
const char* ap_version(void);

typedef struct ap_plan ap_plan; /* opaque, immutable after create */

/*
 * ap_plan_create -- stage the model's profiled costs on `device`.
 * PAPER.md:81 (§III-A "model configs ... runtime statistics"), Alg. 1 line 1
 * ("Get forward time f_i and backward time b_i for block i").
 *   n                 number of sub-layers, 1 <= n <= AP_MAX_N
 *   fwd_ns, bwd_ns    host int64[n], >= 0: forward / backward time of sub-layer i
 *   act_bytes         host int64[n], >= 0: bytes of the activation leaving sub-layer
 *                     i (= the gradient entering it); entry n-1 is ignored
 *   link_bytes_per_s  > 0.  comm_ns[i] = ceil(act_bytes[i]*1e9 / link), 128-bit
 *                     exact ("Comm"; BASELINE north_star "activation
 *                     bytes over link bandwidth"; reading Q4/Q25)
 *   device            CUDA ordinal; must be an sm_100 (B200) device
 *   out               receives the plan
 * Copies the tables host->device once (blocking).  Errors: INVALID, RANGE (a sum
 * that cannot be held in int64), CUDA, NOMEM.
 */
ap_status ap_plan_create(int32_t n, const int64_t* fwd_ns, const int64_t* bwd_ns,
                         const int64_t* act_bytes, uint64_t link_bytes_per_s,
                         int32_t device, ap_plan** out);

/* Release a plan and its device memory.  NULL-safe.  The caller must first make
 * sure no work using the plan is still pending on any stream (synchronise the
 * streams of earlier asynchronous calls); the memory is returned stream-ordered to
 * the library's per-device pool. */
void ap_plan_destroy(ap_plan* plan);

/* Number of sub-layers and comm_ns table (host copy) of a plan.  comm may be NULL. */
ap_status ap_plan_info(const ap_plan* plan, int32_t* n, int64_t* comm_ns);

/*
 * ap_plan_set_memory -- attach the memory model of NEXT N4 (reading R-N4) to
 * a plan, for AP_SEARCH_MEMORY searches and the outer loop over pipeline depth.
 *   static_bytes  host int64[n] >= 0: bytes a sub-layer holds for the whole iteration
 *                 on its stage (weights, gradients, optimizer state).
 *   stash_bytes   host int64[n] >= 0: bytes it keeps per in-flight micro-batch between
 *                 FP and BP (with activation checkpointing: its input).
 *   cap_bytes     per-GPU capacity available to these two terms.
 * Replaces a previous model.  Not synchronised with searches running on the plan.
 * Errors: INVALID (NULL, negative), RANGE (sum(static) + 32*sum(stash) >= 2^62), NOMEM.
 */
ap_status ap_plan_set_memory(ap_plan* plan, const int64_t* static_bytes,
                             const int64_t* stash_bytes, int64_t cap_bytes);

/* C(n-1, p-1): the size of the partition space.  RANGE when it
 * is >= 2^63.  INVALID unless 1 <= p <= n. */
ap_status ap_count(int32_t n, int32_t p, uint64_t* out);

/*
 * ap_eval_batch -- iteration time (and master stage) of `count` candidates.
 * The pipeline simulator of PAPER.md:103-125 (§III-B-1): 1F1B with m micro-batches
 * (warm-up simulated exactly, reading Q1), Comm charged on the receiving stage
 * (PAPER.md:115, :123), micro-batch 0's forward split into k pieces
 * (PAPER.md:202-204 Slicer; BASELINE north_star).  T = end of the last backward of
 * stage 0.  master = stage most visited by the unique critical path
 * in the 1F1B phase (readings Q10, Q11).
 *   p in [1, min(n, AP_MAX_P)], m >= 1 (m <= 1<<20)
 *   cuts     device int32 [count][p-1], row-major, each row a valid cut vector
 *   k        device int32 [count] in [1, AP_MAX_K], or NULL for k = 1
 *   count    >= 0
 *   time_ns  device int64 [count] (written)
 *   master   device int32 [count] (written) or NULL to skip the critical path
 * Asynchronous on `stream`.  INVALID cut vectors or k produce time_ns = -1 and
 * master = -1 for that row (validated on the device, the call still returns OK).
 * RANGE if the overflow guard m*(sum f + sum b) + 2m(p-1)*max comm >= 2^62 trips.
 */
ap_status ap_eval_batch(const ap_plan* plan, int32_t p, int32_t m, const int32_t* cuts,
                        const int32_t* k, int64_t count, int64_t* time_ns, int32_t* master,
                        ap_stream_t stream);

/*
 * ap_eval_batch_ex -- ap_eval_batch that also reports how many rows were invalid (the
 * rows it writes as time_ns = -1, master = -1: a cut vector that is not strictly
 * increasing in [1, n-1], or k outside [1, AP_MAX_K]), so a caller can tell "some
 * candidates were malformed" apart from a plain OK without scanning the outputs.
 *   n_invalid  device int64 [1] or NULL; zeroed and then incremented on `stream`
 *              (stream-ordered: read it after the stream has reached this call).
 * Everything else as ap_eval_batch (which is ap_eval_batch_ex with n_invalid = NULL).
 */
ap_status ap_eval_batch_ex(const ap_plan* plan, int32_t p, int32_t m, const int32_t* cuts,
                           const int32_t* k, int64_t count, int64_t* time_ns, int32_t* master,
                           int64_t* n_invalid, ap_stream_t stream);

/*
 * ap_search_exhaustive -- exact argmin over a contiguous slice of the search space.
 * Simulates every partition with lex rank in [rank_lo, rank_hi) for every
 * k in [k_lo, k_hi] (each (partition, k) pair fully simulated, no pruning) and
 * writes ONE packed int64 key to device memory:
 *     key = T << rb | (rank*(k_hi-k_lo+1) + k - k_lo),  rb = bitlen(N*K - 1),
 * N = C(n-1,p-1), K = k_hi-k_lo+1, or INT64_MAX if the slice holds no candidate
 * with T < T_ref+1, where T_ref = min over k in [k_lo, k_hi] of T(Algorithm 1
 * partition, k) is an attained upper bound on the optimum.  The minimum key over all slices is
 * the lexicographic min of (T, rank, k) ("Return the partition scheme
 * with minimum iteration time"; reading Q15), so the keys of disjoint slices on
 * different GPUs combine with one all_reduce(MIN) (BASELINE north_star).
 *   key     device int64[1] (written); AP_KEY_RANGE if T_ref << rb does not fit in 63
 *           bits (then no candidate is simulated: use ap_search_exhaustive2)
 * Asynchronous on `stream` (T_ref, S and the u32 clamp schedule are computed on the
 * device by a one-thread kernel the sweep reads).
 * Errors: INVALID (p, m, k range, empty or out-of-range rank slice), RANGE (overflow
 * guard), CUDA, NOMEM.
 */
ap_status ap_search_exhaustive(const ap_plan* plan, int32_t p, int32_t m, int32_t k_lo,
                               int32_t k_hi, uint64_t rank_lo, uint64_t rank_hi,
                               int64_t* key, ap_stream_t stream);

/*
 * ap_search_exhaustive_mode -- ap_search_exhaustive with a choice of evaluation
 * strategy.  Every mode returns the SAME key (the exact argmin); they differ only in
 * how much work is done per candidate:
 *   AP_SEARCH_FULL     every (partition, k) pair is row-swept in full (the
 *                      candidates/s metric is defined on this mode).
 *   AP_SEARCH_KFACTOR  exact max-plus factoring over k: one reversed sweep per
 *                      partition gives the longest path G_x from the end of each
 *                      stage's first forward to the sink; T(k) = max_x FF_x(k) + G_x
 *                      where FF(k) is micro-batch 0's k-piece forward.
 *   AP_SEARCH_PRUNED   KFACTOR, skipping partitions whose valid lower bound
 *                      (a stage's 2m ops back to back plus the fill and
 *                      drain chains) exceeds T_ref; a labelled time-to-plan mode.
 * Modes 1 and 2 apply to the p-specialised kernel (p <= 8, 10, 12, 16 and m >= p);
 * elsewhere the call falls back to the full sweep.
 */
#define AP_SEARCH_FULL 0
#define AP_SEARCH_KFACTOR 1
#define AP_SEARCH_PRUNED 2
/* AP_SEARCH_MEMORY (NEXT N4; reading R-N4): the full sweep restricted to the
 * partitions that fit the plan's memory model (ap_plan_set_memory; INVALID without it):
 * every stage x must satisfy  sum(static) + min(p-x, m) * sum(stash) <= cap  over its
 * sub-layers (min(p-x, m) = the micro-batches 1F1B keeps in flight on stage x).  Runs
 * on the generic exact kernel.  T_ref is the Alg.-1 partition's T at k_lo when it
 * fits, else the overflow guard's bound on any T (then the packed key usually does not
 * fit and ap_search_exhaustive2 applies).  INT64_MAX when nothing fits. */
#define AP_SEARCH_MEMORY 4
ap_status ap_search_exhaustive_mode(const ap_plan* plan, int32_t p, int32_t m, int32_t k_lo,
                                    int32_t k_hi, uint64_t rank_lo, uint64_t rank_hi,
                                    int32_t mode, int64_t* key, ap_stream_t stream);

/*
 * ap_search_exhaustive2 -- the same search as ap_search_exhaustive_mode, reduced as
 * a two-word key for the cases where T << rb | index does not fit in 63 bits (SURVEY
 * §8d key packing, NEXT N3 "two-phase key reduction").  Same shard, modes, T_ref
 * bound and exactness; no RANGE failure from key packing.
 *   out   device int64[2] (written): out[0] = least T over this shard's candidates
 *         with T <= T_ref, out[1] = the least index = rank*K + (k - k_lo) among them;
 *         both INT64_MAX when the shard holds none (it cannot hold the winner).
 * Each CTA stores its lexicographic min (T, index); one more single-CTA kernel
 * reduces those records.  Multi-GPU: all_reduce(MIN) a copy of out[0] -> T*, then
 * ap_key2_select(out, T*, idx) and all_reduce(MIN) idx; decode with ap_decode mode 2.
 * Asynchronous on `stream`.  Errors as ap_search_exhaustive_mode (no AP_KEY_RANGE).
 */
ap_status ap_search_exhaustive2(const ap_plan* plan, int32_t p, int32_t m, int32_t k_lo,
                                int32_t k_hi, uint64_t rank_lo, uint64_t rank_hi, int32_t mode,
                                int64_t* out, ap_stream_t stream);

/*
 * ap_search_exhaustive_bounded -- ap_search_exhaustive2 with a caller-supplied bound:
 * only candidates with T <= min(T_ref, t_bound) are kept (the same u32 saturation and,
 * in AP_SEARCH_PRUNED, the same lower-bound pruning, now at min(T_ref, t_bound) + 1).
 * With t_bound an ATTAINED iteration time -- e.g. the heuristic's result
 * (ap_search_heuristic) -- the global optimum T* <= t_bound is kept,
 * so the reduced out over all shards is exactly the exhaustive argmin (SURVEY §8c O7,
 * O11) while the pruning is as tight as the best plan already known.  With t_bound < T*
 * every shard returns INT64_MAX.
 *   t_bound  >= 0 (INVALID otherwise); INT64_MAX = ap_search_exhaustive2.
 *   out      device int64[2], as ap_search_exhaustive2 (decode with ap_decode mode 2).
 * Errors as ap_search_exhaustive2.
 */
ap_status ap_search_exhaustive_bounded(const ap_plan* plan, int32_t p, int32_t m, int32_t k_lo,
                                       int32_t k_hi, uint64_t rank_lo, uint64_t rank_hi,
                                       int32_t mode, int64_t t_bound, int64_t* out,
                                       ap_stream_t stream);

/*
 * ap_key2_select -- phase 2 of the two-phase reduction, stream-ordered on `stream`:
 * *idx = local[1] if local[0] == *t_star (and is not INT64_MAX), else INT64_MAX.
 *   local  device int64[2] from ap_search_exhaustive2; t_star, idx device int64[1].
 * Errors: INVALID (NULL pointer), CUDA.
 */
ap_status ap_key2_select(const int64_t* local, const int64_t* t_star, int64_t* idx,
                         ap_stream_t stream);

/*
 * ap_search_heuristic -- AutoPipe's boundary-shifting heuristic (PAPER.md:147-198,
 * steps 1, 3, 4; adjust_mode 1 adds step 2 / Eq. (1)), run as
 * independent deterministic restarts r in [r_lo, r_hi), one GPU lane each.
 * Restart 0 starts at the Algorithm 1 partition; restart r >= 1 at
 * the seeded perturbation of DESIGN.md reading Q21 (splitmix64(seed ^ r<<32 ^ x),
 * offsets in [-radius, radius]).  Each restart walks: if the master stage i is 0,
 * stop; else simulate the children "move the first block of stage i to i-1"
 * (+/- Algorithm 1 on the first i-1 stages) and "move the last block of stage i to
 * i+1" (+/- Algorithm 1 on the first i stages); move to the
 * child with master <= i and least (T, child order); stop if none.  A restart's
 * result is the first-visited partition of least T among all it simulated.  k = 1.
 *   key   device int64[1]: min over restarts of (T << 20 | r), INT64_MAX if none.
 *   adjust_mode 1 (reading Q19/Q20): before each step, for s = i+1..p-2 while
 *   sum_{j=i+1..s}(F_j+B_j) > (s-i)*B_i and stage s has >= 2 blocks, move its last
 *   block to s+1 and re-simulate; stop adjusting when the master changes.  Because the
 *   master can then rise, the walk also stops when its post-adjustment scheme repeats
 *   one of its last 32 (splitmix64 hash of the cut vector); the n*p step cap holds.
 *   0 <= r_lo < r_hi <= 2^20, 0 <= radius <= 1<<20, adjust_mode in {0, 1}.
 * Asynchronous on `stream`.  RANGE when a simulated T could reach 2^43 (the overflow
 * guard m*(sum f + sum b) + 2m(p-1)*max comm >= 2^43): the key holds T in 43 bits.
 */
ap_status ap_search_heuristic(const ap_plan* plan, int32_t p, int32_t m, uint64_t seed,
                              int32_t radius, uint32_t r_lo, uint32_t r_hi,
                              int32_t adjust_mode, int64_t* key, ap_stream_t stream);

/*
 * ap_search_reachable -- the literal reading of PAPER.md:196 "partition schemes with a
 * master <= i will be processed" (reading R-N1): every
 * qualifying child is processed, not only the best one.  Per restart r (same start as
 * ap_search_heuristic: Alg. 1 for r = 0, the seeded perturbation otherwise), a
 * breadth-first search: a scheme with master i > 0 generates its children a, a', b,
 * b' (as in ap_search_heuristic); a child not evaluated before is simulated and joins
 * the evaluated set in that order, and joins the queue if its master is <= i.  The
 * restart stops when the queue is empty or when vmax schemes have been evaluated
 * (ap_last_truncated counts those).  Its result is the first-evaluated scheme with
 * the least T; never worse than ap_search_heuristic's greedy walk, whose path lies
 * inside the evaluated set.  One 4-lane group per restart on the device.
 *   key   device int64[1]: min over restarts of (T << 20 | r), INT64_MAX if none.
 *   0 <= r_lo < r_hi <= 2^20, 0 <= radius <= 2^20, 1 <= vmax <= 2^20; k = 1.
 * Scratch from the plan's pool: (restart groups in flight) x vmax x (2*P + 8) bytes.
 * Asynchronous on `stream`.
 * Errors: INVALID, RANGE (overflow guard; as ap_search_heuristic, T must stay below
 * 2^43), NOMEM (scratch), CUDA.
 */
ap_status ap_search_reachable(const ap_plan* plan, int32_t p, int32_t m, uint64_t seed,
                              int32_t radius, uint32_t r_lo, uint32_t r_hi, int32_t vmax,
                              int64_t* key, ap_stream_t stream);

typedef struct {
  int64_t time_ns;          /* T of the decoded candidate                     */
  uint64_t rank;            /* lex rank (mode 0) / rank of the cut vector (1) */
  uint32_t restart;         /* winning restart (mode 1), 0 for mode 0         */
  int32_t k;                /* slice pieces of micro-batch 0                  */
  int32_t master;           /* master stage of the decoded candidate          */
  int32_t p;                /* stages                                         */
  int32_t cuts[AP_MAX_P - 1];
} ap_result;

/*
 * ap_decode -- turn a reduced key into a plan (blocking).
 *   mode 0: key from ap_search_exhaustive(k_lo, k_hi): unrank on the device and
 *           re-simulate (T must equal the key's T; master from the critical path).
 *   mode 1: key from ap_search_heuristic(seed, radius, adjust_mode): replay the
 *           winning restart on the device to recover its cut vector.
 *   mode 2: key = the reduced index rank*K + (k - k_lo) of ap_search_exhaustive2
 *           (k_lo, k_hi as in the search): unrank and re-simulate; time_ns is the
 *           re-simulated T (the caller holds T* from phase 1 to compare).
 * INVALID if key == INT64_MAX (empty search) or is not decodable.
 */
ap_status ap_decode(const ap_plan* plan, int32_t mode, int32_t p, int32_t m, int32_t k_lo,
                    int32_t k_hi, uint64_t seed, int32_t radius, int32_t adjust_mode,
                    int64_t key, ap_result* out);

/*
 * ap_decode_reachable -- decode a key of ap_search_reachable (same seed, radius, vmax):
 * replays the winning restart on the device, re-simulates its best scheme with the
 * critical path (T must equal the key's T).  Blocking.  INVALID for an empty key.
 */
ap_status ap_decode_reachable(const ap_plan* plan, int32_t p, int32_t m, uint64_t seed,
                              int32_t radius, int32_t vmax, int64_t key, ap_result* out);

/*
 * ap_slice_sweep -- the Slicer's choice for one partition (§III-C;
 * BASELINE north_star "micro-batch 0 sliced into k pieces"): T(k) for k = 1..k_max,
 * best_k = argmin (T, k) (smallest k on ties).  Blocking.
 *   cuts     host int32[p-1];  time_ns host int64[k_max] (written)
 *   k_max in [1, AP_MAX_K]
 */
ap_status ap_slice_sweep(const ap_plan* plan, int32_t p, int32_t m, const int32_t* cuts,
                         int32_t k_max, int64_t* time_ns, int32_t* best_k);

/*
 * ap_slice_sweep_paper -- the paper's own Slicer form (Fig. 8): the
 * forwards of the first s micro-batches are split into k pieces each (k = 2: halves)
 * and BP is never sliced.  T(s) for s = 0..s_max (s = 0: no slicing); best_s =
 * argmin (T, s).  T only (no critical path for s > 1).  Blocking.
 *   cuts host int32[p-1]; time_ns host int64[s_max+1]; 0 <= s_max <= m.
 */
ap_status ap_slice_sweep_paper(const ap_plan* plan, int32_t p, int32_t m, const int32_t* cuts,
                               int32_t k, int32_t s_max, int64_t* time_ns, int32_t* best_s);

/*
 * ap_slicer_alg2 -- Algorithm 2, the Slicer's analytic number mb of
 * leading micro-batches to slice in halves, transcribed on the device.  The printed
 * pseudocode is garbled; readings in DESIGN.md §2 (Q22-Q24).  reading 0 = the
 * pseudocode's stop test (line 34, "tempt <= endt[0][1]"), reading 1 = the text's
 * ("start of the unbroken micro-batch >= end of the second half").
 * Blocking.  cuts host int32[p-1]; *mb in [1, p].
 */
ap_status ap_slicer_alg2(const ap_plan* plan, int32_t p, const int32_t* cuts, int32_t reading,
                         int32_t* mb);

typedef struct {
  int32_t stage;       /* x                                        */
  int32_t kind;        /* 0 = forward (FP), 1 = backward (BP)      */
  int32_t microbatch;  /* micro-batch index j                      */
  int32_t piece;       /* slice piece q of micro-batch 0's FP, else 0 */
  int64_t start_ns;    /* compute start (after the receive Comm)   */
  int64_t end_ns;      /* compute end                              */
} ap_op;

/*
 * ap_critical_path -- the unique critical path (Fig. 4: the longest
 * path of the AOE network, "closest to the last pipeline stage in the 1F1B phase";
 * reading Q10) from F(0, mb 0, piece 0) to B(0, m-1), its master stage and T.
 * Blocking.  cuts host int32[p-1]; ops host ap_op[cap] written source -> sink;
 * *len = path length (also on CAPACITY, so the caller can retry).
 */
ap_status ap_critical_path(const ap_plan* plan, int32_t p, int32_t m, int32_t k,
                           const int32_t* cuts, ap_op* ops, int32_t cap, int32_t* len,
                           int32_t* master, int64_t* time_ns);

/*
 * ap_alg1 -- Algorithm 1: the min-max balanced partition of the
 * n sub-layers into p stages by f+b (Comm unused, reading Q16; ties -> smallest
 * split point).  Runs on the device; blocking.  cuts host int32[p-1]; value =
 * the max stage load of that partition.
 */
ap_status ap_alg1(const ap_plan* plan, int32_t p, int32_t* cuts, int64_t* value);

/*
 * ap_min_lower_bound -- certified lower bound on the optimum T over every partition
 * and every slicing k <= K (reading R-LB).
 * The O11 bound LB_x = fill_x + m(F_x+B_x+C_in+C_out) + sum_{i<x}(B_i+C_i) (PAPER.md:
 * 113-125: stage x runs m FPs and m BPs with their receives, after its fill and before
 * the BP chain back to stage 0) is relaxed to depend only on (x, c_x, c_{x+1}), and
 * min over partitions of max_x of it is a bottleneck DP over (x, c_x, c_{x+1}),
 * O(p n^2) on one CTA.  Exact min_c max_x LB_x(c) when K = 1 and Comm is uniform.
 * Blocking.  lb: host int64 (T* >= *lb for every partition, every k <= K);
 * cuts: host int32[p-1] or NULL, a partition attaining the relaxed bound (smallest
 * split point on ties).  Errors: INVALID for p outside [1, min(n, AP_MAX_P)], m < 1,
 * K outside [1, AP_MAX_K].
 */
ap_status ap_min_lower_bound(const ap_plan* plan, int32_t p, int32_t m, int32_t K, int64_t* lb,
                             int32_t* cuts);

/* Details of the last ap_search_exhaustive launch on this thread (for benches):
 * which sweep variant ran and its grid.  t_ref, fast_u32 and the clamp fields are
 * computed on the device; this call waits for the last search to read them. */
typedef struct {
  int32_t fast_u32;        /* 1: exact u32 saturating sweep, 0: int64 sweep        */
  int32_t exact_p;         /* 1: kernel specialised for this p, 0: generic        */
  int32_t blocks, threads; /* grid                                                */
  uint64_t chunk;          /* ranks per thread                                    */
  int64_t t_ref;           /* min_k T(Algorithm 1 partition, k), k in [k_lo,k_hi] */
  int32_t rank_bits;       /* rb                                                  */
  int32_t launches;        /* kernels launched by the call                        */
  int32_t clamp_rows;      /* u32 path: steady rows between saturating clamps      */
  int32_t clamp_first;     /* u32 path: steady rows before the first clamp (0 = clamp
                              right after the warm-up; > m-p = no clamp at all)     */
  int32_t clamp_final;     /* u32 path: 1 = clamp once more before the cool-down    */
} ap_launch_info;
void ap_last_launch(ap_launch_info* info);

/* Device time (ms) of the dominant kernel of the last ap_search_exhaustive /
 * ap_search_heuristic call on this thread (the sweep or restart kernel alone),
 * from CUDA events the library records around that launch on the caller's stream.
 * Valid once the stream has passed the launch; AP_ERR_INVALID before that or if
 * no search ran. */
ap_status ap_last_kernel_ms(float* ms);

/* Number of kernels this library has launched since it was loaded (every thread and
 * device; a host-side counter bumped at each launch).  Benches take the difference
 * around a timed region to state how many of the library's kernels ran in it. */
uint64_t ap_kernel_launches(void);

/* Simulations run by the last ap_search_exhaustive / ap_search_heuristic call on this
 * thread: (rank_hi-rank_lo)*(k_hi-k_lo+1) for the sweep; counted on the device for the
 * heuristic (blocks until that kernel has finished). */
ap_status ap_last_sims(uint64_t* sims);

/* Restarts of the last ap_search_reachable call on this thread that stopped at vmax
 * evaluated schemes (blocks until that kernel has finished); 0 after any other search. */
ap_status ap_last_truncated(uint64_t* truncated);

#ifdef __cplusplus
}
#endif
#endif /* AP_H_ */
