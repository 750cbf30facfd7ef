// ap_host.cu -- C-ABI implementation of include/ap.h.
//
// Host side only validates, allocates, launches and copies.  Every step of the
// method (prefix sums, Algorithm 1, simulation, critical path, search, unranking,
// restarts) runs in the kernels of ap_kernels.cu.  There is no CPU fallback: with
// no sm_100 device every call fails with AP_ERR_CUDA.
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <algorithm>
#include <cstring>
#include <atomic>
#include <mutex>
#include <string>
#include <vector>

#include "../../include/ap.h"
#include "ap_launch.h"

namespace {

thread_local std::string g_err;
thread_local ap_launch_info g_last{};

// CUDA events bracketing the dominant kernel of the last search on this thread.
struct KernelTimer {
  cudaEvent_t ev[2] = {nullptr, nullptr};
  int dev = -1;
  bool armed = false;
  cudaError_t record(int which, cudaStream_t s, int device) {
    if (dev != device) {
      // events belong to the device current at creation
      for (auto& e : ev)
        if (e) cudaEventDestroy(e);
      ev[0] = ev[1] = nullptr;
      dev = device;
    }
    for (auto& e : ev)
      if (!e) {
        cudaError_t r = cudaEventCreate(&e);
        if (r != cudaSuccess) return r;
      }
    armed = (which == 1);
    if (which == 0) truncated_valid = false;
    return cudaEventRecord(ev[which], s);
  }
  // simulations of the last search: known on the host (exhaustive) or counted on
  // the device (heuristic, d_sims valid once ev[1] has completed)
  uint64_t host_sims = 0;
  bool sims_on_device = false;
  bool truncated_valid = false;  // the last search was ap_search_reachable
  unsigned long long* d_sims = nullptr;
  int d_sims_dev = -1;
  // SweepDev of the last exhaustive search (written by k_sweep_prep on the device);
  // ap_last_launch reads it once the search has completed
  apk::SweepDev* d_sweep = nullptr;
  int d_sweep_dev = -1;
  bool sweep_pending = false;
  cudaError_t sweep_buffer(int device, apk::SweepDev** out) {
    if (d_sweep_dev != device) {
      d_sweep = nullptr;  // (a buffer of another device is leaked; one per thread/device switch)
      cudaError_t e = cudaMalloc((void**)&d_sweep, sizeof(apk::SweepDev));
      if (e != cudaSuccess) return e;
      d_sweep_dev = device;
    }
    *out = d_sweep;
    return cudaSuccess;
  }
  cudaError_t sims_buffer(int device, unsigned long long** out) {
    if (d_sims_dev != device) {
      d_sims = nullptr;  // (a buffer of another device is leaked; one per thread/device switch)
      cudaError_t e = cudaMalloc((void**)&d_sims, 16);
      if (e != cudaSuccess) return e;
      d_sims_dev = device;
    }
    *out = d_sims;
    return cudaSuccess;
  }
};
thread_local KernelTimer g_timer;

// Per-thread record of the last heuristic search: each restart's best cut vector, so
// ap_decode(mode 1) can read the winner's cuts instead of replaying its walk.
struct HeurCache {
  uint64_t plan_gen = 0;
  int p = 0, m = 0, radius = 0, dev = -1, adjust_mode = 0;
  uint64_t seed = 0;
  uint32_t r_lo = 0, r_hi = 0;
  int16_t* d_best = nullptr;
  size_t cap = 0;
  bool valid = false;
  cudaEvent_t done = nullptr;  // recorded after the search that filled d_best (its device)
};
thread_local HeurCache g_hcache;

ap_status fail(ap_status st, const char* fmt, ...) {
  char buf[512];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof buf, fmt, ap);
  va_end(ap);
  g_err = buf;
  return st;
}

#define AP_CUDA(expr)                                                                 \
  do {                                                                                \
    cudaError_t e__ = (expr);                                                         \
    if (e__ != cudaSuccess)                                                           \
      return fail(e__ == cudaErrorMemoryAllocation ? AP_ERR_NOMEM : AP_ERR_CUDA,      \
                  "%s: %s (%s:%d)", #expr, cudaGetErrorString(e__), __FILE__, __LINE__); \
  } while (0)

struct DeviceGuard {
  int prev = -1;
  explicit DeviceGuard(int dev) {
    if (cudaGetDevice(&prev) != cudaSuccess) prev = -1;
    if (prev != dev) cudaSetDevice(dev);
  }
  ~DeviceGuard() {
    int cur = -1;
    if (prev >= 0 && cudaGetDevice(&cur) == cudaSuccess && cur != prev) cudaSetDevice(prev);
  }
};

// Per-call device scratch from the device's library pool (release threshold = max,
// so stream-ordered frees never unmap memory at a synchronisation), released
// stream-ordered.
struct Scratch {
  cudaStream_t s;
  cudaMemPool_t pool;
  std::vector<void*> ptrs;
  Scratch(cudaStream_t st, cudaMemPool_t pl) : s(st), pool(pl) {}
  cudaError_t get(void** p, size_t bytes) {
    cudaError_t e = cudaMallocFromPoolAsync(p, bytes < 16 ? 16 : bytes, pool, s);
    if (e == cudaSuccess) ptrs.push_back(*p);
    return e;
  }
  ~Scratch() {
    for (void* p : ptrs) cudaFreeAsync(p, s);
  }
};

// One library-owned memory pool per device (created on first use, release threshold =
// max so stream-ordered frees never unmap memory at a synchronisation; never destroyed).
std::mutex g_pool_mu;
cudaMemPool_t g_pools[64] = {nullptr};
cudaError_t device_pool(int device, cudaMemPool_t* out) {
  if (device < 0 || device >= 64) return cudaErrorInvalidDevice;
  std::lock_guard<std::mutex> lk(g_pool_mu);
  if (!g_pools[device]) {
    cudaMemPoolProps props = {};
    props.allocType = cudaMemAllocationTypePinned;
    props.location.type = cudaMemLocationTypeDevice;
    props.location.id = device;
    cudaError_t e = cudaMemPoolCreate(&g_pools[device], &props);
    if (e != cudaSuccess) {
      g_pools[device] = nullptr;
      return e;
    }
    uint64_t thr = UINT64_MAX;
    e = cudaMemPoolSetAttribute(g_pools[device], cudaMemPoolAttrReleaseThreshold, &thr);
    if (e != cudaSuccess) return e;
  }
  *out = g_pools[device];
  return cudaSuccess;
}

// Per-thread pinned host staging buffer (grown on demand, never freed).
cudaError_t pinned_staging(size_t bytes, int64_t** out) {
  thread_local int64_t* buf = nullptr;
  thread_local size_t cap = 0;
  if (cap < bytes) {
    if (buf) cudaFreeHost(buf);
    buf = nullptr;
    cap = 0;
    cudaError_t e = cudaHostAlloc((void**)&buf, bytes, cudaHostAllocDefault);
    if (e != cudaSuccess) return e;
    cap = bytes;
  }
  *out = buf;
  return cudaSuccess;
}

// One internal non-blocking stream per (thread, device) for the blocking calls.
cudaError_t internal_stream(int device, cudaStream_t* out) {
  thread_local cudaStream_t streams[64] = {nullptr};
  if (device < 0 || device >= 64) return cudaErrorInvalidDevice;
  if (!streams[device]) {
    cudaError_t e = cudaStreamCreateWithFlags(&streams[device], cudaStreamNonBlocking);
    if (e != cudaSuccess) return e;
  }
  *out = streams[device];
  return cudaSuccess;
}

int bitlen(unsigned __int128 v) {
  int b = 0;
  while (v) {
    ++b;
    v >>= 1;
  }
  return b;
}

uint64_t binom_sat(int a, int b) {
  if (b < 0 || b > a) return 0;
  unsigned __int128 r = 1;
  for (int i = 1; i <= b; ++i) {
    r = r * (unsigned)(a - b + i) / (unsigned)i;
    if (r > (unsigned __int128)UINT64_MAX) return UINT64_MAX;
  }
  return (uint64_t)r;
}

}  // namespace

std::atomic<uint64_t> g_plan_gen{1};

struct ap_plan {
  uint64_t gen = 0;  // unique id (never reused) for caches keyed by plan
  int n = 0, npad = 0, device = 0;
  std::vector<int64_t> f, b, act, comm;
  int64_t sum_f = 0, sum_b = 0, max_comm = 0;
  uint64_t link = 0;
  int64_t* d_tab = nullptr;
  uint64_t* d_binom = nullptr;
  cudaMemPool_t pool = nullptr;
  // memory model (ap_plan_set_memory, NEXT N4): prefix sums of static and stash bytes
  bool has_mem = false;
  std::vector<int64_t> mem_pw, mem_ps;  // [n+1]
  int64_t mem_cap = 0;
  int64_t* d_mem = nullptr;  // device [2][n+1]: PW, PS
  apk::DevTables dev() const { return apk::DevTables{d_tab, d_binom, n, npad}; }
  bool feasible(int p, int m, const int32_t* cuts) const {
    for (int x = 0; x < p; ++x) {
      const int lo = x == 0 ? 0 : cuts[x - 1], hi = x == p - 1 ? n : cuts[x];
      const int64_t inflight = (p - x < m) ? p - x : m;
      if (mem_pw[hi] - mem_pw[lo] + inflight * (mem_ps[hi] - mem_ps[lo]) > mem_cap) return false;
    }
    return true;
  }
};

extern "C" {

const char* ap_last_error(void) { return g_err.c_str(); }

const char* ap_version(void) { return "autopipe-b200 0.1 (sm_100a)"; }

void ap_last_launch(ap_launch_info* info) {
  if (g_timer.sweep_pending && g_timer.d_sweep) {
    // the T_ref-dependent fields come from the device (k_sweep_prep): wait for the
    // search, then read them once
    apk::SweepDev d{};
    if (cudaEventSynchronize(g_timer.ev[1]) == cudaSuccess &&
        cudaMemcpy(&d, g_timer.d_sweep, sizeof(d), cudaMemcpyDeviceToHost) == cudaSuccess) {
      g_last.t_ref = d.tref;
      g_last.fast_u32 = g_last.fast_u32 && d.u32;
      g_last.clamp_rows = g_last.fast_u32 ? d.clamp_rows : 0;
      g_last.clamp_first = g_last.fast_u32 ? d.clamp_first : 0;
      g_last.clamp_final = g_last.fast_u32 ? d.clamp_final : 0;
    }
    g_timer.sweep_pending = false;
  }
  if (info) *info = g_last;
}

ap_status ap_last_sims(uint64_t* sims) {
  if (!sims) return fail(AP_ERR_INVALID, "sims is NULL");
  if (!g_timer.armed) return fail(AP_ERR_INVALID, "no search launched on this thread");
  if (!g_timer.sims_on_device) {
    *sims = g_timer.host_sims;
    return AP_OK;
  }
  cudaError_t e = cudaEventSynchronize(g_timer.ev[1]);
  unsigned long long v = 0;
  if (e == cudaSuccess) e = cudaMemcpy(&v, g_timer.d_sims, 8, cudaMemcpyDeviceToHost);
  if (e != cudaSuccess) return fail(AP_ERR_CUDA, "sims read: %s", cudaGetErrorString(e));
  *sims = v;
  return AP_OK;
}

uint64_t ap_kernel_launches(void) { return apk::kernel_launches(); }

ap_status ap_last_kernel_ms(float* ms) {
  if (!ms) return fail(AP_ERR_INVALID, "ms is NULL");
  if (!g_timer.armed) return fail(AP_ERR_INVALID, "no search launched on this thread");
  if (cudaEventQuery(g_timer.ev[1]) != cudaSuccess)
    return fail(AP_ERR_INVALID, "last search kernel not complete");
  cudaError_t e = cudaEventElapsedTime(ms, g_timer.ev[0], g_timer.ev[1]);
  if (e != cudaSuccess) return fail(AP_ERR_CUDA, "elapsed: %s", cudaGetErrorString(e));
  return AP_OK;
}

ap_status ap_plan_create(int32_t n, const int64_t* fwd_ns, const int64_t* bwd_ns,
                         const int64_t* act_bytes, uint64_t link_bytes_per_s, int32_t device,
                         ap_plan** out) {
  g_err.clear();
  if (!out) return fail(AP_ERR_INVALID, "out is NULL");
  *out = nullptr;
  if (n < 1 || n > AP_MAX_N) return fail(AP_ERR_INVALID, "n=%d outside [1, %d]", n, AP_MAX_N);
  if (!fwd_ns || !bwd_ns || !act_bytes) return fail(AP_ERR_INVALID, "NULL table");
  if (link_bytes_per_s == 0) return fail(AP_ERR_INVALID, "link_bytes_per_s = 0");
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0)
    return fail(AP_ERR_CUDA, "no CUDA device (the library has no CPU fallback)");
  if (device < 0 || device >= ndev) return fail(AP_ERR_INVALID, "device %d of %d", device, ndev);
  int major = 0, minor = 0;
  AP_CUDA(cudaDeviceGetAttribute(&major, cudaDevAttrComputeCapabilityMajor, device));
  AP_CUDA(cudaDeviceGetAttribute(&minor, cudaDevAttrComputeCapabilityMinor, device));
  if (major != 10)
    return fail(AP_ERR_CUDA, "device %d is sm_%d%d; this library is built for sm_100a", device,
                major, minor);
  ap_plan* P = new ap_plan();
  P->gen = g_plan_gen.fetch_add(1);
  P->n = n;
  P->npad = (n + 1) & ~1;  // even => 16-byte multiple per array (TMA bulk copy)
  P->device = device;
  P->link = link_bytes_per_s;
  P->f.assign(fwd_ns, fwd_ns + n);
  P->b.assign(bwd_ns, bwd_ns + n);
  P->act.assign(act_bytes, act_bytes + n);
  P->comm.assign(n, 0);
  unsigned __int128 sf = 0, sb = 0;
  for (int i = 0; i < n; ++i) {
    if (fwd_ns[i] < 0 || bwd_ns[i] < 0 || act_bytes[i] < 0) {
      delete P;
      return fail(AP_ERR_INVALID, "negative entry at sub-layer %d", i);
    }
    sf += (uint64_t)fwd_ns[i];
    sb += (uint64_t)bwd_ns[i];
    // Comm = ceil(bytes * 1e9 / bandwidth), exact in 128 bits (reading Q4, Q25)
    const unsigned __int128 num = (unsigned __int128)(uint64_t)act_bytes[i] * 1000000000u;
    const unsigned __int128 q = (num + link_bytes_per_s - 1) / link_bytes_per_s;
    if (q >= ((unsigned __int128)1 << 62)) {
      delete P;
      return fail(AP_ERR_RANGE, "comm of sub-layer %d overflows", i);
    }
    if (i < n - 1) P->comm[i] = (int64_t)q;
  }
  if (sf >= ((unsigned __int128)1 << 62) || sb >= ((unsigned __int128)1 << 62)) {
    delete P;
    return fail(AP_ERR_RANGE, "sum of f or b >= 2^62");
  }
  P->sum_f = (int64_t)sf;
  P->sum_b = (int64_t)sb;
  for (int i = 0; i < n - 1; ++i) P->max_comm = P->comm[i] > P->max_comm ? P->comm[i] : P->max_comm;
  std::vector<int64_t> tab(3 * (size_t)P->npad, 0);
  for (int i = 0; i < n; ++i) {
    tab[i] = P->f[i];
    tab[P->npad + i] = P->b[i];
    tab[2 * P->npad + i] = P->comm[i];
  }
  // binomials C(a, b), a <= n, b <= 32, by Pascal's rule (saturating at 2^64-1), laid
  // out right after the tables so one allocation and one copy stage the whole plan
  const size_t nb = (size_t)(n + 1) * 33;
  tab.resize(tab.size() + nb, 0);
  uint64_t* binom = reinterpret_cast<uint64_t*>(tab.data() + 3 * (size_t)P->npad);
  for (int a = 0; a <= n; ++a) {
    binom[(size_t)a * 33] = 1;
    for (int bb = 1; bb <= 32 && bb <= a; ++bb) {
      const uint64_t x = binom[(size_t)(a - 1) * 33 + bb - 1];
      const uint64_t y = (bb <= a - 1) ? binom[(size_t)(a - 1) * 33 + bb] : 0;
      binom[(size_t)a * 33 + bb] = (x > UINT64_MAX - y) ? UINT64_MAX : x + y;
    }
  }
  DeviceGuard g(device);
  cudaStream_t s0 = nullptr;
  cudaError_t e = device_pool(device, &P->pool);
  if (e == cudaSuccess) e = internal_stream(device, &s0);
  if (e == cudaSuccess) e = cudaMallocFromPoolAsync((void**)&P->d_tab, tab.size() * 8, P->pool, s0);
  // stage through a per-thread pinned buffer so the copy is a plain DMA
  int64_t* pinned = nullptr;
  if (e == cudaSuccess) e = pinned_staging(tab.size() * 8, &pinned);
  if (e == cudaSuccess) {
    memcpy(pinned, tab.data(), tab.size() * 8);
    e = cudaMemcpyAsync(P->d_tab, pinned, tab.size() * 8, cudaMemcpyHostToDevice, s0);
  }
  if (e == cudaSuccess) e = cudaStreamSynchronize(s0);
  if (e == cudaSuccess) P->d_binom = reinterpret_cast<uint64_t*>(P->d_tab + 3 * (size_t)P->npad);
  if (e != cudaSuccess) {
    ap_plan_destroy(P);
    return fail(e == cudaErrorMemoryAllocation ? AP_ERR_NOMEM : AP_ERR_CUDA, "plan upload: %s",
                cudaGetErrorString(e));
  }
  *out = P;
  return AP_OK;
}

void ap_plan_destroy(ap_plan* plan) {
  if (!plan) return;
  {
    DeviceGuard g(plan->device);
    // the caller guarantees no call on the plan is still running (include/ap.h)
    cudaStream_t s0 = nullptr;
    if (plan->d_tab && internal_stream(plan->device, &s0) == cudaSuccess) {
      cudaFreeAsync(plan->d_tab, s0);
      if (plan->d_mem) cudaFreeAsync(plan->d_mem, s0);
      cudaStreamSynchronize(s0);
    }
  }
  delete plan;
}

ap_status ap_plan_set_memory(ap_plan* plan, const int64_t* static_bytes, const int64_t* stash_bytes,
                             int64_t cap_bytes) {
  g_err.clear();
  if (!plan) return fail(AP_ERR_INVALID, "plan is NULL");
  if (!static_bytes || !stash_bytes) return fail(AP_ERR_INVALID, "NULL table");
  if (cap_bytes < 0) return fail(AP_ERR_INVALID, "cap_bytes < 0");
  const int n = plan->n;
  std::vector<int64_t> pw(n + 1, 0), ps(n + 1, 0);
  unsigned __int128 tw = 0, ts = 0;
  for (int i = 0; i < n; ++i) {
    if (static_bytes[i] < 0 || stash_bytes[i] < 0)
      return fail(AP_ERR_INVALID, "negative memory entry at sub-layer %d", i);
    tw += (uint64_t)static_bytes[i];
    ts += (uint64_t)stash_bytes[i];
    pw[i + 1] = pw[i] + static_bytes[i];
    ps[i + 1] = ps[i] + stash_bytes[i];
  }
  // a stage's footprint is at most sum(static) + AP_MAX_P * sum(stash)
  if (tw + (unsigned __int128)AP_MAX_P * ts >= ((unsigned __int128)1 << 62))
    return fail(AP_ERR_RANGE, "memory tables too large (>= 2^62 bytes)");
  DeviceGuard g(plan->device);
  cudaStream_t s;
  AP_CUDA(internal_stream(plan->device, &s));
  if (!plan->d_mem) {
    cudaError_t e = cudaMallocFromPoolAsync((void**)&plan->d_mem, 2 * (size_t)(n + 1) * 8,
                                            plan->pool, s);
    if (e != cudaSuccess) return fail(AP_ERR_NOMEM, "memory tables");
  }
  std::vector<int64_t> both(2 * (size_t)(n + 1));
  std::copy(pw.begin(), pw.end(), both.begin());
  std::copy(ps.begin(), ps.end(), both.begin() + (n + 1));
  AP_CUDA(cudaMemcpyAsync(plan->d_mem, both.data(), both.size() * 8, cudaMemcpyHostToDevice, s));
  AP_CUDA(cudaStreamSynchronize(s));
  plan->mem_pw = std::move(pw);
  plan->mem_ps = std::move(ps);
  plan->mem_cap = cap_bytes;
  plan->has_mem = true;
  return AP_OK;
}

ap_status ap_plan_info(const ap_plan* plan, int32_t* n, int64_t* comm_ns) {
  if (!plan) return fail(AP_ERR_INVALID, "plan is NULL");
  if (n) *n = plan->n;
  if (comm_ns) memcpy(comm_ns, plan->comm.data(), plan->comm.size() * 8);
  return AP_OK;
}

ap_status ap_count(int32_t n, int32_t p, uint64_t* out) {
  if (!out) return fail(AP_ERR_INVALID, "out is NULL");
  if (n < 1 || p < 1 || p > n) return fail(AP_ERR_INVALID, "need 1 <= p <= n (p=%d, n=%d)", p, n);
  unsigned __int128 r = 1;
  const int a = n - 1, bb = p - 1;
  for (int i = 1; i <= bb; ++i) {
    r = r * (unsigned)(a - bb + i) / (unsigned)i;
    if (r >= ((unsigned __int128)1 << 63)) return fail(AP_ERR_RANGE, "C(%d,%d) >= 2^63", a, bb);
  }
  *out = (uint64_t)r;
  return AP_OK;
}

}  // extern "C"

namespace {

ap_status check_pm(const ap_plan* plan, int p, int m) {
  if (!plan) return fail(AP_ERR_INVALID, "plan is NULL");
  if (p < 1 || p > plan->n || p > AP_MAX_P)
    return fail(AP_ERR_INVALID, "p=%d outside [1, min(n=%d, %d)]", p, plan->n, AP_MAX_P);
  if (m < 1 || m > (1 << 20)) return fail(AP_ERR_INVALID, "m=%d outside [1, 2^20]", m);
  // overflow guard: every finish time is at most the sum of all op weights
  const unsigned __int128 tot = (unsigned __int128)m * (uint64_t)(plan->sum_f + plan->sum_b) +
                                (unsigned __int128)2 * m * (p - 1) * (uint64_t)plan->max_comm;
  if (tot >= ((unsigned __int128)1 << 62)) return fail(AP_ERR_RANGE, "overflow guard: total >= 2^62");
  return AP_OK;
}

// Restart keys pack T << 20 | r (T < 2^43): the overflow guard's bound on any T must fit.
ap_status check_key43(const ap_plan* plan, int p, int m) {
  const unsigned __int128 tot = (unsigned __int128)m * (uint64_t)(plan->sum_f + plan->sum_b) +
                                (unsigned __int128)2 * m * (p - 1) * (uint64_t)plan->max_comm;
  if (tot >= ((unsigned __int128)1 << 43))
    return fail(AP_ERR_RANGE, "restart key packing: a T up to the overflow guard's bound needs "
                "more than 43 bits");
  return AP_OK;
}

cudaStream_t S_(ap_stream_t s) { return reinterpret_cast<cudaStream_t>(s); }

}  // namespace

extern "C" {

}  // extern "C"

namespace {
// u32 fast path of the evaluation kernel: clamping every CR rows at S
// with (CR + p + 2) * W_row <= 2^32-1-S cannot wrap (a segment, the conversion row and
// the p cool-down rows; from 0 the warm-up is shorter), so every candidate with T < S
// is exact and the rest are recomputed in int64.  Used by ap_eval_batch and by every
// internal evaluation (T_ref, decode, Slicer sweep).  AP_EVAL=int64 disables it,
// AP_EVAL_S=<v> lowers S (tests of the fallback).
struct EvalFast {
  uint32_t S;
  int CR, div1;
};
EvalFast eval_fast(const ap_plan* plan, int p) {
  EvalFast ef{0, 16, 0};
  const unsigned __int128 wrow = (unsigned __int128)(plan->sum_f + plan->sum_b) +
                                 (unsigned __int128)2 * (p - 1) * (uint64_t)plan->max_comm + 1;
  const unsigned __int128 need = wrow * (unsigned __int128)(ef.CR + p + 2);
  const unsigned __int128 lim32 = ((unsigned __int128)1 << 32) - 1;
  ef.S = need < lim32 ? (uint32_t)(lim32 - need) : 0u;
  const char* ev = getenv("AP_EVAL");
  if (ev && strcmp(ev, "int64") == 0) ef.S = 0;
  const char* es = getenv("AP_EVAL_S");
  if (es && ef.S > 0) {
    const unsigned long long v = strtoull(es, nullptr, 10);
    if (v > 0 && v < ef.S) ef.S = (uint32_t)v;
  }
  ef.div1 = (plan->sum_f < (1ll << 28) && plan->max_comm < (1ll << 28)) ? 1 : 0;
  return ef;
}
}  // namespace

extern "C" {

ap_status ap_eval_batch(const ap_plan* plan, int32_t p, int32_t m, const int32_t* cuts,
                        const int32_t* k, int64_t count, int64_t* time_ns, int32_t* master,
                        ap_stream_t stream) {
  return ap_eval_batch_ex(plan, p, m, cuts, k, count, time_ns, master, nullptr, stream);
}

ap_status ap_eval_batch_ex(const ap_plan* plan, int32_t p, int32_t m, const int32_t* cuts,
                           const int32_t* k, int64_t count, int64_t* time_ns, int32_t* master,
                           int64_t* n_invalid, ap_stream_t stream) {
  g_err.clear();
  ap_status st = check_pm(plan, p, m);
  if (st != AP_OK) return st;
  if (count < 0) return fail(AP_ERR_INVALID, "count < 0");
  DeviceGuard g(plan->device);
  if (count == 0) {
    if (n_invalid) AP_CUDA(cudaMemsetAsync(n_invalid, 0, sizeof(*n_invalid), S_(stream)));
    return AP_OK;
  }
  if (!time_ns || (p > 1 && !cuts)) return fail(AP_ERR_INVALID, "NULL output/cuts");
  int launches = 0;
  const EvalFast ef = eval_fast(plan, p);
  AP_CUDA(apk::launch_eval(plan->dev(), plan->pool, p, m, p > 1 ? cuts : nullptr, p - 1, k, 1, 0, count,
                           time_ns, master, S_(stream), &launches, 1, 0, ef.S, ef.CR, ef.div1,
                           reinterpret_cast<unsigned long long*>(n_invalid)));
  return AP_OK;
}

}  // extern "C"

namespace {

// Algorithm 1 on the device into scratch; returns device pointers.
ap_status run_alg1(const ap_plan* plan, int p, Scratch& sc, int16_t** d_arg, int32_t** d_cuts,
                   int64_t** d_val) {
  AP_CUDA(sc.get((void**)d_arg, (size_t)(plan->n + 1) * (p + 1) * 2));
  AP_CUDA(sc.get((void**)d_cuts, 4 * 32));
  AP_CUDA(sc.get((void**)d_val, 8));
  AP_CUDA(apk::launch_alg1(plan->dev(), p, *d_arg, *d_cuts, *d_val, sc.s));
  return AP_OK;
}

}  // namespace

extern "C" {

ap_status ap_alg1(const ap_plan* plan, int32_t p, int32_t* cuts, int64_t* value) {
  g_err.clear();
  if (!plan) return fail(AP_ERR_INVALID, "plan is NULL");
  if (p < 1 || p > plan->n || p > AP_MAX_P) return fail(AP_ERR_INVALID, "p=%d", p);
  DeviceGuard g(plan->device);
  cudaStream_t s;
  AP_CUDA(internal_stream(plan->device, &s));
  ap_status st;
  {
    Scratch sc(s, plan->pool);
    int16_t* arg;
    int32_t* dc;
    int64_t* dv;
    st = run_alg1(plan, p, sc, &arg, &dc, &dv);
    if (st == AP_OK) {
      int64_t v = 0;
      std::vector<int32_t> hc(32, 0);
      cudaError_t e = cudaSuccess;
      if (p > 1) e = cudaMemcpyAsync(hc.data(), dc, 4 * (size_t)(p - 1), cudaMemcpyDeviceToHost, s);
      if (e == cudaSuccess) e = cudaMemcpyAsync(&v, dv, 8, cudaMemcpyDeviceToHost, s);
      if (e == cudaSuccess) e = cudaStreamSynchronize(s);
      if (e != cudaSuccess) st = fail(AP_ERR_CUDA, "alg1: %s", cudaGetErrorString(e));
      else {
        if (cuts && p > 1) memcpy(cuts, hc.data(), 4 * (p - 1));
        if (value) *value = v;
      }
    }
  }
  cudaStreamSynchronize(s);
  return st;
}

ap_status ap_min_lower_bound(const ap_plan* plan, int32_t p, int32_t m, int32_t K, int64_t* lb,
                             int32_t* cuts) {
  g_err.clear();
  // every stage term is <= LB_x(c) <= T(c) for a partition c holding that stage,
  // so the plan's overflow guard covers the DP
  ap_status st = check_pm(plan, p, m);
  if (st != AP_OK) return st;
  if (K < 1 || K > AP_MAX_K) return fail(AP_ERR_INVALID, "K=%d outside [1, %d]", K, AP_MAX_K);
  if (!lb) return fail(AP_ERR_INVALID, "lb is NULL");
  DeviceGuard g(plan->device);
  cudaStream_t s;
  AP_CUDA(internal_stream(plan->device, &s));
  {
    Scratch sc(s, plan->pool);
    int16_t* d_arg = nullptr;
    int32_t* d_cuts = nullptr;
    int64_t* d_v = nullptr;
    cudaError_t e = sc.get((void**)&d_arg, (size_t)(plan->n + 1) * (p + 1) * 2);
    if (e == cudaSuccess) e = sc.get((void**)&d_cuts, 4 * 32);
    if (e == cudaSuccess) e = sc.get((void**)&d_v, 8);
    if (e != cudaSuccess) {
      st = fail(AP_ERR_NOMEM, "minlb scratch");
    } else {
      int32_t hc[32] = {0};
      int64_t v = 0;
      e = apk::launch_minlb(plan->dev(), p, m, K, d_arg, d_cuts, d_v, s);
      if (e == cudaSuccess && p > 1)
        e = cudaMemcpyAsync(hc, d_cuts, 4 * (size_t)(p - 1), cudaMemcpyDeviceToHost, s);
      if (e == cudaSuccess) e = cudaMemcpyAsync(&v, d_v, 8, cudaMemcpyDeviceToHost, s);
      if (e == cudaSuccess) e = cudaStreamSynchronize(s);
      if (e != cudaSuccess) {
        st = fail(AP_ERR_CUDA, "minlb: %s", cudaGetErrorString(e));
      } else {
        *lb = v;
        if (cuts && p > 1) memcpy(cuts, hc, 4 * (size_t)(p - 1));
      }
    }
  }
  cudaStreamSynchronize(s);
  return st;
}

ap_status ap_search_exhaustive(const ap_plan* plan, int32_t p, int32_t m, int32_t k_lo,
                               int32_t k_hi, uint64_t rank_lo, uint64_t rank_hi, int64_t* key,
                               ap_stream_t stream) {
  return ap_search_exhaustive_mode(plan, p, m, k_lo, k_hi, rank_lo, rank_hi, AP_SEARCH_FULL, key,
                                   stream);
}

}  // extern "C"

namespace {

// Shared by the packed-key and the two-phase entry points: exactly one of key / out2.
ap_status search_exhaustive_impl(const ap_plan* plan, int32_t p, int32_t m, int32_t k_lo,
                                 int32_t k_hi, uint64_t rank_lo, uint64_t rank_hi, int32_t mode,
                                 int64_t* key, int64_t* out2, ap_stream_t stream,
                                 int64_t t_bound = INT64_MAX) {
  g_err.clear();
  const bool mem = (mode == AP_SEARCH_MEMORY);
  if (!mem && (mode < AP_SEARCH_FULL || mode > AP_SEARCH_PRUNED))
    return fail(AP_ERR_INVALID, "search mode %d", mode);
  ap_status st = check_pm(plan, p, m);
  if (st != AP_OK) return st;
  if (!key && !out2) return fail(AP_ERR_INVALID, "key is NULL");
  if (mem && !plan->has_mem) return fail(AP_ERR_INVALID, "AP_SEARCH_MEMORY without ap_plan_set_memory");
  if (k_lo < 1 || k_hi < k_lo || k_hi > AP_MAX_K)
    return fail(AP_ERR_INVALID, "k range [%d, %d] outside [1, %d]", k_lo, k_hi, AP_MAX_K);
  uint64_t N;
  st = ap_count(plan->n, p, &N);
  if (st != AP_OK) return st;
  if (rank_lo >= rank_hi || rank_hi > N)
    return fail(AP_ERR_INVALID, "rank slice [%llu, %llu) empty or beyond N=%llu",
                (unsigned long long)rank_lo, (unsigned long long)rank_hi, (unsigned long long)N);
  const unsigned __int128 NK = (unsigned __int128)N * (unsigned)(k_hi - k_lo + 1);
  const int rb = bitlen(NK - 1);
  cudaStream_t s = S_(stream);
  DeviceGuard g(plan->device);
  ap_launch_info info{};
  Scratch sc(s, plan->pool);
  int16_t* d_arg;
  int32_t* d_a1;
  int64_t* d_val;
  st = run_alg1(plan, p, sc, &d_arg, &d_a1, &d_val);
  if (st != AP_OK) return st;
  // T_ref = min over k in [k_lo, k_hi] of T(Alg.-1 partition, k): an attained T, so the
  // argmin has T <= T_ref (the memory mode keeps k_lo: its feasibility test is per plan)
  const int nk = mem ? 1 : k_hi - k_lo + 1;
  int64_t* d_tref;
  AP_CUDA(sc.get((void**)&d_tref, 8 * (size_t)nk));
  int launches = 1;
  {
    const EvalFast ef = eval_fast(plan, p);
    AP_CUDA(apk::launch_eval(plan->dev(), plan->pool, p, m, p > 1 ? d_a1 : nullptr, 0, nullptr, k_lo, 1,
                             nk, d_tref, nullptr, s, &launches, 1, 0, ef.S, ef.CR, ef.div1));
  }
  // Everything that depends on T_ref -- S = T_ref + 1, the u32 choice, its clamp
  // schedule, the key-packing test -- is computed on the device (k_sweep_prep) and read
  // by the sweep kernels: no host synchronisation inside the search.
  // The host only decides what cannot depend on T_ref: which kernels exist for this
  // (p, m, mode) and whether a u32 sweep is possible at all (S >= 1).
  const unsigned __int128 wrow = (unsigned __int128)(plan->sum_f + plan->sum_b) +
                                 (unsigned __int128)2 * (p - 1) * (uint64_t)plan->max_comm + 1;
  const unsigned __int128 lim = ((unsigned __int128)1 << 32) - 1;
  // test/bench overrides: AP_SWEEP=int64 disables the u32 path, AP_SWEEP=generic
  // also the p-specialised kernel (both remain exact)
  const char* ov = getenv("AP_SWEEP");
  int force_generic = 0;
  bool allow_u32 = !mem;
  if (ov && strcmp(ov, "int64") == 0) allow_u32 = false;
  if (ov && strcmp(ov, "generic") == 0) {
    allow_u32 = false;
    force_generic = 1;
  }
  if (mem) force_generic = 1;  // memory mode: the generic exact kernel with the filter
  const bool exact = apk::sweep_has_exact(p, m, mem ? AP_SEARCH_FULL : mode, force_generic, mem);
  // u32 needs r_allow = floor((2^32-1-S)/W) >= p + 1 for some S >= 1
  const int try_u32 = (allow_u32 && exact && (unsigned __int128)(p + 2) * wrow < lim) ? 1 : 0;
  apk::SweepDev* d_sweep = nullptr;
  AP_CUDA(g_timer.sweep_buffer(plan->device, &d_sweep));
  if (key) AP_CUDA(apk::launch_init_key(reinterpret_cast<unsigned long long*>(key), nullptr, s));
  {
    apk::PrepArgs pa{};
    pa.trefs = reinterpret_cast<const long long*>(d_tref);
    pa.nk = nk;
    pa.p = p;
    pa.m = m;
    pa.rb = rb;
    pa.try_u32 = try_u32;
    pa.wrow = (unsigned long long)wrow;
    pa.t_bound = t_bound;
    pa.key = reinterpret_cast<unsigned long long*>(key);
    pa.n = plan->n;
    if (mem) {
      // the overflow guard's bound on any T (every candidate stays) if Alg. 1's
      // partition does not fit
      const unsigned __int128 tot = (unsigned __int128)m * (uint64_t)(plan->sum_f + plan->sum_b) +
                                    (unsigned __int128)2 * m * (p - 1) * (uint64_t)plan->max_comm;
      pa.a1 = d_a1;
      pa.mem = plan->d_mem;
      pa.mem_cap = plan->mem_cap;
      pa.mem_tot = (long long)tot;
    }
    AP_CUDA(apk::launch_sweep_prep(pa, d_sweep, s));
    ++launches;
  }
  apk::SweepPlan sp{};
  unsigned long long* rec = nullptr;
  if (!key) AP_CUDA(sc.get((void**)&rec, 16 * (size_t)apk::sweep_max_blocks(plan->device)));
  // warp-dynamic work cursor for the p-specialised sweep;
  // AP_SWEEP_SCHED=static keeps the one-chunk-per-thread split (A/B measurements)
  unsigned long long* ctr = nullptr;
  const char* sched = getenv("AP_SWEEP_SCHED");
  if (!(sched && strcmp(sched, "static") == 0)) AP_CUDA(sc.get((void**)&ctr, 16));
  AP_CUDA(g_timer.record(0, s, plan->device));
  // one-umulhi floor(v/k) for the slice pieces when every divided value (a stage's
  // compute total, a comm) is below 2^28 (ap_kernels.cu divk); AP_DIV1=0 disables it
  const char* dv = getenv("AP_DIV1");
  const int div1 = (plan->sum_f < (1ll << 28) && plan->max_comm < (1ll << 28) &&
                    !(dv && dv[0] == '0')) ? 1 : 0;
  AP_CUDA(apk::launch_sweep(plan->dev(), p, m, k_lo, k_hi, rank_lo, rank_hi, d_sweep, rb, try_u32,
                            force_generic, mem ? AP_SEARCH_FULL : mode,
                            reinterpret_cast<unsigned long long*>(key), s, &sp, rec,
                            mem ? plan->d_mem : nullptr, plan->mem_cap, ctr, div1));
  launches += (exact && try_u32) ? 2 : 1;
  if (rec) {
    AP_CUDA(apk::launch_reduce2(rec, sp.blocks, reinterpret_cast<long long*>(out2), s));
    ++launches;
  }
  AP_CUDA(g_timer.record(1, s, plan->device));
  g_timer.sims_on_device = false;
  g_timer.sweep_pending = true;
  g_timer.host_sims = (rank_hi - rank_lo) * (uint64_t)(k_hi - k_lo + 1);
  if (key) ++launches;  // k_init_key
  info.fast_u32 = sp.fast_u32;
  info.exact_p = sp.exact_p;
  info.blocks = sp.blocks;
  info.threads = sp.threads;
  info.chunk = sp.chunk;
  info.t_ref = -1;       // device values, filled in by ap_last_launch
  info.rank_bits = rb;
  info.launches = launches;
  g_last = info;
  return AP_OK;
}

}  // namespace

extern "C" {

ap_status ap_search_exhaustive_mode(const ap_plan* plan, int32_t p, int32_t m, int32_t k_lo,
                                    int32_t k_hi, uint64_t rank_lo, uint64_t rank_hi,
                                    int32_t mode, int64_t* key, ap_stream_t stream) {
  if (!key) {
    g_err.clear();
    return fail(AP_ERR_INVALID, "key is NULL");
  }
  return search_exhaustive_impl(plan, p, m, k_lo, k_hi, rank_lo, rank_hi, mode, key, nullptr,
                                stream);
}

ap_status ap_search_exhaustive2(const ap_plan* plan, int32_t p, int32_t m, int32_t k_lo,
                                int32_t k_hi, uint64_t rank_lo, uint64_t rank_hi, int32_t mode,
                                int64_t* out, ap_stream_t stream) {
  if (!out) {
    g_err.clear();
    return fail(AP_ERR_INVALID, "out is NULL");
  }
  return search_exhaustive_impl(plan, p, m, k_lo, k_hi, rank_lo, rank_hi, mode, nullptr, out,
                                stream);
}

ap_status ap_search_exhaustive_bounded(const ap_plan* plan, int32_t p, int32_t m, int32_t k_lo,
                                       int32_t k_hi, uint64_t rank_lo, uint64_t rank_hi,
                                       int32_t mode, int64_t t_bound, int64_t* out,
                                       ap_stream_t stream) {
  g_err.clear();
  if (!out) return fail(AP_ERR_INVALID, "out is NULL");
  if (t_bound < 0) return fail(AP_ERR_INVALID, "t_bound %lld < 0", (long long)t_bound);
  return search_exhaustive_impl(plan, p, m, k_lo, k_hi, rank_lo, rank_hi, mode, nullptr, out,
                                stream, t_bound);
}

ap_status ap_key2_select(const int64_t* local, const int64_t* t_star, int64_t* idx,
                         ap_stream_t stream) {
  g_err.clear();
  if (!local || !t_star || !idx) return fail(AP_ERR_INVALID, "NULL pointer");
  AP_CUDA(apk::launch_key2_select(reinterpret_cast<const long long*>(local),
                                  reinterpret_cast<const long long*>(t_star),
                                  reinterpret_cast<long long*>(idx), S_(stream)));
  return AP_OK;
}

// u32 fast path of the restart kernels: every value grows by at most
// W_row per row and is clamped to S every CR rows (the cool-down adds p more rows), so
// S = 2^32-1 - (max(CR,p)+1)*W_row keeps everything exact below S; 0 = no fast path.
// Test overrides: AP_HEUR=int64 disables it; AP_HEUR_S=<v> lowers the bound so that
// simulations saturate and exercise the exact fallbacks.
static uint32_t heur_fast_bound(const ap_plan* plan, int p, int CR) {
  const unsigned __int128 hw = (unsigned __int128)(plan->sum_f + plan->sum_b) +
                               (unsigned __int128)2 * (p - 1) * (uint64_t)plan->max_comm + 1;
  const unsigned __int128 span = hw * (unsigned __int128)((CR > p ? CR : p) + 1);
  const unsigned __int128 lim32 = ((unsigned __int128)1 << 32) - 1;
  uint32_t fastS = 0;
  if (span < lim32) fastS = (uint32_t)(lim32 - span);
  const char* hov = getenv("AP_HEUR");
  if (hov && strcmp(hov, "int64") == 0) fastS = 0;
  const char* hs = getenv("AP_HEUR_S");
  if (hs && fastS > 0) {
    const unsigned long long v = strtoull(hs, nullptr, 10);
    if (v > 0 && v < fastS) fastS = (uint32_t)v;
  }
  return fastS;
}

ap_status ap_search_heuristic(const ap_plan* plan, int32_t p, int32_t m, uint64_t seed,
                              int32_t radius, uint32_t r_lo, uint32_t r_hi, int32_t adjust_mode,
                              int64_t* key, ap_stream_t stream) {
  g_err.clear();
  ap_status st = check_pm(plan, p, m);
  if (st != AP_OK) return st;
  if (!key) return fail(AP_ERR_INVALID, "key is NULL");
  if (adjust_mode != 0 && adjust_mode != 1)
    return fail(AP_ERR_INVALID, "adjust_mode %d (0 none, 1 Eq. (1))", adjust_mode);
  st = check_key43(plan, p, m);
  if (st != AP_OK) return st;
  if (r_lo >= r_hi || r_hi > (1u << 20)) return fail(AP_ERR_INVALID, "restart range [%u, %u)", r_lo, r_hi);
  if (radius < 0 || radius > (1 << 20)) return fail(AP_ERR_INVALID, "radius %d", radius);
  cudaStream_t s = S_(stream);
  DeviceGuard g(plan->device);
  Scratch sc(s, plan->pool);
  int16_t* d_arg;
  int32_t* d_a1;
  int64_t* d_val;
  st = run_alg1(plan, p, sc, &d_arg, &d_a1, &d_val);
  if (st != AP_OK) return st;
  unsigned int* d_ctr;
  AP_CUDA(sc.get((void**)&d_ctr, 4 * (size_t)(3 + (r_hi - r_lo))));
  unsigned long long* d_sims = nullptr;
  AP_CUDA(g_timer.sims_buffer(plan->device, &d_sims));
  AP_CUDA(cudaMemsetAsync(d_sims, 0, 8, s));
  // decode cache: each restart's best cut vector (int16, (r_hi-r_lo) x (p-1))
  const size_t need = (size_t)(r_hi - r_lo) * (size_t)(p > 1 ? p - 1 : 1) * 2;
  g_hcache.valid = false;
  if (g_hcache.dev != plan->device || g_hcache.cap < need) {
    // stream-ordered (no device-wide synchronisation inside the search)
    if (g_hcache.d_best && g_hcache.dev == plan->device) cudaFreeAsync(g_hcache.d_best, s);
    if (g_hcache.done && g_hcache.dev != plan->device) {
      cudaEventDestroy(g_hcache.done);  // an event belongs to the device it was made on
      g_hcache.done = nullptr;
    }
    g_hcache.d_best = nullptr;
    g_hcache.cap = 0;
    AP_CUDA(cudaMallocFromPoolAsync((void**)&g_hcache.d_best, need, plan->pool, s));
    g_hcache.cap = need;
    g_hcache.dev = plan->device;
  }
  const int hCR = 32;
  const uint32_t fastS = heur_fast_bound(plan, p, hCR);
  AP_CUDA(apk::launch_init_key(reinterpret_cast<unsigned long long*>(key), d_ctr, s));
  AP_CUDA(g_timer.record(0, s, plan->device));
  AP_CUDA(apk::launch_heuristic(plan->dev(), p, m, seed, radius, r_lo, r_hi, d_arg, d_a1, d_ctr,
                                reinterpret_cast<unsigned long long*>(key), nullptr, d_sims,
                                g_hcache.d_best, fastS, hCR, adjust_mode, s));
  g_hcache.plan_gen = plan->gen;
  g_hcache.p = p;
  g_hcache.m = m;
  g_hcache.seed = seed;
  g_hcache.radius = radius;
  g_hcache.r_lo = r_lo;
  g_hcache.r_hi = r_hi;
  g_hcache.adjust_mode = adjust_mode;
  if (g_hcache.done == nullptr)  // g_hcache.dev == plan->device here (the buffer's device)
    AP_CUDA(cudaEventCreateWithFlags(&g_hcache.done, cudaEventDisableTiming));
  AP_CUDA(cudaEventRecord(g_hcache.done, s));
  g_hcache.valid = true;
  AP_CUDA(g_timer.record(1, s, plan->device));
  g_timer.sims_on_device = true;
  ap_launch_info info{};
  info.launches = 3;  // alg1, init, restarts
  g_last = info;
  return AP_OK;
}

ap_status ap_search_reachable(const ap_plan* plan, int32_t p, int32_t m, uint64_t seed,
                              int32_t radius, uint32_t r_lo, uint32_t r_hi, int32_t vmax,
                              int64_t* key, ap_stream_t stream) {
  g_err.clear();
  ap_status st = check_pm(plan, p, m);
  if (st != AP_OK) return st;
  if (!key) return fail(AP_ERR_INVALID, "key is NULL");
  st = check_key43(plan, p, m);
  if (st != AP_OK) return st;
  if (r_lo >= r_hi || r_hi > (1u << 20)) return fail(AP_ERR_INVALID, "restart range [%u, %u)", r_lo, r_hi);
  if (radius < 0 || radius > (1 << 20)) return fail(AP_ERR_INVALID, "radius %d", radius);
  if (vmax < 1 || vmax > (1 << 20)) return fail(AP_ERR_INVALID, "vmax %d outside [1, 2^20]", vmax);
  cudaStream_t s = S_(stream);
  DeviceGuard g(plan->device);
  Scratch sc(s, plan->pool);
  int16_t* d_arg;
  int32_t* d_a1;
  int64_t* d_val;
  st = run_alg1(plan, p, sc, &d_arg, &d_a1, &d_val);
  if (st != AP_OK) return st;
  unsigned int* d_ctr;
  AP_CUDA(sc.get((void**)&d_ctr, 16));
  size_t bytes = 0;
  AP_CUDA(apk::reach_scratch_bytes(plan->dev(), p, m, r_hi - r_lo, vmax, &bytes));
  void* d_scr = nullptr;
  if (sc.get(&d_scr, bytes) != cudaSuccess)
    return fail(AP_ERR_NOMEM, "reachable-set scratch: %zu bytes", bytes);
  unsigned long long* d_sims = nullptr;
  AP_CUDA(g_timer.sims_buffer(plan->device, &d_sims));
  AP_CUDA(cudaMemsetAsync(d_sims, 0, 16, s));
  AP_CUDA(apk::launch_init_key(reinterpret_cast<unsigned long long*>(key), d_ctr, s));
  AP_CUDA(g_timer.record(0, s, plan->device));
  AP_CUDA(apk::launch_reach(plan->dev(), p, m, seed, radius, r_lo, r_hi, vmax, d_arg, d_a1, d_ctr,
                            reinterpret_cast<unsigned long long*>(key), d_sims, nullptr, d_scr,
                            s, heur_fast_bound(plan, p, 32)));
  AP_CUDA(g_timer.record(1, s, plan->device));
  g_timer.sims_on_device = true;
  g_timer.truncated_valid = true;
  ap_launch_info info{};
  info.launches = 3;  // alg1, init, search
  g_last = info;
  return AP_OK;
}

ap_status ap_decode_reachable(const ap_plan* plan, int32_t p, int32_t m, uint64_t seed,
                              int32_t radius, int32_t vmax, int64_t key, ap_result* out) {
  g_err.clear();
  ap_status st = check_pm(plan, p, m);
  if (st != AP_OK) return st;
  if (!out) return fail(AP_ERR_INVALID, "out is NULL");
  if (key == INT64_MAX || key < 0) return fail(AP_ERR_INVALID, "empty key (no candidate found)");
  if (vmax < 1 || vmax > (1 << 20)) return fail(AP_ERR_INVALID, "vmax %d", vmax);
  memset(out, 0, sizeof *out);
  out->p = p;
  out->k = 1;
  const int64_t keyT = key >> 20;
  const uint32_t r = (uint32_t)(key & ((1 << 20) - 1));
  out->restart = r;
  DeviceGuard g(plan->device);
  cudaStream_t s;
  AP_CUDA(internal_stream(plan->device, &s));
  ap_status res = AP_OK;
  {
    Scratch sc(s, plan->pool);
    int16_t* d_arg;
    int32_t* d_a1;
    int64_t* d_val;
    int32_t* d_cuts = nullptr;
    int32_t* d_master = nullptr;
    int64_t* d_T = nullptr;
    unsigned int* d_ctr = nullptr;
    unsigned long long* d_key = nullptr;
    void* d_scr = nullptr;
    size_t bytes = 0;
    res = run_alg1(plan, p, sc, &d_arg, &d_a1, &d_val);
    cudaError_t e = cudaSuccess;
    if (res == AP_OK) {
      e = sc.get((void**)&d_cuts, 4 * 32);
      if (e == cudaSuccess) e = sc.get((void**)&d_master, 16);
      if (e == cudaSuccess) e = sc.get((void**)&d_T, 16);
      if (e == cudaSuccess) e = sc.get((void**)&d_ctr, 16);
      if (e == cudaSuccess) e = sc.get((void**)&d_key, 16);
      if (e == cudaSuccess) e = apk::reach_scratch_bytes(plan->dev(), p, m, 1, vmax, &bytes);
      if (e == cudaSuccess) e = sc.get(&d_scr, bytes);
      if (e != cudaSuccess) res = fail(AP_ERR_NOMEM, "decode scratch");
    }
    if (res == AP_OK) {
      // replay restart r alone: its best cut vector (first-evaluated least T)
      e = apk::launch_init_key(d_key, d_ctr, s);
      if (e == cudaSuccess)
        e = apk::launch_reach(plan->dev(), p, m, seed, radius, r, r + 1, vmax, d_arg, d_a1, d_ctr,
                              d_key, nullptr, p > 1 ? d_cuts : nullptr, d_scr, s);
      int launches = 0;
      if (e == cudaSuccess)
        e = apk::launch_eval(plan->dev(), plan->pool, p, m, p > 1 ? d_cuts : nullptr, 0, nullptr, 1,
                             0, 1, d_T, d_master, s, &launches, 1, 0, eval_fast(plan, p).S,
                             eval_fast(plan, p).CR, eval_fast(plan, p).div1);
      int32_t hc[32] = {0};
      int64_t T = -1;
      int32_t M = -1;
      if (e == cudaSuccess && p > 1)
        e = cudaMemcpyAsync(hc, d_cuts, 4 * (size_t)(p - 1), cudaMemcpyDeviceToHost, s);
      if (e == cudaSuccess) e = cudaMemcpyAsync(&T, d_T, 8, cudaMemcpyDeviceToHost, s);
      if (e == cudaSuccess) e = cudaMemcpyAsync(&M, d_master, 4, cudaMemcpyDeviceToHost, s);
      if (e == cudaSuccess) e = cudaStreamSynchronize(s);
      if (e != cudaSuccess) {
        res = fail(AP_ERR_CUDA, "reachable decode: %s", cudaGetErrorString(e));
      } else {
        if (p > 1) memcpy(out->cuts, hc, 4 * (p - 1));
        out->time_ns = T;
        out->master = M;
        if (T != keyT)
          res = fail(AP_ERR_INVALID, "key does not decode: T(key)=%lld, re-simulated %lld",
                     (long long)keyT, (long long)T);
      }
    }
  }
  cudaStreamSynchronize(s);
  return res;
}

ap_status ap_last_truncated(uint64_t* truncated) {
  if (!truncated) return fail(AP_ERR_INVALID, "truncated is NULL");
  if (!g_timer.armed) return fail(AP_ERR_INVALID, "no search launched on this thread");
  if (!g_timer.truncated_valid) {
    *truncated = 0;
    return AP_OK;
  }
  cudaError_t e = cudaEventSynchronize(g_timer.ev[1]);
  unsigned long long v[2] = {0, 0};
  if (e == cudaSuccess) e = cudaMemcpy(v, g_timer.d_sims, 16, cudaMemcpyDeviceToHost);
  if (e != cudaSuccess) return fail(AP_ERR_CUDA, "truncated read: %s", cudaGetErrorString(e));
  *truncated = v[1];
  return AP_OK;
}

ap_status ap_decode(const ap_plan* plan, int32_t mode, int32_t p, int32_t m, int32_t k_lo,
                    int32_t k_hi, uint64_t seed, int32_t radius, int32_t adjust_mode, int64_t key,
                    ap_result* out) {
  g_err.clear();
  ap_status st = check_pm(plan, p, m);
  if (st != AP_OK) return st;
  if (!out) return fail(AP_ERR_INVALID, "out is NULL");
  if (key == AP_KEY_RANGE)
    return fail(AP_ERR_RANGE, "key packing: T_ref << rank bits does not fit in 63 bits "
                "(use ap_search_exhaustive2)");
  if (key == INT64_MAX || key < 0) return fail(AP_ERR_INVALID, "empty key (no candidate found)");
  memset(out, 0, sizeof *out);
  out->p = p;
  DeviceGuard g(plan->device);
  cudaStream_t s;
  AP_CUDA(internal_stream(plan->device, &s));
  ap_status res = AP_OK;
  {
    Scratch sc(s, plan->pool);
    int32_t* d_cuts = nullptr;
    int32_t* d_master = nullptr;
    int64_t* d_T = nullptr;
    int64_t keyT = 0;
    int kk = 1;
    cudaError_t e = sc.get((void**)&d_cuts, 4 * 32);
    if (e == cudaSuccess) e = sc.get((void**)&d_master, 16);
    if (e == cudaSuccess) e = sc.get((void**)&d_T, 16);
    if (e != cudaSuccess) res = fail(AP_ERR_NOMEM, "decode scratch");
    bool checkT = true;
    if (res == AP_OK && (mode == 0 || mode == 2)) {
      uint64_t N;
      res = ap_count(plan->n, p, &N);
      if (res == AP_OK) {
        if (k_lo < 1 || k_hi < k_lo || k_hi > AP_MAX_K) res = fail(AP_ERR_INVALID, "k range");
      }
      if (res == AP_OK) {
        const uint64_t K = (uint64_t)(k_hi - k_lo + 1);
        const int rb = bitlen((unsigned __int128)N * K - 1);
        uint64_t idx;
        if (mode == 0) {
          keyT = (int64_t)((uint64_t)key >> rb);
          idx = (uint64_t)key & ((rb == 0) ? 0ull : ((1ull << rb) - 1));
        } else {  // two-phase: the key is the index itself (ap_search_exhaustive2)
          idx = (uint64_t)key;
          checkT = false;
        }
        const uint64_t rank = idx / K;
        kk = k_lo + (int)(idx % K);
        if (rank >= N) res = fail(AP_ERR_INVALID, "rank %llu >= N", (unsigned long long)rank);
        out->rank = rank;
        out->k = kk;
        if (res == AP_OK && p > 1) {
          e = apk::launch_unrank(plan->dev(), p, rank, d_cuts, s);
          if (e != cudaSuccess) res = fail(AP_ERR_CUDA, "unrank: %s", cudaGetErrorString(e));
        }
      }
    } else if (res == AP_OK && mode == 1) {
      if (adjust_mode != 0 && adjust_mode != 1)
        res = fail(AP_ERR_INVALID, "adjust_mode %d", adjust_mode);
      keyT = key >> 20;
      const uint32_t r = (uint32_t)(key & ((1 << 20) - 1));
      out->restart = r;
      out->k = 1;
      kk = 1;
      int16_t* d_arg;
      int32_t* d_a1;
      int64_t* d_val;
      unsigned int* d_ctr;
      unsigned long long* d_key;
      const bool cached = g_hcache.valid && g_hcache.plan_gen == plan->gen && g_hcache.p == p &&
                          g_hcache.adjust_mode == adjust_mode &&
                          g_hcache.m == m && g_hcache.seed == seed &&
                          g_hcache.radius == radius && r >= g_hcache.r_lo &&
                          r < g_hcache.r_hi && g_hcache.dev == plan->device && p > 1;
      if (res == AP_OK && cached) {
        // the search kernel already wrote restart r's best cuts: order this stream after
        // it and widen them to int32 on the device (no host round trip)
        e = cudaStreamWaitEvent(s, g_hcache.done, 0);
        if (e == cudaSuccess)
          e = apk::launch_widen16(g_hcache.d_best + (size_t)(r - g_hcache.r_lo) * (p - 1), d_cuts,
                                  p - 1, s);
        if (e != cudaSuccess) res = fail(AP_ERR_CUDA, "decode cache: %s", cudaGetErrorString(e));
      } else if (res == AP_OK) res = run_alg1(plan, p, sc, &d_arg, &d_a1, &d_val);
      if (res == AP_OK && !cached) {
        e = sc.get((void**)&d_ctr, 16);
        if (e == cudaSuccess) e = sc.get((void**)&d_key, 16);
        if (e == cudaSuccess) e = apk::launch_init_key(d_key, d_ctr, s);
        if (e == cudaSuccess)
          e = apk::launch_heuristic(plan->dev(), p, m, seed, radius, r, r + 1, d_arg, d_a1, d_ctr,
                                    d_key, d_cuts, nullptr, nullptr, 0, 1, adjust_mode, s);
        if (e != cudaSuccess) res = fail(AP_ERR_CUDA, "replay: %s", cudaGetErrorString(e));
      }
    } else if (res == AP_OK) {
      res = fail(AP_ERR_INVALID, "mode %d", mode);
    }
    if (res == AP_OK) {
      int launches = 0;
      const EvalFast ef = eval_fast(plan, p);
      e = apk::launch_eval(plan->dev(), plan->pool, p, m, p > 1 ? d_cuts : nullptr, 0, nullptr, kk, 0, 1, d_T,
                           d_master, s, &launches, 1, 0, ef.S, ef.CR, ef.div1);
      int32_t hc[32] = {0};
      int64_t T = -1;
      int32_t M = -1;
      if (e == cudaSuccess && p > 1)
        e = cudaMemcpyAsync(hc, d_cuts, 4 * (size_t)(p - 1), cudaMemcpyDeviceToHost, s);
      if (e == cudaSuccess) e = cudaMemcpyAsync(&T, d_T, 8, cudaMemcpyDeviceToHost, s);
      if (e == cudaSuccess) e = cudaMemcpyAsync(&M, d_master, 4, cudaMemcpyDeviceToHost, s);
      if (e == cudaSuccess) e = cudaStreamSynchronize(s);
      if (e != cudaSuccess) {
        res = fail(AP_ERR_CUDA, "decode eval: %s", cudaGetErrorString(e));
      } else {
        if (p > 1) memcpy(out->cuts, hc, 4 * (p - 1));
        out->time_ns = T;
        out->master = M;
        if (checkT && T != keyT)
          res = fail(AP_ERR_INVALID, "key does not decode: T(key)=%lld, re-simulated %lld",
                     (long long)keyT, (long long)T);
        if (mode == 1 && res == AP_OK) {
          // rank of the heuristic winner, for reference (host arithmetic on the result)
          uint64_t r = 0;
          int prev = 0;
          for (int x = 1; x <= p - 1; ++x) {
            for (int v = prev + 1; v <= hc[x - 1] - 1; ++v) r += binom_sat(plan->n - 1 - v, p - 1 - x);
            prev = hc[x - 1];
          }
          out->rank = r;
        }
      }
    }
  }
  cudaStreamSynchronize(s);
  return res;
}

ap_status ap_slice_sweep(const ap_plan* plan, int32_t p, int32_t m, const int32_t* cuts,
                         int32_t k_max, int64_t* time_ns, int32_t* best_k) {
  g_err.clear();
  ap_status st = check_pm(plan, p, m);
  if (st != AP_OK) return st;
  if (k_max < 1 || k_max > AP_MAX_K) return fail(AP_ERR_INVALID, "k_max=%d", k_max);
  if (!time_ns || !best_k || (p > 1 && !cuts)) return fail(AP_ERR_INVALID, "NULL argument");
  DeviceGuard g(plan->device);
  cudaStream_t s;
  AP_CUDA(internal_stream(plan->device, &s));
  ap_status res = AP_OK;
  {
    Scratch sc(s, plan->pool);
    int32_t* d_cuts;
    int64_t* d_T;
    cudaError_t e = sc.get((void**)&d_cuts, 4 * 32);
    if (e == cudaSuccess) e = sc.get((void**)&d_T, 8 * (size_t)k_max);
    if (e == cudaSuccess && p > 1)
      e = cudaMemcpyAsync(d_cuts, cuts, 4 * (size_t)(p - 1), cudaMemcpyHostToDevice, s);
    int launches = 0;
    if (e == cudaSuccess)
      e = apk::launch_eval(plan->dev(), plan->pool, p, m, p > 1 ? d_cuts : nullptr, 0, nullptr, 1, 1, k_max,
                           d_T, nullptr, s, &launches, 1, 0, eval_fast(plan, p).S,
                           eval_fast(plan, p).CR, eval_fast(plan, p).div1);
    if (e == cudaSuccess)
      e = cudaMemcpyAsync(time_ns, d_T, 8 * (size_t)k_max, cudaMemcpyDeviceToHost, s);
    if (e == cudaSuccess) e = cudaStreamSynchronize(s);
    if (e != cudaSuccess) res = fail(AP_ERR_CUDA, "slice sweep: %s", cudaGetErrorString(e));
  }
  cudaStreamSynchronize(s);
  if (res != AP_OK) return res;
  if (time_ns[0] < 0) return fail(AP_ERR_INVALID, "invalid cut vector");
  int bk = 1;
  for (int q = 2; q <= k_max; ++q)
    if (time_ns[q - 1] < time_ns[bk - 1]) bk = q;  // min (T, k)
  *best_k = bk;
  return AP_OK;
}

ap_status ap_slice_sweep_paper(const ap_plan* plan, int32_t p, int32_t m, const int32_t* cuts,
                               int32_t k, int32_t s_max, int64_t* time_ns, int32_t* best_s) {
  g_err.clear();
  ap_status st = check_pm(plan, p, m);
  if (st != AP_OK) return st;
  if (k < 1 || k > AP_MAX_K) return fail(AP_ERR_INVALID, "k=%d", k);
  if (s_max < 0 || s_max > m) return fail(AP_ERR_INVALID, "s_max=%d outside [0, m]", s_max);
  if (!time_ns || !best_s || (p > 1 && !cuts)) return fail(AP_ERR_INVALID, "NULL argument");
  DeviceGuard g(plan->device);
  cudaStream_t s;
  AP_CUDA(internal_stream(plan->device, &s));
  ap_status res = AP_OK;
  {
    Scratch sc(s, plan->pool);
    int32_t* d_cuts;
    int64_t* d_T;
    cudaError_t e = sc.get((void**)&d_cuts, 4 * 32);
    if (e == cudaSuccess) e = sc.get((void**)&d_T, 8 * (size_t)(s_max + 1));
    if (e == cudaSuccess && p > 1)
      e = cudaMemcpyAsync(d_cuts, cuts, 4 * (size_t)(p - 1), cudaMemcpyHostToDevice, s);
    int launches = 0;
    if (e == cudaSuccess)
      e = apk::launch_eval(plan->dev(), plan->pool, p, m, p > 1 ? d_cuts : nullptr, 0, nullptr, k, 0,
                           s_max + 1, d_T, nullptr, s, &launches, 0, 1);
    if (e == cudaSuccess)
      e = cudaMemcpyAsync(time_ns, d_T, 8 * (size_t)(s_max + 1), cudaMemcpyDeviceToHost, s);
    if (e == cudaSuccess) e = cudaStreamSynchronize(s);
    if (e != cudaSuccess) res = fail(AP_ERR_CUDA, "paper slice sweep: %s", cudaGetErrorString(e));
  }
  cudaStreamSynchronize(s);
  if (res != AP_OK) return res;
  if (time_ns[0] < 0) return fail(AP_ERR_INVALID, "invalid cut vector");
  int bs = 0;
  for (int q = 1; q <= s_max; ++q)
    if (time_ns[q] < time_ns[bs]) bs = q;  // min (T, s)
  *best_s = bs;
  return AP_OK;
}

ap_status ap_slicer_alg2(const ap_plan* plan, int32_t p, const int32_t* cuts, int32_t reading,
                         int32_t* mb) {
  g_err.clear();
  if (!plan) return fail(AP_ERR_INVALID, "plan is NULL");
  if (p < 1 || p > plan->n || p > AP_MAX_P) return fail(AP_ERR_INVALID, "p=%d", p);
  if (reading != 0 && reading != 1) return fail(AP_ERR_INVALID, "reading %d", reading);
  if (!mb || (p > 1 && !cuts)) return fail(AP_ERR_INVALID, "NULL argument");
  DeviceGuard g(plan->device);
  cudaStream_t s;
  AP_CUDA(internal_stream(plan->device, &s));
  ap_status res = AP_OK;
  int32_t h = -1;
  {
    Scratch sc(s, plan->pool);
    int32_t *d_cuts, *d_mb;
    cudaError_t e = sc.get((void**)&d_cuts, 4 * 32);
    if (e == cudaSuccess) e = sc.get((void**)&d_mb, 16);
    if (e == cudaSuccess && p > 1)
      e = cudaMemcpyAsync(d_cuts, cuts, 4 * (size_t)(p - 1), cudaMemcpyHostToDevice, s);
    if (e == cudaSuccess) e = apk::launch_alg2(plan->dev(), p, d_cuts, reading, d_mb, s);
    if (e == cudaSuccess) e = cudaMemcpyAsync(&h, d_mb, 4, cudaMemcpyDeviceToHost, s);
    if (e == cudaSuccess) e = cudaStreamSynchronize(s);
    if (e != cudaSuccess) res = fail(AP_ERR_CUDA, "alg2: %s", cudaGetErrorString(e));
  }
  cudaStreamSynchronize(s);
  if (res != AP_OK) return res;
  if (h < 0) return fail(AP_ERR_INVALID, "invalid cut vector");
  *mb = h;
  return AP_OK;
}

ap_status ap_critical_path(const ap_plan* plan, int32_t p, int32_t m, int32_t k,
                           const int32_t* cuts, ap_op* ops, int32_t cap, int32_t* len,
                           int32_t* master, int64_t* time_ns) {
  g_err.clear();
  ap_status st = check_pm(plan, p, m);
  if (st != AP_OK) return st;
  if (k < 1 || k > AP_MAX_K) return fail(AP_ERR_INVALID, "k=%d", k);
  if (cap < 0 || (cap > 0 && !ops) || (p > 1 && !cuts)) return fail(AP_ERR_INVALID, "NULL argument");
  static_assert(sizeof(ap_op) == sizeof(apk::OpRec), "ap_op layout");
  DeviceGuard g(plan->device);
  cudaStream_t s;
  AP_CUDA(internal_stream(plan->device, &s));
  ap_status res = AP_OK;
  int32_t lm[2] = {-1, -1};
  int64_t T = -1;
  {
    Scratch sc(s, plan->pool);
    int32_t *d_cuts, *d_lm;
    int64_t* d_T;
    apk::OpRec* d_ops;
    void* d_scr;
    const int cap_dev = cap > 0 ? cap : 1;
    cudaError_t e = sc.get((void**)&d_cuts, 4 * 32);
    if (e == cudaSuccess) e = sc.get((void**)&d_lm, 16);
    if (e == cudaSuccess) e = sc.get((void**)&d_T, 16);
    if (e == cudaSuccess) e = sc.get((void**)&d_ops, sizeof(apk::OpRec) * (size_t)cap_dev);
    if (e == cudaSuccess) e = sc.get(&d_scr, apk::cpath_scratch_bytes(p, m));
    if (e == cudaSuccess && p > 1)
      e = cudaMemcpyAsync(d_cuts, cuts, 4 * (size_t)(p - 1), cudaMemcpyHostToDevice, s);
    if (e == cudaSuccess)
      e = apk::launch_cpath(plan->dev(), p, m, k, d_cuts, d_ops, cap, d_lm, d_T, d_scr, s);
    if (e == cudaSuccess) e = cudaMemcpyAsync(lm, d_lm, 8, cudaMemcpyDeviceToHost, s);
    if (e == cudaSuccess) e = cudaMemcpyAsync(&T, d_T, 8, cudaMemcpyDeviceToHost, s);
    if (e == cudaSuccess) e = cudaStreamSynchronize(s);
    if (e == cudaSuccess && lm[0] > 0 && lm[0] <= cap)
      e = cudaMemcpyAsync(ops, d_ops, sizeof(ap_op) * (size_t)lm[0], cudaMemcpyDeviceToHost, s);
    if (e == cudaSuccess) e = cudaStreamSynchronize(s);
    if (e != cudaSuccess) res = fail(AP_ERR_CUDA, "critical path: %s", cudaGetErrorString(e));
  }
  cudaStreamSynchronize(s);
  if (res != AP_OK) return res;
  if (lm[0] < 0) return fail(AP_ERR_INVALID, "invalid cut vector");
  if (len) *len = lm[0];
  if (master) *master = lm[1];
  if (time_ns) *time_ns = T;
  if (lm[0] > cap) return fail(AP_ERR_CAPACITY, "path has %d ops, cap %d", lm[0], cap);
  return AP_OK;
}

}  // extern "C"
