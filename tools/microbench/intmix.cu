// Per-instruction issue rate on sm_100a (warp instructions / clock / SMSP) for the
// candidate SASS forms of a max-plus op.  8 independent chains per thread so the
// pipes, not latency, bound each loop.  Verify the SASS with cuobjdump.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
#define N 8
__device__ __forceinline__ uint32_t opaque(uint32_t v) { asm volatile("" : "+r"(v)); return v; }

template <int MODE>
__global__ void __launch_bounds__(512) kern(uint32_t* out, uint32_t w, uint32_t one, int iters) {
  uint32_t a[N], b[N], c[N];
#pragma unroll
  for (int i = 0; i < N; i++) { a[i] = threadIdx.x * (i + 1); b[i] = threadIdx.x ^ (i * 77); c[i] = i; }
  for (int it = 0; it < iters; it++) {
#pragma unroll
    for (int r = 0; r < 8; r++) {
#pragma unroll
      for (int i = 0; i < N; i++) {
        if (MODE == 0) { a[i] = max(a[i], b[i]); b[i] = max(b[i], c[i]); c[i] = max(c[i], a[i]); } // VIMNMX x3 (counted as 2)
        if (MODE == 1) { a[i] = __vimax3_u32(a[i], b[i], c[i]); b[i] = __vimax3_u32(b[i], a[i], w); }  // VIMNMX3 x2
        if (MODE == 2) { a[i] = __viaddmax_u32(a[i], w, b[i]); b[i] = __viaddmax_u32(b[i], w, a[i]); } // VIADDMNMX x2
        if (MODE == 3) { asm volatile("add.u32 %0, %0, %1;" : "+r"(a[i]) : "r"(w)); asm volatile("add.u32 %0, %0, %1;" : "+r"(b[i]) : "r"(a[i])); }
        if (MODE == 4) { a[i] = a[i] * one + b[i]; b[i] = b[i] * one + a[i]; }             // IMAD
        if (MODE == 5) { a[i] = a[i] + b[i] + w; b[i] = b[i] + a[i] + c[i]; }              // IADD3
        if (MODE == 6) { a[i] = max(a[i], b[i]) + w; b[i] = max(b[i], a[i]) + w; }         // VIMNMX + add (compiler)
        if (MODE == 7) { uint32_t t = a[i] * one + w; a[i] = __viaddmax_u32(b[i], w, t); b[i] = b[i] * one + a[i]; } // VIADDMNMX + 2 IMAD
        if (MODE == 8) { uint32_t t; asm volatile("add.u32 %0, %1, %2;" : "=r"(t) : "r"(a[i]), "r"(w)); a[i] = __viaddmax_u32(b[i], w, t);
                         asm volatile("add.u32 %0, %1, %2;" : "=r"(t) : "r"(b[i]), "r"(a[i])); b[i] = t; } // VIADDMNMX + 2 add
      }
    }
  }
  uint32_t s = 0;
#pragma unroll
  for (int i = 0; i < N; i++) s += a[i] + b[i] + c[i];
  if (s == 0x12345678u) out[0] = s;
}
template <int M> float run(uint32_t* out, int blocks, int threads, int iters) {
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  float ms = 0;
  for (int rep = 0; rep < 3; rep++) {
    cudaEventRecord(e0);
    kern<M><<<blocks, threads>>>(out, 3, 1, iters);
    cudaEventRecord(e1); cudaEventSynchronize(e1);
    cudaEventElapsedTime(&ms, e0, e1);
  }
  return ms;
}
int main() {
  cudaDeviceProp pr; cudaGetDeviceProperties(&pr, 0);
  uint32_t* out; cudaMalloc(&out, 4);
  int iters = 4096, blocks = pr.multiProcessorCount * 4, threads = 512;
  const char* names[] = {"VIMNMX", "VIMNMX3", "VIADDMNMX", "add.u32(ptx)", "IMAD", "IADD3", "max+add", "VIADDMNMX+2IMAD", "VIADDMNMX+2add"};
  float ms[9];
  ms[0] = run<0>(out, blocks, threads, iters); ms[1] = run<1>(out, blocks, threads, iters);
  ms[2] = run<2>(out, blocks, threads, iters); ms[3] = run<3>(out, blocks, threads, iters);
  ms[4] = run<4>(out, blocks, threads, iters); ms[5] = run<5>(out, blocks, threads, iters);
  ms[6] = run<6>(out, blocks, threads, iters); ms[7] = run<7>(out, blocks, threads, iters);
  ms[8] = run<8>(out, blocks, threads, iters);
  double clk = 1.965e9;  // report per nominal max clock; the clock line is printed by the caller
  for (int m = 0; m < 9; m++) {
    double src_lines = (double)blocks * threads / 32 * iters * 8 * N * 2;  // warp-level source statements
    double per_smsp_clk = src_lines / (ms[m] * 1e-3) / (pr.multiProcessorCount * 4) / clk;
    printf("{\"mode\":\"%s\",\"ms\":%.3f,\"stmts_per_clk_per_smsp\":%.3f}\n", names[m], ms[m], per_smsp_clk);
  }
  return 0;
}
