// Integer-pipe microbenchmark for the roofline denominator.
// Measures warp-instruction throughput of the max-plus building blocks on sm_100a:
//   mode 0: u32 max only (VIMNMX)          mode 1: u32 add only (VIADD/IADD3)
//   mode 2: max+add pairs (the max-plus op) mode 3: max + IMAD-forced add
//   mode 4: 64-bit max+add (int64 form)
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
#define ILP 8
template <int MODE>
__global__ void __launch_bounds__(512) kern(uint32_t* out, uint32_t w, uint32_t one, int iters) {
  uint32_t a[ILP], b[ILP];
  unsigned long long a64[ILP], b64[ILP];
#pragma unroll
  for (int i = 0; i < ILP; i++) { a[i] = threadIdx.x * (i + 1); b[i] = threadIdx.x ^ (i * 77); a64[i] = a[i]; b64[i] = b[i]; }
  for (int it = 0; it < iters; it++) {
#pragma unroll
    for (int r = 0; r < 16; r++) {
#pragma unroll
      for (int i = 0; i < ILP; i++) {
        if (MODE == 0) { a[i] = max(a[i], b[i]); b[i] = max(b[i], a[i] ^ w); }
        if (MODE == 1) { a[i] = a[i] + b[i]; b[i] = b[i] + w; }
        if (MODE == 2) { a[i] = max(a[i], b[i]) + w; b[i] = max(b[i], a[i]) + w; }
        if (MODE == 3) { a[i] = max(a[i], b[i]) * one + w; b[i] = max(b[i], a[i]) * one + w; }
        if (MODE == 4) { a64[i] = max(a64[i], b64[i]) + w; b64[i] = max(b64[i], a64[i]) + w; }
      }
    }
  }
  uint32_t s = 0;
#pragma unroll
  for (int i = 0; i < ILP; i++) s += a[i] + b[i] + (uint32_t)(a64[i] + b64[i]);
  if (s == 0x12345678u) out[0] = s;
}
int main() {
  int dev = 0; cudaDeviceProp pr; cudaGetDeviceProperties(&pr, dev);
  int clk; cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, dev);
  printf("{\"gpu\":\"%s\",\"sms\":%d,\"clock_khz_attr\":%d}\n", pr.name, pr.multiProcessorCount, clk);
  uint32_t* out; cudaMalloc(&out, 4);
  int iters = 4096; int blocks = pr.multiProcessorCount * 4, threads = 512;
  const char* names[] = {"max_u32", "add_u32", "maxplus_u32", "maxplus_u32_imad", "maxplus_u64"};
  for (int mode = 0; mode < 5; mode++) {
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    for (int rep = 0; rep < 3; rep++) {
      cudaEventRecord(e0);
      switch (mode) {
        case 0: kern<0><<<blocks, threads>>>(out, 3, 1, iters); break;
        case 1: kern<1><<<blocks, threads>>>(out, 3, 1, iters); break;
        case 2: kern<2><<<blocks, threads>>>(out, 3, 1, iters); break;
        case 3: kern<3><<<blocks, threads>>>(out, 3, 1, iters); break;
        case 4: kern<4><<<blocks, threads>>>(out, 3, 1, iters); break;
      }
      cudaEventRecord(e1); cudaEventSynchronize(e1);
    }
    float ms; cudaEventElapsedTime(&ms, e0, e1);
    double ops = (double)blocks * threads * iters * 16 * ILP * 2;  // source-level ops (each line = 2 ops/elt for modes 0,1; 2 max-plus for 2-4)
    printf("{\"mode\":\"%s\",\"ms\":%.3f,\"src_ops_per_s\":%.4e}\n", names[mode], ms, ops / (ms * 1e-3));
  }
  return 0;
}
