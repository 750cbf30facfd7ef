// Steady-row (mstep) throughput in isolation: P=8 u32, variants of the add form.
//   V0: plain '+' (compiler chooses IADD3 / IMAD.IADD / VIADD)
//   V1: mad.lo with opaque one (IMAD)         V2: explicit __viaddmax + '+'
// Reports rows/clk/SM and instructions per row from the SASS (inspect separately).
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
constexpr int P = 8;
template <int MODE> __device__ __forceinline__ uint32_t ad(uint32_t a, uint32_t b, uint32_t one) {
  if (MODE == 1) { uint32_t d; asm("mad.lo.u32 %0, %1, %2, %3;" : "=r"(d) : "r"(a), "r"(one), "r"(b)); return d; }
  if (MODE == 4) { uint32_t d; asm("mad.lo.u32 %0, %1, 1, %2;" : "=r"(d) : "r"(a), "r"(b)); return d; }
  return a + b;
}
template <int MODE> __device__ __forceinline__ uint32_t amx(uint32_t a, uint32_t b, uint32_t c) {
  if (MODE == 0) { uint32_t t = a + b; return t > c ? t : c; }
  return __viaddmax_u32(a, b, c);
}
// MODE 3: offset ("potential") form: P-1 signed VIADDMNMX per row, outputs renamed
__global__ void __launch_bounds__(256) k3(const uint32_t* w, uint32_t* out, int rows, uint32_t one) {
  int32_t H[P], c[P];
  for (int x = 0; x < P; x++) { H[x] = threadIdx.x * x; c[x] = (int32_t)w[x] - (int32_t)w[P]; }
  for (int r = 0; r < rows; r += 8) {
#pragma unroll
    for (int u = 0; u < 8; u++) {
      int32_t nH[P];
      int32_t M = __viaddmax_s32(H[P - 1], c[P - 2], H[P - 2]);
      nH[P - 1] = M;
#pragma unroll
      for (int x = P - 3; x >= 0; --x) { M = __viaddmax_s32(M, c[x], H[x]); nH[x + 1] = M; }
      nH[0] = M;
#pragma unroll
      for (int x = 0; x < P; x++) H[x] = nH[x];
    }
  }
  int32_t s = 0;
  for (int x = 0; x < P; x++) s ^= H[x];
  if (s == 0x12345) out[0] = s;
}
template <int MODE>
__global__ void __launch_bounds__(256) k(const uint32_t* w, uint32_t* out, int rows, uint32_t one) {
  uint32_t FF[P], wF[P], wB[P];
  for (int x = 0; x < P; x++) { FF[x] = threadIdx.x * x; wF[x] = w[x]; wB[x] = w[P + x]; }
  const uint32_t wBF0 = wB[0] + wF[0];
  for (int r = 0; r < rows; r += 8) {
#pragma unroll
    for (int u = 0; u < 8; u++) {
      uint32_t nF[P];
      uint32_t M = amx<MODE>(FF[P - 1], wB[P - 1], FF[P - 2]);
      nF[P - 1] = ad<MODE>(M, wF[P - 1], one);
#pragma unroll
      for (int x = P - 3; x >= 0; --x) { M = amx<MODE>(M, wB[x + 1], FF[x]); nF[x + 1] = ad<MODE>(M, wF[x + 1], one); }
      nF[0] = ad<MODE>(M, wBF0, one);
#pragma unroll
      for (int x = 0; x < P; x++) FF[x] = nF[x];
    }
  }
  uint32_t s = 0;
  for (int x = 0; x < P; x++) s ^= FF[x];
  if (s == 0x12345) out[0] = s;
}
template <int MODE> void run(const char* name, uint32_t* w, uint32_t* out, int blocksPerSM) {
  cudaDeviceProp pr; cudaGetDeviceProperties(&pr, 0);
  int blocks = pr.multiProcessorCount * blocksPerSM, rows = 1 << 14;
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  float ms = 0;
  for (int rep = 0; rep < 3; rep++) {
    cudaEventRecord(e0);
    if (MODE == 3) k3<<<blocks, 256>>>(w, out, rows, 1u); else k<MODE><<<blocks, 256>>>(w, out, rows, 1u);
    cudaEventRecord(e1); cudaEventSynchronize(e1);
    cudaEventElapsedTime(&ms, e0, e1);
  }
  double warps_rows = (double)blocks * 8 * rows;
  double cyc = ms * 1e-3 * 1.965e9;
  printf("{\"variant\":\"%s\",\"blocks_per_sm\":%d,\"ms\":%.3f,\"cycles_per_row_per_smsp_warp\":%.2f}\n", name, blocksPerSM, ms,
         cyc * pr.multiProcessorCount * 4 / warps_rows);
}
int main() {
  uint32_t *w, *out; cudaMalloc(&w, 64 * 4); cudaMalloc(&out, 4);
  uint32_t hw[16] = {3, 5, 7, 11, 13, 17, 19, 23, 29, 31, 37, 41, 43, 47, 53, 59};
  cudaMemcpy(w, hw, sizeof hw, cudaMemcpyHostToDevice);
  for (int b : {2, 3, 4, 6, 8}) {
    run<0>("plus", w, out, b); run<1>("imad", w, out, b); run<4>("imad_imm1", w, out, b); run<3>("offset", w, out, b);
  }
  return 0;
}
