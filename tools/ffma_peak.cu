// FFMA throughput microbenchmark (measurement tool, not product code): the register-blocked
// 8x8 outer product of the fp32 GEMM inner loop (3-register FFMA, operands reused across the
// row/column) versus the immediate form, on all SMs.  Prints TFLOP/s per variant.
#include <cstdio>
#include <cuda_runtime.h>

template <int MODE>
__global__ void __launch_bounds__(256, 2) ffma_kernel(float *out, int iters, float seed) {
  float a[8], b[8], acc[8][8];
#pragma unroll
  for (int i = 0; i < 8; ++i) { a[i] = seed * (threadIdx.x + i); b[i] = seed * (i + 1); }
#pragma unroll
  for (int i = 0; i < 8; ++i)
#pragma unroll
    for (int j = 0; j < 8; ++j) acc[i][j] = 0.f;
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int u = 0; u < 4; ++u)
#pragma unroll
      for (int i = 0; i < 8; ++i)
#pragma unroll
        for (int j = 0; j < 8; ++j) {
          if (MODE == 0) acc[i][j] = fmaf(a[i], b[j], acc[i][j]);
          else if (MODE == 1) acc[i][j] = fmaf(acc[i][j], 1.0001f, 0.5f);
          else if (MODE == 2 && (j & 1) == 0) {   // packed pair over columns, A broadcast
            float2 r = __ffma2_rn(make_float2(a[i], a[i]), make_float2(b[j], b[j + 1]),
                                  make_float2(acc[i][j], acc[i][j + 1]));
            acc[i][j] = r.x; acc[i][j + 1] = r.y;
          }
        }
  }
  float s = 0.f;
#pragma unroll
  for (int i = 0; i < 8; ++i)
#pragma unroll
    for (int j = 0; j < 8; ++j) s += acc[i][j];
  if (s == 12345.f) out[threadIdx.x] = s;
}

int main() {
  float *out;
  cudaMalloc(&out, 4096);
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  const int iters = 20000;
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  for (int mode = 0; mode < 3; ++mode) {
    for (int rep = 0; rep < 3; ++rep) {
      const int grid = sms * 2;
      cudaEventRecord(e0);
      if (mode == 0) ffma_kernel<0><<<grid, 256>>>(out, iters, 1e-7f);
      else if (mode == 1) ffma_kernel<1><<<grid, 256>>>(out, iters, 1e-7f);
      else ffma_kernel<2><<<grid, 256>>>(out, iters, 1e-7f);
      cudaEventRecord(e1);
      cudaEventSynchronize(e1);
      float ms;
      cudaEventElapsedTime(&ms, e0, e1);
      const double flop = 2.0 * grid * 256.0 * iters * 4 * 64;
      printf("%s rep %d: %.3f ms  %.2f TFLOP/s\n", mode == 0 ? "3-reg outer product" : mode == 1 ? "imm form" : "FFMA2 pairs over columns", rep, ms,
             flop / ms / 1e9);
    }
  }
  return 0;
}
