// FFMA throughput microbenchmark (measurement tool, not product code): the register-blocked
// 8x8 outer product of the fp32 GEMM inner loop (3-register FFMA, operands reused across the
// row/column) versus the immediate form, on all SMs.  Prints TFLOP/s per variant.
#include <cstdint>
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


// Mode 3: the fp32 GEMM kernel's inner loop (8x8 sub-tile, FFMA2, A from a 128-B swizzled
// [128][32] slice read as LDS.128 over 4 k, B from [32][32] boxes read as LDS.128), fed from
// shared memory only: the ceiling of the inner loop without any load or barrier waits.
__global__ void __launch_bounds__(256, 2) smem_loop_kernel(float *out, int iters) {
  __shared__ __align__(1024) float sm[2 * 4096];
  for (int i = threadIdx.x; i < 2 * 4096; i += 256) sm[i] = 1e-7f * (i & 63);
  __syncthreads();
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int wy = warp / 2, wx = warp % 2, ly = lane / 8, lx = lane % 8;
  const int rb = wy * 32 + ly, x0 = rb & 7;
  const uint32_t sa = (uint32_t)__cvta_generic_to_shared(sm) + rb * 128;
  const uint32_t sb = (uint32_t)__cvta_generic_to_shared(sm + 4096) + wx * 2 * 4096 + lx * 16;
  float acc[8][8];
#pragma unroll
  for (int i = 0; i < 8; ++i)
#pragma unroll
    for (int j = 0; j < 8; ++j) acc[i][j] = 0.f;
  for (int it = 0; it < iters; ++it) {
#pragma unroll 1
    for (int k4 = 0; k4 < 32; k4 += 4) {
      const uint32_t ce = (uint32_t)(((k4 >> 2) ^ x0) << 4);
      const uint32_t a_even = sa + ce, a_odd = sa + (ce ^ 64u);
      float fa[8][4];
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        float4 v;
        asm volatile("ld.shared.v4.f32 {%0, %1, %2, %3}, [%4];" : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w)
                     : "r"((i & 1 ? a_odd : a_even) + i * 512));
        fa[i][0] = v.x; fa[i][1] = v.y; fa[i][2] = v.z; fa[i][3] = v.w;
      }
      const uint32_t bk = sb + k4 * 128;
#pragma unroll
      for (int kk = 0; kk < 4; ++kk) {
        float fb[8];
#pragma unroll
        for (int gj = 0; gj < 2; ++gj)
          asm volatile("ld.shared.v4.f32 {%0, %1, %2, %3}, [%4];"
                       : "=f"(fb[gj * 4 + 0]), "=f"(fb[gj * 4 + 1]), "=f"(fb[gj * 4 + 2]), "=f"(fb[gj * 4 + 3])
                       : "r"(bk + kk * 128 + gj * 4096));
#pragma unroll
        for (int i = 0; i < 8; ++i)
#pragma unroll
          for (int j = 0; j < 8; j += 2) {
            const float2 r = __ffma2_rn(make_float2(fa[i][kk], fa[i][kk]), make_float2(fb[j], fb[j + 1]),
                                        make_float2(acc[i][j], acc[i][j + 1]));
            acc[i][j] = r.x; acc[i][j + 1] = r.y;
          }
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
  for (int rep = 0; rep < 3; ++rep) {
    const int grid = sms * 2, it2 = 2000;
    cudaEventRecord(e0);
    smem_loop_kernel<<<grid, 256>>>(out, it2);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    const double flop = 2.0 * grid * 256.0 * it2 * 32 * 64;
    printf("smem-fed GEMM inner loop rep %d: %.3f ms  %.2f TFLOP/s\n", rep, ms, flop / ms / 1e9);
  }
  return 0;
}
