// Device input generator (the artifact's gen_data, PAPER.md P428): the counter-hash draw
// documented in vbinputs/__init__.py, implemented independently here so synthetic batches
// of tens of GB never go through host memory.  Tests check it bit-for-bit against vbinputs.
#include <cuda_bf16.h>
#include <cuda_fp16.h>
#include <cuda_runtime.h>
#include <stdint.h>

namespace vb {
namespace fill {

constexpr uint64_t kSalt = 0x632BE59BD9B4E019ull;

__host__ __device__ __forceinline__ uint64_t splitmix64(uint64_t x) {
  uint64_t z = x + 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

__host__ __device__ __forceinline__ uint64_t matrix_key(uint64_t seed, uint64_t gemm, uint32_t operand) {
  return splitmix64(splitmix64(seed + kSalt) ^ ((gemm << 3) | operand));
}

template <int DT>   // 0 = f32, 1 = bf16, 2 = f16
__global__ void fill_kernel(const int32_t *rows, const int32_t *cols, const int32_t *ld, void *const *ptrs,
                            const int64_t *gemm_id, uint64_t seed, uint32_t operand) {
  const int i = blockIdx.x;
  const int64_t R = rows[i], Cc = cols[i], L = ld[i];
  const int64_t n = R * Cc;
  if (n <= 0) return;
  const uint64_t key = matrix_key(seed, (uint64_t)gemm_id[i], operand);
  const int64_t stride = (int64_t)blockDim.x * gridDim.y;
  for (int64_t idx = (int64_t)blockIdx.y * blockDim.x + threadIdx.x; idx < n; idx += stride) {
    const int64_t r = idx / Cc, c = idx - r * Cc;
    const uint64_t h = splitmix64(key + (uint64_t)idx);
    const float v = (float)(uint32_t)(h >> 40) * 0x1p-23f - 1.0f;
    const int64_t off = r * L + c;
    if constexpr (DT == 0) {
      static_cast<float *>(ptrs[i])[off] = v;
    } else if constexpr (DT == 1) {
      static_cast<__nv_bfloat16 *>(ptrs[i])[off] = __float2bfloat16_rn(v);
    } else {
      static_cast<__half *>(ptrs[i])[off] = __float2half_rn(v);
    }
  }
}

__global__ void alpha_beta_kernel(int batch, const int64_t *gemm_id, uint64_t seed, float *alpha, float *beta) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= batch) return;
  const uint64_t g = (uint64_t)gemm_id[i];
  const uint64_t ha = splitmix64(matrix_key(seed, g, 3) + 0);
  const uint64_t hb = splitmix64(matrix_key(seed, g, 4) + 0);
  alpha[i] = 0.5f + (float)(uint32_t)(ha >> 41) * 0x1p-23f;
  beta[i] = (float)(uint32_t)(hb >> 40) * 0x1p-23f - 1.0f;
}

}  // namespace fill

cudaError_t launch_fill(int dt, int batch, const int32_t *rows, const int32_t *cols, const int32_t *ld,
                        void *const *ptrs, const int64_t *gemm_id, uint64_t seed, int operand, int64_t total_elems,
                        cudaStream_t stream) {
  if (batch <= 0) return cudaSuccess;
  const int64_t avg = total_elems / batch;
  int gy = (int)((avg + 256 * 32 - 1) / (256 * 32));
  gy = gy < 1 ? 1 : (gy > 512 ? 512 : gy);
  dim3 grid((unsigned)batch, (unsigned)gy);
  if (dt == 0)
    fill::fill_kernel<0><<<grid, 256, 0, stream>>>(rows, cols, ld, ptrs, gemm_id, seed, (uint32_t)operand);
  else if (dt == 1)
    fill::fill_kernel<1><<<grid, 256, 0, stream>>>(rows, cols, ld, ptrs, gemm_id, seed, (uint32_t)operand);
  else
    fill::fill_kernel<2><<<grid, 256, 0, stream>>>(rows, cols, ld, ptrs, gemm_id, seed, (uint32_t)operand);
  return cudaGetLastError();
}

cudaError_t launch_alpha_beta(int batch, const int64_t *gemm_id, uint64_t seed, float *alpha, float *beta,
                              cudaStream_t stream) {
  if (batch <= 0) return cudaSuccess;
  fill::alpha_beta_kernel<<<(batch + 255) / 256, 256, 0, stream>>>(batch, gemm_id, seed, alpha, beta);
  return cudaGetLastError();
}

}  // namespace vb
