// TMA descriptor-cache microbenchmark (measurement tool, not product code).
// Like tma_bench.cu, but every stage loads one box through one of R tensor maps kept in global
// memory (one map per region of the footprint, as the GEMM kernel keeps one map per GEMM).
// Measures what per-GEMM tensor maps cost the TMA load stream: R = 1 vs 64 vs 65536 maps, with
// and without prefetch.tensormap D stages ahead.
//   tma_maps <R> <prefetch distance (0 = none)> <boxes per stage> <stages> <producers> [L2 promotion] [split]
#include <cuda.h>
#include <cuda_runtime.h>
#include <cudaTypedefs.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>

#include <vector>

#include "../paper_conf_ppopp_li0yjl19_b200/csrc/sm100.cuh"

using namespace vb;

struct Args {
  const uint8_t *maps;
  int R, rows_per_region, cols, box_w, box_h, bps, stages, iters, producers, pf, split;
  uint32_t stage_bytes;
};

__device__ __forceinline__ uint32_t hash32(uint32_t x) {
  x ^= x >> 16; x *= 0x7feb352dU; x ^= x >> 15; x *= 0x846ca68bU; x ^= x >> 16;
  return x;
}

__global__ void __launch_bounds__(256, 1) tma_maps_stream(const __grid_constant__ Args a) {
  extern __shared__ uint8_t raw[];
  uint8_t *smem = raw + ((1024u - (ptx::smem_u32(raw) & 1023u)) & 1023u);
  __shared__ uint64_t full[32], empty[32];
  if (threadIdx.x == 0) {
    for (int i = 0; i < a.stages; ++i) {
      ptx::mbar_init(&full[i], 1);
      ptx::mbar_init(&empty[i], 1);
    }
    ptx::fence_mbar_init();
  }
  __syncthreads();
  const int tiles_w = a.cols / a.box_w / a.bps / (a.split > 0 ? 2 : 1), tiles_h = a.rows_per_region / a.box_h;
  const int P = a.producers, per = a.stages / P;
  const int w = threadIdx.x / 32, lane = threadIdx.x % 32;
  const int pid = w / 2;
  if (lane == 0 && pid < P && (w % 2) == 0) {
    int st = 0;
    uint32_t ph = 0;
    const uint32_t seed = blockIdx.x * 7919u + pid * 104729u;
    const int n = a.iters / P;
    for (int it = 0; it < n; ++it) {
      const int s = pid * per + st;
      if (a.pf > 0 && it + a.pf < n) {
        const uint32_t hm = hash32(seed * 2654435761u + (uint32_t)(it + a.pf));
        ptx::prefetch_tmap(a.maps + (size_t)(hm % (uint32_t)a.R) * 128);
      }
      // split > 0: stage `it` loads the left 128-B strip of a 256-B pair and stage it+split the right
      // strip of the same pair (k-block strips of one A row band issued `split` stages apart)
      const int base_it = a.split > 0 ? ((it / (2 * a.split)) * 2 * a.split + (it % a.split)) : it;
      const int side = a.split > 0 ? (it / a.split) & 1 : 0;
      const uint32_t h = hash32(seed * 2654435761u + (uint32_t)base_it);
      const uint8_t *map = a.maps + (size_t)(h % (uint32_t)a.R) * 128;
      const uint32_t h2 = hash32(h ^ 0x9e3779b9u);
      const int tile = (int)(h2 % (uint32_t)(tiles_w * tiles_h));
      ptx::mbar_wait(&empty[s], ph ^ 1u);
      ptx::mbar_arrive_expect_tx(&full[s], a.stage_bytes);
      for (int b = 0; b < a.bps; ++b) {
        const int x = (((tile % tiles_w) * a.bps + b) * (a.split > 0 ? 2 : 1) + side) * a.box_w, y = (tile / tiles_w) * a.box_h;
        ptx::tma_load_2d(smem + (size_t)s * a.stage_bytes + (size_t)b * a.box_w * a.box_h * 2, map, &full[s], x, y);
      }
      if (++st == per) {
        st = 0;
        ph ^= 1u;
      }
    }
  } else if (lane == 0 && pid < P && (w % 2) == 1) {
    int st = 0;
    uint32_t ph = 0;
    for (int it = 0; it < a.iters / P; ++it) {
      const int s = pid * per + st;
      ptx::mbar_wait(&full[s], ph);
      ptx::mbar_arrive(&empty[s]);
      if (++st == per) {
        st = 0;
        ph ^= 1u;
      }
    }
  }
}

int main(int argc, char **argv) {
  const int R = argc > 1 ? atoi(argv[1]) : 1;
  const int pf = argc > 2 ? atoi(argv[2]) : 0;
  const int bps = argc > 3 ? atoi(argv[3]) : 1;
  const int stages = argc > 4 ? atoi(argv[4]) : 12;
  const int producers = argc > 5 ? atoi(argv[5]) : 4;
  const int promo = argc > 6 ? atoi(argv[6]) : 3;   // 0 none, 1 64B, 2 128B, 3 256B
  const int split = argc > 7 ? atoi(argv[7]) : 0;
  const int iters = 4000;
  const int cols = 512, box_w = 64, box_h = 128;
  const size_t foot = (size_t)8 << 30;
  const int rows_per_region = (int)(foot / R / (cols * 2)) / box_h * box_h;
  uint8_t *buf;
  cudaMalloc(&buf, foot);
  cudaMemset(buf, 0, foot);
  PFN_cuTensorMapEncodeTiled_v12000 enc = nullptr;
  cudaDriverEntryPointQueryResult q;
  cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", reinterpret_cast<void **>(&enc), cudaEnableDefault, &q);
  std::vector<CUtensorMap> maps(R);
  for (int r = 0; r < R; ++r) {
    cuuint64_t dims[2] = {(cuuint64_t)cols, (cuuint64_t)rows_per_region};
    cuuint64_t strides[1] = {(cuuint64_t)cols * 2};
    cuuint32_t box[2] = {(cuuint32_t)box_w, (cuuint32_t)box_h};
    cuuint32_t es[2] = {1, 1};
    CUresult e = enc(&maps[r], CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, buf + (size_t)r * rows_per_region * cols * 2, dims,
                     strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                     (CUtensorMapL2promotion)promo, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (e != CUDA_SUCCESS) {
      printf("encode failed %d\n", (int)e);
      return 1;
    }
  }
  uint8_t *dmaps;
  cudaMalloc(&dmaps, (size_t)R * 128);
  cudaMemcpy(dmaps, maps.data(), (size_t)R * 128, cudaMemcpyHostToDevice);
  Args a{dmaps, R, rows_per_region, cols, box_w, box_h, bps, stages, iters, producers, pf, split,
         (uint32_t)(box_w * box_h * 2 * bps)};
  const size_t smem = (size_t)a.stage_bytes * stages + 1024;
  cudaFuncSetAttribute(tma_maps_stream, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  for (int rep = 0; rep < 2; ++rep) tma_maps_stream<<<sms, 256, smem>>>(a);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  cudaEventRecord(e0);
  tma_maps_stream<<<sms, 256, smem>>>(a);
  cudaEventRecord(e1);
  cudaEventSynchronize(e1);
  float ms;
  cudaEventElapsedTime(&ms, e0, e1);
  const double bytes = (double)sms * (iters / producers * producers) * a.stage_bytes;
  printf("promo %d split %d maps %d prefetch %d box %dx%d x%d stages %d prod %d (in flight %.0f KB/SM): %.1f GB/s  (%s)\n", promo, split, R, pf, box_w,
         box_h, bps, stages, producers, stages * a.stage_bytes / 1024.0, bytes / ms / 1e6,
         cudaGetErrorString(cudaGetLastError()));
  return 0;
}
