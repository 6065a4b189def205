// TMA load throughput microbenchmark (measurement tool, not product code).
// 148 persistent CTAs; one thread streams 2D TMA boxes into a ring of stages, another thread
// releases them (no compute).  Reports GB/s for a given box shape, stage depth and footprint
// (L2-resident when the footprint < 126 MB).
#include <cuda.h>
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>

#include "../paper_conf_ppopp_li0yjl19_b200/csrc/sm100.cuh"

using namespace vb;

struct Args {
  int rows_total, cols_total, box_w, box_h, boxes_per_stage, stages, iters, producers, sequential;
  uint32_t stage_bytes;
};

__global__ void __launch_bounds__(256, 1) tma_stream(const __grid_constant__ CUtensorMap map, Args a) {
  extern __shared__ uint8_t raw[];
  uint8_t *smem = reinterpret_cast<uint8_t *>((reinterpret_cast<uintptr_t>(raw) + 1023) & ~uintptr_t(1023));
  __shared__ uint64_t full[32], empty[32];
  if (threadIdx.x == 0) {
    for (int i = 0; i < a.stages; ++i) {
      ptx::mbar_init(&full[i], 1);
      ptx::mbar_init(&empty[i], 1);
    }
    ptx::fence_mbar_init();
  }
  __syncthreads();
  const int tiles_w = a.cols_total / a.box_w, tiles_h = a.rows_total / a.box_h;
  const int ntiles = tiles_w * tiles_h;
  // producer p (warp 2p, lane 0) owns stages [p*S/P, (p+1)*S/P); consumer p is warp 2p+1
  const int P = a.producers, per = a.stages / P;
  const int w = threadIdx.x / 32, lane = threadIdx.x % 32;
  const int pid = w / 2;
  if (lane == 0 && pid < P && (w % 2) == 0) {
    int st = 0;
    uint32_t ph = 0;
    unsigned t = blockIdx.x * 7919u + pid * 104729u;
    int pair_next = 0;
    for (int it = 0; it < a.iters / P; ++it) {
      const int s = pid * per + st;
      ptx::mbar_wait(&empty[s], ph ^ 1u);
      ptx::mbar_arrive_expect_tx(&full[s], a.stage_bytes);
      for (int b = 0; b < a.boxes_per_stage; ++b) {
        int tile;
        if (a.sequential == 1) tile = (int)((t++) % (unsigned)ntiles);
        else if (a.sequential == 2) {        // stage = bps consecutive boxes along a row band, stages random
          if (b == 0) { t = t * 1664525u + 1013904223u; }
          const int groups_w = tiles_w / a.boxes_per_stage;
          const int g = (int)(t % (unsigned)(groups_w * tiles_h));
          tile = (g / groups_w) * tiles_w + (g % groups_w) * a.boxes_per_stage + b;
        } else if (a.sequential >= 3) {      // pairs of adjacent boxes in consecutive stages
          if ((it & 1) == 0) {
            t = t * 1664525u + 1013904223u;
            const int groups_w = tiles_w / 2;
            const int g = (int)(t % (unsigned)(groups_w * tiles_h));
            tile = (g / groups_w) * tiles_w + (g % groups_w) * 2;
            if (a.sequential == 3) {          // 3: L2-prefetch the adjacent box with this one
              const int tx = ((tile + 1) % tiles_w) * a.box_w, ty = ((tile + 1) / tiles_w) * a.box_h;
              ptx::tma_prefetch_2d(&map, tx, ty);
            }
            pair_next = tile + 1;
          } else {
            tile = pair_next;                 // 4: the adjacent box one stage later, no prefetch
          }
        } else { t = t * 1664525u + 1013904223u; tile = (int)(t % (unsigned)ntiles); }
        const int x = (tile % tiles_w) * a.box_w, y = (tile / tiles_w) * a.box_h;
        ptx::tma_load_2d(smem + (size_t)s * a.stage_bytes + (size_t)b * a.box_w * a.box_h * 2, &map, &full[s], x, y);
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
  const int box_w = argc > 1 ? atoi(argv[1]) : 64;       // elements (bf16)
  const int box_h = argc > 2 ? atoi(argv[2]) : 64;
  const int bps = argc > 3 ? atoi(argv[3]) : 1;          // boxes per stage
  const int stages = argc > 4 ? atoi(argv[4]) : 8;
  const size_t foot_mb = argc > 5 ? atoll(argv[5]) : 4096;
  const int iters = argc > 6 ? atoi(argv[6]) : 4000;
  const int producers = argc > 7 ? atoi(argv[7]) : 1;
  const int sequential = argc > 8 ? atoi(argv[8]) : 0;
  const int cols = argc > 9 ? atoi(argv[9]) : 4096;   // row length (elements): the row stride
  const int rows = (int)(foot_mb * 1024 * 1024 / (cols * 2));
  void *buf;
  cudaMalloc(&buf, (size_t)rows * cols * 2);
  cudaMemset(buf, 0, (size_t)rows * cols * 2);
  CUtensorMap map;
  // TMA_INNER < cols: the map's row length is shorter than the stride, so the last box of each
  // row is partly out of bounds (zero-filled), like the K tail of an A matrix
  const int inner = getenv("TMA_INNER") ? atoi(getenv("TMA_INNER")) : cols;
  cuuint64_t dims[2] = {(cuuint64_t)inner, (cuuint64_t)rows};
  cuuint64_t strides[1] = {(cuuint64_t)cols * 2};
  cuuint32_t box[2] = {(cuuint32_t)box_w, (cuuint32_t)box_h};
  cuuint32_t es[2] = {1, 1};
  const int sw = box_w * 2;
  CUtensorMapSwizzle swz = sw == 128 ? CU_TENSOR_MAP_SWIZZLE_128B : sw == 64 ? CU_TENSOR_MAP_SWIZZLE_64B
                                                                             : CU_TENSOR_MAP_SWIZZLE_32B;
  CUresult r = cuTensorMapEncodeTiled(&map, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, buf, dims, strides, box, es,
                                      CU_TENSOR_MAP_INTERLEAVE_NONE, swz, getenv("TMA_PROMO") ? (CUtensorMapL2promotion)atoi(getenv("TMA_PROMO")) : CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                                      CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) {
    printf("encode failed %d\n", (int)r);
    return 1;
  }
  Args a{rows, cols, box_w, box_h, bps, stages, iters, producers, sequential, (uint32_t)(box_w * box_h * 2 * bps)};
  const size_t smem = (size_t)a.stage_bytes * stages + 1024;
  cudaFuncSetAttribute(tma_stream, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  for (int rep = 0; rep < 2; ++rep) tma_stream<<<sms, 256, smem>>>(map, a);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  cudaEventRecord(e0);
  tma_stream<<<sms, 256, smem>>>(map, a);
  cudaEventRecord(e1);
  cudaEventSynchronize(e1);
  float ms;
  cudaEventElapsedTime(&ms, e0, e1);
  const double bytes = (double)sms * iters * a.stage_bytes;
  printf("cols %d box %dx%d x%d stages %d prod %d seq %d (in flight %.0f KB/SM) footprint %zu MB: %.1f GB/s  (%s)\n", cols, box_w, box_h, bps, stages, producers, sequential,
         stages * a.stage_bytes / 1024.0, foot_mb, bytes / ms / 1e6, cudaGetErrorString(cudaGetLastError()));
  return 0;
}
