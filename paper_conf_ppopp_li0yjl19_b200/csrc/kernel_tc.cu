// bf16 / fp16 path: persistent, warp-specialised sm_100a kernel that walks the batching
// engine's work lists (Fig. 7, P294-312) with TMA-staged operands and tcgen05
// tensor-core MMA accumulating in TMEM.
//
// One CTA per SM (grid = min(Block_NUM, #SMs)), 8 warps:
//   warp 0      scheduler + A/B producer: atomically takes the next block (work list) b,
//               publishes it in a 4-deep smem ring, then streams every tile of b through a
//               3-stage ring of (A: BY x 64, B: 64 x BX) bf16 k-blocks with TMA.
//   warp 1      MMA issuer: one thread issues tcgen05.mma (M = BY, N = BX, K = 16) into one
//               of two TMEM accumulators (2 x 256 fp32 columns), commits stage releases and
//               "accumulator full" to mbarriers.
//   warp 2      TMEM allocator (512 columns).
//   warp 3      C producer: TMA-loads C_old chunks (BY x 64) into a 4-slot smem ring when
//               beta != 0 (C is never read when beta == 0, reading C-16).
//   warps 4-7   epilogue: tcgen05.ld the accumulator (warp w owns TMEM lanes 32*(w%4)..),
//               C = alpha*acc + beta*C_old in fp32, round-to-nearest-even to bf16/fp16,
//               write back into the swizzled smem chunk and TMA-store it (OOB clipped).
// The Fig. 2 double buffering (P147) becomes the TMA/mbarrier rings; the paper's "unified
// thread structure" (P181) becomes a runtime MMA instruction descriptor per tile, so one
// kernel serves every strategy of the table.
#include <cuda.h>
#include <cuda_bf16.h>
#include <cuda_fp16.h>
#include <cuda_runtime.h>
#include <stdint.h>

#include "plan_types.h"
#include "sm100.cuh"

namespace vb {
namespace tck {

constexpr int kThreads = 256;
constexpr int kBK = 64;                    // bf16 elements per k-block = one 128-B swizzle row
constexpr int kStages = 3;
constexpr int kABytes = 128 * kBK * 2;     // 16 KB (largest BY)
constexpr int kStageBytes = kABytes + 256 * kBK * 2;   // + 32 KB (largest BX)
constexpr int kCSlots = 4;
constexpr int kCSlotBytes = 128 * 128;     // BY rows x 128 B
constexpr int kSched = 4;
constexpr int kTmemCols = 512;
constexpr int kAccCols = 256;
constexpr int kEpiThreads = 128;
constexpr uint32_t kSchedConsumers = 1 + 1 + 4;   // MMA thread, C producer, 4 epilogue warps

struct Bars {
  uint64_t full[kStages], empty[kStages];
  uint64_t tfull[2], tempty[2];
  uint64_t cfull[kCSlots], cempty[kCSlots];
  uint64_t sfull[kSched], sempty[kSched];
  int32_t sched[kSched];
  uint32_t tmem_base;
};

constexpr size_t kSmemBytes = 1024 /*align slack*/ + (size_t)kStages * kStageBytes + (size_t)kCSlots * kCSlotBytes +
                              ((sizeof(Bars) + 127) / 128) * 128;

__device__ __forceinline__ int row_BY(int packed) { return (packed >> 8) & 0xFF; }
__device__ __forceinline__ int row_BX(int packed) { return packed >> 16; }

template <typename Ring>
__device__ __forceinline__ void advance(Ring &idx, uint32_t &phase, int n) {
  if (++idx == n) {
    idx = 0;
    phase ^= 1u;
  }
}

// ------------------------------------------------------------------------- epilogue math
template <int AB_FMT>
__device__ __forceinline__ void unpack8(uint4 w, float (&f)[8]) {
  const uint32_t u[4] = {w.x, w.y, w.z, w.w};
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    if constexpr (AB_FMT == 1) {
      __nv_bfloat162 h = *reinterpret_cast<const __nv_bfloat162 *>(&u[i]);
      float2 v = __bfloat1622float2(h);
      f[2 * i] = v.x;
      f[2 * i + 1] = v.y;
    } else {
      __half2 h = *reinterpret_cast<const __half2 *>(&u[i]);
      float2 v = __half22float2(h);
      f[2 * i] = v.x;
      f[2 * i + 1] = v.y;
    }
  }
}

template <int AB_FMT>
__device__ __forceinline__ uint32_t pack2(float lo, float hi) {
  if constexpr (AB_FMT == 1) {
    __nv_bfloat162 h = __floats2bfloat162_rn(lo, hi);
    return *reinterpret_cast<uint32_t *>(&h);
  } else {
    __half2 h = __floats2half2_rn(lo, hi);
    return *reinterpret_cast<uint32_t *>(&h);
  }
}

// Process NU 16-byte units (8 outputs each) of this thread's row of one C chunk.
template <int AB_FMT, int NU>
__device__ __forceinline__ void epi_row(uint8_t *cb, int row, int c_swz, const uint32_t *acc, float alpha,
                                        float beta) {
#pragma unroll
  for (int u = 0; u < NU; ++u) {
    const uint32_t off = ptx::swz((uint32_t)(row * c_swz + u * 16), c_swz);
    uint4 *p = reinterpret_cast<uint4 *>(cb + off);
    float o[8];
    if (beta != 0.f) {
      float old[8];
      unpack8<AB_FMT>(*p, old);
#pragma unroll
      for (int e = 0; e < 8; ++e) o[e] = fmaf(alpha, __uint_as_float(acc[u * 8 + e]), beta * old[e]);
    } else {
#pragma unroll
      for (int e = 0; e < 8; ++e) o[e] = alpha * __uint_as_float(acc[u * 8 + e]);
    }
    uint4 w;
    w.x = pack2<AB_FMT>(o[0], o[1]);
    w.y = pack2<AB_FMT>(o[2], o[3]);
    w.z = pack2<AB_FMT>(o[4], o[5]);
    w.w = pack2<AB_FMT>(o[6], o[7]);
    *p = w;
  }
}

// --------------------------------------------------------------------------------- kernel
template <int AB_FMT>
__global__ void __launch_bounds__(kThreads, 1) vb_tc_kernel(const __grid_constant__ TcArgs p) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t *smem = reinterpret_cast<uint8_t *>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t *stage_base = smem;
  uint8_t *cbuf = smem + (size_t)kStages * kStageBytes;
  Bars *bars = reinterpret_cast<Bars *>(cbuf + (size_t)kCSlots * kCSlotBytes);
  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;

  if (threadIdx.x == 0) {
    for (int i = 0; i < kStages; ++i) {
      ptx::mbar_init(&bars->full[i], 1);
      ptx::mbar_init(&bars->empty[i], 1);
    }
    for (int i = 0; i < 2; ++i) {
      ptx::mbar_init(&bars->tfull[i], 1);
      ptx::mbar_init(&bars->tempty[i], 4);
    }
    for (int i = 0; i < kCSlots; ++i) {
      ptx::mbar_init(&bars->cfull[i], 1);
      ptx::mbar_init(&bars->cempty[i], 1);
    }
    for (int i = 0; i < kSched; ++i) {
      ptx::mbar_init(&bars->sfull[i], 1);
      ptx::mbar_init(&bars->sempty[i], kSchedConsumers);
    }
    ptx::fence_mbar_init();
  }
  if (warp == 2) ptx::tmem_alloc(&bars->tmem_base, kTmemCols);
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem_base = bars->tmem_base;
  const uint8_t *tmaps = reinterpret_cast<const uint8_t *>(p.tmaps);

  if (warp == 0) {
    // ===================================================== scheduler + A/B TMA producer
    if (lane == 0) {
      int stage = 0, si = 0;
      uint32_t phase = 0, sph = 0;
      for (;;) {
        const int b = atomicAdd(p.counter, 1);
        ptx::mbar_wait(&bars->sempty[si], sph ^ 1u);
        bars->sched[si] = b < p.n_blocks ? b : -1;
        ptx::mbar_arrive(&bars->sfull[si]);
        advance(si, sph, kSched);
        if (b >= p.n_blocks) break;
        const int s1 = p.block_ptr[b + 1];
        for (int s = p.block_ptr[b]; s < s1; ++s) {
          const TileSlot ts = p.slots[s];
          const GemmParam gp = p.gemms[ts.gemm];
          if (gp.kblocks == 0) continue;
          const int BY = row_BY(gp.row), BX = row_BX(gp.row);
          const TcGeom geo = tc_geom(BY, BX);
          const uint8_t *mapA = tmaps + (size_t)ts.gemm * 384;
          const uint8_t *mapB = mapA + 128;
          ptx::tmap_acquire(mapA);
          ptx::tmap_acquire(mapB);
          const uint32_t bytes = (uint32_t)(BY + BX) * kBK * 2;
          const int y0 = ts.y * BY, x0 = ts.x * BX;
          for (int kb = 0; kb < gp.kblocks; ++kb) {
            ptx::mbar_wait(&bars->empty[stage], phase ^ 1u);
            ptx::mbar_arrive_expect_tx(&bars->full[stage], bytes);
            uint8_t *sa = stage_base + (size_t)stage * kStageBytes;
            uint8_t *sb = sa + kABytes;
            ptx::tma_load_2d(sa, mapA, &bars->full[stage], kb * kBK, y0);
            for (int j = 0; j < geo.b_boxes; ++j)
              ptx::tma_load_2d(sb + j * kBK * geo.b_swz, mapB, &bars->full[stage], x0 + j * (geo.b_swz / 2), kb * kBK);
            advance(stage, phase, kStages);
          }
        }
      }
    }
  } else if (warp == 1) {
    // ===================================================== MMA issuer (single thread)
    if (lane == 0) {
      int stage = 0, si = 0;
      uint32_t phase = 0, sph = 0, t = 0;
      for (;;) {
        ptx::mbar_wait(&bars->sfull[si], sph);
        const int b = bars->sched[si];
        ptx::mbar_arrive(&bars->sempty[si]);
        advance(si, sph, kSched);
        if (b < 0) break;
        const int s1 = p.block_ptr[b + 1];
        for (int s = p.block_ptr[b]; s < s1; ++s, ++t) {
          const TileSlot ts = p.slots[s];
          const GemmParam gp = p.gemms[ts.gemm];
          const int BY = row_BY(gp.row), BX = row_BX(gp.row);
          const TcGeom geo = tc_geom(BY, BX);
          const uint32_t buf = t & 1u, aph = (t >> 1) & 1u;
          ptx::mbar_wait(&bars->tempty[buf], aph ^ 1u);
          ptx::tc_fence_after();
          const uint32_t d_tmem = tmem_base + buf * kAccCols;
          const uint32_t idesc = ptx::idesc_f16((uint32_t)AB_FMT, BY, BX);
          const uint32_t blayout = ptx::swizzle_layout_code(geo.b_swz);
          for (int kb = 0; kb < gp.kblocks; ++kb) {
            ptx::mbar_wait(&bars->full[stage], phase);
            ptx::tc_fence_after();
            const uint32_t sa = ptx::smem_u32(stage_base + (size_t)stage * kStageBytes);
            const uint32_t sb = sa + kABytes;
#pragma unroll
            for (int kk = 0; kk < kBK / 16; ++kk) {
              // A: K-major, 128-B swizzle, 8-row atoms 1024 B apart; K step of 16 = +32 B.
              const uint64_t adesc = ptx::smem_desc(sa + kk * 32, 16, 1024, 2);
              // B: MN-major, b_swz swizzle; 8-row (K) atoms 8*b_swz apart (SBO), MN blocks of
              // b_swz/2 elements 64*b_swz apart (LBO); K step of 16 rows = +16*b_swz bytes.
              const uint64_t bdesc = ptx::smem_desc(sb + kk * 16 * geo.b_swz, kBK * geo.b_swz, 8 * geo.b_swz, blayout);
              ptx::mma_f16_ss(d_tmem, adesc, bdesc, idesc, (kb | kk) != 0 ? 1u : 0u);
            }
            ptx::mma_commit(&bars->empty[stage]);   // frees the smem stage when the MMAs retire
            advance(stage, phase, kStages);
          }
          ptx::mma_commit(&bars->tfull[buf]);       // accumulator ready for the epilogue
        }
      }
    }
  } else if (warp == 3) {
    // ===================================================== C_old producer (beta != 0)
    if (lane == 0) {
      int cs = 0, si = 0;
      uint32_t cph = 0, sph = 0;
      for (;;) {
        ptx::mbar_wait(&bars->sfull[si], sph);
        const int b = bars->sched[si];
        ptx::mbar_arrive(&bars->sempty[si]);
        advance(si, sph, kSched);
        if (b < 0) break;
        const int s1 = p.block_ptr[b + 1];
        for (int s = p.block_ptr[b]; s < s1; ++s) {
          const TileSlot ts = p.slots[s];
          const GemmParam gp = p.gemms[ts.gemm];
          const int BY = row_BY(gp.row), BX = row_BX(gp.row);
          const TcGeom geo = tc_geom(BY, BX);
          const float beta = p.beta[ts.gemm];
          const uint8_t *mapC = tmaps + (size_t)ts.gemm * 384 + 256;
          if (beta != 0.f) ptx::tmap_acquire(mapC);
          for (int ch = 0; ch < geo.c_chunks; ++ch) {
            ptx::mbar_wait(&bars->cempty[cs], cph ^ 1u);
            if (beta != 0.f) {
              ptx::mbar_arrive_expect_tx(&bars->cfull[cs], (uint32_t)(BY * geo.c_cols * 2));
              ptx::tma_load_2d(cbuf + (size_t)cs * kCSlotBytes, mapC, &bars->cfull[cs], ts.x * BX + ch * geo.c_cols,
                               ts.y * BY);
            } else {
              ptx::mbar_arrive(&bars->cfull[cs]);
            }
            advance(cs, cph, kCSlots);
          }
        }
      }
    }
  } else if (warp >= 4) {
    // ===================================================== epilogue (128 threads)
    const int q = warp & 3;   // TMEM lane quarter this warp may access
    const bool store_thread = (warp == 4 && lane == 0);
    int cs = 0, si = 0;
    uint32_t cph = 0, sph = 0, t = 0;
    for (;;) {
      ptx::mbar_wait(&bars->sfull[si], sph);
      const int b = bars->sched[si];
      __syncwarp();
      if (lane == 0) ptx::mbar_arrive(&bars->sempty[si]);
      advance(si, sph, kSched);
      if (b < 0) break;
      const int s1 = p.block_ptr[b + 1];
      for (int s = p.block_ptr[b]; s < s1; ++s, ++t) {
        const TileSlot ts = p.slots[s];
        const GemmParam gp = p.gemms[ts.gemm];
        const int BY = row_BY(gp.row), BX = row_BX(gp.row);
        const TcGeom geo = tc_geom(BY, BX);
        const float alpha = p.alpha[ts.gemm], beta = p.beta[ts.gemm];
        const uint8_t *mapC = tmaps + (size_t)ts.gemm * 384 + 256;
        if (store_thread) ptx::tmap_acquire(mapC);
        const uint32_t buf = t & 1u, aph = (t >> 1) & 1u;
        ptx::mbar_wait(&bars->tfull[buf], aph);
        ptx::tc_fence_after();
        // M = 128: tile row 32q + lane lives in TMEM lane 32q + lane.
        // M = 64 : tile row 16q + i lives in TMEM lane 32q + i, i < 16 (half sub-partitions).
        const int row = BY == 128 ? q * 32 + lane : q * 16 + lane;
        const bool row_ok = BY == 128 || lane < 16;
        for (int ch = 0; ch < geo.c_chunks; ++ch) {
          uint32_t acc[64];
          if (gp.kblocks > 0) {
            const uint32_t taddr = tmem_base + ((uint32_t)(q * 32) << 16) + buf * kAccCols + ch * geo.c_cols;
            ptx::tmem_ld_32x32b_x32(taddr, *reinterpret_cast<uint32_t(*)[32]>(&acc[0]));
            if (geo.c_cols == 64) ptx::tmem_ld_32x32b_x32(taddr + 32, *reinterpret_cast<uint32_t(*)[32]>(&acc[32]));
            ptx::tmem_ld_wait();
          } else {
#pragma unroll
            for (int i = 0; i < 64; ++i) acc[i] = 0u;   // K == 0: C = beta * C
          }
          ptx::mbar_wait(&bars->cfull[cs], cph);
          uint8_t *cb = cbuf + (size_t)cs * kCSlotBytes;
          if (row_ok) {
            if (geo.c_cols == 64)
              epi_row<AB_FMT, 8>(cb, row, geo.c_swz, acc, alpha, beta);
            else
              epi_row<AB_FMT, 4>(cb, row, geo.c_swz, acc, alpha, beta);
          }
          const int col0 = ts.x * BX + ch * geo.c_cols;
          if (col0 + geo.c_cols <= gp.N || (gp.N & 7) == 0) {
            // TMA store; rows >= M and whole 16-byte granules >= N are clipped by the TMA unit.
            ptx::fence_proxy_async_smem();
            ptx::named_bar_sync(1, kEpiThreads);
            if (store_thread) {
              ptx::tma_store_2d(mapC, cb, col0, ts.y * BY);
              ptx::bulk_commit();
              ptx::bulk_wait_read0();
              ptx::mbar_arrive(&bars->cempty[cs]);
            }
          } else {
            // The chunk ends inside a 16-byte granule of the row (N % 8 != 0): a TMA store would
            // write the whole granule, i.e. past N into the caller's padding.  Store this chunk
            // from the thread's own row with exact per-element bounds instead.
            const int grow = ts.y * BY + row;
            if (row_ok && grow < gp.M) {
              uint8_t *crow = static_cast<uint8_t *>(p.C[ts.gemm]) + ((size_t)grow * gp.ldc + col0) * 2;
              const int ncol = gp.N - col0;
              for (int u = 0; u * 8 < ncol && u * 8 < geo.c_cols; ++u) {
                const uint4 w = *reinterpret_cast<const uint4 *>(cb + ptx::swz((uint32_t)(row * geo.c_swz + u * 16),
                                                                                  geo.c_swz));
                if (u * 8 + 8 <= ncol) {
                  *reinterpret_cast<uint4 *>(crow + u * 16) = w;
                } else {
                  const uint16_t *h = reinterpret_cast<const uint16_t *>(&w);
                  for (int e = 0; e < ncol - u * 8; ++e) reinterpret_cast<uint16_t *>(crow + u * 16)[e] = h[e];
                }
              }
            }
            ptx::named_bar_sync(1, kEpiThreads);
            if (store_thread) ptx::mbar_arrive(&bars->cempty[cs]);
          }
          advance(cs, cph, kCSlots);
        }
        ptx::tc_fence_before();
        __syncwarp();
        if (lane == 0) ptx::mbar_arrive(&bars->tempty[buf]);
      }
    }
    if (store_thread) ptx::bulk_wait0();
  }
  __syncwarp();
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  if (warp == 2) ptx::tmem_dealloc(tmem_base, kTmemCols);
  // The last CTA to finish resets the work-list counter, so back-to-back launches of the
  // same bound plan need no reset kernel.  Every CTA fetched past n_blocks before getting here.
  if (threadIdx.x == 0) {
    __threadfence();
    if (atomicAdd(&p.counter[1], 1) == (int)gridDim.x - 1) {
      atomicExch(&p.counter[0], 0);
      atomicExch(&p.counter[1], 0);
      __threadfence();
    }
  }
}

// Exec-time prep: patch the global address of every per-GEMM tensor map (A, B, C) with the
// caller's pointers (tensormap.replace), and reset the dynamic work-list counter.
__global__ void vb_tc_prep(uint8_t *tmaps, const void *const *A, const void *const *B, void *const *C,
                           const GemmParam *gemms, int batch, int32_t *counter) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i == 0) {
    counter[0] = 0;
    counter[1] = 0;
  }
  if (i >= batch * 3) return;
  const int g = i / 3, w = i % 3;
  const GemmParam gp = gemms[g];
  if (gp.M <= 0 || gp.N <= 0) return;
  if (w < 2 && gp.K <= 0) return;
  const void *ptr = w == 0 ? A[g] : (w == 1 ? B[g] : static_cast<const void *>(C[g]));
  ptx::tmap_replace_address(tmaps + (size_t)i * 128, ptr);
  ptx::tmap_release();
}

}  // namespace tck

size_t tc_smem_bytes() { return tck::kSmemBytes; }

cudaError_t tc_configure() {
  cudaError_t e = cudaFuncSetAttribute(tck::vb_tc_kernel<1>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                       (int)tck::kSmemBytes);
  if (e != cudaSuccess) return e;
  return cudaFuncSetAttribute(tck::vb_tc_kernel<0>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                              (int)tck::kSmemBytes);
}

cudaError_t launch_tc_prep(uint8_t *tmaps, const void *const *A, const void *const *B, void *const *C,
                           const GemmParam *gemms, int batch, int32_t *counter, cudaStream_t stream) {
  const int n = batch * 3;
  tck::vb_tc_prep<<<n > 0 ? (n + 255) / 256 : 1, 256, 0, stream>>>(tmaps, A, B, C, gemms, batch, counter);
  return cudaGetLastError();
}

cudaError_t launch_tc(const TcArgs &args, int grid, bool bf16, cudaStream_t stream) {
  if (grid <= 0) return cudaSuccess;
  if (bf16)
    tck::vb_tc_kernel<1><<<grid, tck::kThreads, tck::kSmemBytes, stream>>>(args);
  else
    tck::vb_tc_kernel<0><<<grid, tck::kThreads, tck::kSmemBytes, stream>>>(args);
  return cudaGetLastError();
}

}  // namespace vb
