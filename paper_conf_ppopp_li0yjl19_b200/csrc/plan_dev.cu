// Plan-time device kernels: expansion of the compact schedule into the per-slot records the
// GEMM kernels walk, and construction of the per-GEMM tensor maps from a few host-encoded
// templates.  Both run once per vb_plan_* call (not per exec).
//
// The host planner uploads only what the tiling and batching engines decide (§6,
// P282): Tile[] (block_ptr), the slot -> tile order (absent when it is the identity, i.e. for
// threshold batching and one-tile blocks), the GEMM segments of the tile enumeration and the
// per-GEMM parameters (Tiling[] inside GemmParam.row).  Each thread here decodes one slot into
// (GEMM, Y_Coord, X_Coord) -- Fig. 7 lines 6-15 done once at plan time -- and writes the 32-byte
// TileDesc of the tensor-core kernel or the 8-byte TileSlot of the FFMA kernel.
#include <cuda.h>
#include <cuda_runtime.h>
#include <stdint.h>

#include "plan_types.h"
#include "sm100.cuh"

namespace vb {
namespace pdev {

__global__ void vb_plan_expand(ExpandArgs a) {
  for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < a.n_slots;
       k += (int64_t)gridDim.x * blockDim.x) {
    const int32_t t = a.slot_tile ? a.slot_tile[k] : (int32_t)k;
    // segment j with seg_start[j] <= t < seg_start[j + 1] (segments are non-empty, ascending)
    int lo = 0, hi = a.n_seg - 1;
    while (lo < hi) {
      const int mid = (lo + hi + 1) >> 1;
      if (a.seg_start[mid] <= t)
        lo = mid;
      else
        hi = mid - 1;
    }
    const int g = a.seg_gemm[lo];
    const int local = t - a.seg_start[lo];
    const GemmParam gp = a.gemms[g];
    const int r = gp.row & 0xFF;
    const int BY = a.row_by[r], BX = a.row_bx[r];
    const int gx = (gp.N + BX - 1) / BX;
    const int y = local / gx, x = local - y * gx;
    if (a.slots) a.slots[k] = TileSlot{(uint32_t)g, (uint16_t)y, (uint16_t)x};
    if (!a.tiles) continue;
    TileDesc d;
    d.gemm = g;
    d.m0 = y * BY;
    d.kblocks = gp.kblocks;
    d.M = gp.M;
    if ((a.row_swap >> r) & 1) {   // swap-AB tiles keep the fixed split (their epilogue tests N per column)
      d.n0 = x * BX;
      d.N = gp.N;
    } else {
      tile_cols(x, gp.N, BX, d.n0, d.N);
    }
    d.ldc = gp.ldc;
    d.geo = (uint16_t)((BY / 16) | ((BX / 16) << 8));
    d.flags = 0;
    if (gp.row & kGemmConv) {   // implicit GEMM: taps x channel blocks, every k-block full
      const ConvParam c = a.conv[g];
      d.kblocks = gp.K > 0 ? (gp.K / c.Cin) * c.ncb : 0;
      d.flags |= kFlagConv;
      const int last = c.Cin - 64 * (c.ncb - 1);   // channels in each tap's last block
      if (last < 64) d.flags |= (uint16_t)(((last + 15) / 16) << 8);
    } else if (gp.K % 64) {
      d.flags |= (uint16_t)(((gp.K % 64 + 15) / 16) << 8);   // MMA K-steps of the last k-block
    }
    // the tile's last C chunk ends inside a 16-byte granule of the row: stored directly
    const bool last_col = ((a.row_swap >> r) & 1) ? d.n0 + BX > gp.N : d.N == gp.N;   // the GEMM's last column tile
    if ((gp.N & 7) != 0 && last_col && d.n0 < gp.N) d.flags |= 1;
    if ((a.row_swap >> r) & 1) d.flags |= kFlagSwap;
    a.tiles[k] = d;
  }
}

__device__ __forceinline__ void replace_dims(uint8_t *m, uint32_t inner, uint32_t outer, uint64_t stride_bytes) {
  asm volatile("tensormap.replace.tile.global_dim.global.b1024.b32 [%0], 0, %1;" ::"l"(m), "r"(inner) : "memory");
  asm volatile("tensormap.replace.tile.global_dim.global.b1024.b32 [%0], 1, %1;" ::"l"(m), "r"(outer) : "memory");
  asm volatile("tensormap.replace.tile.global_stride.global.b1024.b64 [%0], 0, %1;" ::"l"(m), "l"(stride_bytes)
               : "memory");
}

// One thread per (GEMM, map): copy the map's template (same box, swizzle, element type, L2
// promotion as the host encoder would use) and set its global dims and row stride.  The global
// address stays the template's placeholder until vb_plan_bind patches it.
__global__ void vb_tmaps_build(MapBuildArgs a) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= a.batch * kMapsPerGemm) return;
  const int g = i / kMapsPerGemm, w = i % kMapsPerGemm;
  const GemmParam gp = a.gemms[g];
  const int BYc = (gp.row >> 8) & 0xFF;
  const int outer = tc_map_outer(w, gp.M, gp.N, gp.K, BYc);
  uint8_t *m = a.tmaps + (size_t)i * 128;
  const bool is_a = w <= 1, is_b = w == 2 || w == 3;
  const uint64_t es = (uint64_t)a.es;
#ifdef VB_EXP_C_RMW
  // experiment (timing only): C_old loaded and C stored through whole 16-byte granules
  const uint32_t inner = is_a ? gp.K : is_b ? gp.N : (uint32_t)((gp.N + 7) & ~7);
#else
  const uint32_t inner = is_a ? gp.K : is_b ? gp.N : w == MAP_C ? gp.N : (gp.N & ~7);
#endif
  const uint32_t rows = is_a ? gp.M : is_b ? gp.K : gp.M;
  const uint64_t stride = (uint64_t)(is_a ? gp.lda : is_b ? gp.ldb : gp.ldc) * es;
  const int c = outer ? a.tidx[tmap_key(w, gp.row & 0xFF, outer, (rows - 1) * stride + inner * es < kTmapSmallBytes)]
                      : -1;
  if (c < 0) {                      // map not used: zero, like the host encoder's unused slots
    uint4 *z = reinterpret_cast<uint4 *>(m);
#pragma unroll
    for (int q = 0; q < 8; ++q) z[q] = make_uint4(0, 0, 0, 0);
    return;
  }
  const uint4 *src = reinterpret_cast<const uint4 *>(a.templates + (size_t)c * 128);
  uint4 *dst = reinterpret_cast<uint4 *>(m);
#pragma unroll
  for (int q = 0; q < 8; ++q) dst[q] = src[q];
  replace_dims(m, inner, rows, stride);
  ptx::tmap_release();
}

}  // namespace pdev

cudaError_t launch_plan_expand(const ExpandArgs &a, cudaStream_t s) {
  if (a.n_slots <= 0) return cudaSuccess;
  const int64_t blocks = (a.n_slots + 255) / 256;
  pdev::vb_plan_expand<<<(int)(blocks < 4096 ? blocks : 4096), 256, 0, s>>>(a);
  return cudaGetLastError();
}

cudaError_t launch_tmaps_build(const MapBuildArgs &a, cudaStream_t s) {
  const int n = a.batch * kMapsPerGemm;
  if (n <= 0) return cudaSuccess;
  pdev::vb_tmaps_build<<<(n + 255) / 256, 256, 0, s>>>(a);
  return cudaGetLastError();
}

}  // namespace vb
