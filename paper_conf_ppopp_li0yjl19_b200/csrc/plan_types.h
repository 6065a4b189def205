// Device-visible plan layout shared by the host C-ABI (capi.cu) and the kernels.
//
// The five auxiliary arrays of PAPER.md §6 (P282, Fig. 6) are packed as:
//   block_ptr[n_blocks+1]           == Tile[]                      (CSR over tile slots)
//   TileSlot{gemm, y, x}[n_slots]   == GEMM[], Y_Coord[], X_Coord[] (8 bytes per slot)
//   GemmParam[batch].row            == Tiling[] (per GEMM, reading C-12)
#pragma once
#include <stdint.h>

namespace vb {

struct alignas(8) TileSlot {
  uint32_t gemm;
  uint16_t y;   // tile row index along M   (element origin y * BY)
  uint16_t x;   // tile column index along N (element origin x * BX)
};
static_assert(sizeof(TileSlot) == 8, "TileSlot must stay 8 bytes");

struct alignas(16) GemmParam {
  int32_t M, N, K;
  int32_t lda, ldb, ldc;
  int32_t row;       // bits 0-7: strategy row in the plan's table; 8-15: per-CTA BY; 16-25: BX;
                     // bit 30 (kGemmConv): implicit-GEMM convolution (im2col A, no B K-tail map)
  int32_t kblocks;   // ceil(K / BK)
};
static_assert(sizeof(GemmParam) == 32, "GemmParam must stay 32 bytes");
constexpr int32_t kGemmConv = 1 << 30;

// Kernel arguments (by value).
struct F32Args {
  const int32_t *block_ptr;
  const TileSlot *slots;
  const GemmParam *gemms;
  const float *const *A;
  const float *const *B;
  float *const *C;
  const float *alpha;
  const float *beta;
  const int32_t *order;   // claim order of the blocks, heaviest first (execution detail, not part of the plan)
  const void *tmaps;      // CUtensorMap[batch][kF32MapsPerGemm] (A, B), 128-byte aligned
  int32_t *counter;       // [0] work-list counter, [1] finished CTAs (reset by the last CTA to finish)
  int32_t n_blocks;
};
// fp32 tensor maps per GEMM: A (box 32 x BY, 128-byte swizzle) and B (box min(BX,32) x 32).
constexpr int kF32MapsPerGemm = 2;

// Per tile slot, precomputed by the planner for the tensor-core kernel: the five arrays of
// Fig. 6 joined with the per-GEMM sizes, so the kernel reads one 32-byte record per tile.
struct alignas(16) TileDesc {
  int32_t gemm;
  int32_t m0;        // element row of the tile origin    (Y_Coord * BY)
  int32_t n0;        // element column of the tile origin (balanced: see tile_cols below)
  int32_t kblocks;   // ceil(K / 64)
  int32_t M;         // GEMM rows
  int32_t N;         // end column of the tile (the GEMM's N for its last column tile)
  int32_t ldc;       // elements
  uint16_t geo;      // (BY / 16) | (BX / 16) << 8
  uint16_t flags;    // bit 0: the tile's last C chunk ends inside a 16-byte granule (N % 8 != 0):
                     //        its columns [N & ~7, N) are stored directly, not by TMA
                     // bits 8-10: K=16 MMA steps of the last k-block (1..4), 0 = 4
};
// Balanced column split of a tensor-core GEMM (reading C-26): the ceil(N / BX) column
// tiles of a GEMM share its ceil(N / G) column chunks (G = 64, or BX when narrower) as evenly as
// whole chunks allow, instead of BX columns each plus a ragged last tile.  Tiles that share an A
// row panel then stream it at the same speed, so its re-reads hit in L2 (a 256-column edge tile
// of a 768-wide GEMM beside a 512-column one ran twice as fast and re-read A from DRAM).  The
// plan (tile (y, x), Eq. 1 counts) is unchanged; chunk boundaries stay 64-column aligned, so no
// TMA store box crosses into a neighbouring tile.  Returns [n0, end) of column tile x.
#ifndef VB_BALANCED_N
#define VB_BALANCED_N 1
#endif
__host__ __device__ inline void tile_cols(int x, int N, int BX, int &n0, int &end) {
#if VB_BALANCED_N
  const int G = BX < 64 ? BX : 64;
  const int q = (N + G - 1) / G, nx = (N + BX - 1) / BX;
  n0 = (int)((int64_t)x * q / nx) * G;
  end = (int)((int64_t)(x + 1) * q / nx) * G;
  if (end > N) end = N;
#else
  n0 = x * BX;
  end = n0 + BX < N ? n0 + BX : N;
#endif
}
// inverse of tile_cols: the column tile whose range starts at n0 (q >= nx, so n0 is strictly
// increasing in x)
__host__ __device__ inline int tile_col_index(int n0, int N, int BX) {
#if VB_BALANCED_N
  const int G = BX < 64 ? BX : 64;
  const int q = (N + G - 1) / G, nx = (N + BX - 1) / BX;
  return (int)(((int64_t)(n0 / G) * nx + q - 1) / q);
#else
  return n0 / BX;
#endif
}

// Tensor maps per GEMM (128 bytes each): A, A row-tail, B, B K-tail, C (loads), C store.  The
// tail maps have boxes that stop at the matrix edge, because out-of-bounds box rows are
// zero-filled but still cost L2 request bandwidth.  The C store map is N & ~7 columns wide:
// a TMA store writes whole 16-byte granules, so clipping at N itself would write past N.
constexpr int kMapsPerGemm = 6;
enum MapIndex { MAP_A = 0, MAP_A_TAIL = 1, MAP_B = 2, MAP_B_TAIL = 3, MAP_C = 4, MAP_C_ST = 5 };
static_assert(sizeof(TileDesc) == 32, "TileDesc must stay 32 bytes");

// Implicit-GEMM convolution parameters per GEMM (vb_plan_conv).  A tile whose
// TileDesc.flags has kFlagConv set loads A with TMA im2col copies: k-block kb covers filter tap
// kb / ncb (tap = kh * KW + kw) and input channels [64 * (kb % ncb), +64); its B rows start at
// tap * Cin + 64 * (kb % ncb).  Flags bits 8-10 then give the MMA K=16 steps of each tap's last
// channel block (0 = 4).
struct alignas(16) ConvParam {
  int32_t Hout, Wout;   // output image size (pixels of one image = Hout * Wout)
  int32_t Cin, KW;
  int32_t pad;
  int32_t ncb;          // channel blocks per tap: ceil(Cin / 64)
  int32_t pad_[2];
};
static_assert(sizeof(ConvParam) == 32, "ConvParam must stay 32 bytes");
constexpr uint16_t kFlagConv = 1u << 12;
// TileDesc.flags: swap-AB tile (C^T = B^T A^T): the MMA's A operand is the tile's B panel
// (MN-major, M = BX = 128), its B operand the A rows (K-major, N = BY rounded to 16); the
// accumulator holds C^T (TMEM lane = C column) and the epilogue stores it with direct stores.
constexpr uint16_t kFlagSwap = 1u << 13;

struct TcArgs {
  const int32_t *block_ptr;
  const TileDesc *tiles;    // [n_slots]
  const void *tmaps;        // CUtensorMap[batch][kMapsPerGemm], 128-byte aligned
  void *const *C;           // C pointers (direct stores of row tails that TMA cannot clip)
  const float *alpha;
  const float *beta;
  int32_t *counter;         // [0] work-list counter, [1] finished CTAs (reset by the last CTA to finish)
  int32_t n_blocks;
  long long *trace;         // VB_TRACE builds only: per-role wait cycles (else nullptr)
  const ConvParam *conv;    // [batch] for convolution plans (vb_plan_conv), else nullptr
};

// Plan-time expansion of the compact schedule (csrc/plan_dev.cu).
struct ExpandArgs {
  const int32_t *slot_tile;   // [n_slots] slot -> tile in enumeration order; nullptr = identity
  const int32_t *seg_start;   // [n_seg + 1] first tile of each GEMM segment (enumeration order)
  const int32_t *seg_gemm;    // [n_seg] GEMM of each segment (GEMMs without tiles have none)
  int32_t n_seg;
  int64_t n_slots;
  const GemmParam *gemms;
  const ConvParam *conv;      // [batch] for convolution plans, else nullptr
  TileDesc *tiles;            // tensor-core plans: TileDesc[n_slots] (else nullptr)
  TileSlot *slots;            // FFMA plans: TileSlot[n_slots] (else nullptr)
  int16_t row_by[16], row_bx[16];   // full tile extents (BY, BX) of each table row
  uint16_t row_swap;                // bit r: table row r is a swap-AB strategy
};

// Plan-time construction of the per-GEMM tensor maps from host-encoded templates.
// A map's template is tidx[map][row][box_outer / 8][small] (kTmapKeys entries, -1 = none):
// the box follows from the strategy row, the tail rows of A (M % BY) and B (K % 64), and `small`
// is the encoder's size class (tensor spans < kTmapSmallBytes from first to last element).
constexpr int kTmapKeys = 6 * 16 * 33 * 2;
constexpr uint64_t kTmapSmallBytes = 128 * 1024;
__host__ __device__ inline int tmap_key(int w, int row, int box_outer, bool small) {
  return ((w * 16 + row) * 33 + box_outer / 8) * 2 + (small ? 1 : 0);
}
struct MapBuildArgs {
  uint8_t *tmaps;             // CUtensorMap[batch][kMapsPerGemm]
  const uint8_t *templates;   // CUtensorMap[n_templates]
  const int16_t *tidx;        // [kTmapKeys] template index by tmap_key
  const GemmParam *gemms;
  int32_t batch;
  int32_t es;                 // element bytes
};

// Box rows (outer extent) of map w of a tensor-core GEMM, or 0 when the map is not used
// (the conditions of the kernels' map selection and of the bind-time prep kernel).
__host__ __device__ inline int tc_map_outer(int w, int M, int N, int K, int BYc) {
  if (M <= 0 || N <= 0) return 0;
  switch (w) {
    case 0: return K > 0 ? BYc : 0;                                              // A
    case 1: return (K > 0 && M % BYc) ? (M % BYc + 7) / 8 * 8 : 0;               // A row tail
    case 2: return K > 0 ? 64 : 0;                                               // B
    case 3: return (K > 0 && K % 64) ? (K % 64 + 15) / 16 * 16 : 0;              // B K tail
    case 4: return BYc / 4;                                                      // C (loads)
    default: return N >= 8 ? BYc / 4 : 0;                                        // C store
  }
}

// Debug coverage-counter build (-DVB_COVERAGE, libvbgemm_cov.so): every element
// an epilogue thread stores also bumps an int32 counter at the same element offset of a
// caller-supplied counter arena (vb_debug_set_coverage), so a test can check that the tiles of
// a plan write every C element exactly once and nothing outside the matrices.  Each kernel
// translation unit keeps its own copy of the pointers (no relocatable device code).
#ifdef VB_COVERAGE
static __device__ int32_t *g_cov_counts;
static __device__ const uint8_t *g_cov_cbase;
static __device__ int32_t g_cov_es;
__device__ __forceinline__ void cov_add(const void *elem) {
  if (g_cov_counts)
    atomicAdd(g_cov_counts + ((const uint8_t *)elem - g_cov_cbase) / g_cov_es, 1);
}
#define VB_COV_SETTER(name)                                                                    \
  cudaError_t name(int32_t *counts, const void *c_base, int es) {                             \
    cudaError_t e = cudaMemcpyToSymbol(g_cov_counts, &counts, sizeof(counts));                 \
    if (e == cudaSuccess) e = cudaMemcpyToSymbol(g_cov_cbase, &c_base, sizeof(c_base));        \
    if (e == cudaSuccess) e = cudaMemcpyToSymbol(g_cov_es, &es, sizeof(es));                   \
    return e;                                                                                  \
  }
#endif

// Tensor-core strategy geometry derived from a table row (BY, BX): TMA boxes and swizzles.
struct TcGeom {
  int BY, BX;
  int b_swz;       // bytes of one swizzled B row segment (32/64/128) = box inner extent
  int b_boxes;     // B boxes per k-block (BX / (b_swz/2))
  int c_cols;      // C chunk width in elements (one TMA box)
  int c_swz;       // bytes of one swizzled C row segment
  int c_chunks;    // BX / c_cols
};

__host__ __device__ inline TcGeom tc_geom(int BY, int BX) {
  TcGeom g;
  g.BY = BY;
  g.BX = BX;
  g.b_swz = BX >= 64 ? 128 : BX * 2;
  g.b_boxes = BX >= 64 ? BX >> 6 : 1;      // BX / (b_swz / 2), without an integer division
  g.c_cols = BX >= 64 ? 64 : BX;
  g.c_swz = g.c_cols * 2;
  g.c_chunks = BX >= 64 ? BX >> 6 : 1;     // BX / c_cols
  return g;
}

}  // namespace vb
