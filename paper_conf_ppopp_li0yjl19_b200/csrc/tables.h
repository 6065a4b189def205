// Strategy tables of the product path.  The oracle keeps its own,
// independently restated copy (oracle/plan_ref.py); the two are compared only by tests.
#pragma once
#include <stdint.h>

namespace vb {

struct StrategyRow {
  const char *name;
  int BY;   // C-tile rows    (along M)
  int BX;   // C-tile columns (along N)
  int BK;   // K step of one main-loop iteration
  int ctas;   // CTAs (SMs) that execute one tile: 2 = tcgen05 cta_group::2 pair tile
  int swap;   // 1 = swap-AB tile (tcgen05): computes C^T = B^T A^T, MMA M = BX (the N side), MMA N = BY
};

constexpr int kMaxRows = 16;
constexpr int kMaxVersions = 2;

struct TableDef {
  int id;
  const char *name;
  int n_rows;
  StrategyRow rows[kMaxRows];
  int n_versions;
  int versions[kMaxVersions];   // thread counts T, preferred (more TLP) first — P247
  int64_t tlp_threshold;        // P253 / P290 (platform constant)
  int theta;                    // P259 / P290 (platform constant)
  // Availability floor (reading C-1b): a strategy is available for a GEMM when
  // BY <= max(M, min_BY) and BX <= max(N, min_BX).  0 for the paper's tables (P249 exactly).
  // tcgen05 table: min_BY = 128 because an M = 64 MMA takes as many cycles as M = 128 (the
  // pacing floor max(M,128)*N/256) and the rows past M are neither loaded (row-tail map) nor
  // stored; min_BX = 256 because a tile at the right edge of a GEMM only pays for the columns
  // it has (MMA N trimmed to N, TMEM columns by MMA width, B boxes past N skipped), so the
  // widest strategy costs a narrow GEMM nothing and covers whole B / C rows in one tile (fewer
  // tiles and A re-reads: measured +3 % on C5 and C4 against min_BX = 64).
  int min_BY;
  int min_BX;
};

// PAPER.md Table 2 (P204-214): small 16x16, medium 32x32, large 64x64, tall 128x64,
// wide 64x128, huge 128x128; BK = 8 (P243); 256- and 128-thread versions (P181, P198).
#define VB_TABLE2_ROWS                                                              \
  {{"small", 16, 16, 8, 1}, {"medium", 32, 32, 8, 1}, {"large", 64, 64, 8, 1},      \
   {"tall", 128, 64, 8, 1}, {"wide", 64, 128, 8, 1}, {"huge", 128, 128, 8, 1}}

// V100 profile: the paper's constants (P255, P290).
constexpr TableDef kTableV100 = {1, "v100_table2", 6, VB_TABLE2_ROWS, 2, {256, 128}, 65536, 256, 0, 0};

// B200 FFMA profile (fp32): Table 2's shapes with its 128-thread sub-tiles (an FFMA design that
// still holds on sm_100a), threshold re-set for 148 SMs (reading C-22).  Calibrated on B200
// (DESIGN.md §4, §6.2): the 128-thread version without the 128x128 row (16x8 sub-tiles need
// 255 registers) runs four CTAs per SM -- one warp per SMSP per CTA, so the warps that share an
// operand ring have equal scheduler priority -- and measured 6 % faster on C2 than the
// 256-thread version at two CTAs per SM (0.312 vs 0.332 ms), which in turn beat the full
// 128-thread version at one CTA per SM by 13 %.  TLP threshold 2 * 148 * 256 threads (= 4 tiles
// of 128 threads per SM: one wave at four CTAs per SM) and theta 64 from the grid calibration on
// this table (scripts/calibrate_grid.py, profiles/calibration_grid_f32_r02.json: geometric-mean
// time over the best pair 1.042, against 1.226 for the round-1 constants calibrated on the
// 256-thread table; theta 1 scores 1.023 but would switch K-batching off); C1/C2 are insensitive.
constexpr TableDef kTableB200Ffma = {2, "b200_ffma", 5,
                                     {{"small", 16, 16, 8, 1}, {"medium", 32, 32, 8, 1}, {"large", 64, 64, 8, 1},
                                      {"tall", 128, 64, 8, 1}, {"wide", 64, 128, 8, 1}},
                                     1, {128, 0}, 2 * 148 * 256, 64, 0, 0};

// B200 tcgen05 profile (bf16/fp16): C tiles for tcgen05.mma with M in {64,128}; BK = 64 =
// one 128-byte swizzled row of bf16; 256 threads per tile in Eq. 1.  Besides the paper's
// square/tall/wide family it has the skinny shapes 128x32 and 64x256 that variable-size
// batches need once short GEMMs may take the 64-row MMA (min_BY = 64), and three 2-SM pair
// tiles (cta_group::2, M = 256: each SM holds 128 rows of A and half of B, so a 256x256 pair
// moves 33% fewer bytes per SM per k-block than 128x256) — the B200 "second version" of P198.
#ifndef VB_TC_MIN_BX
#define VB_TC_MIN_BX 256
#endif
// Constants calibrated on B200 over the Fig. 8/9 grid + C3/C4/C5 (scripts/calibrate_grid.py,
// profiles/calibration_grid_bf16_r01.json): TLP threshold 148 * 256 (one tile per SM: the
// persistent kernel overlaps the tiles of an SM), theta 64 (one BK = 64 k-block).
// Rows S16..S64 are swap-AB tiles for GEMMs with M <= 64 (NEXT-2): C^T = B^T A^T with the
// MMA's M = 128 on the N side and its N = 16..64 on the M side, so a 16-row GEMM issues a
// 128 x 16 MMA instead of a 128 x 256 one whose rows past M are discarded.
// Row W2 (256 x 512, 2-SM) is the widest pair tile: each SM holds 128 rows of A and two
// 128-column halves of B and issues two N = 256 MMAs per K step into all 512 TMEM columns, so a
// k-block carries twice the MMA work of H2 for 1.5x its bytes (the latency its operand ring
// covers grows by 1.5x at equal shared memory) -- the shape cuBLAS's own heuristic runs for
// large bf16 GEMMs on B200 (nvjet_tst_256x256_64x4_2x1_2cta: 256 x 256 C elements per CTA).
constexpr TableDef kTableB200Tc = {3, "b200_tcgen05", 16,
                                   {{"s", 64, 32, 64, 1}, {"n", 128, 32, 64, 1}, {"m", 64, 64, 64, 1},
                                    {"t", 128, 64, 64, 1}, {"w", 64, 128, 64, 1}, {"l", 128, 128, 64, 1},
                                    {"x", 64, 256, 64, 1}, {"h", 128, 256, 64, 1},
                                    {"T2", 256, 64, 64, 2}, {"L2", 256, 128, 64, 2}, {"H2", 256, 256, 64, 2},
                                    {"S16", 16, 128, 64, 1, 1}, {"S32", 32, 128, 64, 1, 1}, {"S48", 48, 128, 64, 1, 1},
                                    {"S64", 64, 128, 64, 1, 1}, {"W2", 256, 512, 64, 2}},
                                   1, {256, 0}, 148 * 256, 64, 128, VB_TC_MIN_BX};

#undef VB_TABLE2_ROWS

inline const TableDef *table_by_id(int id) {
  switch (id) {
    case 1: return &kTableV100;
    case 2: return &kTableB200Ffma;
    case 3: return &kTableB200Tc;
    default: return nullptr;
  }
}

}  // namespace vb
