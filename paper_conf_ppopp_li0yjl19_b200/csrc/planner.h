// Host planner: tiling engine (§4.2.3), tile enumeration, batching engine (§5),
// five-array encoding (§6) and the LPT GEMM->rank sharder.  Pure integer C++.
#pragma once
#include <stdint.h>

#include <string>
#include <vector>

#include "tables.h"

namespace vb {

struct TilerRound {
  int64_t tlp;
  int version_T;
};

struct TilingOut {
  std::vector<int> row;            // chosen table row per GEMM
  int version_T = 0;
  std::vector<TilerRound> trace;
};

struct TileRec {
  int32_t gemm, y, x, K;
};

struct Schedule {                  // the five auxiliary arrays of Fig. 6 (P282)
  std::vector<int32_t> block_ptr;  // Tile[]  (Block_NUM + 1)
  std::vector<int32_t> slot_tile;  // slot -> tile index (enumeration order)
};

// Eq. 1 (P220) with ceil tile counts (reading C-5); a 2-SM pair tile counts twice.
int64_t tlp_eq1(const int32_t *M, const int32_t *N, int batch, const std::vector<int> &row,
                const TableDef &t, int T);

// §4.2.3 steps 1-3 and the two exceptions (P249-253; readings C-1..C-8).
TilingOut tiling_engine(const int32_t *M, const int32_t *N, int batch, const TableDef &t,
                        int64_t threshold, bool pairs_allowed = true);

// Reading C-7b: offer the 2-SM pair strategies only to batches with arithmetic intensity
// 2*sum(MNK) / sum(es*(MK+KN) + 2*es*MN) >= 128 flop/byte.
bool pairs_allowed(const int32_t *M, const int32_t *N, const int32_t *K, int batch, int elem_bytes);

// GEMM-major, row-major (y, x) tiles (P133-135, P157, P284; C-11, C-13).
std::vector<TileRec> enumerate_tiles(const int32_t *M, const int32_t *N, const int32_t *K,
                                     int batch, const std::vector<int> &row, const TableDef &t);

// Threshold batching (P261, reading C-9), binary batching (P263-270, Eq. 5, reading C-10),
// and one tile per block.
Schedule batch_threshold(const std::vector<TileRec> &tiles, int T, int64_t tlp_threshold, int theta);
Schedule batch_binary(const std::vector<TileRec> &tiles, int theta);
Schedule batch_none(const std::vector<TileRec> &tiles);

// LPT on 2*M*N*K (BASELINE.json; reading C-23).
std::vector<int32_t> shard_lpt(const int32_t *M, const int32_t *N, const int32_t *K, int batch,
                               int n_ranks);

}  // namespace vb
