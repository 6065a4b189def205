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

struct Schedule {                  // the batching scheme (Fig. 6, P282)
  std::vector<int32_t> block_ptr;  // Tile[]  (Block_NUM + 1)
  std::vector<int32_t> slot_tile;  // slot -> tile (enumeration order); EMPTY = identity (threshold, none)
};

// The tile enumeration in compact form: GEMM gemm[j] owns tiles [start[j], start[j+1]) in
// row-major (y, x) order.  Segments [0, n_pair) are the GEMMs on 2-SM pair strategies.
struct Segments {
  std::vector<int32_t> gemm;
  std::vector<int64_t> start;      // [n_seg + 1]
  int n_pair = 0;
  int64_t n_pair_tiles = 0;
  int64_t n_tiles() const { return start.empty() ? 0 : start.back(); }
  int64_t find(int64_t tile) const;
};

// Eq. 1 (P220) with ceil tile counts (reading C-5); a 2-SM pair tile counts twice.
int64_t tlp_eq1(const int32_t *M, const int32_t *N, int batch, const std::vector<int> &row,
                const TableDef &t, int T);

// §4.2.3 steps 1-3 and the two exceptions (P249-253; readings C-1..C-8).
TilingOut tiling_engine(const int32_t *M, const int32_t *N, int batch, const TableDef &t,
                        int64_t threshold, bool pairs_allowed = true);

// Reading C-1d (B200 tcgen05 table): after the tiling engine, spend TLP left below the threshold
// on the longest-K GEMMs by halving their tile width (one more trace entry when it applies).
void tlp_fill(const int32_t *M, const int32_t *N, const int32_t *K, int batch, const TableDef &t, int64_t threshold,
              TilingOut &out);

// Reading C-7b: offer the 2-SM pair strategies only to batches with arithmetic intensity
// 2*sum(MNK) / sum(es*(MK+KN) + 2*es*MN) >= 128 flop/byte.
bool pairs_allowed(const int32_t *M, const int32_t *N, const int32_t *K, int batch, int elem_bytes);

// GEMM-major, row-major (y, x) tiles (P133-135, P157, P284; C-11, C-13), pair-strategy GEMMs
// first (reading C-7b), as segments.
Segments build_segments(const int32_t *M, const int32_t *N, int batch, const std::vector<int> &row,
                        const TableDef &t);
// (GEMM, Y, X, K) of one tile of the enumeration (host mirror of the device expansion).
TileRec decode_tile(const Segments &sg, const int32_t *N, const int32_t *K, const std::vector<int> &row,
                    const TableDef &t, int64_t tile);

// Batching of one launch's tiles (part 0: pair tiles, 1: 1-SM tiles), appended to s
// (s.block_ptr must already hold its leading entry): threshold batching (P261, reading C-9),
// binary batching (P263-270, Eq. 5, reading C-10) and one tile per block.  Threshold and none
// keep the enumeration order (s.slot_tile stays empty); binary fills s.slot_tile.
void batch_threshold(const Segments &sg, const int32_t *K, int part, int T, int64_t tlp_threshold, int theta,
                     Schedule &s);
void batch_binary(const Segments &sg, const int32_t *K, int part, int theta, Schedule &s);
void batch_none(const Segments &sg, int part, Schedule &s);

// LPT on 2*M*N*K (BASELINE.json; reading C-23).
std::vector<int32_t> shard_lpt(const int32_t *M, const int32_t *N, const int32_t *K, int batch,
                               int n_ranks);

}  // namespace vb
