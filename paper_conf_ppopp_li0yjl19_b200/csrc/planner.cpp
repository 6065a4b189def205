// Host planner.  Follows PAPER.md §4.2.3 (tiling), §5 (batching) and §6 (encoding).
// Readings of silent or garbled passages are numbered as in DESIGN.md §3.
#include "planner.h"

#include <algorithm>
#include <numeric>
#include <queue>
#include <utility>

namespace vb {

static inline int64_t cdiv(int64_t a, int64_t b) { return (a + b - 1) / b; }

// Priority order of a table: smaller C tile first (P249), ties by table row (C-3).
static std::vector<int> priority_order(const TableDef &t) {
  std::vector<int> o(t.n_rows);
  std::iota(o.begin(), o.end(), 0);
  std::stable_sort(o.begin(), o.end(), [&](int a, int b) {
    return t.rows[a].BY * t.rows[a].BX < t.rows[b].BY * t.rows[b].BX;
  });
  return o;
}

int64_t tlp_eq1(const int32_t *M, const int32_t *N, int batch, const std::vector<int> &row,
                const TableDef &t, int T) {
  int64_t tiles = 0;
  for (int i = 0; i < batch; ++i) {
    const StrategyRow &s = t.rows[row[i]];
    tiles += cdiv(M[i], s.BY) * cdiv(N[i], s.BX) * s.ctas;   // a pair tile occupies two CTAs
  }
  return tiles * (int64_t)T;
}

bool pairs_allowed(const int32_t *M, const int32_t *N, const int32_t *K, int batch, int elem_bytes) {
  // exact in 128-bit integers (sums up to ~1e15 flops for 2^31 GEMMs of 2^20 x 2^20 x 2^31)
  __int128 flops = 0, bytes = 0;
  for (int i = 0; i < batch; ++i) {
    flops += (__int128)2 * M[i] * N[i] * K[i];
    if (M[i] > 0 && N[i] > 0)
      bytes += (__int128)elem_bytes * ((int64_t)M[i] * K[i] + (int64_t)K[i] * N[i]) + (__int128)2 * elem_bytes * M[i] * N[i];
  }
#ifndef VB_PAIR_MIN_AI
#define VB_PAIR_MIN_AI 128
#endif
  return bytes > 0 && flops >= (__int128)VB_PAIR_MIN_AI * bytes;
}

TilingOut tiling_engine(const int32_t *M, const int32_t *N, int batch, const TableDef &t,
                        int64_t threshold, bool allow_pairs) {
  std::vector<int> order = priority_order(t);
  if (!allow_pairs) {   // C-7b: the 1-SM version only
    std::vector<int> o1;
    for (int r : order)
      if (t.rows[r].ctas == 1) o1.push_back(r);
    order = o1;
  }
  // Step 1 (P249): per-GEMM queue of strategies with BY <= M and BX <= N (C-1, with the
  // table's MMA floor C-1b); if none
  // fits, the smallest strategy alone (C-4).  A queue is a [head, end) window of `order`
  // restricted to fitting rows, so pop = advance head, top = read head.
  std::vector<std::vector<int>> q(batch);
  for (int i = 0; i < batch; ++i) {
    const int mf = std::max<int>(M[i], t.min_BY), nf = std::max<int>(N[i], t.min_BX);   // C-1b floor
    for (int r : order)
      if (t.rows[r].BY <= mf && t.rows[r].BX <= nf) q[i].push_back(r);
    if (q[i].empty()) q[i].push_back(order[0]);
  }
  std::vector<size_t> head(batch, 0);
  int vi = 0;
  TilingOut out;
  out.row.assign(batch, 0);
  for (;;) {
    // Step 2: pop one strategy per GEMM, or top when a single one is left (exception 1, C-2).
    bool single_before = true;
    for (int i = 0; i < batch; ++i)
      if (q[i].size() - head[i] > 1) single_before = false;
    bool all_single = true;
    for (int i = 0; i < batch; ++i) {
      out.row[i] = q[i][head[i]];
      if (q[i].size() - head[i] > 1) ++head[i];
      if (q[i].size() - head[i] > 1) all_single = false;
    }
    const int T = t.versions[vi];
    const int64_t tlp = tlp_eq1(M, N, batch, out.row, t, T);
    out.trace.push_back({tlp, T});
    out.version_T = T;
    // Step 3: compare with the threshold (strict, C-6).
    if (tlp <= threshold) return out;
    // Exception 2 (C-7): about to repeat step 2 while every queue holds one strategy:
    // switch to the next thread version and repeat.  With no further version, repeat once
    // more if this round popped (the largest strategies get evaluated); if this round already
    // took every queue's top, nothing larger exists and the solution stands.
    if (all_single) {
      if (vi + 1 < t.n_versions)
        ++vi;
      else if (single_before)
        return out;
    }
  }
}

std::vector<TileRec> enumerate_tiles(const int32_t *M, const int32_t *N, const int32_t *K,
                                     int batch, const std::vector<int> &row, const TableDef &t) {
  int64_t total = 0;
  for (int i = 0; i < batch; ++i)
    if (M[i] > 0 && N[i] > 0) total += cdiv(M[i], t.rows[row[i]].BY) * cdiv(N[i], t.rows[row[i]].BX);
  std::vector<TileRec> tiles;
  tiles.reserve((size_t)total);
  for (int i = 0; i < batch; ++i) {
    if (M[i] <= 0 || N[i] <= 0) continue;
    const StrategyRow &s = t.rows[row[i]];
    const int gy = (int)cdiv(M[i], s.BY), gx = (int)cdiv(N[i], s.BX);
    for (int y = 0; y < gy; ++y)
      for (int x = 0; x < gx; ++x) tiles.push_back({i, y, x, K[i]});
  }
  return tiles;
}

Schedule batch_threshold(const std::vector<TileRec> &tiles, int T, int64_t tlp_threshold, int theta) {
  // P261 (garbled; reading C-9): before opening a block, TLP = (unassigned + assigned
  // blocks) * T.  If TLP > threshold/2, fill the block in enumeration order until the sum
  // of K is not less than theta; otherwise every remaining tile is its own block.  A tile's
  // K-workload counts at least 1 (C-11): a K = 0 tile still runs its C = beta*C epilogue, so
  // theta also bounds how many of them one persistent CTA takes.
  Schedule s;
  const int64_t n = (int64_t)tiles.size();
  s.block_ptr.push_back(0);
  s.slot_tile.reserve((size_t)n);
  int64_t i = 0, nblocks = 0;
  while (i < n) {
    const int64_t tlp = ((n - i) + nblocks) * (int64_t)T;
    if (2 * tlp > tlp_threshold) {           // TLP > threshold / 2, exact in integers
      int64_t sk = 0;
      while (i < n && sk < theta) {
        s.slot_tile.push_back((int32_t)i);
        sk += std::max<int64_t>(tiles[(size_t)i].K, 1);
        ++i;
      }
      s.block_ptr.push_back((int32_t)s.slot_tile.size());
      ++nblocks;
    } else {
      for (; i < n; ++i) {
        s.slot_tile.push_back((int32_t)i);
        s.block_ptr.push_back((int32_t)s.slot_tile.size());
        ++nblocks;
      }
    }
  }
  return s;
}

Schedule batch_binary(const std::vector<TileRec> &tiles, int theta) {
  // P263-270 / Eq. 5 (reading C-10): tiles sorted by K ascending (ties: enumeration
  // order); pair min-K with max-K; a max-K tile with K >= theta and an odd middle go alone.
  Schedule s;
  const int64_t n = (int64_t)tiles.size();
  std::vector<int32_t> ord((size_t)n);
  std::iota(ord.begin(), ord.end(), 0);
  std::stable_sort(ord.begin(), ord.end(),
                   [&](int32_t a, int32_t b) { return tiles[(size_t)a].K < tiles[(size_t)b].K; });
  s.block_ptr.push_back(0);
  s.slot_tile.reserve((size_t)n);
  int64_t lo = 0, hi = n - 1;
  while (lo <= hi) {
    if (lo == hi) {
      s.slot_tile.push_back(ord[(size_t)lo]);
      s.block_ptr.push_back((int32_t)s.slot_tile.size());
      break;
    }
    if (tiles[(size_t)ord[(size_t)hi]].K >= theta) {
      s.slot_tile.push_back(ord[(size_t)hi]);
      --hi;
    } else {
      s.slot_tile.push_back(ord[(size_t)lo]);
      s.slot_tile.push_back(ord[(size_t)hi]);
      ++lo;
      --hi;
    }
    s.block_ptr.push_back((int32_t)s.slot_tile.size());
  }
  return s;
}

Schedule batch_none(const std::vector<TileRec> &tiles) {
  Schedule s;
  s.block_ptr.resize(tiles.size() + 1);
  s.slot_tile.resize(tiles.size());
  for (size_t i = 0; i <= tiles.size(); ++i) s.block_ptr[i] = (int32_t)i;
  for (size_t i = 0; i < tiles.size(); ++i) s.slot_tile[i] = (int32_t)i;
  return s;
}

std::vector<int32_t> shard_lpt(const int32_t *M, const int32_t *N, const int32_t *K, int batch,
                               int n_ranks) {
  std::vector<int64_t> work((size_t)batch);
  for (int i = 0; i < batch; ++i) work[(size_t)i] = 2 * (int64_t)M[i] * (int64_t)N[i] * (int64_t)K[i];
  std::vector<int32_t> ord((size_t)batch);
  std::iota(ord.begin(), ord.end(), 0);
  std::stable_sort(ord.begin(), ord.end(),
                   [&](int32_t a, int32_t b) { return work[(size_t)a] > work[(size_t)b]; });
  // min-heap of (load, rank): least-loaded first, ties to the lowest rank
  using LR = std::pair<int64_t, int32_t>;
  std::priority_queue<LR, std::vector<LR>, std::greater<LR>> heap;
  for (int r = 0; r < n_ranks; ++r) heap.push({0, r});
  std::vector<int32_t> rank_of((size_t)batch, 0);
  for (int32_t g : ord) {
    LR top = heap.top();
    heap.pop();
    rank_of[(size_t)g] = top.second;
    top.first += work[(size_t)g];
    heap.push(top);
  }
  return rank_of;
}

}  // namespace vb
