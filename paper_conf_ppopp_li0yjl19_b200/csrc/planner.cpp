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

// Tiles of one strategy row for an M x N GEMM: ceil(M/BY) * ceil(N/BX) * ctas (C-5).  Every
// table's BY and BX are powers of two, so the divisions are shifts (checked, with a fallback).
struct RowCount {
  int sy = -1, sx = -1, by = 1, bx = 1, ctas = 1;
  explicit RowCount(const StrategyRow &s) : by(s.BY), bx(s.BX), ctas(s.ctas) {
    if ((s.BY & (s.BY - 1)) == 0) sy = __builtin_ctz((unsigned)s.BY);
    if ((s.BX & (s.BX - 1)) == 0) sx = __builtin_ctz((unsigned)s.BX);
  }
  RowCount() = default;
  inline int64_t gy(int64_t m) const { return sy >= 0 ? (m + by - 1) >> sy : (m + by - 1) / by; }
  inline int64_t gx(int64_t n) const { return sx >= 0 ? (n + bx - 1) >> sx : (n + bx - 1) / bx; }
  inline int64_t ctas_for(int64_t m, int64_t n) const { return gy(m) * gx(n) * ctas; }
};

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
  std::vector<int> order;
  for (int r : priority_order(t)) {
    if (t.rows[r].swap) continue;                     // swap-AB rows: forced schedules only (for now)
    if (!allow_pairs && t.rows[r].ctas != 1) continue;   // C-7b: the 1-SM version only
    order.push_back(r);
  }
  RowCount rc[kMaxRows];
  for (int r = 0; r < t.n_rows; ++r) rc[r] = RowCount(t.rows[r]);
  // Step 1 (P249): per-GEMM queue of strategies with BY <= M and BX <= N (C-1, with the
  // table's MMA floor C-1b); if none fits, the smallest strategy alone (C-4).  The queues are
  // stored flat (no = |order| slots per GEMM, rows in priority order); pop = advance head[i],
  // top = read the head.
  const int no = (int)order.size();
#ifdef VB_EXP_FLOOR_BY
  const int floor_by = t.min_BY > 0 ? VB_EXP_FLOOR_BY : 0;   // experiment build: another row floor
#else
  const int floor_by = t.min_BY;
#endif
  std::vector<uint8_t> q((size_t)batch * (size_t)no), qlen((size_t)batch), head((size_t)batch, 0);
  int64_t n_multi = 0;   // queues holding more than one strategy
  for (int i = 0; i < batch; ++i) {
    const int mf = std::max<int>(M[i], floor_by), nf = std::max<int>(N[i], t.min_BX);   // C-1b floor
    uint8_t *qi = &q[(size_t)i * no];
    int n = 0;
    for (int r : order)
      if (t.rows[r].BY <= mf && t.rows[r].BX <= nf) qi[n++] = (uint8_t)r;
    if (n == 0) qi[n++] = (uint8_t)order[0];
    qlen[(size_t)i] = (uint8_t)n;
    n_multi += n > 1;
  }
  int vi = 0;
  TilingOut out;
  out.row.assign(batch, 0);
  int *row = out.row.data();
  for (;;) {
    // Step 2: pop one strategy per GEMM, or top when a single one is left (exception 1, C-2).
    const bool single_before = n_multi == 0;
    int64_t ctas = 0;
    for (int i = 0; i < batch; ++i) {
      const int h = head[(size_t)i], len = qlen[(size_t)i];
      const int r = q[(size_t)i * no + h];
      row[i] = r;
      if (len - h > 1) {
        head[(size_t)i] = (uint8_t)(h + 1);
        if (len - h == 2) --n_multi;   // now a single strategy is left
      }
      ctas += rc[r].ctas_for(M[i], N[i]);
    }
    const bool all_single = n_multi == 0;
    const int T = t.versions[vi];
    const int64_t tlp = ctas * (int64_t)T;
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

void tlp_fill(const int32_t *M, const int32_t *N, const int32_t *K, int batch, const TableDef &t, int64_t threshold,
              TilingOut &out) {
  // Reading C-1d (B200 tcgen05 table): the tiling engine stops at the first round whose TLP is
  // within the threshold, all GEMMs moving together.  When that round leaves TLP below the
  // threshold (the SMs of one wave are not all used), the spare TLP goes to the critical path:
  // the GEMMs whose tiles carry the most operand bytes (K * (min(BY, M) + min(BX, N))) all split their tiles --
  // half the width (same BY) if that gives the GEMM more tiles, else half the height (same BX)
  // -- only if every one of them can and the TLP stays within the threshold; the step repeats
  // on the new maximum.
  if (out.trace.empty() || out.trace.back().tlp > threshold) return;
  const int T = out.version_T;
  int64_t tlp = out.trace.back().tlp;
  bool moved = false;
  auto tiles = [&](int g, int r) { return cdiv(M[g], t.rows[r].BY) * cdiv(N[g], t.rows[r].BX) * t.rows[r].ctas; };
  // the strategy a GEMM's tiles split into: half the width if that gives the GEMM more tiles,
  // else half the height; -1 if neither exists or adds tiles
  auto half_of = [&](int g) {
    const StrategyRow &s = t.rows[out.row[(size_t)g]];
    for (int dim = 0; dim < 2; ++dim)
      for (int q = 0; q < t.n_rows; ++q) {
        const StrategyRow &c = t.rows[q];
        if (c.ctas != s.ctas || c.swap != s.swap) continue;
        const bool fits = dim == 0 ? (c.BY == s.BY && 2 * c.BX == s.BX) : (c.BX == s.BX && 2 * c.BY == s.BY);
        if (fits && tiles(g, q) > tiles(g, out.row[(size_t)g])) return q;
      }
    return -1;
  };
  auto work = [&](int g) {   // operand bytes per k-block of the GEMM's (interior) tile, ~ K (BY + BX)
    const StrategyRow &s = t.rows[out.row[(size_t)g]];
    return (int64_t)K[g] * (std::min<int64_t>(s.BY, M[g]) + std::min<int64_t>(s.BX, N[g]));
  };
  for (;;) {
    int64_t wmax = -1;
    for (int g = 0; g < batch; ++g)
      if (M[g] > 0 && N[g] > 0 && K[g] > 0) wmax = std::max(wmax, work(g));
    if (wmax <= 0) break;
    int64_t add = 0;
    bool ok = true;
    for (int g = 0; g < batch && ok; ++g) {
      if (M[g] <= 0 || N[g] <= 0 || K[g] <= 0 || work(g) != wmax) continue;
      const int h = half_of(g);
      if (h < 0) ok = false;
      else add += tiles(g, h) - tiles(g, out.row[(size_t)g]);
    }
    if (!ok || tlp + add * (int64_t)T > threshold) break;
    std::vector<int> target((size_t)batch, -1);
    for (int g = 0; g < batch; ++g)
      if (M[g] > 0 && N[g] > 0 && K[g] > 0 && work(g) == wmax) target[(size_t)g] = half_of(g);
    for (int g = 0; g < batch; ++g)
      if (target[(size_t)g] >= 0) out.row[(size_t)g] = target[(size_t)g];
    tlp += add * (int64_t)T;
    moved = true;
  }
  if (moved) out.trace.push_back({tlp, T});   // the filled plan's TLP, reported as one more round
}

Segments build_segments(const int32_t *M, const int32_t *N, int batch, const std::vector<int> &row,
                        const TableDef &t) {
  // Tile enumeration (P133-135, P157, P284) in compact form: GEMM g with strategy (BY, BX)
  // owns ceil(M/BY) x ceil(N/BX) consecutive tiles, row-major (y, x).  GEMMs on a 2-SM pair
  // strategy come first (reading C-7b: they run in their own launch), each part ascending.
  RowCount rc[kMaxRows];
  for (int r = 0; r < t.n_rows; ++r) rc[r] = RowCount(t.rows[r]);
  Segments sg;
  sg.gemm.reserve((size_t)batch);
  sg.start.reserve((size_t)batch + 1);
  int64_t at = 0;
  for (int part = 0; part < 2; ++part) {
    for (int i = 0; i < batch; ++i) {
      if (M[i] <= 0 || N[i] <= 0) continue;
      const RowCount &c = rc[row[i]];
      if ((c.ctas == 2) != (part == 0)) continue;
      sg.gemm.push_back(i);
      sg.start.push_back(at);
      at += c.gy(M[i]) * c.gx(N[i]);
    }
    if (part == 0) {
      sg.n_pair = (int)sg.gemm.size();
      sg.n_pair_tiles = at;
    }
  }
  sg.start.push_back(at);
  return sg;
}

int64_t Segments::find(int64_t tile) const {
  // the segment j with start[j] <= tile < start[j + 1]
  return (int64_t)(std::upper_bound(start.begin(), start.end() - 1, tile) - start.begin()) - 1;
}

TileRec decode_tile(const Segments &sg, const int32_t *N, const int32_t *K, const std::vector<int> &row,
                    const TableDef &t, int64_t tile) {
  const int64_t j = sg.find(tile);
  const int g = sg.gemm[(size_t)j];
  const int64_t local = tile - sg.start[(size_t)j];
  const int64_t gx = cdiv(N[g], t.rows[row[g]].BX);
  return TileRec{g, (int32_t)(local / gx), (int32_t)(local % gx), K[g]};
}

static inline void part_range(const Segments &sg, int part, int &j0, int &j1) {
  j0 = part ? sg.n_pair : 0;
  j1 = part ? (int)sg.gemm.size() : sg.n_pair;
}

void batch_threshold(const Segments &sg, const int32_t *K, int part, int T, int64_t tlp_threshold, int theta,
                     Schedule &s) {
  // P261 (garbled; reading C-9): before opening a block, TLP = (unassigned + assigned
  // blocks) * T.  If TLP > threshold/2, fill the block in enumeration order until the sum
  // of K is not less than theta; otherwise every remaining tile is its own block.  A tile's
  // K-workload counts at least 1 (C-11): a K = 0 tile still runs its C = beta*C epilogue, so
  // theta also bounds how many of them one persistent CTA takes.  Blocks are runs of
  // consecutive tiles, so the slot order is the enumeration order (no slot_tile array); the
  // tiles of one GEMM share K, so a fill takes whole runs of a segment at once.
  int j0, j1;
  part_range(sg, part, j0, j1);
  const int64_t t0 = sg.start[(size_t)j0], n = sg.start[(size_t)j1] - t0;
  int64_t i = 0, nblocks = 0;
  int j = j0;
  while (i < n) {
    const int64_t tlp = ((n - i) + nblocks) * (int64_t)T;
    if (2 * tlp > tlp_threshold) {           // TLP > threshold / 2, exact in integers
      int64_t sk = 0;
      while (i < n && sk < theta) {
        while (sg.start[(size_t)j + 1] <= t0 + i) ++j;
        const int64_t kw = std::max<int64_t>(K[sg.gemm[(size_t)j]], 1);
        const int64_t left = sg.start[(size_t)j + 1] - (t0 + i);
        const int64_t need = (theta - sk + kw - 1) / kw;   // tiles until sk >= theta
        const int64_t m = std::min(left, need);
        i += m;
        sk += m * kw;
      }
      s.block_ptr.push_back((int32_t)(t0 + i));
      ++nblocks;
    } else {
      for (; i < n; ++i) s.block_ptr.push_back((int32_t)(t0 + i + 1));
    }
  }
}

// Segments j0..j1-1 stably sorted by the K of their GEMM (K >= 0): LSD radix sort on two
// 16-bit digits for large batches, std::stable_sort for small ones.
static std::vector<int32_t> stable_order_by_k(const Segments &sg, const int32_t *K, int j0, int j1) {
  const size_t n = (size_t)(j1 - j0);
  std::vector<int32_t> ord(n);
  for (size_t q = 0; q < n; ++q) ord[q] = j0 + (int32_t)q;
  auto key = [&](int32_t j) { return (uint32_t)K[sg.gemm[(size_t)j]]; };
  if (n < 4096) {
    std::stable_sort(ord.begin(), ord.end(), [&](int32_t a, int32_t b) { return key(a) < key(b); });
    return ord;
  }
  std::vector<int32_t> tmp(n);
  std::vector<uint32_t> cnt(65537);
  for (int shift = 0; shift < 32; shift += 16) {
    std::fill(cnt.begin(), cnt.end(), 0u);
    bool trivial = true;
    for (size_t q = 0; q < n; ++q) {
      const uint32_t d = (key(ord[q]) >> shift) & 0xFFFF;
      ++cnt[d + 1];
      trivial &= d == 0;
    }
    if (trivial) continue;                       // every digit 0: the pass keeps the order
    for (size_t d = 1; d <= 65536; ++d) cnt[d] += cnt[d - 1];
    for (size_t q = 0; q < n; ++q) tmp[cnt[(key(ord[q]) >> shift) & 0xFFFF]++] = ord[q];
    ord.swap(tmp);
  }
  return ord;
}

void batch_binary(const Segments &sg, const int32_t *K, int part, int theta, Schedule &s) {
  // P263-270 / Eq. 5 (reading C-10): tiles sorted by K ascending (ties: enumeration
  // order); pair min-K with max-K; a max-K tile with K >= theta and an odd middle go alone.
  // A GEMM's tiles share K and are consecutive, so the stable sort of the tiles is the stable
  // sort of the GEMM segments, walked by two cursors.
  int j0, j1;
  part_range(sg, part, j0, j1);
  std::vector<int32_t> ord = stable_order_by_k(sg, K, j0, j1);
  const int64_t n = sg.start[(size_t)j1] - sg.start[(size_t)j0];
  if (n == 0) return;
  auto seg_n = [&](int q) { return sg.start[(size_t)ord[(size_t)q] + 1] - sg.start[(size_t)ord[(size_t)q]]; };
  int qa = 0, qb = (int)ord.size() - 1;        // cursor segments (in sorted order)
  int64_t oa = 0, ob = seg_n(qb) - 1;          // offsets inside them
  auto tile_of = [&](int q, int64_t o) { return (int32_t)(sg.start[(size_t)ord[(size_t)q]] + o); };
  auto k_of = [&](int q) { return K[sg.gemm[(size_t)ord[(size_t)q]]]; };
  auto next_lo = [&]() {
    if (++oa == seg_n(qa)) { ++qa; oa = 0; }
  };
  auto next_hi = [&]() {
    if (--ob < 0 && --qb >= 0) ob = seg_n(qb) - 1;
  };
  int64_t lo = 0, hi = n - 1;
  while (lo <= hi) {
    if (lo == hi) {
      s.slot_tile.push_back(tile_of(qa, oa));
      s.block_ptr.push_back((int32_t)s.slot_tile.size());
      break;
    }
    if (k_of(qb) >= theta) {
      s.slot_tile.push_back(tile_of(qb, ob));
      next_hi();
      --hi;
    } else {
      s.slot_tile.push_back(tile_of(qa, oa));
      s.slot_tile.push_back(tile_of(qb, ob));
      next_lo();
      next_hi();
      ++lo;
      --hi;
    }
    s.block_ptr.push_back((int32_t)s.slot_tile.size());
  }
}

void batch_none(const Segments &sg, int part, Schedule &s) {
  int j0, j1;
  part_range(sg, part, j0, j1);
  for (int64_t i = sg.start[(size_t)j0]; i < sg.start[(size_t)j1]; ++i) s.block_ptr.push_back((int32_t)(i + 1));
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
