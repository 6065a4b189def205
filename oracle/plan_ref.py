"""ORACLE (test infrastructure only): reference tiling engine, batching engine, encoding, sharder.

Plain Python, step by step in the paper's order and notation.  Shares no code, table or
constant generator with the C++ planner in ``paper_conf_ppopp_li0yjl19_b200/csrc``; the
tables below are restated here from PAPER.md Table 2 (P204–214) and DESIGN.md §4.

Readings of silent / garbled passages are numbered C-1 … C-24 as in DESIGN.md §3.
"""
from __future__ import annotations

from dataclasses import dataclass, field
from math import ceil
from typing import List, Sequence, Tuple


# ----------------------------------------------------------------------------------------
# Strategy tables
# ----------------------------------------------------------------------------------------
@dataclass(frozen=True)
class Strategy:
    name: str
    BY: int      # tile rows    (along M)
    BX: int      # tile columns (along N)
    BK: int      # K step of one main-loop iteration
    ctas: int = 1  # CTAs executing one tile (2 = tcgen05 cta_group::2 pair tile)
    swap: int = 0  # 1 = swap-AB tile (C^T = B^T A^T on tcgen05; same C tile, same enumeration)


@dataclass(frozen=True)
class Table:
    name: str
    rows: Tuple[Strategy, ...]           # table row order (ids are derived from it)
    versions: Tuple[int, ...]            # thread counts T, first = preferred (more TLP)
    tlp_threshold: int                   # default TLP threshold (P253, P290)
    theta: int                           # default batching threshold θ (P259, P290)

    def order(self) -> List[int]:
        """Priority order: smaller tile first (P249); ties by table row (reading C-3)."""
        return sorted(range(len(self.rows)), key=lambda r: (self.rows[r].BY * self.rows[r].BX, r))

    def strategy_id(self, row: int, T: int) -> int:
        """Reading C-14: id = version_index * n_rows + row ("0-11" for Table 2, P282)."""
        return self.versions.index(T) * len(self.rows) + row


# PAPER.md Table 2 (P204–214), the V100 profile: six shapes, BK = 8 (P243),
# 256- and 128-thread versions (P181, P198); TLP threshold 65536 and θ = 256 (P255, P290).
V100 = Table("v100_table2", (
    Strategy("small", 16, 16, 8), Strategy("medium", 32, 32, 8), Strategy("large", 64, 64, 8),
    Strategy("tall", 128, 64, 8), Strategy("wide", 64, 128, 8), Strategy("huge", 128, 128, 8)),
    versions=(256, 128), tlp_threshold=65536, theta=256)

# B200 FFMA (fp32) profile: the Table 2 shapes (an FFMA design) without the 128x128 row, one
# version with T = 128 threads; platform constants re-set for 148 SMs (calibrated on B200,
# DESIGN.md §4 and §6.2, reading C-22).
B200_F32 = Table("b200_ffma", V100.rows[:5], versions=(128,), tlp_threshold=2 * 148 * 256, theta=64)

# B200 tcgen05 (bf16/fp16) profile: C-tile shapes sized for tcgen05.mma
# (M in {64,128}), BK = 64 (one 128-byte swizzle row of bf16), plus the skinny shapes
# 128x32 and 64x256, plus 2-SM pair tiles 256x{64,128,256,512} (ctas = 2, cta_group::2).  One
# kernel "version" with T = 256 threads.  Its step 1 is the B200 pre-pass
# ``b200_step1`` below (readings C-1b, C-7b), not P249's literal rule.
B200_TC = Table("b200_tcgen05", (
    Strategy("s", 64, 32, 64), Strategy("n", 128, 32, 64), Strategy("m", 64, 64, 64), Strategy("t", 128, 64, 64),
    Strategy("w", 64, 128, 64), Strategy("l", 128, 128, 64), Strategy("x", 64, 256, 64),
    Strategy("h", 128, 256, 64), Strategy("T2", 256, 64, 64, 2), Strategy("L2", 256, 128, 64, 2),
    Strategy("H2", 256, 256, 64, 2), Strategy("S16", 16, 128, 64, 1, 1), Strategy("S32", 32, 128, 64, 1, 1),
    Strategy("S48", 48, 128, 64, 1, 1), Strategy("S64", 64, 128, 64, 1, 1), Strategy("W2", 256, 512, 64, 2)),
    versions=(256,), tlp_threshold=148 * 256, theta=64)

TABLES = {1: V100, 2: B200_F32, 3: B200_TC}


# ----------------------------------------------------------------------------------------
# Tiling engine (§4.2.3, P245–255)
# ----------------------------------------------------------------------------------------
def tlp(Ms, Ns, rows: Sequence[int], table: Table, T: int) -> int:
    """Eq. 1 (P220): TLP = sum_i (M_i*N_i)/(BY_i*BX_i) * T, tiles counted with ceil (C-5)."""
    total = 0
    for M, N, r in zip(Ms, Ns, rows):
        s = table.rows[r]
        total += ceil(M / s.BY) * ceil(N / s.BX) * s.ctas      # a pair tile occupies two CTAs
    return total * T


@dataclass
class TilingResult:
    rows: List[int]            # chosen table row per GEMM
    T: int                     # chosen version (threads per block)
    trace: List[Tuple[List[int], int, int]] = field(default_factory=list)  # (rows, T, TLP) per round
    filled: bool = False       # the last trace entry is the TLP fill post-pass (reading C-1d)

    def ids(self, table: Table) -> List[int]:
        return [table.strategy_id(r, self.T) for r in self.rows]


def step1_p249(Ms, Ns, table: Table) -> List[List[int]]:
    """Step 1 of §4.2.3 exactly as P249 states it: a GEMM's available strategies are the
    table's strategies with BY <= M and BX <= N, in a priority queue, smaller tile first
    (ties by table row, C-3).  If none fits, the smallest strategy alone (C-4)."""
    order = table.order()
    queues = []
    for M, N in zip(Ms, Ns):
        q = [r for r in order if table.rows[r].BY <= M and table.rows[r].BX <= N]
        queues.append(q if q else [order[0]])
    return queues


# B200 pre-pass constants (readings C-1b and C-7b; hardware facts, not paper claims).
TC_MMA_MIN_ROWS = 128     # a 64-row tcgen05.mma issues in the cycles of a 128-row one
TC_EDGE_FREE_COLS = 256   # an edge tile's MMA N, TMEM columns and B boxes stop at the GEMM's N
PAIR_MIN_AI = 128         # flop per compulsory byte at which the 2-SM version is offered


def b200_availability(M: int, N: int) -> Tuple[int, int]:
    """Reading C-1b (B200 tcgen05 table only): the extents a strategy is tested against.

    A tile row count below 128 saves no MMA time (an M = 64 MMA costs the cycles of M = 128) and
    rows past M are neither loaded nor stored, so availability sees at least 128 rows; an edge
    tile's MMA N, TMEM columns and B boxes end at the GEMM's N, so a tile up to 256 columns wide
    costs a narrow GEMM nothing and availability sees at least 256 columns."""
    return max(M, TC_MMA_MIN_ROWS), max(N, TC_EDGE_FREE_COLS)


def pairs_allowed(Ms, Ns, Ks, es: int = 2) -> bool:
    """Reading C-7b: the 2-SM pair version (cta_group::2) is offered only to batches whose
    arithmetic intensity 2*sum(MNK) / sum(es*(MK + KN) + 2*es*MN) is at least 128 flop/B, i.e.
    batches near the compute side of the B200 ridge (~265 flop/B); memory-bound batches keep
    the 1-SM version so that their compute- and memory-heavy tiles overlap in one kernel.
    (The C term counts a read and a write of C whatever β is: a batch-level platform rule.)"""
    flops = sum(2 * m * n * k for m, n, k in zip(Ms, Ns, Ks))
    nbytes = sum(es * (m * k + k * n) + 2 * es * m * n for m, n, k in zip(Ms, Ns, Ks) if m > 0 and n > 0)
    return nbytes > 0 and flops >= PAIR_MIN_AI * nbytes


def b200_step1(Ms, Ns, table: Table, allow_pairs: bool) -> List[List[int]]:
    """The B200 tcgen05 pre-pass that replaces P249's step 1 for that table only:
    P249's rule applied to the extents of ``b200_availability`` (C-1b), over the 1-SM
    strategies only unless ``allow_pairs`` (C-7b).  Pinned by hand-derived plans in
    ``tests/golden/b200_examples.json``."""
    order = [r for r in table.order() if (allow_pairs or table.rows[r].ctas == 1) and not table.rows[r].swap]
    queues = []
    for M, N in zip(Ms, Ns):
        mf, nf = b200_availability(M, N)
        q = [r for r in order if table.rows[r].BY <= mf and table.rows[r].BX <= nf]
        queues.append(q if q else [order[0]])
    return queues


def tiling_engine(Ms, Ns, table: Table, threshold: int | None = None,
                  queues: List[List[int]] | None = None) -> TilingResult:
    """The three steps and two exceptions of P249–253.

    1. Per GEMM, a priority queue of available strategies (``queues``; default: P249's
       literal rule, ``step1_p249``).
    2. Take one strategy per GEMM: pop, or top if only one is left (exception 1, C-2);
       TLP by Eq. 1 with the current version T.
    3. If TLP > threshold (strict, C-6) repeat step 2; otherwise this is the solution.
       Exception 2 (C-7): if step 2 is to be repeated while every queue holds a single
       strategy, switch to the next version (128 threads) and repeat step 2.  With no
       further version, step 2 is still repeated once if this round popped (so the last,
       largest strategy of each queue is evaluated); if this round already took the top of
       every queue there is nothing larger to try and the current solution stands.
    """
    thr = table.tlp_threshold if threshold is None else threshold
    queues = [list(q) for q in (step1_p249(Ms, Ns, table) if queues is None else queues)]
    vi = 0
    T = table.versions[vi]
    trace = []
    while True:
        single_before = all(len(q) == 1 for q in queues)
        cur = [q.pop(0) if len(q) > 1 else q[0] for q in queues]       # step 2
        t = tlp(Ms, Ns, cur, table, T)
        trace.append((list(cur), T, t))
        if t <= thr:                                                   # step 3
            return TilingResult(cur, T, trace)
        if all(len(q) == 1 for q in queues):                           # exception 2
            if vi + 1 < len(table.versions):
                vi += 1
                T = table.versions[vi]
            elif single_before:
                return TilingResult(cur, T, trace)


def tlp_fill(Ms, Ns, Ks, table: Table, threshold: int, tr: TilingResult) -> TilingResult:
    """Reading C-1d, the B200 tcgen05 post-pass on the tiling engine's solution.  When the
    final round's TLP is within the threshold (the wave is not full): take the GEMMs whose
    tiles carry the most operand bytes, K * (min(BY, M) + min(BX, N)); if every one of them can split its tiles
    -- the strategy with the same BY and half the BX (same CTA count) if that gives it more
    tiles, else the one with the same BX and half the BY -- and the TLP with all of them moved
    stays <= threshold, move them all and repeat; otherwise stop.  The filled
    TLP is appended to the trace when some GEMM moved."""
    rows, T = list(tr.rows), tr.T
    t = tr.trace[-1][2]
    if t > threshold:
        return tr

    def tiles(g, r):
        s = table.rows[r]
        return ceil(Ms[g] / s.BY) * ceil(Ns[g] / s.BX) * s.ctas

    def split(g):
        """Half the width (same BY) if that gives GEMM g more tiles, else half the height."""
        s = table.rows[rows[g]]
        for same_by in (True, False):
            for q, x in enumerate(table.rows):
                if x.ctas != s.ctas or x.swap != s.swap:
                    continue
                fits = (x.BY == s.BY and 2 * x.BX == s.BX) if same_by else (x.BX == s.BX and 2 * x.BY == s.BY)
                if fits and tiles(g, q) > tiles(g, rows[g]):
                    return q
        return None

    live = [g for g in range(len(rows)) if Ms[g] > 0 and Ns[g] > 0 and Ks[g] > 0]
    moved = False
    while live:
        work = {g: Ks[g] * (min(table.rows[rows[g]].BY, Ms[g]) + min(table.rows[rows[g]].BX, Ns[g])) for g in live}
        top = [g for g in live if work[g] == max(work.values())]
        targets = [split(g) for g in top]
        if any(h is None for h in targets):
            break
        add = sum(tiles(g, h) - tiles(g, rows[g]) for g, h in zip(top, targets))
        if t + add * T > threshold:
            break
        for g, h in zip(top, targets):
            rows[g] = h
        t += add * T
        moved = True
    trace = tr.trace + ([(list(rows), T, t)] if moved else [])
    return TilingResult(rows, T, trace, moved)


# ----------------------------------------------------------------------------------------
# Tile enumeration (P133–135, P157, P284)
# ----------------------------------------------------------------------------------------
@dataclass(frozen=True)
class Tile:
    gemm: int
    y: int        # tile row index along M   (C-13)
    x: int        # tile column index along N
    K: int        # K-workload of the tile = K of its GEMM (C-11)


def enumerate_tiles(Ms, Ns, Ks, rows: Sequence[int], table: Table) -> List[Tile]:
    """GEMM-major, then row-major (y, x): ceil(M/BY) x ceil(N/BX) tiles per GEMM."""
    tiles = []
    for g, (M, N, K, r) in enumerate(zip(Ms, Ns, Ks, rows)):
        s = table.rows[r]
        if M <= 0 or N <= 0:
            continue
        for y in range(ceil(M / s.BY)):
            for x in range(ceil(N / s.BX)):
                tiles.append(Tile(g, y, x, int(K)))
    return tiles


# ----------------------------------------------------------------------------------------
# Batching engine (§5, P259–270)
# ----------------------------------------------------------------------------------------
def threshold_batching(tiles: Sequence[Tile], T: int, tlp_threshold: int, theta: int) -> List[List[int]]:
    """Threshold batching, TLP first (P261; garbled passage, reading C-9).

    Before opening each new block: TLP = (#unassigned tiles + #assigned blocks) * T.
    If TLP > threshold / 2, fill the new block with tiles (enumeration order) until the sum
    of their K-workloads is not less than θ; otherwise every remaining tile gets its own block.
    A tile's K-workload is its K, counted as at least 1 (reading C-11: a K = 0 tile still
    runs its epilogue C = βC, so θ also bounds the number of K = 0 tiles in one block).
    """
    n = len(tiles)
    blocks: List[List[int]] = []
    i = 0
    while i < n:
        t = ((n - i) + len(blocks)) * T
        if t > tlp_threshold / 2:
            blk, sk = [], 0
            while i < n and sk < theta:
                blk.append(i)
                sk += max(tiles[i].K, 1)
                i += 1
            blocks.append(blk)
        else:
            while i < n:
                blocks.append([i])
                i += 1
    return blocks


def binary_batching(tiles: Sequence[Tile], theta: int) -> List[List[int]]:
    """Binary batching, ILP first (P263–270, Eq. 5; reading C-10).

    Sort tiles by K ascending (stable: ties keep enumeration order); repeatedly pair the
    first (minimal K) with the last (maximal K).  A last tile with K >= θ goes alone (a
    pair containing it can only increase Eq. 5's objective); an odd middle tile goes alone.
    """
    order = sorted(range(len(tiles)), key=lambda t: (tiles[t].K, t))
    blocks: List[List[int]] = []
    lo, hi = 0, len(order) - 1
    while lo <= hi:
        if lo == hi:
            blocks.append([order[lo]])
            break
        if tiles[order[hi]].K >= theta:
            blocks.append([order[hi]])
            hi -= 1
        else:
            blocks.append([order[lo], order[hi]])
            lo += 1
            hi -= 1
    return blocks


def no_batching(tiles: Sequence[Tile]) -> List[List[int]]:
    """One tile per block (the un-batched baseline: "a thread block is responsible for a single tile", P259)."""
    return [[i] for i in range(len(tiles))]


def eq5_objective(tiles: Sequence[Tile], blocks: Sequence[Sequence[int]], theta: int) -> int:
    """Eq. 5 (P267): sum over two-tile blocks of |K_i + K_j - θ|."""
    return sum(abs(tiles[b[0]].K + tiles[b[1]].K - theta) for b in blocks if len(b) == 2)


# ----------------------------------------------------------------------------------------
# Programming interface: the five auxiliary arrays (§6, P282–284, Fig. 6 / Fig. 7)
# ----------------------------------------------------------------------------------------
@dataclass
class Encoded:
    Tile: List[int]          # CSR offsets, Block_NUM + 1 entries
    GEMM: List[int]          # per tile slot: source GEMM
    Y: List[int]             # per tile slot: tile row index
    X: List[int]             # per tile slot: tile column index
    Tiling: List[int]        # per GEMM: strategy id (C-12)


def encode(tiles: Sequence[Tile], blocks: Sequence[Sequence[int]], gemm_strategy_ids: Sequence[int]) -> Encoded:
    """Block b owns tile slots [Tile[b], Tile[b+1]) (P282); slots follow block order."""
    Tl, G, Y, X = [0], [], [], []
    for blk in blocks:
        for t in blk:
            G.append(tiles[t].gemm)
            Y.append(tiles[t].y)
            X.append(tiles[t].x)
        Tl.append(len(G))
    return Encoded(Tl, G, Y, X, list(gemm_strategy_ids))


# ----------------------------------------------------------------------------------------
# Whole plan
# ----------------------------------------------------------------------------------------
POLICY_THRESHOLD, POLICY_BINARY, POLICY_NONE = 0, 1, 2


@dataclass
class Plan:
    table: Table
    tiling: TilingResult
    tiles: List[Tile]
    blocks: List[List[int]]
    enc: Encoded


def plan(Ms, Ns, Ks, table: Table, policy: int = POLICY_THRESHOLD,
         tlp_threshold: int | None = None, theta: int | None = None, es: int = 2, allow_pairs: bool = True) -> Plan:
    """The whole host phase: tiling engine, tile enumeration, batching engine, encoding.

    Tables with pair tiles (the B200 tcgen05 table) take step 1 from the B200 pre-pass
    ``b200_step1``; every other table uses P249 literally.  allow_pairs=False: 1-SM
    strategies only (the implicit-GEMM convolution plans).

    Reading C-7b (launch split): pair tiles run in their own cluster launch, enqueued before
    the 1-SM launch on the same stream.  The two launches never run concurrently, so the
    batching engine sees two batches: it packs the pair tiles and the 1-SM tiles separately
    (each in enumeration order; P261's TLP counts the thread blocks of one launch) and the
    pair blocks come first in Tile[].
    """
    thr = table.tlp_threshold if tlp_threshold is None else tlp_threshold
    th = table.theta if theta is None else theta
    Ms = [int(v) for v in Ms]; Ns = [int(v) for v in Ns]; Ks = [int(v) for v in Ks]
    if table is B200_TC:
        q = b200_step1(Ms, Ns, table, allow_pairs and pairs_allowed(Ms, Ns, Ks, es))
    else:
        q = step1_p249(Ms, Ns, table)
    tr = tiling_engine(Ms, Ns, table, thr, q)
    if table is B200_TC:
        tr = tlp_fill(Ms, Ns, Ks, table, thr, tr)
    all_tiles = enumerate_tiles(Ms, Ns, Ks, tr.rows, table)
    is_pair = [table.rows[tr.rows[t.gemm]].ctas == 2 for t in all_tiles]
    tiles = [t for t, pp in zip(all_tiles, is_pair) if pp] + [t for t, pp in zip(all_tiles, is_pair) if not pp]
    n_pair = sum(is_pair)
    blocks = []
    for lo, hi in ((0, n_pair), (n_pair, len(tiles))):
        part = tiles[lo:hi]
        if policy == POLICY_THRESHOLD:
            b = threshold_batching(part, tr.T, thr, th)
        elif policy == POLICY_BINARY:
            b = binary_batching(part, th)
        elif policy == POLICY_NONE:
            b = no_batching(part)
        else:
            raise ValueError(policy)
        blocks += [[lo + i for i in blk] for blk in b]
    enc = encode(tiles, blocks, tr.ids(table))
    return Plan(table, tr, tiles, blocks, enc)


# ----------------------------------------------------------------------------------------
# Multi-GPU: FLOP-balanced GEMM -> rank assignment (BASELINE.json north_star; C-23)
# ----------------------------------------------------------------------------------------
def shard_lpt(Ms, Ns, Ks, n_ranks: int) -> List[int]:
    """Longest-processing-time first on work 2*M*N*K: GEMMs by (-work, index) each go to
    the least-loaded rank, ties to the lowest rank."""
    if n_ranks <= 0:
        raise ValueError("n_ranks must be positive")
    work = [2 * int(m) * int(n) * int(k) for m, n, k in zip(Ms, Ns, Ks)]
    order = sorted(range(len(work)), key=lambda g: (-work[g], g))
    load = [0] * n_ranks
    rank_of = [0] * len(work)
    for g in order:
        r = min(range(n_ranks), key=lambda q: (load[q], q))
        rank_of[g] = r
        load[r] += work[g]
    return rank_of
