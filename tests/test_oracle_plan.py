"""Pins for the reference tiling / batching / encoding / sharding (oracle/plan_ref.py).

Pinned to values the paper prints (tests/golden/paper_examples.json, each with its
PAPER.md line), to table arithmetic, to consistency with P352, to derived values of the
worked examples and to invariants on random batches.
"""
import itertools
from math import ceil

import numpy as np
import pytest
from hypothesis import given, settings, strategies as st

from oracle import plan_ref as pr
from oracle.checks import check_plan_invariants, coverage

V = pr.V100


def _names(table, rows):
    return [table.rows[r].name for r in rows]


# ---------------------------------------------------------------------------- T1 (P255)
def test_w3_tiler_trace_matches_paper(golden):
    w = golden["W3_tiler"]
    M, N, K = zip(*w["gemms_MNK"])
    tr = pr.tiling_engine(M, N, V, w["threshold"])
    assert tr.T == w["T"]
    assert len(tr.trace) == len(w["rounds"])
    for (rows, T, tlp), exp in zip(tr.trace, w["rounds"]):
        assert _names(V, rows) == exp["strategies"]
        assert tlp == exp["TLP"]
    assert _names(V, tr.rows) == w["final"]


def test_w3_or_reading_would_disagree(golden):
    # C-1: the "BY<=M or BX<=N" reading gives (medium, medium, medium) with TLP 17664 != 17920
    w = golden["W3_tiler"]
    M, N, _ = zip(*w["gemms_MNK"])
    tlp_or = pr.tlp(M, N, [1, 1, 1], V, 256)
    assert tlp_or == 17664 and tlp_or != w["rounds"][1]["TLP"]


# ---------------------------------------------------------------------------- T2 (P157)
def test_w1_grid_orientation(golden):
    w = golden["W1_magma_tiles"]
    one = pr.Table("t16", (pr.Strategy("s16", 16, 16, 8),), versions=(256,), tlp_threshold=0, theta=256)
    M, N, K = zip(*w["gemms_MNK"])
    tiles = pr.enumerate_tiles(M, N, K, [0, 0, 0], one)
    for g, (r, c) in enumerate(w["grids_rows_cols"]):
        mine = [t for t in tiles if t.gemm == g]
        assert len(mine) == r * c
        assert max(t.y for t in mine) + 1 == r and max(t.x for t in mine) + 1 == c
        # row-major order inside the GEMM
        assert [(t.y, t.x) for t in mine] == [(y, x) for y in range(r) for x in range(c)]


# ---------------------------------------------------------------------------- T3 (P282-284)
def test_w4_encoding(golden):
    w = golden["W4_encoding"]
    # GEMM0: 256x128 with 128x128 tiles -> 2 tiles; GEMM1: 256x256 with 128x64 tiles -> 8 tiles
    Ms, Ns, Ks = [256, 256], [128, 256], [64, 64]
    rows = [5, 3]                                   # huge, tall
    tiles = pr.enumerate_tiles(Ms, Ns, Ks, rows, V)
    assert [sum(1 for t in tiles if t.gemm == g) for g in (0, 1)] == w["tiles_per_gemm"]
    blocks = [[0], [1], [2, 3], [4, 5], [6, 7], [8, 9]]
    enc = pr.encode(tiles, blocks, [V.strategy_id(r, 256) for r in rows])
    assert len(enc.Tile) - 1 == w["n_blocks"]
    assert enc.Tile == [0, 1, 2, 4, 6, 8, 10]
    assert enc.GEMM == [0, 0, 1, 1, 1, 1, 1, 1, 1, 1]
    lo, hi = w["block2_slots"]
    assert (enc.Tile[2], enc.Tile[3]) == (lo, hi)
    assert all(enc.GEMM[s] == w["block2_gemm"] for s in range(lo, hi))
    assert [[enc.Y[s], enc.X[s]] for s in range(lo, hi)] == w["block2_coords"]


# ---------------------------------------------------------------------------- T4 (Tables 1, 2)
def test_table2_matches_paper_and_unified_threads(golden):
    t2 = golden["table2"]
    assert [(s.name, s.BY, s.BX, s.BK) for s in V.rows] == [tuple(r[:4]) for r in t2["rows"]]
    for name, BY, BX, BK, sub128, sub256 in t2["rows"]:
        # "unified thread structure" (P181): every strategy has the same thread count
        assert (BY // sub128[0]) * (BX // sub128[1]) == 128
        assert (BY // sub256[0]) * (BX // sub256[1]) == 256
        assert BY % sub128[0] == 0 and BX % sub128[1] == 0
    assert set(V.versions) == set(t2["versions"]) and V.versions[0] == 256   # 256 first (P247)
    c = golden["constants"]
    assert V.tlp_threshold == c["tlp_threshold"] and V.theta == c["theta"]
    assert all(s.BK == c["BK"] for s in V.rows)


def test_table1_threads_and_eq4():
    # Table 1 rows (P187-196); threads = BY*BX/sub-tile (P179); Eq. 4 = Eq. 3 / Eq. 2 (P228-239)
    rows = [("small", 16, 16, 32, (4, 2)), ("medium", 32, 32, 64, (4, 4)), ("large", 64, 64, 64, (8, 8)),
            ("tall", 128, 64, 128, (8, 8)), ("wide", 64, 128, 128, (8, 8)), ("huge", 128, 128, 256, (8, 8))]
    for _, BY, BX, T, sub in rows:
        assert BY * BX // (sub[0] * sub[1]) == T
        BK, lw = 8, 4
        num_load = (BY * BK + BK * BX) / (lw * T)
        num_fma = BY * BX * BK / T
        assert abs(num_fma / num_load - 4 * BY * BX / (BY + BX)) < 1e-9


def test_priority_order_is_by_area():
    for tab in (pr.V100, pr.B200_TC):
        areas = [tab.rows[r].BY * tab.rows[r].BX for r in tab.order()]
        assert areas == sorted(areas)


# ---------------------------------------------------------------------------- T5 (P202, P324)
def test_tile_counts(golden):
    w5, w6 = golden["W5_single_gemm_tiles"], golden["W6_tiling_blocks"]
    M, N, K = w5["MNK"]
    assert len(pr.enumerate_tiles([M], [N], [K], [5], V)) == w5["tiles"] < w5["v100_sms"]
    m, n = w6["MN"]
    b = w6["batch"]
    assert len(pr.enumerate_tiles([m] * b, [n] * b, [64] * b, [5] * b, V)) == w6["huge_blocks"]
    assert len(pr.enumerate_tiles([m] * b, [n] * b, [64] * b, [0] * b, V)) == w6["small_blocks"]


# ---------------------------------------------------------------------------- T6 (P352)
def _inception(nb, module):
    from vbinputs import googlenet_shapes
    sh = googlenet_shapes(nb, first_stage_only=True, module=module)
    return [s[1] for s in sh], [s[2] for s in sh], [s[3] for s in sh]


def test_googlenet_anchor_shape(golden):
    from vbinputs import googlenet_shapes
    g = {name: (m, n, k) for name, m, n, k in googlenet_shapes(1)}
    assert list(g["3a/5x5_reduce"]) == golden["googlenet_anchor"]["MNK"]


def test_googlenet_3a_batches_and_3b_does_not():
    # P352: for 3a "the batching engine can batch two tiles along K" (K=192 < θ=256);
    # for the other layers "K ... large enough, so the benefit only comes from tiling" (3b: K=256)
    for nb in (1, 2, 4):
        M, N, K = _inception(nb, "3a")
        for pol in (pr.POLICY_THRESHOLD, pr.POLICY_BINARY):
            p = pr.plan(M, N, K, V, pol)
            assert max(len(b) for b in p.blocks) == 2
        M, N, K = _inception(nb, "3b")
        for pol in (pr.POLICY_THRESHOLD, pr.POLICY_BINARY):
            p = pr.plan(M, N, K, V, pol)
            assert max(len(b) for b in p.blocks) == 1      # pins "not less than θ" (C-9) and K>=θ alone (C-10)


def test_googlenet_3a_m16_gets_small_128_threads():
    # P352: "the second GEMM is with M = 16 ... we can choose small tile strategy with 128-thread version"
    M, N, K = _inception(3, "3a")
    tr = pr.tiling_engine(M, N, V)
    g16 = M.index(16)
    assert V.rows[tr.rows[g16]].name == "small" and tr.T == 128


def test_googlenet_nb1_derived_plans():
    # SURVEY.md Appendix A derived values (V100 profile, readings C-1..C-11)
    M, N, K = _inception(1, "3a")
    p = pr.plan(M, N, K, V, pr.POLICY_THRESHOLD)
    assert _names(V, p.tiling.rows) == ["medium", "medium", "small", "medium"] and p.tiling.T == 256
    assert len(p.tiles) == 199
    assert len(p.blocks) == 128 and sum(1 for b in p.blocks if len(b) == 2) == 71
    assert len(pr.plan(M, N, K, V, pr.POLICY_BINARY).blocks) == 100


# ---------------------------------------------------------------------------- T7 (derived, W3)
def test_w3_derived_plans(golden):
    M, N, K = zip(*golden["W3_tiler"]["gemms_MNK"])
    pt = pr.plan(M, N, K, V, pr.POLICY_THRESHOLD)
    assert len(pt.tiles) == 70 and len(pt.blocks) == 70 and all(len(b) == 1 for b in pt.blocks)
    pb = pr.plan(M, N, K, V, pr.POLICY_BINARY)
    assert len(pb.blocks) == 35 and all(len(b) == 2 for b in pb.blocks)
    first = [(pb.tiles[t].gemm, pb.tiles[t].y, pb.tiles[t].x, pb.tiles[t].K) for t in pb.blocks[0]]
    assert first == [(1, 0, 0, 64), (0, 0, 1, 128)]
    last = [(pb.tiles[t].gemm, pb.tiles[t].y, pb.tiles[t].x) for t in pb.blocks[-1]]
    assert last == [(2, 3, 6), (2, 3, 7)]
    assert pr.eq5_objective(pb.tiles, pb.blocks, 256) == 2 * 64 + 33 * 128


def test_threshold_batching_fill_mode_small_example():
    # hand-checked: T=1, threshold 100 -> fill while (unassigned+blocks) > 50
    tiles = [pr.Tile(0, 0, i, k) for i, k in enumerate([100] * 60)]
    blocks = pr.threshold_batching(tiles, 1, 100, 256)
    # each fill block takes 3 tiles (300 >= 256); block b opened when (60-3b)+b > 50 <=> b < 5
    assert [len(b) for b in blocks[:5]] == [3] * 5
    assert all(len(b) == 1 for b in blocks[5:]) and len(blocks) == 5 + 45


# ---------------------------------------------------------------------------- invariants
sizes = st.lists(st.tuples(st.integers(0, 300), st.integers(0, 300), st.integers(0, 700)), min_size=0, max_size=24)


@settings(max_examples=60, deadline=None)
@given(sizes, st.sampled_from([1, 2, 3]), st.sampled_from([0, 1, 2]),
       st.sampled_from([0, 1000, 65536, 10 ** 9]), st.sampled_from([1, 64, 256, 1024]))
def test_plan_invariants_random(sz, table_id, policy, thr, theta):
    tab = pr.TABLES[table_id]
    M = [s[0] for s in sz]; N = [s[1] for s in sz]; K = [s[2] for s in sz]
    p = pr.plan(M, N, K, tab, policy, thr, theta)
    check_plan_invariants(p, M, N, K, policy, theta)


# ---------------------------------------------------------------------------- LPT
def _opt_makespan(work, m):
    best = None
    for assign in itertools.product(range(m), repeat=len(work)):
        loads = [0] * m
        for w, r in zip(work, assign):
            loads[r] += w
        best = max(loads) if best is None else min(best, max(loads))
    return best


@pytest.mark.parametrize("seed", range(12))
def test_lpt_graham_bound(seed):
    rng = np.random.default_rng(seed)
    n = int(rng.integers(1, 9)); m = int(rng.integers(1, 4))
    Ms, Ns, Ks = (rng.integers(1, 40, n) for _ in range(3))
    rank = pr.shard_lpt(Ms, Ns, Ks, m)
    assert len(rank) == n and all(0 <= r < m for r in rank)
    work = [2 * int(a) * int(b) * int(c) for a, b, c in zip(Ms, Ns, Ks)]
    loads = [sum(w for w, r in zip(work, rank) if r == q) for q in range(m)]
    opt = _opt_makespan(work, m)
    assert max(loads) <= (4 / 3 - 1 / (3 * m)) * opt + 1e-9


def test_lpt_example():
    # works 16,12,10,8,6 on 2 ranks: 16->0, 12->1, 10->1 (12<16), 8->0 (16<22), 6->0 (24 > 22? no: 24 vs 22 -> 1)
    # loads: r0 = 16+8 = 24, r1 = 12+10 = 22 -> 6 goes to r1
    M = [8, 6, 5, 4, 3]; N = [1] * 5; K = [1] * 5
    assert pr.shard_lpt(M, N, K, 2) == [0, 1, 1, 0, 1]
