"""Pins for the B200 departures of the plan oracle (oracle/plan_ref.py), against plans derived
by hand in tests/golden/b200_examples.json (every number there is pencil arithmetic, written
out next to it):

* the tcgen05 availability pre-pass ``b200_step1`` / ``b200_availability`` (reading C-1b),
  contrasted with P249's literal step 1 on the same GEMMs;
* the pair-version gate ``pairs_allowed`` (C-7b) on both sides of 128 flop/B;
* the per-launch batching of pair and 1-SM tiles (C-7b launch split) under both heuristics;
* the K-workload floor of threshold batching (C-11);
* the W2 pair row (256 x 512): its availability and its place at the end of the priority order
  (E3), in the oracle and in the product planner.
"""
import json
import os

import pytest

import vbinputs
from oracle import plan_ref as pr

TC = pr.B200_TC
GOLD = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden", "b200_examples.json")


@pytest.fixture(scope="module")
def g():
    with open(GOLD) as f:
        return json.load(f)


def _names(rows):
    return [TC.rows[r].name for r in rows]


def _mnk(g):
    return [list(c) for c in zip(*g["E1_gemms"]["gemms_MNK"])]


def test_pairs_allowed_e1(g):
    M, N, K = _mnk(g)
    assert pr.pairs_allowed(M, N, K) == g["E1_gemms"]["pairs_allowed"]


@pytest.mark.parametrize("i", [0, 1])
def test_pairs_allowed_both_sides_of_128(g, i):
    x, exp = g["pairs_allowed_cubes"]["cases"][i]
    assert pr.pairs_allowed([x], [x], [x]) is exp


def test_pairs_allowed_configs():
    # C5 (AI ~60 flop/B) keeps the 1-SM version; C4 (AI ~205) is offered the pairs
    assert not pr.pairs_allowed(*vbinputs.config_sizes("C5"))
    assert pr.pairs_allowed(*vbinputs.config_sizes("C4"))


def test_b200_queues(g):
    M, N, _ = _mnk(g)
    q = pr.b200_step1(M, N, TC, allow_pairs=True)
    assert [_names(x) for x in q] == g["E1_gemms"]["b200_queues"]
    q = pr.step1_p249(M, N, TC)
    assert [_names(x) for x in q] == g["E1_gemms"]["p249_queues"]


@pytest.mark.parametrize("key", ["E1_tiler_thr5120", "E1_tiler_thr2048"])
def test_b200_tiler_rounds(g, key):
    M, N, _ = _mnk(g)
    e = g[key]
    tr = pr.tiling_engine(M, N, TC, e["threshold"], pr.b200_step1(M, N, TC, True))
    assert [[_names(r), t] for r, _, t in tr.trace] == [[a, b] for a, b in e["rounds"]]
    assert _names(tr.rows) == e["final"] and tr.T == 256


def test_p249_literal_tiler_rounds(g):
    M, N, _ = _mnk(g)
    e = g["E1_tiler_thr5120"]
    tr = pr.tiling_engine(M, N, TC, e["threshold"])          # default step 1 = P249 literally
    assert [[_names(r), t] for r, _, t in tr.trace] == [[a, b] for a, b in e["p249_rounds"]]
    assert _names(tr.rows) == e["p249_final"]


def test_b200_tiler_without_pairs(g):
    M, N, _ = _mnk(g)
    e = g["E1_tiler_thr2048"]
    tr = pr.tiling_engine(M, N, TC, e["threshold"], pr.b200_step1(M, N, TC, False))
    assert _names(tr.rows) == e["no_pairs_final"] and len(tr.trace) == e["no_pairs_rounds"]


def _blocks(p):
    return [[[p.tiles[t].gemm, p.tiles[t].y, p.tiles[t].x] for t in blk] for blk in p.blocks]


def test_plan_routes_tc_table_through_prepass(g):
    M, N, K = _mnk(g)
    e = g["E1_batching_thr2048_theta10000"]
    p = pr.plan(M, N, K, TC, pr.POLICY_THRESHOLD, tlp_threshold=e["threshold"], theta=e["theta"])
    assert _names(p.tiling.rows) == g["E1_tiler_thr2048"]["final"]
    assert _blocks(p) == e["threshold_blocks"]
    assert p.enc.Tile == e["threshold_Tile"]


def test_binary_batching_per_launch(g):
    M, N, K = _mnk(g)
    e = g["E1_batching_thr2048_theta10000"]
    p = pr.plan(M, N, K, TC, pr.POLICY_BINARY, tlp_threshold=e["threshold"], theta=e["theta"])
    assert _blocks(p) == e["binary_blocks"]


def test_kworkload_floor(g):
    e = g["kworkload_zero"]
    tiles = [pr.Tile(0, i, 0, 0) for i in range(e["zero_tiles"])]
    assert [len(b) for b in pr.threshold_batching(tiles, 256, 0, 64)] == e["zero_block_sizes"]
    tiles = [pr.Tile(0, i, 0, k) for i, k in enumerate(e["mixed_K"])]
    assert [len(b) for b in pr.threshold_batching(tiles, 256, 0, 64)] == e["mixed_block_sizes"]


def test_tlp_fill_post_pass(g):
    e = g["E2_tlp_fill"]
    M, N, K = [list(c) for c in zip(*e["gemms_MNK"])]
    assert pr.pairs_allowed(M, N, K) is False
    tr = pr.tiling_engine(M, N, TC, e["threshold"], pr.b200_step1(M, N, TC, False))
    assert _names(tr.rows) == e["tiler_final"]
    filled = pr.tlp_fill(M, N, K, TC, e["threshold"], tr)
    assert _names(filled.rows) == e["final"] and filled.trace[-1][2] == e["final_tlp"]
    assert len(filled.trace) == e["rounds"]
    p = pr.plan(M, N, K, TC, pr.POLICY_THRESHOLD, tlp_threshold=e["threshold"])
    assert _names(p.tiling.rows) == e["final"]


def test_w2_row_availability_and_priority(g):
    e = g["E3_w2"]
    M, N, K = [list(c) for c in zip(*e["gemms_MNK"])]
    assert pr.pairs_allowed(M, N, K) is e["pairs_allowed"]
    assert TC.rows[e["w2_table_row"]].name == "W2"
    q = pr.b200_step1(M, N, TC, allow_pairs=True)
    assert [_names(x) for x in q] == e["b200_queues"]
    tr = pr.tiling_engine(M, N, TC, 5000, q)
    assert [[_names(r), t] for r, _, t in tr.trace] == [[a, b] for a, b in e["rounds"]]
    assert _names(tr.rows) == e["final_thr5000"]
    tr = pr.tiling_engine(M, N, TC, 5632, pr.b200_step1(M, N, TC, allow_pairs=True))
    assert _names(tr.rows) == e["final_thr5632"]


@pytest.mark.parametrize("thr,key", [(5000, "final_thr5000"), (5632, "final_thr5632")])
def test_w2_row_product_planner(g, thr, key):
    """The C++ tiling engine picks the same rows as the hand derivation (host plan, no GPU)."""
    import numpy as np
    import paper_conf_ppopp_li0yjl19_b200 as vb
    e = g["E3_w2"]
    M, N, K = (np.array(c) for c in zip(*e["gemms_MNK"]))
    ld = (N + 7) // 8 * 8                     # 16-byte rows
    p = vb.plan_vbatched(M, N, K, K, ld, ld, "bf16", vb.VB_BATCH_THRESHOLD, device=-1,
                         table_id=vb.VB_TABLE_B200_TC, tlp_threshold=thr)
    rows = [int(s) % len(TC.rows) for s in p.export()["gemm_strategy"]]
    assert _names(rows) == e[key]
