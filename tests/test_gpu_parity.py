"""GPU parity: the CUDA path (through the C-ABI) against the fp64 oracle, element by element,
on the same seeded inputs (regenerated on the host by vbinputs; never read back from the GPU).
Tolerances (BASELINE.json north_star): normwise max relative error 1e-5 fp32, 2e-2 bf16/fp16."""
import numpy as np
import pytest
import torch

import vbinputs
from oracle import plan_ref as pr
from gpu_helpers import check_batch, check_bound, check_recorded, to_f64

pytestmark = pytest.mark.gpu

if torch.cuda.is_available():
    from paper_conf_ppopp_li0yjl19_b200.batch import DeviceBatch
    import paper_conf_ppopp_li0yjl19_b200 as vb

SEED = 0


def _run(M, N, K, dtype, policy=0, ab="random", seed=SEED, ld_extra=0, table_id=0, thr=0, theta=0, c_sentinel=True):
    db = DeviceBatch(M, N, K, dtype, ld_extra=ld_extra)
    if c_sentinel:
        db.C.fill_(float("nan"))
    db.fill(seed, ab)
    plan = db.plan(policy, table_id=table_id, tlp_threshold=thr, theta=theta)
    db.run(plan)
    torch.cuda.synchronize()
    return db, plan


def _padding_untouched(db):
    # row padding [N, ldc) of rows 0 .. M-2 (the last row's padding lies past the matrix's
    # allocation and may hold the next matrix)
    for g in range(db.batch):
        m, n, ld = int(db.M[g]), int(db.N[g]), int(db.ldc[g])
        if m <= 1 or n == 0 or ld == n:
            continue
        full = torch.as_strided(db.C, (m - 1, ld), (ld, 1), int(db.offC[g]))
        assert torch.isnan(full[:, n:]).all(), f"GEMM {g}: padding of C was written"


def test_device_fill_matches_host_generator():
    for dtype in ("f32", "bf16", "f16"):
        M = np.array([1, 7, 33, 130]); N = np.array([3, 16, 65, 9]); K = np.array([5, 64, 17, 200])
        db = DeviceBatch(M, N, K, dtype, gemm_ids=[11, 0, 5, 70000], ld_extra=1)
        db.fill(seed=123)
        torch.cuda.synchronize()
        for g in range(4):
            gid = int(db.gemm_ids[g])
            for view, op, r, c in ((db.a(g), 0, M[g], K[g]), (db.b(g), 1, K[g], N[g]), (db.c(g), 2, M[g], N[g])):
                ref_store, ref64 = vbinputs.matrix(123, gid, op, int(r), int(c), dtype)
                assert np.array_equal(to_f64(view), ref64), (dtype, g, op)
        al, be = vbinputs.alpha_beta(123, db.gemm_ids)
        assert np.array_equal(db.alpha.cpu().numpy(), al) and np.array_equal(db.beta.cpu().numpy(), be)


@pytest.mark.parametrize("policy", [0, 1, 2])
def test_c1_fp32_full(policy):
    M, N, K = vbinputs.config_sizes("C1")
    db, _ = _run(M, N, K, "f32", policy)
    check_batch(db, range(db.batch), SEED, "random")
    _padding_untouched(db)


def test_c1_fp32_v100_profile_and_128_threads():
    # force the 128-thread version: tiny threshold makes the tiler walk to the largest tiles
    M, N, K = vbinputs.config_sizes("C1")
    db, plan = _run(M, N, K, "f32", 0, table_id=vb.VB_TABLE_V100, thr=1)
    assert plan.info()["version_T"] == 128
    check_batch(db, range(db.batch), SEED, "random")


def test_c2_fp32_full():
    M, N, K = vbinputs.config_sizes("C2")
    db, _ = _run(M, N, K, "f32", 0)
    check_recorded("C2/threshold-full", db, range(db.batch), SEED, "random")
    _padding_untouched(db)


def test_fp32_every_strategy_both_versions():
    rng = np.random.default_rng(3)
    M = rng.integers(1, 300, 40); N = rng.integers(1, 300, 40); K = rng.integers(1, 300, 40)
    for table_id in (1, 2):
        for thr in (1, 10 ** 4, 10 ** 5, 10 ** 9):
            db, plan = _run(M, N, K, "f32", 0, table_id=table_id, thr=thr)
            check_batch(db, range(db.batch), SEED, "random")


@pytest.mark.parametrize("dtype", ["bf16", "f16"])
def test_c3_googlenet_full(dtype):
    for nb in (1, 4):
        M, N, K = vbinputs.config_sizes("C3", nb=nb)
        db, _ = _run(M, N, K, dtype, 0, ab="conv")
        check_batch(db, range(db.batch), SEED, "conv")
        _padding_untouched(db)


EDGE = [(1, 1, 1), (5, 3, 7), (64, 32, 64), (65, 33, 65), (127, 63, 1), (129, 65, 129), (128, 256, 64),
        (200, 300, 100), (17, 257, 640), (300, 31, 33), (0, 16, 16), (16, 0, 16), (40, 24, 0), (1000, 8, 8),
        (8, 1000, 8), (513, 129, 2048)]


@pytest.mark.parametrize("dtype", ["bf16", "f16"])
@pytest.mark.parametrize("policy", [0, 1, 2])
def test_tc_edge_shapes(dtype, policy):
    M, N, K = (np.array(c) for c in zip(*EDGE))
    db, _ = _run(M, N, K, dtype, policy)
    check_recorded(f"edge/{dtype}/p{policy}", db, range(db.batch), SEED, "random")
    _padding_untouched(db)


def _forced_rows_plan(db, rows, table, table_id):
    """Device plan with the given strategy row per GEMM, one tile per block (plan_from_schedule)."""
    tiles = pr.enumerate_tiles(db.M, db.N, db.K, rows, table)
    pair = [table.rows[rows[t.gemm]].ctas == 2 for t in tiles]     # 2-SM pair blocks first
    tiles = [t for t, q in zip(tiles, pair) if q] + [t for t, q in zip(tiles, pair) if not q]
    return vb.plan_from_schedule(db.M, db.N, db.K, db.lda, db.ldb, db.ldc, rows, table.versions[0],
                                 list(range(len(tiles) + 1)), [t.gemm for t in tiles], [t.y for t in tiles],
                                 [t.x for t in tiles], dtype=db.dtype, device=0, table_id=table_id)


@pytest.mark.parametrize("dtype", ["bf16", "f16", "f32"])
def test_every_strategy_row_forced(dtype):
    # every row of the table on ragged shapes, including shapes smaller than the tile
    rng = np.random.default_rng(4)
    n = 48
    M = rng.integers(1, 400, n); N = rng.integers(1, 400, n); K = rng.integers(0, 600, n)
    db = DeviceBatch(M, N, K, dtype)
    db.C.fill_(float("nan"))
    db.fill(SEED)
    table, tid = (pr.B200_TC, 3) if dtype != "f32" else (pr.B200_F32, 2)
    rows = [g % len(table.rows) for g in range(n)]
    db.run(_forced_rows_plan(db, rows, table, tid))
    torch.cuda.synchronize()
    check_batch(db, range(n), SEED, "random")
    check_bound(db, range(n), SEED, "random")
    _padding_untouched(db)


def test_fp32_edge_shapes():
    M, N, K = (np.array(c) for c in zip(*EDGE))
    db, _ = _run(M, N, K, "f32", 0, ld_extra=1)
    check_batch(db, range(db.batch), SEED, "random")
    _padding_untouched(db)


@pytest.mark.parametrize("dtype", ["f32", "bf16"])
def test_beta_zero_never_reads_c(dtype):
    M = np.array([70, 130, 5]); N = np.array([64, 200, 9]); K = np.array([33, 256, 3])
    db = DeviceBatch(M, N, K, dtype)
    db.fill(SEED, "conv")
    db.C.fill_(float("nan"))
    db.run(db.plan())
    torch.cuda.synchronize()
    for g in range(3):
        assert torch.isfinite(db.c(g)).all()
    check_batch(db, range(3), SEED, "conv", c_old=[np.zeros((int(m), int(n))) for m, n in zip(M, N)])


@pytest.mark.parametrize("dtype", ["f32", "bf16"])
def test_alpha_zero_scales_c(dtype):
    M = np.array([70, 130]); N = np.array([64, 200]); K = np.array([33, 256])
    db = DeviceBatch(M, N, K, dtype)
    db.fill(SEED)
    db.alpha.zero_()
    c_old = [to_f64(db.c(g)).copy() for g in range(2)]
    be = db.beta.cpu().numpy().astype(np.float64)
    db.run(db.plan())
    torch.cuda.synchronize()
    tol = 1e-6 if dtype == "f32" else 4e-3
    for g in range(2):
        ref = be[g] * c_old[g]
        assert np.max(np.abs(to_f64(db.c(g)) - ref)) <= tol * max(1.0, np.abs(ref).max())


def _sampled(cfg, n_sample, policy=0):
    M, N, K = vbinputs.config_sizes(cfg)
    db, plan = _run(M, N, K, "bf16", policy, c_sentinel=False)
    work = 2 * M * N * K
    rng = np.random.default_rng(7)
    idx = sorted(set([int(np.argmax(work)), int(np.argmin(work)), 0, len(M) - 1] +
                     list(rng.choice(len(M), n_sample, replace=False))))
    return check_recorded(f"{cfg}-sampled/p{policy}", db, idx, SEED, "random")


def test_c4_sampled_full_size():
    _sampled("C4", 10)


@pytest.mark.parametrize("policy", [0, 1])
def test_c5_sampled_full_size(policy):
    _sampled("C5", 60, policy)


def test_device_plan_export_matches_oracle():
    for cfg, tab in (("C2", pr.B200_F32), ("C3", pr.B200_TC), ("C4", pr.B200_TC)):
        M, N, K = vbinputs.config_sizes(cfg)
        dtype = vbinputs.CONFIGS[cfg]["dtype"]
        for pol in (0, 1):
            db = DeviceBatch(M, N, K, dtype)
            ex = db.plan(pol).export()        # decoded from the DEVICE copy
            ref = pr.plan(M, N, K, tab, pol).enc
            assert list(ex["block_ptr"]) == ref.Tile and list(ex["tile_gemm"]) == ref.GEMM
            assert list(ex["tile_y"]) == ref.Y and list(ex["tile_x"]) == ref.X
            assert list(ex["gemm_strategy"]) == ref.Tiling


@pytest.mark.parametrize("dtype", ["f32", "bf16"])
def test_bitwise_deterministic_and_reexecutable(dtype):
    M, N, K = vbinputs.config_sizes("C2")
    M, N, K = M[:64], N[:64], K[:64]
    db = DeviceBatch(M, N, K, dtype)
    db.fill(SEED)
    plan = db.plan()
    c0 = db.C.clone()
    db.run(plan)
    r1 = db.C.clone()
    db.C.copy_(c0)
    db.run(plan)
    torch.cuda.synchronize()
    assert torch.equal(r1.view(torch.uint8), db.C.view(torch.uint8))      # no split-K: bitwise reproducible
    # re-execute the same plan on its own output: C <- a*AB + b*C1 (exec is stream-ordered, stateless)
    c1 = [to_f64(db.c(g)).copy() for g in range(len(M))]
    db.run(plan)
    torch.cuda.synchronize()
    # beta close to -1 makes C2 = (1+beta)*alpha*AB + beta^2*C0 cancel, so the normwise
    # measure is not meaningful here; check the elementwise forward-error bound instead
    check_bound(db, range(len(M)), SEED, "random", c_old=c1)


@pytest.mark.parametrize("dtype", ["f32", "bf16"])
def test_bind_then_exec_bound_repeatedly(dtype):
    # exec_bound launches only the GEMM kernel; the kernel resets its own work counter, so
    # back-to-back launches must each process the whole batch
    M, N, K = vbinputs.config_sizes("C2")
    M, N, K = M[:48], N[:48], K[:48]
    db = DeviceBatch(M, N, K, dtype)
    db.fill(SEED)
    plan = db.plan()
    db.bind(plan)
    c_prev = None
    for it in range(3):
        c_prev = [to_f64(db.c(g)).copy() for g in range(len(M))]
        db.run_bound(plan)
        torch.cuda.synchronize()
        check_bound(db, range(len(M)), SEED, "random", c_old=c_prev)
    with pytest.raises(vb.VbError):
        db.plan().exec_bound(db.alpha.data_ptr(), db.beta.data_ptr(), 0)   # never bound


@pytest.mark.parametrize("dtype", ["bf16", "f16", "f32"])
def test_rebind_alternating_buffers_never_uses_stale_descriptors(dtype):
    # one plan, two batches with identical shapes in different arenas; re-bind back and forth
    # (tensor maps are patched in place by the prep kernel) and check every result
    M, N, K = vbinputs.config_sizes("C2")
    M, N, K = M[:40], N[:40], K[:40]
    dbs = [DeviceBatch(M, N, K, dtype), DeviceBatch(M, N, K, dtype)]
    seeds = [11, 12]
    for db, sd in zip(dbs, seeds):
        db.fill(sd)
    plan = dbs[0].plan()
    c0 = [db.C.clone() for db in dbs]
    for rnd in range(4):
        i = rnd % 2
        db = dbs[i]
        db.C.copy_(c0[i])
        db.run(plan)                   # bind (patch maps) + GEMM kernel
        torch.cuda.synchronize()
        check_batch(db, range(len(M)), seeds[i], "random")


@pytest.mark.parametrize("dtype", ["bf16", "f16"])
def test_pair_tiles_selected_for_compute_bound_batch(dtype):
    # arithmetic intensity ~200 flop/B >= 128: the tiler offers the 2-SM pair strategies (C-7b);
    # shapes include row/column/K tails and a GEMM too short for a pair tile
    M = np.array([512, 300, 777, 1024, 100, 256]); N = np.array([512, 260, 640, 1000, 96, 512])
    K = np.array([2048, 1500, 1900, 4096, 3000, 2000])
    db = DeviceBatch(M, N, K, dtype)
    db.C.fill_(float("nan"))
    db.fill(SEED)
    plan = db.plan(tlp_threshold=1)        # small batch: let the tiler reach the largest tiles
    ids = plan.export()["gemm_strategy"]
    assert (ids >= 8).sum() >= 4 and plan.info()["launches_per_exec"] == 3, (ids, plan.info())
    db.run(plan)
    torch.cuda.synchronize()
    check_batch(db, range(len(M)), SEED, "random")
    _padding_untouched(db)


@pytest.mark.parametrize("dtype", ["bf16", "f16"])
def test_w2_tiles_forced(dtype):
    """W2 (256 x 512 pair tile: two N <= 256 MMAs per K step into 512 TMEM columns) forced on
    every GEMM: N tails inside the first half (N - n0 <= 256: one MMA), inside the second half
    (the pair splits each half evenly, CTA 1's share of half 1 possibly empty), row tails on
    either CTA, K tails and K = 0, beta != 0; alternating with H2 so that 512-column and
    256-column accumulators share the TMEM ring."""
    N = np.array([512, 300, 260, 289, 511, 513, 700, 1000, 1024, 257, 33, 640, 768, 520])
    M = np.array([256, 300, 129, 512, 255, 100, 384, 777, 1024, 256, 256, 130, 17, 600])
    K = np.array([64, 100, 4096, 0, 1000, 63, 1500, 17, 2048, 640, 128, 300, 700, 1])
    db = DeviceBatch(M, N, K, dtype)
    db.C.fill_(float("nan"))
    db.fill(SEED)
    rows = [15 if g % 3 else 10 for g in range(len(M))]
    db.run(_forced_rows_plan(db, rows, pr.B200_TC, 3))
    torch.cuda.synchronize()
    check_batch(db, range(len(M)), SEED, "random")
    check_bound(db, range(len(M)), SEED, "random")
    _padding_untouched(db)


def test_pair_kernel_repeated_and_graph_replays():
    """The pair kernel's cross-CTA protocol (mirrored tile ring, the peer's release forwarder,
    relaxed accumulator releases, just-in-time claims) over repeated launches of one bound plan
    and CUDA-graph replays: W2 + H2 + 1-SM tiles, beta != 0, every result checked."""
    M = np.array([512, 300, 777, 1024, 100, 256, 640]); N = np.array([512, 260, 640, 1000, 96, 512, 700])
    K = np.array([2048, 1500, 1900, 4096, 3000, 2000, 33])
    db = DeviceBatch(M, N, K, "bf16")
    db.fill(SEED)
    c0 = db.C.clone()
    plan = db.plan(tlp_threshold=1)
    assert plan.info()["launches_per_exec"] == 3
    db.bind(plan)
    for _ in range(3):
        db.C.copy_(c0)
        db.run_bound(plan)
        torch.cuda.synchronize()
        check_batch(db, range(len(M)), SEED, "random")
    s = torch.cuda.Stream()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.stream(s):
        db.run_bound(plan, s)
        torch.cuda.synchronize()
        with torch.cuda.graph(g, stream=s):
            db.run_bound(plan, s)
    for _ in range(3):
        db.C.copy_(c0)
        torch.cuda.synchronize()
        g.replay()
        torch.cuda.synchronize()
        check_batch(db, range(len(M)), SEED, "random")


# ------------------------------------------------------------------ policy selection (P272-274)
@pytest.mark.parametrize("dtype", ["bf16", "f32"])
def test_auto_policy_parity(dtype):
    """VB_BATCH_AUTO (random-forest choice) runs the chosen heuristic and stays exact."""
    rng = np.random.default_rng(3)
    M, N, K = (rng.integers(1, 300, 40) for _ in range(3))
    db, plan = _run(M, N, K, dtype, vb.VB_BATCH_AUTO)
    assert plan.policy() in (vb.VB_BATCH_THRESHOLD, vb.VB_BATCH_BINARY)
    check_batch(db, range(db.batch), SEED, "random")
    _padding_untouched(db)


@pytest.mark.parametrize("dtype", ["bf16", "f32"])
def test_plan_tune_keeps_faster_and_is_exact(dtype):
    """vb_plan_tune (P272: try both heuristics on a fixed batch, keep the better one)."""
    rng = np.random.default_rng(4)
    M, N, K = (rng.integers(16, 400, 64) for _ in range(3))
    db = DeviceBatch(M, N, K, dtype)
    db.fill(SEED, "random")
    plan, ms = db.plan_tune(reps=3)
    assert ms[0] > 0 and ms[1] > 0
    assert plan.policy() == (vb.VB_BATCH_BINARY if ms[1] < ms[0] else vb.VB_BATCH_THRESHOLD)
    db.fill(SEED, "random")          # tuning used C as scratch: restore C_old, then run the kept plan
    db.run(plan)
    torch.cuda.synchronize()
    check_batch(db, range(db.batch), SEED, "random")


@pytest.mark.parametrize("dtype", ["bf16", "f32"])
def test_cuda_graph_replays_of_exec_bound(dtype):
    # vb_exec_bound captured alone in a CUDA graph: every replay must claim all work lists again
    # (the kernels reset their work-list counter themselves), and give the same exact result
    M, N, K = vbinputs.config_sizes("C2")
    M, N, K = M[:48], N[:48], K[:48]
    db = DeviceBatch(M, N, K, dtype)
    db.fill(SEED)
    plan = db.plan()
    c0 = db.C.clone()
    db.bind(plan)
    torch.cuda.synchronize()
    s = torch.cuda.Stream()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.stream(s):
        db.run_bound(plan, s)                 # warm-up outside the capture
        torch.cuda.synchronize()
        db.C.copy_(c0)
        torch.cuda.synchronize()
        with torch.cuda.graph(g, stream=s):
            db.run_bound(plan, s)
    torch.cuda.synchronize()
    first = None
    for rep in range(4):
        db.C.copy_(c0)
        torch.cuda.synchronize()
        g.replay()
        torch.cuda.synchronize()
        got = [db.c(g).clone() for g in range(len(M))]   # the matrices (arena padding is undefined)
        if first is None:
            first = got
            check_batch(db, range(len(M)), SEED, "random")
        else:
            assert all(torch.equal(a, b) for a, b in zip(first, got)), f"replay {rep} differs"


@pytest.mark.parametrize("dtype", ["bf16", "f16", "f32"])
@pytest.mark.parametrize("policy", [0, 1])
def test_random_ragged_shapes(dtype, policy):
    # 160 GEMMs with M, N, K drawn from [1, 600] (every size class: 1-wide, sub-tile, ragged
    # multi-tile, K tails), C pre-filled with NaN outside the matrices: every GEMM within the
    # tolerance and the padding of C never written
    rng = np.random.default_rng(1234 + policy)
    r = rng.integers(1, 601, (160, 3))
    r[:10, 0] = 1
    r[10:20, 1] = 1
    r[20:30, 2] = 1
    db, _ = _run(r[:, 0], r[:, 1], r[:, 2], dtype, policy=policy, seed=5)
    check_recorded(f"ragged160/{dtype}/p{policy}", db, range(db.batch), 5, "random")
    _padding_untouched(db)


@pytest.mark.parametrize("cfg", ["C4", "ragged"])
def test_device_built_tensor_maps_equal_host_encoded(cfg, monkeypatch):
    """Plan-time tensor maps built on the device (templates + tensormap.replace of the global
    dims and stride) are bit-identical to cuTensorMapEncodeTiled's maps for every GEMM and map,
    once both plans are bound to the same buffers (the bind patches the address)."""
    if cfg == "C4":
        M, N, K = vbinputs.config_sizes("C4")
    else:
        r = np.random.default_rng(21).integers(1, 700, (300, 3))
        r[:20, 2] = 0
        r[20:40, 1] = np.random.default_rng(2).integers(1, 8, 20)
        # tensors spanning just below / exactly / above 128 KiB (rows x row stride), with and
        # without row padding: the encoder's size class
        edge = np.array([[1024, 40, 64], [1023, 40, 64], [1024, 40, 63], [1025, 40, 63], [40, 64, 1024],
                         [40, 64, 1023], [40, 63, 1024], [1024, 64, 40], [1023, 64, 40], [1024, 57, 40]])
        r = np.concatenate([r, edge])
        M, N, K = r[:, 0], r[:, 1], r[:, 2]
    db = DeviceBatch(M, N, K, "bf16")
    db.fill(SEED)
    dev_plan = db.plan()
    monkeypatch.setenv("VB_TMAPS_HOST", "1")
    host_plan = db.plan()
    monkeypatch.delenv("VB_TMAPS_HOST")
    for p in (dev_plan, host_plan):
        db.bind(p)
    torch.cuda.synchronize()
    a, b = dev_plan.debug_tmaps(), host_plan.debug_tmaps()
    assert a.shape == b.shape and a.shape[0] == len(M)
    bad = np.nonzero((a != b).any(axis=2))
    assert bad[0].size == 0, f"{bad[0].size} maps differ, first GEMM {bad[0][:5]} map {bad[1][:5]}"
    db.run(dev_plan)
    torch.cuda.synchronize()
    check_batch(db, range(0, len(M), max(1, len(M) // 60)), SEED, "random")


@pytest.mark.parametrize("dtype", ["bf16", "f16"])
@pytest.mark.parametrize("ab", ["random", "conv"])
def test_swap_ab_tiles_small_m(dtype, ab):
    """Swap-AB strategies (S16..S64: C^T = B^T A^T, NEXT-2) forced on small-M GEMMs with N and K
    tails, K = 0, 1-wide shapes; beta = 0 runs on NaN-poisoned C (C must not be read); elementwise
    bound and C padding untouched."""
    rng = np.random.default_rng(8)
    n = 64
    M = rng.integers(1, 65, n); N = rng.integers(1, 700, n); K = rng.integers(0, 900, n)
    M[:4] = [1, 16, 64, 17]; N[:4] = [1, 7, 129, 256]; K[4:8] = 0
    db = DeviceBatch(M, N, K, dtype)
    db.C.fill_(float("nan"))
    db.fill(SEED, ab)
    if ab == "conv":
        db.C.fill_(float("nan"))           # beta = 0: C_old must never be read
    table = pr.B200_TC
    row = {s.name: i for i, s in enumerate(table.rows)}
    rows = [row[f"S{min(64, (int(m) + 15) // 16 * 16)}"] for m in M]
    db.run(_forced_rows_plan(db, rows, table, 3))
    torch.cuda.synchronize()
    c_old = [np.zeros((int(m), int(k))) for m, k in zip(M, N)] if ab == "conv" else None
    check_recorded(f"swapAB/{dtype}/{ab}", db, range(n), SEED, ab, c_old=c_old)
    _padding_untouched(db)


def test_replanning_loop_reuses_workspaces_and_stays_exact():
    """The paper's on-line case (P272): sizes vary per call and every call plans again.  Forty
    plans of varying batches (bf16 and fp32) are built, executed and destroyed in turn (the
    workspaces cycle through the per-device pool); every result is checked."""
    rng = np.random.default_rng(31)
    for it in range(40):
        dtype = "bf16" if it % 3 else "f32"
        n = int(rng.integers(1, 40))
        M, N, K = (rng.integers(1, 400, n) for _ in range(3))
        db = DeviceBatch(M, N, K, dtype)
        db.C.fill_(float("nan"))
        db.fill(it)
        plan = db.plan(vb.VB_BATCH_AUTO)
        db.run(plan)
        torch.cuda.synchronize()
        check_batch(db, range(n), it, "random")
        _padding_untouched(db)
        del plan, db
