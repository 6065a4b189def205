"""CPU tests of the C-ABI library: symbol exports, validation, and bit-exact parity of the
C++ planner (host-only plans, device = -1) with the reference planner in oracle/plan_ref.py.
No compute call is made here (no GPU)."""
import ctypes
import subprocess

import numpy as np
import pytest
from hypothesis import given, settings, strategies as st

import vbinputs
from oracle import plan_ref as pr
import paper_conf_ppopp_li0yjl19_b200 as vb
from paper_conf_ppopp_li0yjl19_b200 import _native as nv

TABLES = {1: pr.V100, 2: pr.B200_F32, 3: pr.B200_TC}


def test_library_exports_every_header_symbol():
    syms = nv.header_symbols()
    assert len(syms) >= 14
    out = subprocess.check_output(["nm", "-D", "--defined-only", nv.LIB_PATH]).decode()
    exported = {line.split()[-1] for line in out.splitlines() if line.strip()}
    missing = [s for s in syms if s not in exported]
    assert not missing, missing
    for s in syms:
        getattr(nv.lib, s)   # resolvable through ctypes
    assert "sm_100a" in vb.version()


def _host_plan(M, N, K, dtype, policy, table_id, thr=0, theta=0):
    ld = lambda c: vbinputs.padded_ld(c, dtype)  # noqa: E731
    return nv.plan_vbatched(M, N, K, ld(K), ld(N), ld(N), dtype, policy, device=-1, table_id=table_id,
                            tlp_threshold=thr, theta=theta)


def _assert_same(plan, ref: pr.Plan):
    ex = plan.export()
    enc = ref.enc
    assert list(ex["block_ptr"]) == enc.Tile
    assert list(ex["tile_gemm"]) == enc.GEMM
    assert list(ex["tile_y"]) == enc.Y
    assert list(ex["tile_x"]) == enc.X
    assert list(ex["gemm_strategy"]) == enc.Tiling
    assert ex["version_T"] == ref.tiling.T
    assert plan.tiler_trace() == [(t, T) for (_, T, t) in ref.tiling.trace]


def test_w3_trace_through_the_abi(golden):
    w = golden["W3_tiler"]
    M, N, K = (np.array(c) for c in zip(*w["gemms_MNK"]))
    p = _host_plan(M, N, K, "f32", vb.VB_BATCH_THRESHOLD, vb.VB_TABLE_V100)
    assert [t for t, _ in p.tiler_trace()] == [r["TLP"] for r in w["rounds"]]
    names = [pr.V100.rows[s % 6].name for s in p.export()["gemm_strategy"]]
    assert names == w["final"]


def test_w4_schedule_roundtrip(golden):
    M, N, K = [256, 256], [128, 256], [64, 64]
    p = nv.plan_from_schedule(M, N, K, [64, 64], [128, 256], [128, 256], gemm_row=[5, 3], version_T=256,
                              block_ptr=[0, 1, 2, 4, 6, 8, 10], tile_gemm=[0, 0, 1, 1, 1, 1, 1, 1, 1, 1],
                              tile_y=[0, 1, 0, 0, 0, 0, 1, 1, 1, 1], tile_x=[0, 0, 0, 1, 2, 3, 0, 1, 2, 3],
                              dtype="f32", device=-1, table_id=vb.VB_TABLE_V100)
    ex = p.export()
    assert list(ex["block_ptr"]) == [0, 1, 2, 4, 6, 8, 10]
    assert list(ex["tile_gemm"][2:4]) == [1, 1] and [(0, 0), (0, 1)] == list(zip(ex["tile_y"][2:4], ex["tile_x"][2:4]))


def test_schedule_validation_rejects_double_cover_and_gaps():
    base = dict(M=[64], N=[64], K=[8], lda=[8], ldb=[64], ldc=[64], gemm_row=[2], version_T=256, dtype="f32",
                device=-1, table_id=vb.VB_TABLE_V100)
    with pytest.raises(vb.VbError):   # tile covered twice
        nv.plan_from_schedule(block_ptr=[0, 2], tile_gemm=[0, 0], tile_y=[0, 0], tile_x=[0, 0], **base)
    with pytest.raises(vb.VbError):   # tile missing
        nv.plan_from_schedule(block_ptr=[0, 0], tile_gemm=[], tile_y=[], tile_x=[], **base)
    with pytest.raises(vb.VbError):   # outside the GEMM
        nv.plan_from_schedule(block_ptr=[0, 1], tile_gemm=[0], tile_y=[1], tile_x=[0], **base)


def test_schedule_pair_blocks_with_empty_blocks():
    """an empty block before the pair blocks must not shift the pair/1-SM split.
    GEMM 0 runs H2 (row 10, 2-SM pair tile), GEMM 1 runs h (row 7, 1-SM)."""
    base = dict(M=[256, 128], N=[256, 256], K=[64, 64], lda=[64, 64], ldb=[256, 256], ldc=[256, 256],
                gemm_row=[10, 7], version_T=256, dtype="bf16", device=-1, table_id=vb.VB_TABLE_B200_TC)
    one = dict(M=[256], N=[256], K=[64], lda=[64], ldb=[256], ldc=[256], gemm_row=[10], version_T=256,
               dtype="bf16", device=-1, table_id=vb.VB_TABLE_B200_TC)
    # [empty, pair]: one pair launch only (prep + pair kernel)
    p = nv.plan_from_schedule(block_ptr=[0, 0, 1], tile_gemm=[0], tile_y=[0], tile_x=[0], **one)
    assert p.info()["launches_per_exec"] == 2
    # [empty, pair, single, empty]: prep + pair + 1-SM
    p = nv.plan_from_schedule(block_ptr=[0, 0, 1, 2, 2], tile_gemm=[0, 1], tile_y=[0, 0], tile_x=[0, 0], **base)
    assert p.info()["launches_per_exec"] == 3
    with pytest.raises(vb.VbError):   # a 1-SM block before a pair block
        nv.plan_from_schedule(block_ptr=[0, 1, 1, 2], tile_gemm=[1, 0], tile_y=[0, 0], tile_x=[0, 0], **base)
    with pytest.raises(vb.VbError):   # a block mixing the two versions
        nv.plan_from_schedule(block_ptr=[0, 2], tile_gemm=[0, 1], tile_y=[0, 0], tile_x=[0, 0], **base)


def test_fill_rejects_unknown_dtype():
    st = nv.lib.vb_fill_uniform_batch(7, 0, None, None, None, None, None, 0, 0, 0, None)
    assert st == vb.VB_ERR_INVALID_ARG


def test_int32_range_checked_before_the_abi():
    with pytest.raises(ValueError):
        nv.plan_vbatched([8], [8], [2**32 + 16], [8], [8], [8], "bf16", device=-1)


def test_validation_errors():
    with pytest.raises(vb.VbError) as e:
        nv.plan_vbatched([8], [8], [8], [9], [8], [8], "bf16", device=-1)   # lda*2 not a 16-B multiple
    assert e.value.status == vb.VB_ERR_ALIGNMENT
    with pytest.raises(vb.VbError) as e:
        nv.plan_vbatched([8], [8], [-1], [8], [8], [8], "bf16", device=-1)
    assert e.value.status == vb.VB_ERR_INVALID_ARG
    with pytest.raises(vb.VbError) as e:
        nv.plan_vbatched([8], [16], [8], [8], [8], [16], "bf16", device=-1)  # ldb < N
    assert e.value.status == vb.VB_ERR_INVALID_ARG
    p = nv.plan_vbatched([8], [8], [8], [8], [8], [8], "bf16", device=-1)
    with pytest.raises(vb.VbError) as e:
        p.exec(0, 0, 0, 0, 0, 0)
    assert e.value.status == vb.VB_ERR_UNSUPPORTED
    empty = nv.plan_vbatched([], [], [], [], [], [], "bf16", device=-1)
    assert empty.info()["n_tiles"] == 0 and empty.info()["n_blocks"] == 0


@pytest.mark.parametrize("cfg", ["C1", "C2", "C3", "C4"])
@pytest.mark.parametrize("policy", [0, 1, 2])
def test_config_plans_match_oracle(cfg, policy):
    M, N, K = vbinputs.config_sizes(cfg)
    dtype = vbinputs.CONFIGS[cfg]["dtype"]
    tid = 2 if dtype == "f32" else 3
    p = _host_plan(M, N, K, dtype, policy, tid)
    _assert_same(p, pr.plan(M, N, K, TABLES[tid], policy))


@pytest.mark.slow
@pytest.mark.parametrize("policy", [0, 1])
def test_c5_plan_matches_oracle(policy):
    M, N, K = vbinputs.config_sizes("C5")
    p = _host_plan(M, N, K, "bf16", policy, 3)
    _assert_same(p, pr.plan(M, N, K, pr.B200_TC, policy))


def test_v100_profile_on_googlenet():
    for nb in (1, 3, 8):
        sh = vbinputs.googlenet_shapes(nb, first_stage_only=True)
        M, N, K = (np.array([s[i] for s in sh]) for i in (1, 2, 3))
        for pol in (0, 1):
            _assert_same(_host_plan(M, N, K, "f32", pol, 1), pr.plan(M, N, K, pr.V100, pol))


sizes = st.lists(st.tuples(st.integers(0, 700), st.integers(0, 700), st.integers(0, 900)), min_size=0, max_size=40)


@settings(max_examples=80, deadline=None)
@given(sizes, st.sampled_from([1, 2, 3]), st.sampled_from([0, 1, 2]),
       st.sampled_from([0, 1, 5000, 65536, 600000]), st.sampled_from([1, 100, 256, 512, 3000]))
def test_random_plans_match_oracle(sz, tid, policy, thr, theta):
    M = np.array([s[0] for s in sz], np.int64); N = np.array([s[1] for s in sz], np.int64)
    K = np.array([s[2] for s in sz], np.int64)
    dtype = "f32" if tid != 3 else "bf16"
    p = _host_plan(M, N, K, dtype, policy, tid, thr, theta)
    _assert_same(p, pr.plan(M, N, K, TABLES[tid], policy, thr if thr > 0 else None, theta if theta > 0 else None))


@settings(max_examples=40, deadline=None)
@given(st.lists(st.tuples(st.integers(0, 2000), st.integers(0, 2000), st.integers(0, 2000)), min_size=0,
                max_size=60), st.integers(1, 8))
def test_lpt_matches_oracle(sz, ranks):
    M = [s[0] for s in sz]; N = [s[1] for s in sz]; K = [s[2] for s in sz]
    assert list(nv.shard_lpt(M, N, K, ranks)) == pr.shard_lpt(M, N, K, ranks)


@pytest.mark.parametrize("nb", [1, 4, 32])
@pytest.mark.parametrize("policy", [vb.VB_BATCH_THRESHOLD, vb.VB_BATCH_BINARY])
def test_conv_plan_is_the_oracle_plan_of_its_gemm_view(nb, policy):
    # vb_plan_conv plans the GEMM view M = nb*Hout*Wout, N = Cout, K = KH*KW*Cin with 1-SM strategies
    convs = vbinputs.googlenet_convs(nb=nb)
    descs = [dict(c, ldb=int(vbinputs.padded_ld(c["Cout"], "bf16")), ldc=int(vbinputs.padded_ld(c["Cout"], "bf16")))
             for c in convs]
    plan = nv.plan_conv(descs, "bf16", policy, device=-1)
    M = [c["nb"] * c["H"] * c["W"] for c in convs]
    N = [c["Cout"] for c in convs]
    K = [c["KH"] * c["KW"] * c["Cin"] for c in convs]
    ref = pr.plan(M, N, K, pr.B200_TC, policy, allow_pairs=False)
    _assert_same(plan, ref)
    assert all(pr.B200_TC.rows[r].ctas == 1 for r in ref.tiling.rows)


def test_conv_plan_validation_on_host():
    good = dict(nb=2, H=8, W=8, Cin=16, Cout=24, KH=3, KW=3, pad=1, ldb=24, ldc=32)
    assert nv.plan_conv([good], "bf16", device=-1).info()["n_tiles"] >= 1
    bad_cases = [dict(good, Cin=12), dict(good, KW=5), dict(good, pad=3), dict(good, ldc=16),
                 dict(good, KH=9, KW=9), dict(good, nb=0), dict(good, H=1, W=1, pad=0), dict(good, ldb=20)]
    for bad in bad_cases:
        with pytest.raises(vb.VbError):
            nv.plan_conv([bad], "bf16", device=-1)
    with pytest.raises(vb.VbError):
        nv.plan_conv([good], "f32", device=-1)
    assert nv.plan_conv([], "bf16", device=-1).info()["n_tiles"] == 0


def test_balanced_column_split_c26():
    """Reading C-26 through the product's own function (vb_debug_tile_cols): the column tiles of
    a GEMM cover [0, N) exactly once, in order, every interior boundary 64-column aligned (no TMA
    store box crosses into a neighbour), no tile wider than BX, widths within one chunk of each
    other, and the export decodes each tile's index back from its origin."""
    import ctypes
    f = nv.lib.vb_debug_tile_cols
    f.argtypes = [ctypes.c_int32] * 3 + [ctypes.POINTER(ctypes.c_int32)] * 3
    a, b, xb = ctypes.c_int32(), ctypes.c_int32(), ctypes.c_int32()
    for BX in (32, 64, 128, 256, 512):
        G = min(64, BX)
        for N in list(range(1, 1100, 7)) + [BX, 2 * BX, 3 * BX - 1, 768, 700, 4096, 4097]:
            nx = -(-N // BX)
            prev, widths = 0, []
            for x in range(nx):
                assert f(x, N, BX, ctypes.byref(a), ctypes.byref(b), ctypes.byref(xb)) == vb.VB_OK
                assert a.value == prev and b.value > a.value and b.value - a.value <= BX, (BX, N, x)
                assert a.value % G == 0 and (b.value == N or b.value % G == 0), (BX, N, x)
                assert xb.value == x
                widths.append(b.value - a.value)
                prev = b.value
            assert prev == N
            full = widths[:-1] if N % G else widths
            assert not full or max(full) - min(full) <= G, (BX, N, widths)
    assert f(1, 100, 128, ctypes.byref(a), ctypes.byref(b), ctypes.byref(xb)) == vb.VB_ERR_INVALID_ARG
    assert f(0, 100, 100, ctypes.byref(a), ctypes.byref(b), ctypes.byref(xb)) == vb.VB_ERR_INVALID_ARG
