"""GPU parity of the implicit-GEMM convolution path (vb_plan_conv)
against the fp64 convolution oracle (oracle/conv_ref.py), on inputs regenerated on the host
by vbinputs.  Tolerance: the bf16/fp16 normwise 2e-2 of BASELINE.json's north_star."""
import numpy as np
import pytest
import torch

import vbinputs
from oracle import conv_ref as cr
from oracle.checks import TOL, normwise_error

pytestmark = pytest.mark.gpu

if torch.cuda.is_available():
    from paper_conf_ppopp_li0yjl19_b200.batch import ConvBatch
    import paper_conf_ppopp_li0yjl19_b200 as vb

SEED = 0


def _to_f64(t):
    return t.detach().to("cpu", torch.float64).numpy()


def check_convs(db, idx, seed, ab_mode):
    al, be = vbinputs.alpha_beta(seed, db.gemm_ids[list(idx)], ab_mode)
    worst = 0.0
    for t, g in enumerate(idx):
        c = db.convs[g]
        gid = int(db.gemm_ids[g])
        x = vbinputs.matrix(seed, gid, vbinputs.OP_A, int(db.P[g]), c["Cin"], db.dtype)[1]
        wt = vbinputs.matrix(seed, gid, vbinputs.OP_B, int(db.K[g]), c["Cout"], db.dtype)[1]
        c_old = vbinputs.matrix(seed, gid, vbinputs.OP_C, int(db.M[g]), c["Cout"], db.dtype)[1]
        ref = cr.conv_gemm(x.reshape(c["nb"], c["H"], c["W"], c["Cin"]),
                           wt.reshape(c["KH"], c["KW"], c["Cin"], c["Cout"]), c_old, float(al[t]), float(be[t]),
                           c["pad"])
        got = _to_f64(db.c(g))
        err = normwise_error(got, ref)
        worst = max(worst, err)
        assert err <= TOL[db.dtype], f"conv {g} {c}: normwise error {err:.3e}"
    return worst


def _run(convs, dtype="bf16", ab="conv", policy=0, seed=SEED):
    db = ConvBatch(convs, dtype)
    db.C.fill_(float("nan"))
    db.fill(seed, ab)
    plan = db.plan(policy)
    db.run(plan)
    torch.cuda.synchronize()
    return db, plan


@pytest.mark.parametrize("dtype", ["bf16", "f16"])
def test_googlenet_inception_convs_nb1(dtype):
    convs = vbinputs.googlenet_convs(nb=1)
    db, _ = _run(convs, dtype)
    check_convs(db, range(db.batch), SEED, "conv")


def test_googlenet_inception_3a_nb4_both_policies():
    convs = vbinputs.googlenet_convs(nb=4, module="3a")
    for pol in (0, 1):
        db, _ = _run(convs, "bf16", policy=pol)
        check_convs(db, range(db.batch), SEED, "conv")


@pytest.mark.parametrize("conv", [
    dict(nb=2, H=9, W=7, Cin=8, Cout=24, KH=3, KW=3, pad=1),      # tiny channel count, ragged tiles
    dict(nb=1, H=5, W=6, Cin=72, Cout=40, KH=3, KW=3, pad=0),     # valid conv, Cin % 64 != 0
    dict(nb=3, H=4, W=4, Cin=136, Cout=8, KH=5, KW=5, pad=2),     # 5x5 wider than the image
    dict(nb=1, H=1, W=1, Cin=16, Cout=16, KH=3, KW=3, pad=1),     # single pixel
    dict(nb=2, H=11, W=13, Cin=64, Cout=300, KH=1, KW=1, pad=0),  # 1x1, N tail
    dict(nb=1, H=30, W=30, Cin=32, Cout=136, KH=7, KW=7, pad=3),  # 7x7, many taps
])
def test_edge_convolutions_random_alpha_beta(conv):
    db, _ = _run([conv], "bf16", ab="random", seed=3)
    check_convs(db, [0], 3, "random")


def test_plan_shape_is_the_gemm_view():
    convs = vbinputs.googlenet_convs(nb=2, module="4a")
    plan = vb.plan_conv([dict(c, ldb=c["Cout"], ldc=c["Cout"]) for c in convs], "bf16")
    inf = plan.info()
    db = ConvBatch(convs, "bf16")
    assert inf["n_tiles"] >= db.batch
    assert list(db.M) == [2 * 14 * 14] * len(convs)


def test_invalid_descriptors_rejected():
    good = dict(nb=1, H=8, W=8, Cin=16, Cout=16, KH=3, KW=3, pad=1, ldb=16, ldc=16)
    for bad in (dict(good, Cin=12), dict(good, KW=5), dict(good, pad=3), dict(good, ldc=8), dict(good, KH=9, KW=9)):
        with pytest.raises(vb.VbError):
            vb.plan_conv([bad], "bf16")
    with pytest.raises(vb.VbError):
        vb.plan_conv([good], "f32")


def test_googlenet_nb32_sampled_convs():
    # the bench's C3i size at nb = 32 (every branch, 25 088 output pixels per conv); the oracle
    # checks a sample of the convolutions (largest K, a 5x5, a 1x1, the first and the last)
    convs = vbinputs.googlenet_convs(nb=32)
    db, _ = _run(convs, "bf16")
    ks = [c["KH"] * c["KW"] * c["Cin"] for c in convs]
    pick = sorted({0, len(convs) - 1, int(np.argmax(ks)),
                   next(i for i, c in enumerate(convs) if c["KH"] == 5),
                   next(i for i, c in enumerate(convs) if c["KH"] == 1 and c["Cin"] > 500)})
    check_convs(db, pick, SEED, "conv")
