"""Small cases for compute-sanitizer (SURVEY.md §4 GPU row, §5): each case runs the CUDA path
through the C-ABI and checks the result against the fp64 oracle, so a sanitizer run also
proves the instrumented kernels still compute the right thing.

    compute-sanitizer --tool memcheck python tests/tools/sanitize_cases.py [case ...]

cases: c1 (C1 fp32, 3 policies), ragged_bf16 / ragged_f32 (48 GEMMs, M, N, K in [1, 600]),
pair (2-SM cta_group::2 tiles incl. W2 + 1-SM tiles, two GEMM launches), w2 (W2 / H2 pair tiles
forced on ragged shapes: both MMA halves, N tails inside either half, K = 0), conv (GoogleNet 3a implicit
GEMM, TMA im2col), graph (vb_exec_bound captured in a CUDA graph, 3 replays).
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))

import numpy as np  # noqa: E402
import torch  # noqa: E402

import vbinputs  # noqa: E402
from gpu_helpers import check_batch  # noqa: E402
from paper_conf_ppopp_li0yjl19_b200.batch import ConvBatch, DeviceBatch  # noqa: E402
import paper_conf_ppopp_li0yjl19_b200 as vb  # noqa: E402

SEED = 0


def _run(M, N, K, dtype, policy=0, thr=0):
    db = DeviceBatch(M, N, K, dtype)
    db.C.fill_(float("nan"))
    db.fill(SEED)
    plan = db.plan(policy, tlp_threshold=thr)
    db.run(plan)
    torch.cuda.synchronize()
    check_batch(db, range(db.batch), SEED, "random")
    return plan


def case_c1():
    M, N, K = vbinputs.config_sizes("C1")
    for pol in (0, 1, 2):
        _run(M, N, K, "f32", pol)


def _ragged(dtype):
    r = np.random.default_rng(99).integers(1, 601, (48, 3))
    r[:4, 0] = 1
    r[4:8, 1] = 1
    r[8:12, 2] = 1
    for pol in (0, 1):
        _run(r[:, 0], r[:, 1], r[:, 2], dtype, pol)


def case_ragged_bf16():
    _ragged("bf16")


def case_ragged_f32():
    _ragged("f32")


def case_pair():
    M = np.array([512, 300, 777, 100, 256]); N = np.array([512, 260, 640, 96, 512])
    K = np.array([1024, 700, 900, 1000, 600])
    plan = _run(M, N, K, "bf16", 0, thr=1)
    assert plan.info()["launches_per_exec"] == 3, plan.info()


def case_w2():
    from oracle import plan_ref as pr
    N = np.array([512, 300, 260, 289, 511, 700, 1000, 257, 640, 768])
    M = np.array([256, 300, 129, 512, 255, 384, 777, 256, 130, 17])
    K = np.array([64, 100, 700, 0, 300, 150, 17, 640, 300, 1])
    db = DeviceBatch(M, N, K, "bf16")
    db.C.fill_(float("nan"))
    db.fill(SEED)
    rows = [15 if g % 3 else 10 for g in range(len(M))]
    tiles = pr.enumerate_tiles(db.M, db.N, db.K, rows, pr.B200_TC)
    plan = vb.plan_from_schedule(db.M, db.N, db.K, db.lda, db.ldb, db.ldc, rows, 256, list(range(len(tiles) + 1)),
                                 [t.gemm for t in tiles], [t.y for t in tiles], [t.x for t in tiles], dtype="bf16",
                                 device=0, table_id=3)
    db.run(plan)
    torch.cuda.synchronize()
    check_batch(db, range(db.batch), SEED, "random")


def case_conv():
    sys.path.insert(0, os.path.join(ROOT, "tests"))
    from test_gpu_conv import check_convs
    convs = vbinputs.googlenet_convs(nb=1, module="3a")
    db = ConvBatch(convs, "bf16")
    db.C.fill_(float("nan"))
    db.fill(SEED, "conv")
    db.run(db.plan(0))
    torch.cuda.synchronize()
    check_convs(db, range(db.batch), SEED, "conv")


def case_graph():
    for dtype in ("bf16", "f32"):
        M, N, K = (c[:24] for c in vbinputs.config_sizes("C2"))
        db = DeviceBatch(M, N, K, dtype)
        db.fill(SEED)
        plan = db.plan()
        c0 = db.C.clone()
        db.bind(plan)
        s = torch.cuda.Stream()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.stream(s):
            db.run_bound(plan, s)
            torch.cuda.synchronize()
            with torch.cuda.graph(g, stream=s):
                db.run_bound(plan, s)
        torch.cuda.synchronize()
        for _ in range(3):
            db.C.copy_(c0)
            torch.cuda.synchronize()
            g.replay()
            torch.cuda.synchronize()
            check_batch(db, range(db.batch), SEED, "random")


CASES = {k[5:]: v for k, v in globals().items() if k.startswith("case_")}

if __name__ == "__main__":
    names = sys.argv[1:] or list(CASES)
    for n in names:
        CASES[n]()
        print(f"case {n}: parity ok", flush=True)
