"""Context measurement (not product code): the tcgen05 kernel against cuBLAS on the same
batches, in the power-capped steady state.

cuBLAS here is a comparison library only (SURVEY.md §2 OUT as a system): uniform batches go
through torch.bmm (one strided-batched cuBLAS call), variable-size batches through one
torch.mm per GEMM captured in a CUDA graph (no launch overhead from Python).  The cuBLAS arm
computes C = A*B into a separate buffer (beta = 0, no C_old read), which favours it slightly.

Each arm runs STEPS back-to-back launches with CUDA events around each; we report the median
of the first 5 (burst clocks) and of the last half (steady state under the 1000 W cap).
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import vbinputs  # noqa: E402
from paper_conf_ppopp_li0yjl19_b200 import POLICIES  # noqa: E402
from paper_conf_ppopp_li0yjl19_b200.batch import DeviceBatch  # noqa: E402

STEPS = int(os.environ.get("STEPS", "60"))


def timed(fn, steps=STEPS):
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(steps)]
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    for s, e in ev:
        s.record()
        fn()
        e.record()
    torch.cuda.synchronize()
    t = np.array([s.elapsed_time(e) for s, e in ev])
    return float(np.median(t[:5])), float(np.median(t[steps // 2:]))


def ours(db, policy):
    plan = db.plan(POLICIES[policy])
    db.bind(plan)
    burst, steady = timed(lambda: db.run_bound(plan))
    info = plan.info()
    info["policy"] = plan.policy()
    return burst, steady, info


def cublas_uniform(db):
    b, m, n, k = db.batch, int(db.M[0]), int(db.N[0]), int(db.K[0])
    A = torch.stack([db.a(g) for g in range(b)])
    B = torch.stack([db.b(g) for g in range(b)])
    C = torch.empty(b, m, n, dtype=A.dtype, device=A.device)
    return timed(lambda: torch.bmm(A, B, out=C))


def cublas_graph(db):
    outs = [torch.empty(int(db.M[g]), int(db.N[g]), dtype=db.A.dtype, device=db.device) for g in range(db.batch)]
    views = [(db.a(g), db.b(g)) for g in range(db.batch)]
    s = torch.cuda.Stream()
    s.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(s):
        for (a, b), o in zip(views, outs):      # warm cuBLAS heuristics / workspaces
            torch.mm(a, b, out=o)
    torch.cuda.current_stream().wait_stream(s)
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        for (a, b), o in zip(views, outs):
            torch.mm(a, b, out=o)
    return timed(g.replay)


def main():
    cases = [("uniform 64x1024x1024x4096", np.full(64, 1024), np.full(64, 1024), np.full(64, 4096), "auto"),
             ("uniform 16x2048x2048x4096", np.full(16, 2048), np.full(16, 2048), np.full(16, 4096), "auto"),
             ("uniform 256x512x512x2048", np.full(256, 512), np.full(256, 512), np.full(256, 2048), "auto")]
    M, N, K = vbinputs.config_sizes("C4")
    cases.append(("C4", M, N, K, "auto"))
    for name, M, N, K, pol in cases:
        db = DeviceBatch(M, N, K, "bf16")
        db.fill(0, "random")
        flops = db.flops()
        res = dict(case=name, gflop=round(flops / 1e9, 1))
        b, st, info = ours(db, pol)
        res["ours_ms_burst"], res["ours_ms_steady"] = round(b, 4), round(st, 4)
        res["ours_tflops_steady"] = round(flops / st / 1e9, 1)
        res["policy"] = info.get("policy")
        uniform = len(set(M.tolist())) == 1 and len(set(N.tolist())) == 1 and len(set(K.tolist())) == 1
        b2, st2 = cublas_uniform(db) if uniform else cublas_graph(db)
        res["cublas"] = "torch.bmm" if uniform else "torch.mm per GEMM in a CUDA graph"
        res["cublas_ms_burst"], res["cublas_ms_steady"] = round(b2, 4), round(st2, 4)
        res["cublas_tflops_steady"] = round(flops / st2 / 1e9, 1)
        print(json.dumps(res), flush=True)
        del db
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
