"""Experiment: per-GEMM strategy choice by K on C5 (measurement tool).  Builds schedules with
vb_plan_from_schedule -- every GEMM on the 128x256 row ('h'), or the GEMMs with K <= k_max on
128x128 ('l') so that more short-K accumulators fit in TMEM -- one tile per block, and times
them against the library's own plan."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import vbinputs  # noqa: E402
import paper_conf_ppopp_li0yjl19_b200 as vb  # noqa: E402
from paper_conf_ppopp_li0yjl19_b200 import _native as nv  # noqa: E402
from paper_conf_ppopp_li0yjl19_b200.batch import DeviceBatch  # noqa: E402

ROWS = {"l": (5, 128, 128), "h": (7, 128, 256), "t": (3, 128, 64)}
cfg = sys.argv[1] if len(sys.argv) > 1 else "C5"
M, N, K = (np.asarray(x, np.int64) for x in vbinputs.config_sizes(cfg))
db = DeviceBatch(M, N, K, "bf16")
db.fill(0)


def schedule(kmax, short="l", order="gemm"):
    row = np.where(K <= kmax, ROWS[short][0], ROWS["h"][0])
    by = np.where(K <= kmax, ROWS[short][1], 128)
    bx = np.where(K <= kmax, ROWS[short][2], 256)
    gy, gx = -(-M // by), -(-N // bx)
    cnt = gy * gx
    tg = np.repeat(np.arange(len(M)), cnt)
    start = np.concatenate([[0], np.cumsum(cnt)[:-1]])
    local = np.arange(cnt.sum()) - np.repeat(start, cnt)
    ty, tx = local // np.repeat(gx, cnt), local % np.repeat(gx, cnt)
    if order == "kdesc":   # longest K first
        o = np.argsort(-K[tg], kind="stable")
        tg, ty, tx = tg[o], ty[o], tx[o]
    bp = np.arange(len(tg) + 1)
    return nv.plan_from_schedule(M, N, K, db.lda, db.ldb, db.ldc, row, 256, bp, tg, ty, tx, "bf16"), len(tg)


def timeit(plan):
    db.bind(plan)
    for _ in range(3):
        db.run_bound(plan)
    ts = []
    for _ in range(12):
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s.record()
        db.run_bound(plan)
        e.record()
        ts.append((s, e))
    torch.cuda.synchronize()
    return float(np.median([s.elapsed_time(e) for s, e in ts]))


for rep in range(2):
    p = db.plan(vb.VB_BATCH_AUTO)
    print(json.dumps(dict(case="library plan", ms=round(timeit(p), 4), tiles=p.info()["n_tiles"])), flush=True)
    del p
    for kmax, short in ((0, "l"), (64, "l"), (128, "l"), (256, "l"), (10 ** 9, "l"), (64, "t")):
        p, nt = schedule(kmax, short)
        print(json.dumps(dict(case=f"K<={kmax} -> {short}", ms=round(timeit(p), 4), tiles=nt)), flush=True)
        del p
