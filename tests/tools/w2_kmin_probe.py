"""Measurement tool (uses the oracle planner to build schedules, so it lives under tests/tools):
C4 with W2 (256 x 512 pair) tiles only for GEMMs with K >= Kmin, H2 below -- does the W2
epilogue, which cannot overlap the next tile's MMAs (one W2 accumulator fills TMEM), cost more
than W2's operand savings on short-K GEMMs?  Plans are built with the oracle's tiling result,
rows edited, then enumerated and binary-batched per launch exactly like oracle.plan_ref.plan,
and run through vb_plan_from_schedule; timed in interleaved rounds (power drift)."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import vbinputs  # noqa: E402
from oracle import plan_ref as pr  # noqa: E402
from paper_conf_ppopp_li0yjl19_b200 import _native as nv  # noqa: E402
from paper_conf_ppopp_li0yjl19_b200.batch import DeviceBatch  # noqa: E402

TC = pr.B200_TC
W2, H2 = 15, 10
M, N, K = vbinputs.config_sizes("C4")
db = DeviceBatch(M, N, K, "bf16")
db.fill(0)
base = pr.plan(M, N, K, TC, pr.POLICY_BINARY)


def schedule(kmin):
    rows = [H2 if (r == W2 and K[g] < kmin) else r for g, r in enumerate(base.tiling.rows)]
    tiles = pr.enumerate_tiles(M, N, K, rows, TC)
    isp = [TC.rows[rows[t.gemm]].ctas == 2 for t in tiles]
    tiles = [t for t, q in zip(tiles, isp) if q] + [t for t, q in zip(tiles, isp) if not q]
    npair = sum(isp)
    blocks = []
    for lo, hi in ((0, npair), (npair, len(tiles))):
        blocks += [[lo + i for i in b] for b in pr.binary_batching(tiles[lo:hi], TC.theta)]
    order = [i for b in blocks for i in b]
    bp = np.cumsum([0] + [len(b) for b in blocks])
    return nv.plan_from_schedule(db.M, db.N, db.K, db.lda, db.ldb, db.ldc, rows, 256, bp.tolist(),
                                 [tiles[i].gemm for i in order], [tiles[i].y for i in order],
                                 [tiles[i].x for i in order], dtype="bf16", device=0, table_id=3)


kmins = [0, 512, 1024, 2048, 1 << 30]
plans = {k: schedule(k) for k in kmins}
lib = db.plan(nv.VB_BATCH_BINARY)
times = {k: [] for k in ["lib"] + kmins}
for rnd in range(int(os.environ.get("ROUNDS", "8"))):
    for k in ["lib"] + kmins:
        p = lib if k == "lib" else plans[k]
        db.bind(p)
        db.run_bound(p)
        ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(3)]
        for s, e in ev:
            s.record()
            db.run_bound(p)
            e.record()
        torch.cuda.synchronize()
        times[k].append(float(np.median([s.elapsed_time(e) for s, e in ev])))
ref = np.array(times["lib"])
for k, v in times.items():
    print(json.dumps(dict(kmin=str(k), ms_median=round(float(np.median(v)), 4),
                          rel_to_lib=round(float(np.median(np.array(v) / ref)), 4))), flush=True)
