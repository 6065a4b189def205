"""Swap-AB tiles (S16..S64) against the 128x256 tile for the GEMMs with M <= 64 of a batch,
through forced schedules (vb_plan_from_schedule, one tile per block, enumeration order).

    python tests/tools/swap_probe.py [C5|C3|small]
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))), "tests"))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import vbinputs  # noqa: E402
from oracle import plan_ref as pr  # noqa: E402
import paper_conf_ppopp_li0yjl19_b200 as vb  # noqa: E402
from paper_conf_ppopp_li0yjl19_b200.batch import DeviceBatch  # noqa: E402
from gpu_helpers import check_batch  # noqa: E402

T = pr.B200_TC
ROW = {s.name: i for i, s in enumerate(T.rows)}


def forced(db, rows):
    tiles = pr.enumerate_tiles(db.M, db.N, db.K, rows, T)
    n = len(tiles)
    return vb.plan_from_schedule(db.M, db.N, db.K, db.lda, db.ldb, db.ldc, rows, 256, list(range(n + 1)),
                                 [t.gemm for t in tiles], [t.y for t in tiles], [t.x for t in tiles], dtype=db.dtype,
                                 device=0, table_id=3)


def timed(db, plan, reps=10, flush=None):
    db.bind(plan)
    db.run_bound(plan)
    ts = []
    for _ in range(reps):
        if flush is not None:
            flush.fill_(1)
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s.record()
        db.run_bound(plan)
        e.record()
        ts.append((s, e))
    torch.cuda.synchronize()
    return float(np.median([s.elapsed_time(e) for s, e in ts]))


cfg = sys.argv[1] if len(sys.argv) > 1 else "C5"
if cfg == "small":
    rng = np.random.default_rng(5)
    M = rng.integers(8, 65, 2048); N = rng.integers(64, 1025, 2048); K = rng.integers(64, 1025, 2048)
else:
    M, N, K = vbinputs.config_sizes(cfg)
ab = "conv" if cfg == "C3" else "random"
db = DeviceBatch(M, N, K, "bf16")
db.fill(0, ab)
small_l2 = db.arena_bytes() < 4 * 126e6
flush = torch.empty(int(512e6), dtype=torch.uint8, device="cuda") if small_l2 else None
base = [ROW["h"]] * len(M)
swap = [ROW[f"S{min(64, (int(m) + 15) // 16 * 16)}"] if m <= 64 else ROW["h"] for m in M]
print(cfg, "GEMMs with M <= 64:", int((np.asarray(M) <= 64).sum()), "of", len(M), flush=True)
for name, rows in (("h", base), ("swap", swap), ("h", base), ("swap", swap)):
    plan = forced(db, rows)
    ms = timed(db, plan, flush=flush)
    print(f"  {name:5s} tiles {plan.info()['n_tiles']:7d}  {ms:.4f} ms", flush=True)
plan = forced(db, swap)
db.fill(0, ab)
db.run(plan)
torch.cuda.synchronize()
idx = [i for i in range(len(M)) if M[i] <= 64][:40] + [int(np.argmax(M))]
print("parity (normwise) worst", check_batch(db, idx, 0, ab))
