"""C3: the tiler's one-wave plan (128x256 tiles) against 'wave-fill' variants that move the
longest-K GEMMs to 128x128 tiles while the tile count stays within the 148 SMs (forced
schedules, one tile per block, longest tiles first)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import vbinputs  # noqa: E402
from oracle import plan_ref as pr  # noqa: E402
import paper_conf_ppopp_li0yjl19_b200 as vb  # noqa: E402
from paper_conf_ppopp_li0yjl19_b200.batch import DeviceBatch  # noqa: E402

T = pr.B200_TC
ROW = {s.name: i for i, s in enumerate(T.rows)}


def ntiles(M, N, r):
    s = T.rows[r]
    return -(-M // s.BY) * -(-N // s.BX)


def forced(db, rows):
    tiles = pr.enumerate_tiles(db.M, db.N, db.K, rows, T)
    tiles.sort(key=lambda t: -t.K)               # longest first (binary-batching order)
    return vb.plan_from_schedule(db.M, db.N, db.K, db.lda, db.ldb, db.ldc, rows, 256, list(range(len(tiles) + 1)),
                                 [t.gemm for t in tiles], [t.y for t in tiles], [t.x for t in tiles], dtype="bf16",
                                 device=0, table_id=3)


def timed(db, plan, flush, reps=20):
    db.bind(plan)
    db.run_bound(plan)
    ts = []
    for _ in range(reps):
        flush.fill_(1)
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s.record()
        db.run_bound(plan)
        e.record()
        ts.append((s, e))
    torch.cuda.synchronize()
    return float(np.median([s.elapsed_time(e) for s, e in ts]))


nb = int(sys.argv[1]) if len(sys.argv) > 1 else 1
M, N, K = vbinputs.config_sizes("C3", nb=nb)
db = DeviceBatch(M, N, K, "bf16")
db.fill(0, "conv")
flush = torch.empty(int(512e6), dtype=torch.uint8, device="cuda")
auto = db.plan(vb.VB_BATCH_AUTO)
print("auto plan", auto.info(), f"{timed(db, auto, flush):.4f} ms")
base = [ROW["h"]] * len(M)
print("h, longest first", sum(ntiles(m, n, ROW['h']) for m, n in zip(M, N)), f"{timed(db, forced(db, base), flush):.4f} ms")
for alt in ("l", "x", "t"):
    rows = list(base)
    total = sum(ntiles(m, n, r) for m, n, r in zip(M, N, rows))
    for g in sorted(range(len(M)), key=lambda g: -K[g]):
        extra = ntiles(M[g], N[g], ROW[alt]) - ntiles(M[g], N[g], rows[g])
        if total + extra <= 148:
            rows[g] = ROW[alt]
            total += extra
    print(f"wave-fill to {alt}: {total} tiles, {timed(db, forced(db, rows), flush):.4f} ms")
    allr = [ROW[alt]] * len(M)
    print(f"all {alt}: {sum(ntiles(m, n, ROW[alt]) for m, n in zip(M, N))} tiles, {timed(db, forced(db, allr), flush):.4f} ms")
