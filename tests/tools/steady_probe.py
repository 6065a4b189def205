"""Steady-state (power-capped) C5 kernel time: 60 back-to-back bind+exec steps after warm-up,
median of the last 40; variants through VB_LIB (experiment builds, e.g. -DVB_EXP_FLOOR_BY=64 or
-DVB_WAIT_HINT) or --swap (M <= 64 GEMMs on swap-AB tiles through a forced schedule)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import vbinputs  # noqa: E402
import paper_conf_ppopp_li0yjl19_b200 as vb  # noqa: E402
from paper_conf_ppopp_li0yjl19_b200.batch import DeviceBatch  # noqa: E402

cfg = os.environ.get("VB_CFG", "C5")
M, N, K = vbinputs.config_sizes(cfg)
db = DeviceBatch(M, N, K, "bf16")
db.fill(0)
if "--swap" in sys.argv:
    from oracle import plan_ref as pr
    T = pr.B200_TC
    ex = db.plan(vb.VB_BATCH_THRESHOLD).export()
    rows = [int(r) for r in ex["gemm_strategy"]]
    ROW = {s.name: i for i, s in enumerate(T.rows)}
    rows = [ROW[f"S{min(64, (int(m) + 15) // 16 * 16)}"] if m <= 64 else r for m, r in zip(M, rows)]
    tiles = pr.enumerate_tiles(M, N, K, rows, T)
    plan = vb.plan_from_schedule(db.M, db.N, db.K, db.lda, db.ldb, db.ldc, rows, 256, list(range(len(tiles) + 1)),
                                 [t.gemm for t in tiles], [t.y for t in tiles], [t.x for t in tiles], dtype="bf16",
                                 device=0, table_id=3)
else:
    plan = db.plan(vb.VB_BATCH_AUTO)
s = torch.cuda.current_stream()
ts = []
for i in range(70):
    db.bind(plan, s)
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(s)
    db.run_bound(plan, s)
    b.record(s)
    ts.append((a, b))
torch.cuda.synchronize()
v = [a.elapsed_time(b) for a, b in ts]
print(f"{cfg} {os.path.basename(os.environ.get('VB_LIB', 'libvbgemm.so'))} {'swap' if '--swap' in sys.argv else ''} tiles {plan.info()['n_tiles']}: "
      f"first5 {np.median(v[:5]):.3f}  steady {np.median(v[30:]):.3f} ms", flush=True)
