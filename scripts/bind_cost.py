"""GEMM-kernel time on C5 with and without a re-bind (tensor-map address patch) before each launch."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import vbinputs  # noqa: E402
import paper_conf_ppopp_li0yjl19_b200 as vb  # noqa: E402
from paper_conf_ppopp_li0yjl19_b200.batch import DeviceBatch  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "C5"
info = vbinputs.CONFIGS[cfg]
M, N, K = vbinputs.config_sizes(cfg)
db = DeviceBatch(M, N, K, info["dtype"])
db.fill(0, info["ab"])
plan = db.plan(vb.POLICIES["threshold"])
db.bind(plan)
for rebind in (False, True, False, True):
    for _ in range(3):
        if rebind:
            db.bind(plan)
        db.run_bound(plan)
    ts = []
    for _ in range(10):
        if rebind:
            db.bind(plan)
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s.record()
        db.run_bound(plan)
        e.record()
        ts.append((s, e))
    torch.cuda.synchronize()
    print(cfg, "rebind" if rebind else "bound ", round(sum(s.elapsed_time(e) for s, e in ts) / len(ts), 4), "ms", flush=True)
