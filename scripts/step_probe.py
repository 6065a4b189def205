"""Per-step kernel times of C5 (bimodality check): bind+exec steps back to back, exec_bound
only, and with a host sync between steps."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import vbinputs  # noqa: E402
import paper_conf_ppopp_li0yjl19_b200 as vb  # noqa: E402
from paper_conf_ppopp_li0yjl19_b200.batch import DeviceBatch  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "C5"
M, N, K = vbinputs.config_sizes(cfg)
db = DeviceBatch(M, N, K, "bf16")
db.fill(0)
plan = db.plan(vb.VB_BATCH_AUTO)
s = torch.cuda.current_stream()


def run(mode, n=int(os.environ.get("VB_STEPS", "40"))):
    ts = []
    for i in range(n):
        if mode == "bind+exec" or i == 0:
            db.bind(plan, s)
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(s)
        db.run_bound(plan, s)
        b.record(s)
        if mode == "sync":
            torch.cuda.synchronize()
        ts.append((a, b))
    torch.cuda.synchronize()
    v = [a.elapsed_time(b) for a, b in ts]
    print(mode, " ".join(f"{x:.2f}" for x in v))
    print(f"   p10 {np.percentile(v, 10):.3f} p50 {np.percentile(v, 50):.3f} p90 {np.percentile(v, 90):.3f}", flush=True)


for mode in (sys.argv[2].split(",") if len(sys.argv) > 2 else ("bind+exec", "exec", "sync", "bind+exec")):
    run(mode)
