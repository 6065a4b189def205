"""Per-role wait-cycle breakdown of the tensor-core kernel (needs libvbgemm_trace.so).

    VB_LIB=paper_conf_ppopp_li0yjl19_b200/libvbgemm_trace.so python scripts/trace_run.py --config C5
Prints, per CTA (averaged over CTAs), the cycles each role spent waiting on each barrier,
as a fraction of the kernel's cycles."""
import argparse
import ctypes
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import vbinputs  # noqa: E402
import paper_conf_ppopp_li0yjl19_b200 as vb  # noqa: E402
from paper_conf_ppopp_li0yjl19_b200 import _native as nv  # noqa: E402
from paper_conf_ppopp_li0yjl19_b200.batch import DeviceBatch  # noqa: E402

NAMES = ["sched_rempty", "sched_budget", "prod_rfull", "prod_empty", "mma_rfull", "mma_tempty", "mma_full",
         "cprod_rfull", "cprod_cempty", "epi_rfull", "epi_tfull", "epi_cfull", "epi_store", "epi_tmem", "epi_math",
         "total", "tiles", "prod_issue", "mma_issue", "epi_fencebar", "epi_stissue", "epi_loop",
         "epi_tload", "epi_rel", "epi_proc", "epi_head"]
WARPS = {"sched": 1, "prod": 1, "mma": 1, "cprod": 1, "epi": 8, "cprod": 2, "prod": 4}

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C5")
ap.add_argument("--policy", default="threshold")
args = ap.parse_args()
assert "trace" in nv.LIB_PATH or "VB_TRACE" in os.environ, "set VB_LIB to a trace build"
info = vbinputs.CONFIGS[args.config]
M, N, K = vbinputs.config_sizes(args.config)
db = DeviceBatch(M, N, K, info["dtype"])
db.fill(0, info["ab"])
plan = db.plan(vb.POLICIES[args.policy])
db.bind(plan)
db.run_bound(plan)
buf = torch.zeros(32, dtype=torch.int64, device="cuda")
nv.lib.vb_debug_set_trace.argtypes = [ctypes.c_void_p]
nv.lib.vb_debug_set_trace(buf.data_ptr())
db.bind(plan)
s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
s.record()
db.run_bound(plan)
e.record()
torch.cuda.synchronize()
nv.lib.vb_debug_set_trace(None)
v = buf.cpu().tolist()
grid = min(plan.info()["n_blocks"], 148)
total = v[NAMES.index("total")] / (16 * grid)
print(f"{args.config} {args.policy}: {s.elapsed_time(e):.3f} ms, {total:.0f} cycles per CTA, tiles {v[16]}")
for i, n in enumerate(NAMES[:15] + NAMES[17:]):
    i = NAMES.index(n)
    w = WARPS[n.split("_")[0]]
    cyc = v[i] / (w * grid)
    print(f"  {n:14s} {cyc / total * 100:6.1f}%")
