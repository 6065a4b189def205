"""VB_TRACE breakdown of the pair launch of C4 alone (its GEMMs with M >= 256, binary policy):
per-role wait fractions with the scheduler and MMA roles counted per CTA pair (measurement tool).
    VB_LIB=paper_conf_ppopp_li0yjl19_b200/libvbgemm_trace.so python scripts/trace_subset.py"""
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
WARPS = {"sched": 1, "prod": 4, "mma": 1, "cprod": 2, "epi": 8}
M, N, K = vbinputs.config_sizes("C4")
sel = M >= 256
db = DeviceBatch(M[sel], N[sel], K[sel], "bf16")
db.fill(0)
plan = db.plan(vb.VB_BATCH_BINARY)
assert plan.info()["launches_per_exec"] == 2, plan.info()
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
grid = 148
total = v[15] / (16 * grid)
print(f"C4 pair subset ({int(sel.sum())} GEMMs): {s.elapsed_time(e):.3f} ms, {total:.0f} cycles per CTA")
for i, n in enumerate(NAMES):
    if n in ("total", "tiles"):
        continue
    role = n.split("_")[0]
    g = grid // 2 if role in ("sched", "mma") else grid
    print(f"  {n:14s} {v[i] / (WARPS[role] * g) / total * 100:6.1f}%")
