"""VB_TRACE breakdown for a uniform batch (M N K B from argv)."""
import ctypes
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_ppopp_li0yjl19_b200 import _native as nv  # noqa: E402
from paper_conf_ppopp_li0yjl19_b200.batch import DeviceBatch  # noqa: E402

M, N, K, B = (int(x) for x in sys.argv[1:5])
NAMES = ["sched_rempty", "sched_budget", "prod_rfull", "prod_empty", "mma_rfull", "mma_tempty", "mma_full",
         "cprod_rfull", "cprod_cempty", "epi_rfull", "epi_tfull", "epi_cfull", "epi_store", "epi_tmem", "epi_math",
         "total", "tiles", "prod_issue", "mma_issue", "epi_fencebar", "epi_stissue", "epi_loop",
         "epi_tload", "epi_rel", "epi_proc", "epi_head"]
WARPS = {"sched": 1, "prod": 4, "mma": 1, "cprod": 2, "epi": 8}
db = DeviceBatch(np.full(B, M), np.full(B, N), np.full(B, K), "bf16")
db.fill(0)
plan = db.plan()
db.bind(plan)
db.run_bound(plan)
buf = torch.zeros(32, dtype=torch.int64, device="cuda")
nv.lib.vb_debug_set_trace.argtypes = [ctypes.c_void_p]
nv.lib.vb_debug_set_trace(buf.data_ptr())
s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
s.record()
db.run_bound(plan)
e.record()
torch.cuda.synchronize()
nv.lib.vb_debug_set_trace(None)
v = buf.cpu().tolist()
grid = min(plan.info()["n_blocks"], 148)
# a pair plan (launches_per_exec 2 = prep + pair kernel) has one scheduler and MMA thread per CTA pair
leaders = grid // 2 if plan.info()["launches_per_exec"] == 2 and (db.M >= 256).all() and (db.N >= 256).all() else grid
total = v[15] / (16 * grid)
print("tiles per CTA (pair tiles per pair):", plan.info()["n_tiles"] / leaders)
print(f"{B}x {M}x{N}x{K}: {s.elapsed_time(e):.3f} ms, {total:.0f} cycles/CTA, {db.flops() / s.elapsed_time(e) / 1e9:.0f} TF/s")
for i, n in enumerate(NAMES):
    if n in ("total", "tiles"):
        continue
    g = leaders if n.split('_')[0] in ("sched", "mma") else grid
    print(f"  {n:14s} {v[i] / (WARPS[n.split('_')[0]] * g) / total * 100:6.1f}%")
