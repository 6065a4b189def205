"""Probe: does TMA move out-of-bounds (zero-filled) box rows through L2->SM?  Runs a batch of
short GEMMs (M=16) whose 64-row A boxes are 75% out of bounds; compare ncu TMA bytes with the
in-bounds and full-box byte counts printed here."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_ppopp_li0yjl19_b200.batch import DeviceBatch  # noqa: E402

B = 4000
M = np.full(B, 16); N = np.full(B, 256); K = np.full(B, 1024)
db = DeviceBatch(M, N, K, "bf16")
db.fill(0)
plan = db.plan()
db.bind(plan)
for _ in range(2):
    db.run_bound(plan)
torch.cuda.synchronize()
a_real = B * 16 * 1024 * 2
a_box = B * 64 * 1024 * 2 * (256 // 256)
b = B * 1024 * 256 * 2
c = B * 16 * 256 * 2
print(f"plan {plan.info()}  A in-bounds {a_real/1e9:.3f} GB, A full box (64 rows) {a_box/1e9:.3f} GB, "
      f"B {b/1e9:.3f} GB, C_old {c/1e9:.3f} GB")
