"""Quick check of the 2-SM pair kernel on a small batch (run under `timeout`)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))), "tests"))
from gpu_helpers import check_batch  # noqa: E402
from paper_conf_ppopp_li0yjl19_b200.batch import DeviceBatch  # noqa: E402

M = np.array([256, 300, 512, 700, 1024]); N = np.array([256, 260, 128, 333, 1024]); K = np.array([64, 100, 512, 65, 1024])
db = DeviceBatch(M, N, K, "bf16")
db.fill(3)
plan = db.plan(tlp_threshold=1)
print(plan.info(), plan.export()["gemm_strategy"], flush=True)
db.run(plan)
torch.cuda.synchronize()
print("ran", flush=True)
print("worst normwise error", check_batch(db, range(len(M)), 3, "random"))
