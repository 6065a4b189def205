"""Kernel throughput on uniform batches (all GEMMs the same shape): isolates the mainloop /
epilogue efficiency of the tcgen05 kernel from the variable-size effects."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_ppopp_li0yjl19_b200.batch import DeviceBatch  # noqa: E402

for (b, m, n, k, ab) in [(64, 1024, 1024, 4096, "random"), (64, 1024, 1024, 4096, "conv"), (512, 512, 512, 512, "random"),
                         (8192, 128, 128, 128, "random"), (32768, 64, 64, 64, "random")]:
    db = DeviceBatch(np.full(b, m), np.full(b, n), np.full(b, k), "bf16")
    db.fill(0, ab)
    plan = db.plan()
    db.bind(plan)
    for _ in range(3):
        db.run_bound(plan)
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    s.record()
    for _ in range(10):
        db.run_bound(plan)
    e.record()
    torch.cuda.synchronize()
    ms = s.elapsed_time(e) / 10
    nbytes = db.algorithmic_bytes(ab != "conv")
    print(json.dumps(dict(batch=b, M=m, N=n, K=k, ab=ab, ms=round(ms, 4), tflops=round(db.flops() / ms / 1e9, 1),
                          hbm_frac=round(nbytes / ms / 1e6 / 6462.1, 3), tiles=plan.info()["n_tiles"])), flush=True)
    del db, plan
    torch.cuda.empty_cache()
