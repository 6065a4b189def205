"""Single-tile latency of the tcgen05 kernel: one GEMM, one 128-row tile, K swept -- the slope
is the per-k-block time of an isolated tile (the critical path of latency-bound batches like
C3).  Kernel time by CUDA events, median of 20, L2 warm."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ppopp_li0yjl19_b200 as vb  # noqa: E402
from paper_conf_ppopp_li0yjl19_b200.batch import DeviceBatch  # noqa: E402

for N in (64, 256):
    for K in (64, 640, 1728, 6400):
        db = DeviceBatch([128], [N], [K], "bf16")
        db.fill(0, "random")
        plan = db.plan(vb.VB_BATCH_NONE)
        db.bind(plan)
        ts = []
        for it in range(23):
            s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            s.record()
            db.run_bound(plan)
            e.record()
            torch.cuda.synchronize()
            if it >= 3:
                ts.append(s.elapsed_time(e))
        print(f"M=128 N={N} K={K:5d} ({(K + 63) // 64:3d} k-blocks): {np.median(ts) * 1e3:7.1f} us", flush=True)
