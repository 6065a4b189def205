"""Experiment: does the leading-dimension alignment (16 B vs 128 B) change the C5 kernel time?
(Partial 32-byte sectors at row ends cost DRAM read-modify-write on stores.)"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import vbinputs  # noqa: E402
import paper_conf_ppopp_li0yjl19_b200 as vb  # noqa: E402
from paper_conf_ppopp_li0yjl19_b200.batch import DeviceBatch  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C5")
ap.add_argument("--align", default="16,128")
ap.add_argument("--iters", type=int, default=20)
args = ap.parse_args()
orig = vbinputs.padded_ld
for al in [int(a) for a in args.align.split(",")]:
    def padded(cols, dtype, extra=0, al=al):
        q = al // vbinputs.elem_size(dtype)
        cols = np.asarray(cols, dtype=np.int64)
        return ((np.maximum(cols, 1) + q - 1) // q) * q
    vbinputs.padded_ld = padded
    info = vbinputs.CONFIGS[args.config]
    M, N, K = vbinputs.config_sizes(args.config)
    db = DeviceBatch(M, N, K, info["dtype"])
    db.fill(0, info["ab"])
    plan = db.plan(vb.POLICIES["threshold"])
    db.bind(plan)
    for _ in range(3):
        db.run_bound(plan)
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    s.record()
    for _ in range(args.iters):
        db.run_bound(plan)
    e.record()
    torch.cuda.synchronize()
    print(f"align {al}: {s.elapsed_time(e) / args.iters:.3f} ms", flush=True)
    del db, plan
    torch.cuda.empty_cache()
vbinputs.padded_ld = orig
