"""DRAM overfetch by shape: run under ncu (dram__bytes_read.sum) one launch per uniform batch
and compare with the algorithmic read bytes printed here."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_ppopp_li0yjl19_b200.batch import DeviceBatch  # noqa: E402

SHAPES = [(512, 512, 512, 512), (512, 500, 500, 500), (2048, 300, 300, 300), (2048, 256, 256, 256),
          (16384, 100, 100, 100), (16384, 128, 128, 128), (4096, 1000, 100, 100), (4096, 100, 1000, 100),
          (4096, 100, 100, 1000)]
import argparse  # noqa: E402
ap = argparse.ArgumentParser()
ap.add_argument("--shapes", default="")
ap.add_argument("--beta0", action="store_true")
args = ap.parse_args()
sel = [SHAPES[int(i)] for i in args.shapes.split(",")] if args.shapes else SHAPES
for (b, m, n, k) in sel:
    db = DeviceBatch(np.full(b, m), np.full(b, n), np.full(b, k), "bf16")
    db.fill(0, "random")
    if args.beta0:
        db.beta.zero_()
    plan = db.plan()
    db.bind(plan)
    db.run_bound(plan)
    torch.cuda.synchronize()
    rd = b * (m * k + k * n + (0 if args.beta0 else m * n)) * 2
    print(f"SHAPE b={b} {m}x{n}x{k} alg_read_GB={rd / 1e9:.3f} tiles={plan.info()['n_tiles']}", flush=True)
    del db, plan
    torch.cuda.empty_cache()
