"""GoogleNet inception convolutions: explicit conv-as-GEMM shapes (C3, the paper's view, P45 --
the im2col matrix is an input) versus the implicit-GEMM path (vb_plan_conv, TMA im2col; only
input + weights + output move), per image batch nb.  Uses bench.py's timing (CUDA events,
L2 flushed between steps when the arenas fit in L2).  One JSON line per point."""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--nb", default="1,8,32")
ap.add_argument("--steps", type=int, default=20)
ap.add_argument("--policy", default="auto")
a = ap.parse_args()
peaks = bench.load_peaks()
for nb in [int(x) for x in a.nb.split(",")]:
    for cfg in ("C3", "C3i"):
        args = argparse.Namespace(nb=nb, steps=a.steps, warmup=3, policy=a.policy, seed=0, e2e_steps=0)
        r, db, plan = bench.run_config(cfg, args, 1, 0, 0, peaks, None, headline=False)
        print(json.dumps({"cfg": cfg, "nb": nb, "kernel_ms": round(r["kernel_ms"], 4),
                          "step_ms": round(r["step_ms"], 4), "tflops": round(r["kernel_tflops"], 2),
                          "gflop": round(r["flops"] / 1e9, 2), "alg_bytes_MB": round(r["bytes_rank"] / 1e6, 1),
                          "roofline": bench._round(r["roofline"]), "n_tiles": r["plan"]["n_tiles"],
                          "policy": r["policy_chosen"]}), flush=True)
        del db, plan
