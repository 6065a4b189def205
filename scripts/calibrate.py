"""Offline calibration of the two platform constants on B200 (PAPER.md P253, P259, P290).

TLP threshold (P253: "starting with a huge GEMM case and decreasing the TLP iteratively ...
the inflection point with large performance degradation"): batches of identical GEMMs run
with the largest tile (tiling forced by threshold 1), the batch shrunk step by step so the
Eq. 1 TLP (tiles x 256 threads) falls; TFLOP/s against TLP, and the TLP below which the
throughput drops under 90 % of the large-batch plateau.

theta (P259: "if the total K of the tiles assigned to a thread block is larger than theta,
the benefit of batching tiles is not significant"): small-K batches under threshold batching
with theta swept; the theta past which the gain over theta = 0-like (one tile) flattens.

    python scripts/calibrate.py [--out profiles/calibration_r01.json] [--dtype bf16]
"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ppopp_li0yjl19_b200 as vb  # noqa: E402
from paper_conf_ppopp_li0yjl19_b200.batch import DeviceBatch  # noqa: E402


def timed(db, plan, flush, reps=7):
    db.bind(plan)
    for _ in range(2):
        db.run_bound(plan)
    ts = []
    for _ in range(reps):
        flush.fill_(1)
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s.record()
        db.run_bound(plan)
        e.record()
        ts.append((s, e))
    torch.cuda.synchronize()
    v = sorted(s.elapsed_time(e) for s, e in ts)
    return v[len(v) // 2]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default="")
    ap.add_argument("--dtype", default="bf16")
    args = ap.parse_args()
    flush = torch.empty(int(512e6), dtype=torch.uint8, device="cuda")
    out = {"dtype": args.dtype, "tlp": [], "theta": []}
    # ---- TLP threshold: shrinking batches of 512 x 512 x 1024 GEMMs at the largest tile
    size = (512, 512, 1024) if args.dtype != "f32" else (256, 256, 512)
    for b in [512, 384, 256, 192, 128, 96, 64, 48, 32, 24, 16, 12, 8, 4, 2, 1]:
        m, n, k = size
        db = DeviceBatch([m] * b, [n] * b, [k] * b, args.dtype)
        db.fill(0, "random")
        plan = db.plan(vb.POLICIES["none"], tlp_threshold=1)
        inf = plan.info()
        ms = timed(db, plan, flush)
        rec = {"B": b, "tiles": inf["n_tiles"], "tlp": inf["n_tiles"] * 256, "ms": round(ms, 5),
               "tflops": round(db.flops() / ms / 1e9, 2)}
        out["tlp"].append(rec)
        print(json.dumps(rec), flush=True)
        del plan, db
    plateau = max(r["tflops"] for r in out["tlp"])
    # smallest TLP that still reaches 90 % of the plateau: below it TLP is too low
    ok = [r for r in out["tlp"] if r["tflops"] >= 0.9 * plateau]
    out["tlp_inflection"] = min(r["tlp"] for r in ok) if ok else None
    # ---- theta: 4096 small-K GEMMs, threshold batching with theta swept
    for (m, n, k) in [(128, 128, 16), (128, 128, 64), (256, 256, 32), (128, 256, 128)]:
        db = DeviceBatch([m] * 4096, [n] * 4096, [k] * 4096, args.dtype)
        db.fill(0, "random")
        base = None
        for theta in [1, 64, 128, 256, 512, 1024, 2048]:
            plan = db.plan(vb.POLICIES["threshold"], theta=theta)
            inf = plan.info()
            ms = timed(db, plan, flush)
            base = base or ms
            rec = {"M": m, "N": n, "K": k, "theta": theta, "blocks": inf["n_blocks"], "ms": round(ms, 5),
                   "speedup_vs_theta1": round(base / ms, 3)}
            out["theta"].append(rec)
            print(json.dumps(rec), flush=True)
            del plan
        del db
    print(json.dumps({"tlp_inflection": out["tlp_inflection"], "plateau_tflops": plateau}), flush=True)
    if args.out:
        with open(args.out, "w") as f:
            json.dump(out, f, indent=1)


if __name__ == "__main__":
    main()
