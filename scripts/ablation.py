"""Internal ablation over the paper's evaluation grid (§7.1-7.2, Fig. 8 and Fig. 9,
P320-334) on B200, bf16 through the tcgen05 kernel.

Batches of B identical GEMMs, M = N in {128, 256, 512, 1024}, B in {4, 8, 16, 32, 64, 128},
K in {16, 32, ..., 2048} (log grid, P322).  Four variants, each timed with a 512 MB L2 flush
before every launch (cold L2, kernel-only CUDA events):

  fixed      largest available tile, one tile per block: the MAGMA-style baseline (P314)
  tiler      tiling engine (§4.2.3) + one tile per block (Fig. 8: tiling engine alone)
  threshold  tiling + threshold batching (Fig. 9)
  binary     tiling + binary batching

    python scripts/ablation.py [--out profiles/ablation_r01.json] [--quick]
"""
import argparse
import itertools
import json
import math
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ppopp_li0yjl19_b200 as vb  # noqa: E402
from paper_conf_ppopp_li0yjl19_b200.batch import DeviceBatch  # noqa: E402

VARIANTS = {                       # (policy, tlp_threshold): threshold 1 forces the largest tiles
    "fixed": ("none", 1),
    "tiler": ("none", 0),
    "threshold": ("threshold", 0),
    "binary": ("binary", 0),
}


def time_plan(db, plan, flush, reps):
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
    ap.add_argument("--quick", action="store_true")
    ap.add_argument("--reps", type=int, default=7)
    args = ap.parse_args()
    MNs = [128, 256, 512, 1024]
    Bs = [4, 8, 16, 32, 64, 128]
    Ks = [16, 32, 64, 128, 256, 512, 1024, 2048]
    if args.quick:
        MNs, Bs, Ks = [128, 512], [4, 64], [16, 256, 2048]
    flush = torch.empty(int(512e6), dtype=torch.uint8, device="cuda")
    rows = []
    for mn, b, k in itertools.product(MNs, Bs, Ks):
        db = DeviceBatch([mn] * b, [mn] * b, [k] * b, "bf16")
        db.fill(0, "random")
        flops = db.flops()
        rec = {"MN": mn, "B": b, "K": k}
        for name, (pol, thr) in VARIANTS.items():
            plan = db.plan(vb.POLICIES[pol], tlp_threshold=thr)
            ms = time_plan(db, plan, flush, args.reps)
            inf = plan.info()
            rec[name] = {"ms": round(ms, 5), "tflops": round(flops / ms / 1e9, 2), "tiles": inf["n_tiles"],
                         "blocks": inf["n_blocks"]}
            del plan
        rows.append(rec)
        print(json.dumps(rec), flush=True)
        del db
    # geometric-mean speedups (the paper reports averages over the grid, P324 / P332)
    def gmean(xs):
        return math.exp(sum(math.log(x) for x in xs) / len(xs))
    summ = {}
    for v in ("tiler", "threshold", "binary"):
        summ[f"{v}_vs_fixed"] = round(gmean([r["fixed"]["ms"] / r[v]["ms"] for r in rows]), 3)
    summ["best_batching_vs_fixed"] = round(gmean([r["fixed"]["ms"] / min(r["threshold"]["ms"], r["binary"]["ms"])
                                                  for r in rows]), 3)
    summ["best_batching_vs_tiler"] = round(gmean([r["tiler"]["ms"] / min(r["threshold"]["ms"], r["binary"]["ms"])
                                                  for r in rows]), 3)
    summ["threshold_wins"] = sum(r["threshold"]["ms"] <= r["binary"]["ms"] for r in rows)
    summ["binary_wins"] = sum(r["binary"]["ms"] < r["threshold"]["ms"] for r in rows)
    for mn in MNs:
        sub = [r for r in rows if r["MN"] == mn]
        summ[f"MN{mn}_tiler_vs_fixed"] = round(gmean([r["fixed"]["ms"] / r["tiler"]["ms"] for r in sub]), 3)
        summ[f"MN{mn}_best_vs_fixed"] = round(gmean([r["fixed"]["ms"] / min(r["threshold"]["ms"], r["binary"]["ms"])
                                                     for r in sub]), 3)
    print(json.dumps({"summary": summ}), flush=True)
    if args.out:
        with open(args.out, "w") as f:
            json.dump({"grid": {"MN": MNs, "B": Bs, "K": Ks}, "variants": VARIANTS, "summary": summ, "points": rows},
                      f, indent=1)


if __name__ == "__main__":
    main()
