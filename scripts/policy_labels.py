"""Labelled training set for the online batching-policy selector (§5, P272-274).

"We form a training set with more than 400 samples.  We test all the batching algorithms and
label the sample with the best algorithm."  Each sample is a seeded synthetic batch (fixed
size, uniform or log-uniform sizes; batch size log-uniform in [1, 4096]); both heuristics are
planned and timed on the GPU (median of 5 cold-L2 launches) and the faster one is the label.
Features are the paper's: mean M, mean N, mean K and the batch size B.

    python scripts/policy_labels.py --dtype bf16 --n 450 --out profiles/policy_labels_bf16_r01.json
"""
import argparse
import json
import math
import os
import sys
import time

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ppopp_li0yjl19_b200 as vb  # noqa: E402
from paper_conf_ppopp_li0yjl19_b200.batch import DeviceBatch  # noqa: E402


def draw(rng, dtype):
    """One synthetic batch (M, N, K arrays)."""
    es = 4 if dtype == "f32" else 2
    flop_cap = 2e11 if dtype == "f32" else 2e12
    byte_cap = 4e9
    B = int(round(math.exp(rng.uniform(0.0, math.log(4096.0)))))
    kind = rng.choice(["fixed", "uniform", "loguniform"])
    hi_cap = 1024 if dtype == "f32" else 2048

    def dim(lo_min, hi_max):
        lo = math.exp(rng.uniform(math.log(lo_min), math.log(hi_max)))
        hi = math.exp(rng.uniform(math.log(lo), math.log(hi_max)))
        return int(lo), max(int(lo), int(hi))

    if kind == "fixed":
        m = int(math.exp(rng.uniform(math.log(16), math.log(hi_cap))))
        n = m if rng.random() < 0.5 else int(math.exp(rng.uniform(math.log(16), math.log(hi_cap))))
        k = int(math.exp(rng.uniform(math.log(16), math.log(2 * hi_cap))))
        M, N, K = np.full(B, m), np.full(B, n), np.full(B, k)
    else:
        (ml, mh), (nl, nh), (kl, kh) = dim(16, hi_cap), dim(16, hi_cap), dim(16, 2 * hi_cap)
        if kind == "uniform":
            M, N, K = rng.integers(ml, mh + 1, B), rng.integers(nl, nh + 1, B), rng.integers(kl, kh + 1, B)
        else:
            lg = lambda lo, hi: np.floor(np.exp(rng.uniform(math.log(lo), math.log(hi + 1), B))).astype(np.int64)
            M, N, K = lg(ml, mh), lg(nl, nh), lg(kl, kh)
    M, N, K = (np.maximum(x, 1).astype(np.int64) for x in (M, N, K))
    flops = float((2 * M * N * K).sum())
    nbytes = float((es * (M * K + K * N + 2 * M * N)).sum())
    scale = max(flops / flop_cap, nbytes / byte_cap, 1.0)
    if scale > 1.0:
        keep = max(1, int(B / scale))
        M, N, K = M[:keep], N[:keep], K[:keep]
    return str(kind), M, N, K


def timed(db, plan, flush, reps=5):
    db.bind(plan)
    db.run_bound(plan)
    ts = []
    for _ in range(reps):
        if flush is not None:
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
    ap.add_argument("--dtype", default="bf16")
    ap.add_argument("--n", type=int, default=450)
    ap.add_argument("--seed", type=int, default=2019)
    ap.add_argument("--out", default="")
    ap.add_argument("--budget-s", type=float, default=1e9, help="stop after this many seconds")
    args = ap.parse_args()
    rng = np.random.default_rng(args.seed)
    flush = torch.empty(int(512e6), dtype=torch.uint8, device="cuda")
    samples = []
    t0 = time.time()
    for i in range(args.n):
        kind, M, N, K = draw(rng, args.dtype)
        db = DeviceBatch(M, N, K, args.dtype)
        db.fill(i, "random")
        small = db.arena_bytes() < 4 * 126e6
        rec = {"i": i, "kind": kind, "B": int(len(M)), "mean_M": float(M.mean()), "mean_N": float(N.mean()),
               "mean_K": float(K.mean()), "flops": float(db.flops())}
        for pol in ("threshold", "binary"):
            plan = db.plan(vb.POLICIES[pol])
            rec[pol + "_ms"] = round(timed(db, plan, flush if small else None), 5)
            del plan
        rec["label"] = "threshold" if rec["threshold_ms"] <= rec["binary_ms"] else "binary"
        samples.append(rec)
        print(json.dumps(rec), flush=True)
        del db
        if time.time() - t0 > args.budget_s:
            break
    if args.out:
        with open(args.out, "w") as f:
            json.dump({"dtype": args.dtype, "seed": args.seed, "features": ["mean_M", "mean_N", "mean_K", "B"],
                       "samples": samples}, f, indent=0)


if __name__ == "__main__":
    main()
