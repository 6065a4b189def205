"""Randomised parity campaign on the GPU (run under gpurun; test infrastructure, not product code).

Each case draws a random batch -- dtype (bf16 / fp16 / fp32), size distribution (uniform,
log-uniform, skinny, tiny, K = 0 and 1-wide mixes), batch size, policy (threshold / binary /
none / AUTO), optional TLP-threshold and theta overrides, and sometimes a forced schedule of
random strategy rows (pair, 1-SM and swap-AB tiles, blocks of random length) -- runs it through
the C-ABI on NaN-poisoned C and checks every GEMM against the fp64 oracle (normwise tolerance
and the elementwise bound) plus untouched C padding.  Random implicit-GEMM convolution batches
are mixed in.  Prints one JSON line per case and a summary; stops at the first failure.

    python tests/tools/fuzz_parity.py [--minutes 20] [--seed 7] [--out gpurun_out/fuzz.json]
"""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))

import numpy as np  # noqa: E402
import torch  # noqa: E402

import vbinputs  # noqa: E402
from oracle import plan_ref as pr  # noqa: E402
from gpu_helpers import check_recorded, RECORD  # noqa: E402
from test_gpu_conv import check_convs  # noqa: E402
import paper_conf_ppopp_li0yjl19_b200 as vb  # noqa: E402
from paper_conf_ppopp_li0yjl19_b200.batch import ConvBatch, DeviceBatch  # noqa: E402


def draw_sizes(rng):
    kind = rng.choice(["uniform", "loguniform", "skinny", "tiny", "mixed"])
    B = int(rng.integers(1, 200))
    if kind == "uniform":
        hi = int(rng.integers(16, 1200))
        r = rng.integers(1, hi + 1, (B, 3))
    elif kind == "loguniform":
        r = np.floor(np.exp(rng.uniform(0, np.log(1500), (B, 3)))).astype(np.int64)
    elif kind == "skinny":
        r = np.stack([rng.integers(1, 70, B), rng.integers(100, 1500, B), rng.integers(1, 2500, B)], 1)
        if rng.random() < 0.5:
            r = r[:, [1, 0, 2]]
    elif kind == "tiny":
        r = rng.integers(1, 24, (B, 3))
    else:
        r = rng.integers(1, 700, (B, 3))
        z = rng.random(B)
        r[z < 0.1, 2] = 0
        r[(z >= 0.1) & (z < 0.15), 0] = 1
        r[(z >= 0.15) & (z < 0.2), 1] = 1
    return kind, np.maximum(r, 0)


def forced_plan(db, rng, table, tid):
    n_rows = len(table.rows)
    rows = [int(rng.integers(0, n_rows)) for _ in range(db.batch)]
    tiles = pr.enumerate_tiles(db.M, db.N, db.K, rows, table)
    pair = [table.rows[rows[t.gemm]].ctas == 2 for t in tiles]
    order = [i for i, q in enumerate(pair) if q] + [i for i, q in enumerate(pair) if not q]
    n_pair = sum(pair)
    tiles = [tiles[i] for i in order]
    bp, i = [0], 0
    while i < len(tiles):                 # random block lengths, never mixing pair and 1-SM tiles
        lim = n_pair if i < n_pair else len(tiles)
        i = min(lim, i + int(rng.integers(1, 5)))
        bp.append(i)
    return vb.plan_from_schedule(db.M, db.N, db.K, db.lda, db.ldb, db.ldc, rows, table.versions[0], bp,
                                 [t.gemm for t in tiles], [t.y for t in tiles], [t.x for t in tiles],
                                 dtype=db.dtype, device=0, table_id=tid), "forced"


def padding_ok(db):
    """Row padding [N, ldc) of rows 0 .. M-2 is still NaN (the last row's padding lies past the
    matrix's allocation and may hold the next matrix)."""
    for g in range(db.batch):
        m, n, ld = int(db.M[g]), int(db.N[g]), int(db.ldc[g])
        if m > 1 and n and ld != n:
            full = torch.as_strided(db.C, (m - 1, ld), (ld, 1), int(db.offC[g]))
            if not torch.isnan(full[:, n:]).all():
                return False
    return True


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--minutes", type=float, default=20)
    ap.add_argument("--seed", type=int, default=7)
    ap.add_argument("--out", default="")
    args = ap.parse_args()
    rng = np.random.default_rng(args.seed)
    t0 = time.time()
    stats = {"cases": 0, "gemms": 0, "by_kind": {}}
    case = 0
    while time.time() - t0 < args.minutes * 60:
        case += 1
        seed = int(rng.integers(0, 2 ** 31))
        if rng.random() < 0.08:       # implicit-GEMM convolutions
            convs = [c for c in vbinputs.googlenet_convs(nb=int(rng.integers(1, 4)))
                     if rng.random() < 0.3] or vbinputs.googlenet_convs(module="3a")
            dtype = str(rng.choice(["bf16", "f16"]))
            db = ConvBatch(convs, dtype)
            db.C.fill_(float("nan"))
            ab = str(rng.choice(["conv", "random"]))
            db.fill(seed, ab)
            plan = db.plan(int(rng.integers(0, 3)))
            db.run(plan)
            torch.cuda.synchronize()
            check_convs(db, range(db.batch), seed, ab)
            rec = {"case": case, "kind": "conv", "dtype": dtype, "batch": db.batch}
        else:
            kind, r = draw_sizes(rng)
            dtype = str(rng.choice(["bf16", "f16", "f32"], p=[0.45, 0.2, 0.35]))
            ab = str(rng.choice(["random", "conv"], p=[0.8, 0.2]))
            db = DeviceBatch(r[:, 0], r[:, 1], r[:, 2], dtype, ld_extra=int(rng.integers(0, 2)))
            db.C.fill_(float("nan"))
            db.fill(seed, ab)
            if ab == "conv":
                db.C.fill_(float("nan"))        # beta = 0: C must never be read
            how = "planned"
            if rng.random() < 0.25:
                table, tid = (pr.B200_F32, 2) if dtype == "f32" else (pr.B200_TC, 3)
                if dtype == "f32" and rng.random() < 0.4:
                    table, tid = pr.V100, 1
                plan, how = forced_plan(db, rng, table, tid)
            else:
                pol = int(rng.choice([0, 1, 2, vb.VB_BATCH_AUTO]))
                thr = int(rng.choice([0, 0, 1, 148 * 256 // 4, 4 * 148 * 256]))
                theta = int(rng.choice([0, 0, 1, 32, 512]))
                plan = db.plan(pol, tlp_threshold=thr, theta=theta)
            db.run(plan)
            torch.cuda.synchronize()
            c_old = [np.zeros((int(m), int(n))) for m, n in zip(db.M, db.N)] if ab == "conv" else None
            res = check_recorded(f"fuzz{case}", db, range(db.batch), seed, ab, c_old=c_old)
            assert padding_ok(db), f"case {case}: C padding written"
            rec = {"case": case, "kind": kind, "dtype": dtype, "how": how, "batch": db.batch,
                   "tiles": plan.info()["n_tiles"], "normwise_max": res["normwise_max"],
                   "bound_ratio_max": res["bound_ratio_max"]}
            RECORD.pop(f"fuzz{case}", None)
        stats["cases"] += 1
        stats["gemms"] += rec["batch"]
        stats["by_kind"][rec["kind"]] = stats["by_kind"].get(rec["kind"], 0) + 1
        for key in ("normwise_max", "bound_ratio_max"):
            if key in rec:
                k = f"{rec['dtype']}_{key}"
                stats[k] = max(stats.get(k, 0.0), rec[key])
        print(json.dumps(rec), flush=True)
        del db, plan
    stats["minutes"] = round((time.time() - t0) / 60, 1)
    print(json.dumps({"summary": stats}), flush=True)
    if args.out:
        with open(args.out, "w") as f:
            json.dump(stats, f, indent=1)


if __name__ == "__main__":
    main()
