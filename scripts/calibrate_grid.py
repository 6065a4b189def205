"""Grid calibration of the B200 platform constants (TLP threshold, theta) per kernel family.

PAPER.md P253/P290 set both constants offline, once per platform.  Here every
(threshold, theta) pair is timed with threshold and binary batching over the Fig. 8/9 grid
(M = N in {128, 256, 512, 1024}, B in {4, 16, 64}, K in {16, 64, 256, 1024, 2048}) plus the
BASELINE configs of the dtype; the score of a pair is the geometric-mean time relative to the
best pair per point.

    python scripts/calibrate_grid.py --dtype bf16 --out profiles/calibration_grid_bf16_r01.json
"""
import argparse
import itertools
import json
import math
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import vbinputs  # noqa: E402
import paper_conf_ppopp_li0yjl19_b200 as vb  # noqa: E402
from paper_conf_ppopp_li0yjl19_b200.batch import DeviceBatch  # noqa: E402


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
    ap.add_argument("--out", default="")
    args = ap.parse_args()
    sms = 148
    thrs = [1, sms * 256, 2 * sms * 256, 4 * sms * 256, 8 * sms * 256, 16 * sms * 256]
    thetas = [1, 64, 128, 256, 512]
    pols = ["threshold", "binary"]
    combos = [(p, t, th) for p in pols for t in thrs for th in thetas]
    points = []
    hi = 1024 if args.dtype != "f32" else 512
    for mn, b, k in itertools.product([128, 256, 512, hi], [4, 16, 64], [16, 64, 256, 1024, 2048]):
        points.append((f"grid {mn}x{mn}x{k} B{b}", [mn] * b, [mn] * b, [k] * b))
    cfgs = ["C3", "C4", "C5"] if args.dtype != "f32" else ["C1", "C2"]
    for c in cfgs:
        M, N, K = vbinputs.config_sizes(c)
        points.append((c, M, N, K))
    flush = torch.empty(int(512e6), dtype=torch.uint8, device="cuda")
    res = {}
    for name, M, N, K in points:
        db = DeviceBatch(M, N, K, args.dtype)
        db.fill(0, "random")
        small = db.arena_bytes() < 4 * 126e6
        row = {}
        for pol, t, th in combos:
            plan = db.plan(vb.POLICIES[pol], tlp_threshold=t, theta=th)
            row[f"{pol}/{t}/{th}"] = timed(db, plan, flush if small else None, reps=5 if small else 3)
            del plan
        res[name] = row
        print(json.dumps({name: {k: round(v, 4) for k, v in row.items()}}), flush=True)
        del db
    score = {}
    for key in res[next(iter(res))]:
        score[key] = math.exp(sum(math.log(r[key] / min(r.values())) for r in res.values()) / len(res))
    grid_only = {k: math.exp(sum(math.log(r[k] / min(r.values())) for n, r in res.items() if n.startswith("grid"))
                             / sum(1 for n in res if n.startswith("grid"))) for k in score}
    best = sorted(score.items(), key=lambda kv: kv[1])[:10]
    print(json.dumps({"best": best}), flush=True)
    if args.out:
        with open(args.out, "w") as f:
            json.dump({"dtype": args.dtype, "score_all": score, "score_grid": grid_only, "times_ms": res}, f, indent=0)


if __name__ == "__main__":
    main()
