"""Paired A/B timing of several plans of the same batch (measurement tool).  Power and clock
drift on a B200 move single-run C5 times by +-5 %, so the plans are interleaved: each round
binds every plan in turn and times a few launches of it; the report is the median over rounds
of each plan's time relative to the first plan.

    python scripts/plan_ab.py C5 threshold,none,binary [--rounds 12]
Plan names: threshold | binary | none | auto, optionally with ':theta=<t>' or ':thr=<threads>'."""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import vbinputs  # noqa: E402
from paper_conf_ppopp_li0yjl19_b200 import _native as nv  # noqa: E402
from paper_conf_ppopp_li0yjl19_b200.batch import DeviceBatch  # noqa: E402

POL = {"threshold": nv.VB_BATCH_THRESHOLD, "binary": nv.VB_BATCH_BINARY, "none": nv.VB_BATCH_NONE,
       "auto": nv.VB_BATCH_AUTO}
ap = argparse.ArgumentParser()
ap.add_argument("config")
ap.add_argument("plans")
ap.add_argument("--rounds", type=int, default=12)
ap.add_argument("--launches", type=int, default=4)
args = ap.parse_args()
info = vbinputs.CONFIGS[args.config]
M, N, K = vbinputs.config_sizes(args.config)
db = DeviceBatch(M, N, K, info["dtype"])
db.fill(0, info.get("ab", "random"))
plans = []
for spec in args.plans.split(","):
    name, *opts = spec.split(":")
    kw = {k: int(v) for k, v in (o.split("=") for o in opts)}
    plans.append((spec, db.plan(POL[name], theta=kw.get("theta", 0), tlp_threshold=kw.get("thr", 0))))
times = {s: [] for s, _ in plans}
for r in range(args.rounds + 1):
    for spec, p in plans:
        db.bind(p)
        db.run_bound(p)
        ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.launches)]
        for s, e in ev:
            s.record()
            db.run_bound(p)
            e.record()
        torch.cuda.synchronize()
        if r:   # round 0 warms up
            times[spec].append(float(np.median([s.elapsed_time(e) for s, e in ev])))
base = np.array(times[plans[0][0]])
for spec, p in plans:
    t = np.array(times[spec])
    inf = p.info()
    print(json.dumps(dict(config=args.config, plan=spec, ms_median=round(float(np.median(t)), 4),
                          rel_to_first=round(float(np.median(t / base)), 4), tiles=inf["n_tiles"],
                          blocks=inf["n_blocks"])), flush=True)
