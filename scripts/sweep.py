"""Time the GEMM kernel (vb_exec_bound) for configs x policies x tuning; one line per point."""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import vbinputs  # noqa: E402
import paper_conf_ppopp_li0yjl19_b200 as vb  # noqa: E402
from paper_conf_ppopp_li0yjl19_b200.batch import DeviceBatch  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--configs", default="C4,C5")
ap.add_argument("--policies", default="threshold,binary,none")
ap.add_argument("--thr", default="0")
ap.add_argument("--theta", default="0")
ap.add_argument("--iters", type=int, default=10)
args = ap.parse_args()
for cfg in args.configs.split(","):
    info = vbinputs.CONFIGS[cfg]
    M, N, K = vbinputs.config_sizes(cfg)
    db = DeviceBatch(M, N, K, info["dtype"])
    db.fill(0, info["ab"])
    flops = db.flops()
    nbytes = db.algorithmic_bytes(db.beta[:db.batch].cpu().numpy() != 0)
    for pol in args.policies.split(","):
        for thr in [int(x) for x in args.thr.split(",")]:
            for theta in [int(x) for x in args.theta.split(",")]:
                plan = db.plan(vb.POLICIES[pol], tlp_threshold=thr, theta=theta)
                db.bind(plan)
                for _ in range(3):
                    db.run_bound(plan)
                s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                s.record()
                for _ in range(args.iters):
                    db.run_bound(plan)
                e.record()
                torch.cuda.synchronize()
                ms = s.elapsed_time(e) / args.iters
                inf = plan.info()
                print(json.dumps(dict(cfg=cfg, policy=pol, thr=thr, theta=theta, ms=round(ms, 4),
                                      tflops=round(flops / ms / 1e9, 1), hbm_frac=round(nbytes / ms / 1e6 / 6462.1, 4),
                                      tiles=inf["n_tiles"], blocks=inf["n_blocks"])), flush=True)
                del plan
    del db
    torch.cuda.empty_cache()
