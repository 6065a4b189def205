"""Run one config's GEMM kernel a few times (for ncu captures): plan, fill, bind, N launches."""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import vbinputs  # noqa: E402
import paper_conf_ppopp_li0yjl19_b200 as vb  # noqa: E402
from paper_conf_ppopp_li0yjl19_b200.batch import DeviceBatch  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C5")
ap.add_argument("--iters", type=int, default=3)
ap.add_argument("--policy", default="threshold")
ap.add_argument("--nb", type=int, default=1)
ap.add_argument("--thr", type=int, default=0)
ap.add_argument("--theta", type=int, default=0)
args = ap.parse_args()
if args.config == "C3i":   # GoogleNet convolutions as implicit GEMMs (vb_plan_conv)
    from paper_conf_ppopp_li0yjl19_b200.batch import ConvBatch
    db = ConvBatch(vbinputs.googlenet_convs(nb=args.nb), "bf16")
    db.fill(0, "conv")
else:
    info = vbinputs.CONFIGS[args.config]
    M, N, K = vbinputs.config_sizes(args.config, nb=args.nb)
    db = DeviceBatch(M, N, K, info["dtype"])
    db.fill(0, info["ab"])
plan = db.plan(vb.POLICIES[args.policy], tlp_threshold=args.thr, theta=args.theta)
db.bind(plan)
for _ in range(args.iters):
    db.run_bound(plan)
torch.cuda.synchronize()
print(args.config, plan.info(), flush=True)
