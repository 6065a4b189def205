"""Planning cost by phase on the GPU box (VB_PLAN_PROFILE=1 prints the library's phase clock):
    VB_PLAN_PROFILE=1 python scripts/plan_profile.py [C5 ...]"""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import vbinputs  # noqa: E402
from paper_conf_ppopp_li0yjl19_b200 import _native as nv  # noqa: E402
import paper_conf_ppopp_li0yjl19_b200 as vb  # noqa: E402

for cfg in sys.argv[1:] or ["C5", "C4"]:
    dt = vbinputs.CONFIGS[cfg]["dtype"]
    M, N, K = vbinputs.config_sizes(cfg)
    ld = lambda c: vbinputs.padded_ld(c, dt)  # noqa: E731
    for rep in range(3):
        t0 = time.perf_counter()
        p = nv.plan_vbatched(M, N, K, ld(K), ld(N), ld(N), dt, vb.VB_BATCH_AUTO, device=int(os.environ.get("VB_PLAN_DEVICE", "0")))
        print(f"{cfg} rep {rep}: plan_vbatched {(time.perf_counter() - t0) * 1e3:.2f} ms", p.info(), flush=True)
        del p
