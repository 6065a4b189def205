"""How the L2 flush between timed steps affects the small configs (C3, C2): flush by writing a
512 MB buffer (leaves ~126 MB of dirty lines that the next kernel must write back while it
runs), by writing then reading a second 512 MB buffer (L2 left holding clean lines), or no
flush.  Kernel time by CUDA events on the launching stream, median of 30."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import vbinputs  # noqa: E402
import paper_conf_ppopp_li0yjl19_b200 as vb  # noqa: E402
from paper_conf_ppopp_li0yjl19_b200.batch import DeviceBatch  # noqa: E402

wbuf = torch.empty(int(512e6), dtype=torch.uint8, device="cuda")
rbuf = torch.ones(int(512e6) // 4, dtype=torch.float32, device="cuda")
for cfg in ("C3", "C2"):
    info = vbinputs.CONFIGS[cfg]
    M, N, K = vbinputs.config_sizes(cfg)
    db = DeviceBatch(M, N, K, info["dtype"])
    db.fill(0, info["ab"])
    plan = db.plan(vb.VB_BATCH_AUTO)
    db.bind(plan)
    for mode in ("write", "write+read", "none"):
        ts = []
        for it in range(33):
            if mode != "none":
                wbuf.fill_(1)
            if mode == "write+read":
                rbuf.sum()
            s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            s.record()
            db.run_bound(plan)
            e.record()
            torch.cuda.synchronize()
            if it >= 3:
                ts.append(s.elapsed_time(e))
        print(f"{cfg} flush={mode:11s} kernel {np.median(ts) * 1e3:8.1f} us")
