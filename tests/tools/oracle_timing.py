"""The fp64 oracle as it stands, timed on this host: C1-C3 in full with one
thread and with every core (OpenMP over GEMMs x rows), as effective TFLOP/s.  One JSON line per
point; this is a reported baseline, not a target."""
import json
import os
import platform
import sys
import time

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import vbinputs  # noqa: E402
from oracle import gemm as og  # noqa: E402

cpu = platform.processor() or "unknown"
try:
    with open("/proc/cpuinfo") as f:
        cpu = next(l.split(":", 1)[1].strip() for l in f if l.startswith("model name"))
except (OSError, StopIteration):
    pass
for cfg in ("C1", "C2", "C3"):
    info = vbinputs.CONFIGS[cfg]
    M, N, K = vbinputs.config_sizes(cfg)
    As, Bs, Cs = [], [], []
    for g in range(len(M)):
        m, n, k = int(M[g]), int(N[g]), int(K[g])
        As.append(vbinputs.matrix_f64_fast(0, g, vbinputs.OP_A, m, k, info["dtype"]))
        Bs.append(vbinputs.matrix_f64_fast(0, g, vbinputs.OP_B, k, n, info["dtype"]))
        Cs.append(vbinputs.matrix_f64_fast(0, g, vbinputs.OP_C, m, n, info["dtype"]))
    al, be = vbinputs.alpha_beta(0, range(len(M)), info["ab"])
    flops = float((2 * M * N * K).sum())
    for threads in (1, og.max_threads()):
        cw = [c.copy() for c in Cs]
        t0 = time.perf_counter()
        og.gemm_batch(As, Bs, cw, al.astype(np.float64), be.astype(np.float64), nthreads=threads)
        dt = time.perf_counter() - t0
        print(json.dumps({"config": cfg, "threads": threads, "cpu": cpu, "seconds": round(dt, 3),
                          "tflops": round(flops / dt / 1e12, 5)}), flush=True)
