"""DRAM-rate probe of the tcgen05 kernel on uniform and C5-like batches (measurement tool).
Run with VB_LIB pointing at a loads-only build (-DVB_EXP_NOMMA -DVB_EXP_NOMATH -DVB_EXP_NOSTORE)
to see the rate of the operand stream alone, or at the product library.  Prints, per batch, the
kernel time and the compulsory bytes it moves per second: loads only = s(MK + KN + MN) (A, B,
C_old), full kernel = s(MK + KN + 2MN)."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import vbinputs  # noqa: E402
import paper_conf_ppopp_li0yjl19_b200 as vb  # noqa: E402
from paper_conf_ppopp_li0yjl19_b200.batch import DeviceBatch  # noqa: E402

loads_only = "loads" in os.environ.get("VB_LIB", "")
if os.environ.get("VB_LD_ALIGN"):             # leading dimensions rounded to this many bytes
    _al = int(os.environ["VB_LD_ALIGN"])

    def _padded(cols, dtype, extra=0):
        q = _al // vbinputs.elem_size(dtype)
        return ((np.maximum(np.asarray(cols, np.int64), 1) + q - 1) // q) * q + extra * (16 // vbinputs.elem_size(dtype))
    vbinputs.padded_ld = _padded
M5, N5, K5 = vbinputs.config_sizes("C5")
up = lambda a, q: (a + q - 1) // q * q  # noqa: E731
cases = {
    "C5": (M5, N5, K5),
    "C4": vbinputs.config_sizes("C4"),
    "C5_K64": (M5, N5, up(K5, 64)),
    "C5_all64": (up(M5, 64), up(N5, 64), up(K5, 64)),
    "C5_M64": (up(M5, 64), N5, K5),
    "C5_N64": (M5, up(N5, 64), K5),
    "C5_MN64": (up(M5, 64), up(N5, 64), K5),
    "C5_NK64": (M5, up(N5, 64), up(K5, 64)),
    "C5_N32": (M5, up(N5, 32), K5),
    "C5_M128": (up(M5, 128), N5, K5),
    "C5_all128": (up(M5, 128), up(N5, 256), up(K5, 64)),
}
for b, m, n, k in [(4096, 128, 256, 1024), (16384, 256, 256, 256), (16384, 200, 200, 200),
                   (65536, 128, 256, 128), (65536, 100, 100, 100), (65536, 64, 64, 64)]:
    cases[f"u{b}x{m}x{n}x{k}"] = (np.full(b, m), np.full(b, n), np.full(b, k))
# compute-bound uniform batches (tensor-pipe feed of the pair kernel; cuBLAS context in
# scripts/cublas_context.py)
for b, m, n, k in [(64, 1024, 1024, 4096), (16, 2048, 2048, 4096), (256, 512, 512, 2048), (64, 1024, 1024, 1024),
                   (64, 1024, 1024, 256), (64, 1024, 1024, 512), (64, 1024, 1024, 2048), (256, 512, 512, 512),
                   (256, 512, 512, 1024), (256, 512, 512, 4096), (400, 768, 768, 2048), (400, 1000, 1000, 2000),
                   (400, 700, 1024, 2048), (400, 300, 1024, 2048), (400, 600, 700, 1500)]:
    cases[f"c{b}x{m}x{n}x{k}"] = (np.full(b, m), np.full(b, n), np.full(b, k))
for k in (16, 32, 40, 48, 56, 64, 72, 100, 128, 200, 256):
    cases[f"K{k}"] = (np.full(32768, 128), np.full(32768, 256), np.full(32768, k))
for n in (16, 17, 20, 24, 25, 29, 31, 32, 33, 40, 48, 64, 100, 128, 200, 256):
    cases[f"N{n}"] = (np.full(32768, 128), np.full(32768, n), np.full(32768, 256))
for m in (16, 40, 64, 100, 128):
    cases[f"M{m}"] = (np.full(32768, m), np.full(32768, 256), np.full(32768, 256))
only = sys.argv[1].split(",") if len(sys.argv) > 1 else list(cases)
for name in only:
    M, N, K = (np.asarray(x, np.int64) for x in cases[name])
    db = DeviceBatch(M, N, K, "bf16")
    db.fill(0)
    plan = db.plan(vb.POLICIES[os.environ.get("VB_POLICY", "threshold")])
    db.bind(plan)
    for _ in range(3):
        db.run_bound(plan)
    ts = []
    for _ in range(int(os.environ.get("VB_STEPS", "12"))):
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s.record()
        db.run_bound(plan)
        e.record()
        ts.append((s, e))
    torch.cuda.synchronize()
    ms = float(np.median([s.elapsed_time(e) for s, e in ts]))
    mn = (M * N).sum()
    nbytes = 2 * ((M * K).sum() + (K * N).sum() + mn * (1 if loads_only else 2))
    print(json.dumps(dict(case=name, lib=os.path.basename(os.environ.get("VB_LIB", "libvbgemm.so")), ms=round(ms, 4),
                          GB=round(nbytes / 1e9, 2), TBps=round(nbytes / ms / 1e9, 3),
                          TFLOPs=round(2 * (M * N * K).sum() / ms / 1e9, 1),
                          tiles=plan.info()["n_tiles"])), flush=True)
    del db, plan
    torch.cuda.empty_cache()
