"""Timeline of CTA 0 of the tcgen05 kernel (VB_LIB=.../libvbgemm_timeline.so, -DVB_TIMELINE):
%globaltimer stamps of its first tile's events relative to kernel entry, for an isolated
single-tile GEMM and for C3.  Measurement tool only."""
import ctypes
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import vbinputs  # noqa: E402
import paper_conf_ppopp_li0yjl19_b200 as vb  # noqa: E402
from paper_conf_ppopp_li0yjl19_b200 import _native as nv  # noqa: E402
from paper_conf_ppopp_li0yjl19_b200.batch import DeviceBatch  # noqa: E402

EV = ["entry", "setup", "ring1", "kb_armed", "mma_k1", "acc_commit", "epi_acc", "epi_done", "stores", "teardown",
      "exit"]
nv.lib.vb_debug_set_trace.argtypes = [ctypes.c_void_p]
buf = torch.zeros(32, dtype=torch.int64, device="cuda")
cases = [("1 GEMM 128x256x64", [128], [256], [64]), ("1 GEMM 128x256x1728", [128], [256], [1728]),
         ("C3", *vbinputs.config_sizes("C3"))]
for name, M, N, K in cases:
    db = DeviceBatch(M, N, K, "bf16")
    db.fill(0, "random")
    plan = db.plan(vb.VB_BATCH_NONE)
    db.bind(plan)
    for _ in range(3):
        db.run_bound(plan)
    torch.cuda.synchronize()
    buf.zero_()
    nv.lib.vb_debug_set_trace(buf.data_ptr())
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    s.record()
    db.run_bound(plan)
    e.record()
    torch.cuda.synchronize()
    nv.lib.vb_debug_set_trace(None)
    v = buf.cpu().tolist()
    t0 = v[0]
    line = ", ".join(f"{EV[i]} {(v[i] - t0) / 1e3:.2f}" for i in range(len(EV)) if v[i])
    print(f"{name}: events {s.elapsed_time(e) * 1e3:.1f} us | CTA0 (us from entry): {line}", flush=True)
