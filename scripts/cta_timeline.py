"""Entry / exit time of every CTA of the tcgen05 kernel (VB_LIB=.../libvbgemm_ctatl.so built with
-DVB_TIMELINE_ALL): launch-to-first-entry spread, per-CTA busy time, last exit.  L2 flushed."""
import ctypes
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import vbinputs  # noqa: E402
import paper_conf_ppopp_li0yjl19_b200 as vb  # noqa: E402
from paper_conf_ppopp_li0yjl19_b200 import _native as nv  # noqa: E402
from paper_conf_ppopp_li0yjl19_b200.batch import DeviceBatch  # noqa: E402

nv.lib.vb_debug_set_trace.argtypes = [ctypes.c_void_p]
cfg = sys.argv[1] if len(sys.argv) > 1 else "C3"
M, N, K = vbinputs.config_sizes(cfg)
db = DeviceBatch(M, N, K, "bf16")
db.fill(0, vbinputs.CONFIGS[cfg]["ab"])
plan = db.plan(vb.VB_BATCH_AUTO)
ex = plan.export()
flush = torch.empty(int(512e6), dtype=torch.uint8, device="cuda")
buf = torch.zeros(2 * 148 + 8, dtype=torch.int64, device="cuda")
db.bind(plan)
for rep in range(4):
    flush.fill_(1)
    buf.zero_()
    nv.lib.vb_debug_set_trace(buf.data_ptr())
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    s.record()
    db.run_bound(plan)
    e.record()
    torch.cuda.synchronize()
    nv.lib.vb_debug_set_trace(None)
v = buf.cpu().numpy()[:2 * 148].reshape(-1, 2)
v = v[v[:, 0] > 0]
t0 = v[:, 0].min()
ent, ext = (v[:, 0] - t0) / 1e3, (v[:, 1] - t0) / 1e3
busy = ext - ent
print(f"{cfg}: {len(v)} CTAs, event time {s.elapsed_time(e) * 1e3:.1f} us; entry spread {ent.max():.2f} us; "
      f"exit min/median/max {ext.min():.2f}/{np.median(ext):.2f}/{ext.max():.2f} us; busy median {np.median(busy):.2f}")
order = np.argsort(-ext)[:6]
bp = ex["block_ptr"]
for c in order:
    b = int(c)  # static first block = CTA index
    tiles = [(int(ex["tile_gemm"][k]), int(ex["tile_y"][k]), int(ex["tile_x"][k])) for k in range(bp[b], bp[b + 1])]
    g = tiles[0][0]
    print(f"  CTA {c}: entry {ent[c]:.2f} exit {ext[c]:.2f} us, block {b} tiles {tiles[:3]} GEMM {g} MNK {M[g]}x{N[g]}x{K[g]} "
          f"strategy {int(ex['gemm_strategy'][g])}")
