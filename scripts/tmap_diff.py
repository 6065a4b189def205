"""Diagnostic: compare device-built tensor maps with host-encoded ones word by word (GPU box)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import vbinputs  # noqa: E402
from paper_conf_ppopp_li0yjl19_b200.batch import DeviceBatch  # noqa: E402

M, N, K = (a[:64] for a in vbinputs.config_sizes("C4"))
db = DeviceBatch(M, N, K, "bf16")
dev = db.plan()
os.environ["VB_TMAPS_HOST"] = "1"
host = db.plan()
del os.environ["VB_TMAPS_HOST"]
db.bind(dev)
db.bind(host)
torch.cuda.synchronize()
a, b = dev.debug_tmaps(), host.debug_tmaps()
diff = np.nonzero((a != b).any(axis=2))
print("differing maps:", diff[0].size, "of", int((b != 0).any(axis=2).sum()))
for g, w in list(zip(*diff))[:6]:
    wa, wb = a[g, w].view(np.uint32), b[g, w].view(np.uint32)
    print(f"GEMM {g} (M,N,K)=({M[g]},{N[g]},{K[g]}) map {w}")
    for i in np.nonzero(wa != wb)[0]:
        print(f"   word {i:2d}: device {wa[i]:#010x}  host {wb[i]:#010x}")
    print("   host words:", " ".join(f"{x:08x}" for x in wb))

# which host-encoded maps carry word-2 bit 21, against their dims / stride / box
rows = []
for g in range(b.shape[0]):
    for w in range(b.shape[1]):
        wb = b[g, w].view(np.uint32)
        if not wb.any():
            continue
        d0, d1, st = int(wb[8]) + 1, int(wb[9]) + 1, int(wb[3]) * 16
        rows.append((w, d0, d1, st, (int(wb[2]) >> 21) & 1, int(wb[2]), int((a[g, w] != b[g, w]).any())))
for r in sorted(set(rows), key=lambda r: (r[4], r[0], r[1]))[:400]:
    print("map %d dims %5d x %5d stride %6d  bit21 %d  word2 %#010x  differs %d" % r)
