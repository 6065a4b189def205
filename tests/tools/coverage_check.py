"""Coverage-counter check (SURVEY.md §4 GPU row: "debug coverage-counter build: each C element
written exactly once").  Run with the -DVB_COVERAGE library:

    VB_LIB=paper_conf_ppopp_li0yjl19_b200/libvbgemm_cov.so python tests/tools/coverage_check.py

For each batch (both policies): zero an int32 counter per element of the C arena, run
vb_exec_vbatched, and require counter == 1 on every element of every C matrix and 0 everywhere
else (row padding, gaps between matrices).  Cases: ragged random shapes in bf16 / fp16 / fp32
(every size class, K = 0 GEMMs, 1-wide), the 2-SM pair tiles + 1-SM tiles of a compute-bound
batch, a GoogleNet module as implicit-GEMM convolutions, and C4 at full size.
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)
assert "libvbgemm_cov" in os.environ.get("VB_LIB", ""), "run with VB_LIB=.../libvbgemm_cov.so"

import numpy as np  # noqa: E402
import torch  # noqa: E402

import vbinputs  # noqa: E402
from paper_conf_ppopp_li0yjl19_b200 import _native as nv  # noqa: E402
from paper_conf_ppopp_li0yjl19_b200.batch import ConvBatch, DeviceBatch  # noqa: E402


def check(name, db, plan):
    counts = torch.zeros(db.C.numel(), dtype=torch.int32, device=db.C.device)
    nv.debug_set_coverage(0, counts.data_ptr(), db.C.data_ptr(), db.es)
    db.run(plan)
    torch.cuda.synchronize()
    nv.debug_set_coverage(0, 0, 0, 0)
    expect = torch.zeros_like(counts)
    for g in range(db.batch):
        m, n, ld = int(db.M[g]), int(db.N[g]), int(db.ldc[g])
        if m and n:
            torch.as_strided(expect, (m, n), (ld, 1), int(db.offC[g])).fill_(1)
    bad = int((counts != expect).sum())
    res = {"case": name, "elements": int(expect.sum()), "wrong_counts": bad, "max_count": int(counts.max()),
           "n_tiles": plan.info()["n_tiles"], "launches_per_exec": plan.info()["launches_per_exec"]}
    print(json.dumps(res), flush=True)
    return bad == 0


ok = True
rng = np.random.default_rng(77)
r = rng.integers(1, 700, (200, 3))
r[:10, 0] = 1
r[10:20, 1] = 1
r[20:30, 2] = 0
for dtype in ("bf16", "f16", "f32"):
    for pol in (0, 1):
        db = DeviceBatch(r[:, 0], r[:, 1], r[:, 2], dtype)
        db.fill(1)
        ok &= check(f"ragged200/{dtype}/p{pol}", db, db.plan(pol))
M = np.array([512, 300, 777, 1024, 100, 256]); N = np.array([512, 260, 640, 1000, 96, 512])
K = np.array([2048, 1500, 1900, 4096, 3000, 2000])
db = DeviceBatch(M, N, K, "bf16")
db.fill(1)
ok &= check("pair+single/bf16", db, db.plan(0, tlp_threshold=1))
cb = ConvBatch(vbinputs.googlenet_convs(nb=2, module="4e"), "bf16")
cb.fill(1, "conv")
ok &= check("conv-4e-nb2/bf16", cb, cb.plan(0))
# every strategy row of the tcgen05 table forced (pair, 1-SM and swap-AB tiles) on ragged shapes
from oracle import plan_ref as pr  # noqa: E402  (test infrastructure: enumerates the forced tiles)
rows = [g % len(pr.B200_TC.rows) for g in range(len(r))]
db = DeviceBatch(r[:, 0], r[:, 1], np.maximum(r[:, 2], 1), "bf16")
db.fill(1)
tl = pr.enumerate_tiles(db.M, db.N, db.K, rows, pr.B200_TC)
pair = [pr.B200_TC.rows[rows[t.gemm]].ctas == 2 for t in tl]
tl = [t for t, q in zip(tl, pair) if q] + [t for t, q in zip(tl, pair) if not q]
plan = nv.plan_from_schedule(db.M, db.N, db.K, db.lda, db.ldb, db.ldc, rows, 256, list(range(len(tl) + 1)),
                             [t.gemm for t in tl], [t.y for t in tl], [t.x for t in tl], dtype="bf16", device=0,
                             table_id=nv.VB_TABLE_B200_TC)
ok &= check("every-row-forced/bf16", db, plan)
M, N, K = vbinputs.config_sizes("C4")
db = DeviceBatch(M, N, K, "bf16")
db.fill(1)
ok &= check("C4/bf16/auto", db, db.plan(nv.VB_BATCH_AUTO))
sys.exit(0 if ok else 1)
