"""Per-CTA exit spread of C4's two launches (pair launch: GEMMs with M >= 256; 1-SM launch: the
rest), measurement tool; needs the -DVB_TIMELINE_ALL build:
    python paper_conf_ppopp_li0yjl19_b200/build.py -DVB_TIMELINE_ALL --out=libvbgemm_ctatl.so
    VB_LIB=paper_conf_ppopp_li0yjl19_b200/libvbgemm_ctatl.so python scripts/tl_c4.py"""
import ctypes, os, sys
sys.path.insert(0, os.getcwd())
import numpy as np, torch, vbinputs
import paper_conf_ppopp_li0yjl19_b200 as vb
from paper_conf_ppopp_li0yjl19_b200 import _native as nv
from paper_conf_ppopp_li0yjl19_b200.batch import DeviceBatch
nv.lib.vb_debug_set_trace.argtypes = [ctypes.c_void_p]
M, N, K = vbinputs.config_sizes("C4")
for name, sel in (("pair", M >= 256), ("single", M < 256)):
    db = DeviceBatch(M[sel], N[sel], K[sel], "bf16"); db.fill(0)
    plan = db.plan(vb.VB_BATCH_BINARY); db.bind(plan)
    buf = torch.zeros(2 * 148 + 8, dtype=torch.int64, device="cuda")
    for rep in range(3):
        buf.zero_(); nv.lib.vb_debug_set_trace(buf.data_ptr())
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s.record(); db.run_bound(plan); e.record(); torch.cuda.synchronize()
        nv.lib.vb_debug_set_trace(None)
    v = buf.cpu().numpy()[:2 * 148].reshape(-1, 2); v = v[v[:, 0] > 0]
    t0 = v[:, 0].min(); ent = (v[:, 0] - t0) / 1e3; ext = (v[:, 1] - t0) / 1e3
    q = np.percentile(ext, [0, 10, 50, 90, 100])
    print(name, f"event {s.elapsed_time(e)*1e3:.1f} us, CTAs {len(v)}, exit min/p10/p50/p90/max", np.round(q, 1))
    del db, plan; torch.cuda.empty_cache()
