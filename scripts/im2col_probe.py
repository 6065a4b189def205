import sys, os, json, numpy as np, torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import vbinputs
import paper_conf_ppopp_li0yjl19_b200 as vb
from paper_conf_ppopp_li0yjl19_b200.batch import ConvBatch, DeviceBatch

def timeit(db, plan, n=20):
    db.bind(plan); db.run_bound(plan); torch.cuda.synchronize()
    fl = torch.empty(int(512e6), dtype=torch.uint8, device="cuda")
    ts = []
    for _ in range(n):
        fl.fill_(1)
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s.record(); db.run_bound(plan); e.record(); torch.cuda.synchronize()
        ts.append(s.elapsed_time(e))
    return float(np.median(ts))

for nb in (8, 32):
    convs = [c for c in vbinputs.googlenet_convs(nb=nb) if c["KH"] == 1]
    cb = ConvBatch(convs, "bf16"); cb.fill(0, "conv")
    pc = cb.plan(vb.VB_BATCH_THRESHOLD)
    t_conv = timeit(cb, pc)
    M = [c["nb"] * c["H"] * c["W"] for c in convs]; N = [c["Cout"] for c in convs]; K = [c["Cin"] for c in convs]
    db = DeviceBatch(M, N, K, "bf16"); db.fill(0, "conv")
    pg = db.plan(vb.VB_BATCH_THRESHOLD)
    t_gemm = timeit(db, pg)
    print(json.dumps({"nb": nb, "n": len(convs), "im2col_ms": t_conv, "tiled_ms": t_gemm,
                      "tiles_conv": pc.info()["n_tiles"], "tiles_gemm": pg.info()["n_tiles"]}))
    # 3x3 and 5x5 only
    convs = [c for c in vbinputs.googlenet_convs(nb=nb) if c["KH"] > 1]
    cb = ConvBatch(convs, "bf16"); cb.fill(0, "conv")
    pc = cb.plan(vb.VB_BATCH_THRESHOLD)
    t_conv = timeit(cb, pc)
    M = [c["nb"] * c["H"] * c["W"] for c in convs]; N = [c["Cout"] for c in convs]; K = [c["KH"]*c["KW"]*c["Cin"] for c in convs]
    db = DeviceBatch(M, N, K, "bf16"); db.fill(0, "conv")
    pg = db.plan(vb.VB_BATCH_THRESHOLD)
    t_gemm = timeit(db, pg)
    print(json.dumps({"nb": nb, "kxk": len(convs), "im2col_ms": t_conv, "explicit_pixels_x_K_gemm_ms": t_gemm}))
