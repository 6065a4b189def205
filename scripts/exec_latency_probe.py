"""Per-call time of vb_exec_vbatched (bind-time prep kernel + GEMM kernel, no event between them)
on the small configs, L2 flushed before each call, plus the same in a CUDA graph."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import vbinputs  # noqa: E402
import paper_conf_ppopp_li0yjl19_b200 as vb  # noqa: E402
from paper_conf_ppopp_li0yjl19_b200.batch import DeviceBatch  # noqa: E402

flush = torch.empty(int(512e6), dtype=torch.uint8, device="cuda")
for cfg in sys.argv[1:] or ["C3", "C1", "C2"]:
    info = vbinputs.CONFIGS[cfg]
    M, N, K = vbinputs.config_sizes(cfg)
    db = DeviceBatch(M, N, K, info["dtype"])
    db.fill(0, info["ab"])
    plan = db.plan(vb.VB_BATCH_AUTO)
    s = torch.cuda.current_stream()
    for _ in range(3):
        db.run(plan, s)
    ts = []
    for _ in range(50):
        flush.fill_(1)
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(s)
        db.run(plan, s)
        b.record(s)
        ts.append((a, b))
    torch.cuda.synchronize()
    v = [a.elapsed_time(b) * 1e3 for a, b in ts]
    g_stream = torch.cuda.Stream()
    graph = torch.cuda.CUDAGraph()
    g_stream.wait_stream(s)
    with torch.cuda.stream(g_stream):
        db.run(plan, g_stream)
        torch.cuda.synchronize()
        with torch.cuda.graph(graph, stream=g_stream):
            db.run(plan, g_stream)
    torch.cuda.synchronize()
    gs = []
    for _ in range(50):
        flush.fill_(1)
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(s)
        graph.replay()
        b.record(s)
        gs.append((a, b))
    torch.cuda.synchronize()
    w = [a.elapsed_time(b) * 1e3 for a, b in gs]
    print(f"{cfg} {os.path.basename(os.environ.get('VB_LIB', 'libvbgemm.so'))}: exec p50 {np.median(v):.1f} us, "
          f"graph p50 {np.median(w):.1f} us", flush=True)
