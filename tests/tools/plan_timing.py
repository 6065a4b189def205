"""Planning cost per config: the C++ planner (tiling + batching + encoding,
host-only plan: no device upload) against the Python reference planner of oracle/plan_ref.py on
the same batch.  CPU only; prints one JSON line per config and policy."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import vbinputs  # noqa: E402
from oracle import plan_ref as pr  # noqa: E402
import paper_conf_ppopp_li0yjl19_b200 as vb  # noqa: E402
from paper_conf_ppopp_li0yjl19_b200 import _native as nv  # noqa: E402

TABLE = {"f32": (vb.VB_TABLE_B200_FFMA, pr.B200_F32), "bf16": (vb.VB_TABLE_B200_TC, pr.B200_TC)}
for cfg in ("C1", "C2", "C3", "C4", "C5"):
    info = vbinputs.CONFIGS[cfg]
    dt = info["dtype"]
    M, N, K = vbinputs.config_sizes(cfg)
    ld = lambda c: vbinputs.padded_ld(c, dt)  # noqa: E731
    tid, tref = TABLE[dt]
    for pol, pname in ((vb.VB_BATCH_THRESHOLD, "threshold"), (vb.VB_BATCH_BINARY, "binary")):
        reps = 5 if len(M) < 10000 else 2
        t0 = time.perf_counter()
        for _ in range(reps):
            p = nv.plan_vbatched(M, N, K, ld(K), ld(N), ld(N), dt, pol, device=-1, table_id=tid)
        cpp_ms = (time.perf_counter() - t0) / reps * 1e3
        info_p = p.info()
        t0 = time.perf_counter()
        ref = pr.plan(M, N, K, tref, pol, es=vbinputs.elem_size(dt))
        py_ms = (time.perf_counter() - t0) * 1e3
        assert len(ref.tiles) == info_p["n_tiles"]
        print(json.dumps({"config": cfg, "policy": pname, "batch": int(len(M)), "tiles": info_p["n_tiles"],
                          "blocks": info_p["n_blocks"], "cpp_planner_ms": round(cpp_ms, 3),
                          "python_reference_planner_ms": round(py_ms, 1)}), flush=True)
