"""GPU parity on exactly the paths bench.py times, with both error checks.

bench.py runs every config with VB_BATCH_AUTO (the random forest of P272-274 picks the
heuristic): C2 fp32 -> binary, C3 -> threshold, C4 -> binary with the 2-SM pair launch plus
the 1-SM launch, C5 -> threshold.  Each config here is run at its FULL size under AUTO and under
both heuristics explicitly; GEMMs are checked against the fp64 oracle by the normwise
tolerance (BASELINE.json) and by the elementwise forward-error bound (gpu_helpers.check_bound),
and the achieved errors are recorded (conftest writes them to $VB_PARITY_OUT).
The AUTO plan's device copy must also equal the oracle plan of the policy it chose.
"""
import numpy as np
import pytest
import torch

import vbinputs
from oracle import plan_ref as pr
from gpu_helpers import check_recorded

pytestmark = pytest.mark.gpu

if torch.cuda.is_available():
    from paper_conf_ppopp_li0yjl19_b200.batch import DeviceBatch
    import paper_conf_ppopp_li0yjl19_b200 as vb

SEED = 0
POL = {"auto": None, "threshold": 0, "binary": 1}
TAB = {"C2": pr.B200_F32, "C3": pr.B200_TC, "C4": pr.B200_TC, "C5": pr.B200_TC}


def _sample(cfg, M, N, K, plan_rows, table):
    """Every GEMM for C2/C3; for C4/C5 the largest/smallest/first/last GEMMs, random ones, and
    at least 4 GEMMs of every strategy the plan uses (so pair and 1-SM tiles are both checked)."""
    if cfg in ("C2", "C3"):
        return list(range(len(M)))
    work = 2 * M * N * K
    rng = np.random.default_rng(11)
    idx = {int(np.argmax(work)), int(np.argmin(work)), 0, len(M) - 1}
    idx |= set(int(i) for i in rng.choice(len(M), 24 if cfg == "C4" else 40, replace=False))
    rows = np.asarray(plan_rows) % len(table.rows)
    for r in np.unique(rows):
        cand = np.flatnonzero(rows == r)
        idx |= set(int(i) for i in rng.choice(cand, min(4, len(cand)), replace=False))
    return sorted(idx)


@pytest.mark.parametrize("cfg", ["C2", "C3", "C4", "C5"])
@pytest.mark.parametrize("policy", ["auto", "threshold", "binary"])
def test_benched_config_full_size(cfg, policy):
    M, N, K = vbinputs.config_sizes(cfg)
    dtype = vbinputs.CONFIGS[cfg]["dtype"]
    ab = "conv" if cfg == "C3" else "random"
    db = DeviceBatch(M, N, K, dtype)
    db.fill(SEED, ab)
    plan = db.plan(vb.VB_BATCH_AUTO if POL[policy] is None else POL[policy])
    chosen = plan.policy()
    ex = plan.export()
    ref = pr.plan(M, N, K, TAB[cfg], chosen)
    assert list(ex["block_ptr"]) == ref.enc.Tile and list(ex["gemm_strategy"]) == ref.enc.Tiling
    assert list(ex["tile_gemm"]) == ref.enc.GEMM
    assert list(ex["tile_y"]) == ref.enc.Y and list(ex["tile_x"]) == ref.enc.X
    info = plan.info()
    if cfg == "C4":   # the benched C4 path: 2-SM pair launch + 1-SM launch
        assert info["launches_per_exec"] == 3, info
    db.run(plan)
    torch.cuda.synchronize()
    idx = _sample(cfg, M, N, K, ex["gemm_strategy"], TAB[cfg])
    r = check_recorded(f"{cfg}/{policy}", db, idx, SEED, ab)
    r["policy_run"] = {0: "threshold", 1: "binary", 2: "none"}[chosen]
    r["launches_per_exec"] = info["launches_per_exec"]
    r["strategies_checked"] = sorted({TAB[cfg].rows[int(ex['gemm_strategy'][g]) % len(TAB[cfg].rows)].name
                                      for g in idx})
