"""Multi-GPU shard path on one GPU: every LPT shard of the headline C5
batch at N = 2 and N = 8 -- the rank's GEMMs with their GLOBAL ids, drawn by the device
generator keyed on those ids, exactly as bench.py's rank path builds them -- is planned and
executed through the C-ABI and checked against the fp64 oracle; the shards partition the batch."""
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

import bench  # noqa: E402  (repo root is on sys.path via conftest)

SEED = 0


@pytest.mark.parametrize("world", [2, 8])
def test_lpt_shards_of_c5_through_exec(world):
    M, N, K = vbinputs.config_sizes("C5")
    rank_of = vb.shard_lpt(M, N, K, world)
    assert list(rank_of) == pr.shard_lpt(M, N, K, world)
    seen = []
    loads = []
    for rank in range(world):
        idx = bench.shard_indices(M, N, K, world, rank, vb.shard_lpt)
        assert np.all(np.diff(idx) > 0)
        seen.append(idx)
        loads.append(int((2 * M[idx] * N[idx] * K[idx]).sum()))
        db = DeviceBatch(M[idx], N[idx], K[idx], "bf16", gemm_ids=idx)
        db.fill(SEED)
        plan = db.plan(vb.VB_BATCH_AUTO)
        db.run(plan)
        torch.cuda.synchronize()
        w = 2 * db.M * db.N * db.K
        rng = np.random.default_rng(rank)
        local = sorted({0, db.batch - 1, int(np.argmax(w)), int(np.argmin(w))} |
                       set(int(i) for i in rng.choice(db.batch, 8, replace=False)))
        check_recorded(f"C5-shard/N{world}/r{rank}", db, local, SEED, "random")
        del db, plan
        torch.cuda.empty_cache()
    allidx = np.sort(np.concatenate(seen))
    assert np.array_equal(allidx, np.arange(len(M)))           # a partition: every GEMM exactly once
    assert max(loads) / (sum(loads) / world) < 1.02            # FLOP-balanced
