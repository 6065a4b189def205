"""Multi-process (world size 2, gloo on CPU) checks of the multi-GPU host logic in bench.py:
identical LPT shards on every rank (no collective needed to agree), the shards partition the
batch, and the timing gather (max over ranks) / count reduction (sum) helpers."""
import os
import socket

import numpy as np
import torch.distributed as dist
import torch.multiprocessing as mp

import vbinputs


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _worker(rank, world, port, out):
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK=str(rank), WORLD_SIZE=str(world))
    import torch
    import bench
    import paper_conf_ppopp_li0yjl19_b200 as vb
    dist.init_process_group("gloo", rank=rank, world_size=world)
    M, N, K = vbinputs.config_sizes("C5")
    idx = bench.shard_indices(M, N, K, world, rank, vb.shard_lpt)
    # every rank gathers everybody's shard and the work per rank
    sizes = [None] * world
    dist.all_gather_object(sizes, idx.tolist())
    work = float((2 * M[idx] * N[idx] * K[idx]).sum())
    mx = bench.gather_max([float(rank + 1), work], world)
    sm = bench.gather_sum([work, 1.0], world)
    out[rank] = (sizes, mx, sm, work)
    dist.barrier()
    dist.destroy_process_group()


def test_lpt_shards_partition_and_gather_world2():
    world = 2
    port = _free_port()
    mgr = mp.Manager()
    out = mgr.dict()
    mp.spawn(_worker, args=(world, port, out), nprocs=world, join=True)
    M, N, K = vbinputs.config_sizes("C5")
    sizes0, mx0, sm0, w0 = out[0]
    sizes1, mx1, sm1, w1 = out[1]
    assert sizes0 == sizes1                       # both ranks see the same partition
    allg = sorted(sizes0[0] + sizes0[1])
    assert allg == list(range(len(M)))            # disjoint and complete
    total = float((2 * M * N * K).sum())
    assert abs(sm0[0] - total) / total < 1e-12 and sm0[1] == 2.0
    assert mx0[0] == 2.0 and mx0[1] == max(w0, w1)
    assert abs(w0 - w1) / total < 0.01           # FLOP-balanced
