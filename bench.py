#!/usr/bin/env python
"""bench.py — variable-size batched GEMM on B200 (coordinated tiling + batching, PPoPP'19).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference] [--config C5]

One JSON line on rank 0 (BASELINE.json metric: "vbatched GEMM effective TFLOP/s (fp32, bf16)
at 1/2/4/8 B200; % of roofline").

* Workload (headline): C5 = 65536 mixed-size bf16 GEMMs, M, N, K log-uniform on [16, 1024],
  alpha/beta random (beta != 0), FLOP-balanced over the ranks by LPT on 2*M*N*K (no
  collective on the data path; NCCL only for the barrier and the timing gather).
  The total batch is fixed as N grows -> "scaling": "strong".
* step = one vb_exec_vbatched over the rank's shard with inputs resident in HBM:
  vb_plan_bind (tensor-map prep kernel) + vb_exec_bound (the persistent GEMM kernel), with a
  CUDA event between the two that gives the GEMM kernel's own duration for the roofline (the
  event also keeps the GEMM kernel from starting its setup under the prep kernel, as its
  programmatic launch does in a plain vb_exec_vbatched call -- see cuda_graph_step_ms and e2e).
  Planning (tiling + batching engines, descriptor upload) happens once per batch shape and is
  reported separately as plan_ms.  The inputs (30.5 GB) are far larger than L2 (126 MB).
* value = sum over ranks of 2*M*N*K / max over ranks of the timed region (CUDA events on the
  launching stream, barrier + synchronize on both sides).
* e2e = same metric through the same C-ABI call with HOST (pinned) buffers: every step copies
  A, B, C, alpha, beta host->device, runs, and copies C device->host.
* roofline = the GEMM kernel: algorithmic (compulsory) bytes / its event-timed duration vs the
  measured HBM copy bandwidth (MEASURED_PEAKS.json).
* cpu_baseline / --impl reference = the fp64 C oracle (oracle/gemm_ref.c) on the host cores,
  on a bounded random sample of the same GEMMs.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

import vbinputs  # noqa: E402

METRIC = "vbatched GEMM effective TFLOP/s (fp32, bf16) at 1/2/4/8 B200; % of roofline"
UNIT = "TFLOP/s"
PEAKS_FALLBACK = {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0, "bf16_tflops_sustained": 1400.0, "sm_max_mhz": 1965.0}
FFMA_LANES_PER_SM = 128      # fp32 FMA units per SM (Blackwell), 2 flop each


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        d["_source"] = "measured"
        return d
    d = dict(PEAKS_FALLBACK)
    d["_source"] = "fallback"
    return d


# ----------------------------------------------------------------------------- distributed
def dist_env():
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return world, rank, local


def dist_init(world, backend):
    import torch.distributed as dist
    if world > 1 and not dist.is_initialized():
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        os.environ.setdefault("MASTER_PORT", "29511")
        dist.init_process_group(backend=backend)
    return dist


def shard_indices(M, N, K, world, rank, shard_fn):
    """GEMM ids of this rank (ascending); every rank computes the identical LPT map."""
    if world == 1:
        return np.arange(len(M), dtype=np.int64)
    rank_of = np.asarray(shard_fn(M, N, K, world))
    return np.nonzero(rank_of == rank)[0].astype(np.int64)


def gather_max(values, world, device=None):
    """Element-wise max over ranks of a small float vector (NCCL all_gather off the hot path)."""
    if world == 1:
        return list(values)
    import torch
    import torch.distributed as dist
    t = torch.tensor(values, dtype=torch.float64, device=device)
    out = [torch.zeros_like(t) for _ in range(world)]
    dist.all_gather(out, t)
    return [max(float(o[i]) for o in out) for i in range(len(values))]


def gather_sum(values, world, device=None):
    if world == 1:
        return list(values)
    import torch
    import torch.distributed as dist
    t = torch.tensor(values, dtype=torch.float64, device=device)
    dist.all_reduce(t)
    return [float(x) for x in t.tolist()]


# ----------------------------------------------------------------------------- clocks
class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled every 100 ms during the timed region."""
    Q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu_index):
        self.gpu = gpu_index
        self.lines = []
        self.proc = None

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.gpu), f"--query-gpu={self.Q}",
                                          "--format=csv,noheader,nounits", "-lms", "100"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.th = threading.Thread(target=self._read, daemon=True)
            self.th.start()
        except FileNotFoundError:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        time.sleep(0.25)
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except subprocess.TimeoutExpired:
            self.proc.kill()
        sm, smax, reasons, power = [], [], set(), []
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            parts = [p.strip() for p in ln.split(",")]
            if len(parts) < 7:
                continue
            try:
                sm.append(float(parts[0]))
                smax.append(float(parts[1]))
                power.append(float(parts[2]))
            except ValueError:
                continue
            for nm, v in zip(names, parts[3:7]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        loaded = [s for s in sm if smax and s > 0.5 * max(smax)] or sm
        return {"sm_mhz": statistics.median(loaded) if loaded else None,
                "sm_max_mhz": max(smax) if smax else None, "reasons": sorted(reasons),
                "samples": len(sm), "power_w_max": max(power) if power else None}


# ----------------------------------------------------------------------------- roofline
def roofline_for(dtype, flops, nbytes, t_s, peaks, sustained=False):
    """Bound and fraction of the per-batch roofline t_roof = max(F/P, B/BW)."""
    bw = peaks["hbm_gbs"] * 1e9
    if dtype == "f32":
        p = FFMA_LANES_PER_SM * 2 * 148 * peaks.get("sm_max_mhz", 1965.0) * 1e6
        compute_bound = "alu"
    else:
        p = (peaks["bf16_tflops_sustained"] if sustained else peaks["bf16_tflops"]) * 1e12
        compute_bound = "tensor"
    t_c, t_m = flops / p, nbytes / bw
    if t_m >= t_c:
        return {"bound": "hbm", "achieved": nbytes / t_s / 1e9, "peak": peaks["hbm_gbs"], "unit": "GB/s",
                "frac": (nbytes / t_s) / bw, "t_roof_us": t_m * 1e6}
    return {"bound": compute_bound, "achieved": flops / t_s / 1e12, "peak": p / 1e12, "unit": "TFLOP/s",
            "frac": (flops / t_s) / p, "t_roof_us": t_c * 1e6}


def aggregate_roofline(dtype, flops_all, bytes_all, makespan_s, t_roof_max_us, world, peaks):
    """N > 1: the job's roofline is the slowest rank's t_roof; `frac` is the
    whole-job achieved rate over N times the per-GPU peak (= sum of the ranks' bytes or flops /
    makespan / (N * peak)), and `frac_makespan` = max over ranks of t_roof / makespan."""
    r = roofline_for(dtype, flops_all, bytes_all, makespan_s, peaks)
    one = r["peak"]
    r["peak"] = one * world
    r["frac"] = r["achieved"] / r["peak"]
    r["t_roof_us"] = t_roof_max_us
    r["frac_makespan"] = t_roof_max_us * 1e-6 / makespan_s
    r["aggregate"] = f"{world} ranks: achieved = sum over ranks / makespan, peak = {world} x {one}"
    return r


def committed_traffic(cfg):
    """dram read+write bytes per launch from the committed ncu capture (profiles/), or None."""
    p = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if not os.path.exists(p):
        return None
    with open(p) as f:
        d = json.load(f)
    return d.get(cfg, {}).get("dram_bytes_per_launch")


# ----------------------------------------------------------------------------- oracle timing
def oracle_sample(M, N, K, dtype, ab_mode, seed, rng, target_flops):
    """Random GEMMs of the workload (without replacement) until ~target_flops; fp64 inputs."""
    order = rng.permutation(len(M))
    pick, tot = [], 0
    for g in order:
        pick.append(int(g))
        tot += 2 * int(M[g]) * int(N[g]) * int(K[g])
        if tot >= target_flops:
            break
    As, Bs, Cs = [], [], []
    for g in pick:
        m, n, k = int(M[g]), int(N[g]), int(K[g])
        As.append(vbinputs.matrix_f64_fast(seed, g, vbinputs.OP_A, m, k, dtype))
        Bs.append(vbinputs.matrix_f64_fast(seed, g, vbinputs.OP_B, k, n, dtype))
        Cs.append(vbinputs.matrix_f64_fast(seed, g, vbinputs.OP_C, m, n, dtype))
    al, be = vbinputs.alpha_beta(seed, pick, ab_mode)
    return pick, As, Bs, Cs, al.astype(np.float64), be.astype(np.float64), tot


def time_oracle(M, N, K, dtype, ab_mode, seed, seconds=10.0, steps=1, warmup=0):
    """Time the fp64 oracle (as it stands) on a bounded sample; returns a result dict."""
    from oracle import gemm as og
    # every host core: torchrun sets OMP_NUM_THREADS=1 per rank, but the oracle runs on rank 0
    # alone after the GPU work of every rank is done
    cores = os.cpu_count() or og.max_threads()
    rng = np.random.default_rng(12345)
    # calibrate the rate on a small sample, then size the per-step sample for `seconds`
    pick, As, Bs, Cs, al, be, f0 = oracle_sample(M, N, K, dtype, ab_mode, seed, rng, 2e9)
    t0 = time.perf_counter()
    og.gemm_batch(As, Bs, [c.copy() for c in Cs], al, be, nthreads=cores)
    rate = f0 / max(time.perf_counter() - t0, 1e-6)
    pick, As, Bs, Cs, al, be, fl = oracle_sample(M, N, K, dtype, ab_mode, seed, np.random.default_rng(777),
                                                 rate * seconds)
    times = []
    for it in range(warmup + steps):
        cw = [c.copy() for c in Cs]
        t0 = time.perf_counter()
        og.gemm_batch(As, Bs, cw, al, be, nthreads=cores)
        dt = time.perf_counter() - t0
        if it >= warmup:
            times.append(dt)
    tot = sum(times)
    return {"value": fl * len(times) / tot / 1e12, "unit": UNIT, "cores": cores, "kind": "oracle",
            "sample": f"{len(pick)} of {len(M)} GEMMs drawn uniformly at random ({fl / 1e9:.1f} GFLOP, "
                      f"{fl / (2 * (M * N * K).sum()) * 100:.2f}% of the workload's FLOPs), fp64 triple loop, "
                      f"{cores} OpenMP threads", "ms_per_step": tot / len(times) * 1e3}


# ----------------------------------------------------------------------------- our GPU arm
def run_config(cfg, args, world, rank, local, peaks, dist_device, headline=True):
    import torch
    import paper_conf_ppopp_li0yjl19_b200 as vb
    from paper_conf_ppopp_li0yjl19_b200.batch import DeviceBatch

    dev = torch.device("cuda", local)
    if cfg == "C3i":   # the C3 convolutions as implicit GEMMs (vb_plan_conv, NEXT-3)
        from paper_conf_ppopp_li0yjl19_b200.batch import ConvBatch
        dtype, ab = "bf16", "conv"
        convs = vbinputs.googlenet_convs(nb=args.nb)
        idx = np.asarray(shard_indices(np.array([1] * len(convs)), np.array([1] * len(convs)),
                                       np.array([1] * len(convs)), world, rank, vb.shard_lpt)) if world > 1 else \
            np.arange(len(convs))
        db = ConvBatch([convs[i] for i in idx], dtype, device=dev, gemm_ids=idx)
    else:
        info = vbinputs.CONFIGS[cfg]
        dtype, ab = info["dtype"], info["ab"]
        nb = args.nb if cfg == "C3" else 1
        M, N, K = vbinputs.config_sizes(cfg, nb=nb)
        idx = shard_indices(M, N, K, world, rank, vb.shard_lpt)
        db = DeviceBatch(M[idx], N[idx], K[idx], dtype, device=dev, gemm_ids=idx)
    db.fill(args.seed, ab)
    torch.cuda.synchronize(dev)
    # planning cost (host tiling + batching engines, device descriptor expansion, tensor maps):
    # the first plan of the process, then the steady state of re-planning (the paper's on-line
    # case, P272-274), median of 5; the last plan is the one that runs
    plan_times = []
    for _ in range(6):
        t0 = time.perf_counter()
        plan = db.plan(vb.POLICIES[args.policy])
        plan_times.append((time.perf_counter() - t0) * 1e3)
    plan_ms = float(np.median(plan_times[1:]))
    plan_first_ms = plan_times[0]
    pinfo = plan.info()
    flops = db.flops()
    beta_nz = db.beta[:db.batch].cpu().numpy() != 0
    nbytes = db.algorithmic_bytes(beta_nz)
    small = db.arena_bytes() < 4 * 126e6          # inputs not >> L2: flush between steps
    flush = torch.empty(int(512e6), dtype=torch.uint8, device=dev) if small else None
    stream = torch.cuda.current_stream(dev)

    def step():
        db.bind(plan, stream)
        ev_mid = torch.cuda.Event(enable_timing=True)
        ev_mid.record(stream)
        db.run_bound(plan, stream)
        return ev_mid

    steps = args.steps if headline else max(5, min(args.steps, 20))
    for _ in range(max(args.warmup, 3)):
        step()
    torch.cuda.synchronize(dev)
    if world > 1:
        import torch.distributed as dist
        dist.barrier()
    torch.cuda.synchronize(dev)
    clocks = ClockSampler(local) if (headline and rank == 0) else None
    if clocks:
        clocks.start()
        time.sleep(0.3)
    starts, mids, ends = [], [], []
    for _ in range(steps):
        if flush is not None:
            flush.fill_(1)                          # evict L2 between timed iterations
        s = torch.cuda.Event(enable_timing=True)
        s.record(stream)
        m = step()
        e = torch.cuda.Event(enable_timing=True)
        e.record(stream)
        starts.append(s); mids.append(m); ends.append(e)
    torch.cuda.synchronize(dev)
    if world > 1:
        import torch.distributed as dist
        dist.barrier()
    torch.cuda.synchronize(dev)
    clk = clocks.stop() if clocks else None
    step_list = [s.elapsed_time(e) for s, e in zip(starts, ends)]
    kern_list = [m.elapsed_time(e) for m, e in zip(mids, ends)]
    step_ms = sum(step_list) / steps
    kern_ms = sum(kern_list) / steps
    pct = lambda v, q: float(np.percentile(v, q))  # noqa: E731
    dist = {"kernel_ms_p10": pct(kern_list, 10), "kernel_ms_p50": pct(kern_list, 50),
            "kernel_ms_p90": pct(kern_list, 90), "step_ms_p10": pct(step_list, 10),
            "step_ms_p50": pct(step_list, 50), "step_ms_p90": pct(step_list, 90)}
    t_roof_rank = roofline_for(dtype, flops, nbytes, 1.0, peaks)["t_roof_us"]
    step_ms_max, kern_ms_max, plan_ms_max, t_roof_max = gather_max([step_ms, kern_ms, plan_ms, t_roof_rank], world,
                                                                    dist_device)
    flops_all, bytes_all = gather_sum([float(flops), float(nbytes)], world, dist_device)
    res = {
        "cfg": cfg, "dtype": dtype, "flops_rank": flops, "bytes_rank": nbytes, "flops": flops_all,
        "step_ms": step_ms_max, "kernel_ms": kern_ms_max, "plan_ms": plan_ms_max, "plan_first_ms": plan_first_ms,
        "value": flops_all / (step_ms_max * 1e-3) / 1e12,
        "kernel_tflops": flops_all / (kern_ms_max * 1e-3) / 1e12,
        "roofline": roofline_for(dtype, flops, nbytes, kern_ms * 1e-3, peaks) if world == 1 else
        aggregate_roofline(dtype, flops_all, bytes_all, kern_ms_max * 1e-3, t_roof_max, world, peaks),
        "plan": pinfo, "policy_chosen": {0: "threshold", 1: "binary", 2: "none"}.get(plan.policy(), "?"), "l2": "flushed (512 MB write) between steps" if small else
        f"inputs ({db.arena_bytes() / 1e9:.1f} GB per rank) >> L2 (126 MB); no flush",
        "launches": pinfo["launches_per_exec"] * steps, "clocks": clk, "batch_rank": int(db.batch),
        "dist": {k: round(v, 4) for k, v in dist.items()},
    }
    if dtype != "f32" and world == 1:
        # compute-leaning batches (C4): the fraction also against the sustained tensor peak
        rs = roofline_for(dtype, flops, nbytes, kern_ms * 1e-3, peaks, sustained=True)
        res["roofline"]["frac_vs_sustained_tensor_peak"] = rs["frac"]
        res["roofline"]["bound_vs_sustained_tensor_peak"] = rs["bound"]
    if not headline and small and world == 1:
        # the small configs also with the step (bind + exec) captured in one CUDA
        # graph and replayed (launch overhead amortised), L2 flushed outside the graph
        g_stream = torch.cuda.Stream(dev)
        graph = torch.cuda.CUDAGraph()
        g_stream.wait_stream(stream)
        with torch.cuda.stream(g_stream):
            step()
            torch.cuda.synchronize(dev)
            with torch.cuda.graph(graph, stream=g_stream):
                db.bind(plan, g_stream)
                db.run_bound(plan, g_stream)
        torch.cuda.synchronize(dev)
        gts = []
        for _ in range(steps):
            flush.fill_(1)
            s0 = torch.cuda.Event(enable_timing=True)
            e0 = torch.cuda.Event(enable_timing=True)
            s0.record(stream)
            graph.replay()
            e0.record(torch.cuda.current_stream(dev))
            torch.cuda.synchronize(dev)
            gts.append(s0.elapsed_time(e0))
        res["graph_step_ms"] = float(np.median(gts))
        del graph
    if headline and args.e2e_steps > 0:
        res["e2e"] = run_e2e(db, plan, args, world, dist_device, flops_all, stream, dev)
    del flush
    return res, db, plan


def run_e2e(db, plan, args, world, dist_device, flops_all, stream, dev):
    """Same metric through the public API with pinned HOST buffers; copies inside the timing.

    The batch is cut into ``--e2e-chunks`` contiguous GEMM ranges (equal arena bytes), each planned
    once with vb_plan_vbatched; every step then pipelines, per chunk, the H2D copy of its A, B, C,
    alpha, beta (copy stream), vb_exec_vbatched on its sub-plan (compute stream) and the D2H copy
    of its C (a third stream), ordered by CUDA events -- so host->device and device->host PCIe
    traffic overlap each other and the GEMMs.  With one chunk this is the plain sequential
    H2D + exec + D2H."""
    import torch
    import paper_conf_ppopp_li0yjl19_b200 as vb
    hA = torch.empty(db.A.shape, dtype=db.A.dtype, pin_memory=True)
    hB = torch.empty(db.B.shape, dtype=db.B.dtype, pin_memory=True)
    hC = torch.empty(db.C.shape, dtype=db.C.dtype, pin_memory=True)
    hOut = torch.empty(db.C.shape, dtype=db.C.dtype, pin_memory=True)
    hAl = torch.empty(db.alpha.shape, dtype=torch.float32, pin_memory=True)
    hBe = torch.empty(db.beta.shape, dtype=torch.float32, pin_memory=True)
    hA.copy_(db.A); hB.copy_(db.B); hC.copy_(db.C); hAl.copy_(db.alpha); hBe.copy_(db.beta)
    h2d = sum(t.numel() * t.element_size() for t in (hA, hB, hC, hAl, hBe))
    d2h = hOut.numel() * hOut.element_size()

    # chunk boundaries: equal shares of the arena bytes, in GEMM order
    nchunk = max(1, min(args.e2e_chunks, db.batch))
    per = (db.offA + db.offB + db.offC).astype(np.float64)
    cuts = [0] + [int(np.searchsorted(per, per[-1] * c / nchunk)) for c in range(1, nchunk)] + [db.batch]
    cuts = sorted(set(cuts))
    chunks = []
    for g0, g1 in zip(cuts[:-1], cuts[1:]):
        if g1 <= g0:
            continue
        sub = vb.plan_vbatched(db.M[g0:g1], db.N[g0:g1], db.K[g0:g1], db.lda[g0:g1], db.ldb[g0:g1], db.ldc[g0:g1],
                               db.dtype, plan.policy(), device=dev.index or 0)
        rng = {}
        for name, off, arena in (("A", db.offA, db.A), ("B", db.offB, db.B), ("C", db.offC, db.C)):
            lo = int(off[g0])
            hi = int(off[g1]) if g1 < db.batch else arena.numel()
            rng[name] = (lo, hi)
        chunks.append((g0, g1, sub, rng))
    n_up = max(1, int(os.environ.get("VB_E2E_UPLOAD_STREAMS", "1")))
    s_up = [torch.cuda.Stream(dev) for _ in range(n_up)]   # uploads alternate between these
    s_d2h = torch.cuda.Stream(dev)

    def step():
        prev_d2h = []
        for ci, (g0, g1, sub, rng) in enumerate(chunks):
            s_h2d = s_up[ci % n_up]
            with torch.cuda.stream(s_h2d):
                for name, dst, src in (("A", db.A, hA), ("B", db.B, hB), ("C", db.C, hC)):
                    lo, hi = rng[name]
                    dst[lo:hi].copy_(src[lo:hi], non_blocking=True)
                db.alpha[g0:g1].copy_(hAl[g0:g1], non_blocking=True)
                db.beta[g0:g1].copy_(hBe[g0:g1], non_blocking=True)
                ev_in = torch.cuda.Event()
                ev_in.record(s_h2d)
            stream.wait_event(ev_in)
            sub.exec(db.pA[g0:g1].data_ptr(), db.pB[g0:g1].data_ptr(), db.pC[g0:g1].data_ptr(),
                     db.alpha[g0:g1].data_ptr(), db.beta[g0:g1].data_ptr(), stream.cuda_stream)
            ev_out = torch.cuda.Event()
            ev_out.record(stream)
            s_d2h.wait_event(ev_out)
            with torch.cuda.stream(s_d2h):
                lo, hi = rng["C"]
                hOut[lo:hi].copy_(db.C[lo:hi], non_blocking=True)
                ev_done = torch.cuda.Event()
                ev_done.record(s_d2h)
            prev_d2h.append(ev_done)
        for ev in prev_d2h:                          # the step ends when its last result is on the host
            stream.wait_event(ev)

    step()
    torch.cuda.synchronize(dev)
    if world > 1:
        import torch.distributed as dist
        dist.barrier()
    torch.cuda.synchronize(dev)
    s = torch.cuda.Event(enable_timing=True)
    e = torch.cuda.Event(enable_timing=True)
    s.record(stream)
    for su in s_up:
        su.wait_stream(stream)
    for _ in range(args.e2e_steps):
        step()
        for su in s_up:
            su.wait_stream(stream)                   # next step's uploads after this step's results
    e.record(stream)
    torch.cuda.synchronize(dev)
    ms = s.elapsed_time(e) / args.e2e_steps
    (ms_max,) = gather_max([ms], world, dist_device)
    h2d_all, d2h_all = gather_sum([float(h2d), float(d2h)], world, dist_device)
    del hA, hB, hC, hOut, chunks
    return {"value": flops_all / (ms_max * 1e-3) / 1e12, "unit": UNIT, "h2d_bytes_per_step": int(h2d_all),
            "d2h_bytes_per_step": int(d2h_all), "ms_per_step": ms_max, "steps": args.e2e_steps,
            "chunks": len(cuts) - 1,
            "path": "vb_plan_vbatched per chunk (planned once) + per step and chunk: H2D(A,B,C,alpha,beta) on a "
                    "copy stream -> vb_exec_vbatched -> D2H(C) on a second copy stream, pinned host buffers"}


def workload_desc(cfg, args):
    if cfg == "C3i":
        return (f"the 54 GoogleNet inception branch convolutions as batched implicit GEMMs (TMA im2col, "
                f"NHWC x HWIO, bf16, nb={args.nb}); algorithmic bytes = input + weights + output")
    d = vbinputs.CONFIGS[cfg]["desc"]
    return d + (f" (nb={args.nb})" if cfg == "C3" else "")


def main_ours(args):
    import torch
    world, rank, local = dist_env()
    if not torch.cuda.is_available():
        print(json.dumps({"metric": METRIC, "error": "no CUDA device"}))
        return 1
    # VB_BENCH_SHARE_GPU=1 (testing the N > 1 code path on a one-GPU box only): every rank uses
    # cuda:0 and the gloo backend for the barrier and the timing gathers
    share = os.environ.get("VB_BENCH_SHARE_GPU") == "1"
    if share:
        local = 0
    torch.cuda.set_device(local)
    dist_init(world, "gloo" if share else "nccl")
    dist_device = torch.device("cpu") if share else torch.device("cuda", local)
    peaks = load_peaks()
    res, db, plan = run_config(args.config, args, world, rank, local, peaks, dist_device, headline=True)
    aux = {}
    cpu = None
    if world == 1 and not args.no_aux:
        del db, plan
        torch.cuda.empty_cache()
        for cfg in [c for c in ("C1", "C2", "C3", "C3i", "C4") if c != args.config]:
            r, d2, p2 = run_config(cfg, args, world, rank, local, peaks, dist_device, headline=False)
            aux[cfg] = {"workload": workload_desc(cfg, args), "dtype": r["dtype"], "value": round(r["value"], 3),
                        "kernel_tflops": round(r["kernel_tflops"], 3), "ms_per_step": round(r["step_ms"], 4),
                        "plan_ms": round(r["plan_ms"], 2), "roofline": _round(r["roofline"]), "dist": r["dist"],
                        "n_tiles": r["plan"]["n_tiles"], "n_blocks": r["plan"]["n_blocks"], "l2": r["l2"],
                        "policy": r["policy_chosen"]}
            if "graph_step_ms" in r:
                aux[cfg]["cuda_graph_step_ms"] = round(r["graph_step_ms"], 4)
            del d2, p2
            torch.cuda.empty_cache()
    if world > 1:
        import torch.distributed as dist
        dist.barrier()          # every rank's GPU work is done: rank 0 times the oracle on idle cores
    if rank == 0 and not args.no_cpu_baseline:
        info = vbinputs.CONFIGS[args.config]
        M, N, K = vbinputs.config_sizes(args.config, nb=args.nb if args.config == "C3" else 1)
        cpu = time_oracle(M, N, K, info["dtype"], info["ab"], args.seed, seconds=args.cpu_seconds)
        cpu.pop("ms_per_step", None)
    rl = res["roofline"]
    rl["traffic"] = committed_traffic(args.config) if world == 1 else None   # ncu capture is of the 1-GPU launch
    rl_out = _round(rl)
    rl_out["kernel"] = "vb_tc_kernel (persistent tcgen05 GEMM)" if res["dtype"] != "f32" else "vb_f32_kernel (FFMA)"
    rl_out["peak_source"] = f"{peaks['_source']} (MEASURED_PEAKS.json)" if peaks["_source"] == "measured" else \
        "fallback (B200_PROFILING.md)"
    line = {
        "metric": METRIC, "value": round(res["value"], 3), "unit": UNIT, "n_gpus": world, "steps": args.steps,
        "warmup": max(args.warmup, 3), "ms_per_step": round(res["step_ms"], 4), "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": res["dtype"],
        "data": "synthetic: counter-hash uniform[-1,1) inputs drawn on the device (vbinputs recipe, seed "
                f"{args.seed}); shapes per BASELINE.json configs",
        "config": {"workload": f"{args.config}: {workload_desc(args.config, args)}", "batch": int(
            len(vbinputs.config_sizes(args.config, nb=args.nb if args.config == 'C3' else 1)[0])),
            "parallelism": f"gemm-sharded x{world} (LPT on 2MNK, no data-path collective)" if world > 1 else
            "single GPU", "policy": args.policy if args.policy != "auto" else
            f"auto (random forest, P272-274) -> {res['policy_chosen']}", "table": "b200_tcgen05" if res["dtype"] != "f32" else "b200_ffma",
            "l2": res["l2"], "plan_ms": round(res["plan_ms"], 2), "plan_first_ms": round(res["plan_first_ms"], 2),
            "n_tiles_rank0": res["plan"]["n_tiles"],
            "n_blocks_rank0": res["plan"]["n_blocks"], "kernel_ms": round(res["kernel_ms"], 4),
            "kernel_tflops": round(res["kernel_tflops"], 3), "timing_distribution_rank0": res["dist"]},
        "roofline": rl_out,
        "cpu_baseline": cpu,
        "e2e": res.get("e2e"),
        "gpu_launches": res["launches"],
        "clocks": res["clocks"],
    }
    if aux:
        line["aux_configs"] = aux
    if rank == 0:
        print(json.dumps(line), flush=True)
    if world > 1:
        import torch.distributed as dist
        dist.barrier()
        dist.destroy_process_group()
    return 0


def _round(d):
    return {k: (round(v, 4) if isinstance(v, float) else v) for k, v in d.items()}


# ----------------------------------------------------------------------------- reference arm
def main_reference(args):
    world, rank, local = dist_env()
    if rank != 0:
        return 0                                   # rank 0 alone runs and prints
    info = vbinputs.CONFIGS[args.config]
    M, N, K = vbinputs.config_sizes(args.config, nb=args.nb if args.config == "C3" else 1)
    r = time_oracle(M, N, K, info["dtype"], info["ab"], args.seed, seconds=args.ref_step_seconds,
                    steps=args.steps, warmup=max(args.warmup, 3))
    line = {
        "metric": METRIC, "value": round(r["value"], 6), "unit": UNIT, "impl": "reference", "n_gpus": world,
        "steps": args.steps, "warmup": max(args.warmup, 3), "ms_per_step": round(r["ms_per_step"], 2),
        "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f64",
        "data": f"synthetic (vbinputs recipe, seed {args.seed}), host-generated",
        "config": {"workload": f"{args.config}: {workload_desc(args.config, args)}", "batch": int(len(M)),
                   "parallelism": "host CPU (fp64 oracle, OpenMP)", "policy": "n/a", "table": "n/a"},
        "cpu_baseline": {"value": round(r["value"], 6), "unit": UNIT, "cores": r["cores"], "kind": "oracle",
                         "sample": r["sample"]},
        "e2e": {"value": round(r["value"], 6), "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
        "gpu_launches": 0,
    }
    print(json.dumps(line), flush=True)
    return 0


def spawn_ranks(n, argv):
    """`bench.py --gpus N` without a launcher: start N ranks (one process per GPU) through
    torch.distributed.run on 127.0.0.1, exactly as the driver's torchrun launch would, and
    return their exit status (rank 0 prints the JSON line)."""
    import socket
    with socket.socket() as so:
        so.bind(("127.0.0.1", 0))
        port = so.getsockname()[1]
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={n}",
           "--master-addr=127.0.0.1", f"--master-port={port}", os.path.abspath(__file__)] + argv
    return subprocess.call(cmd)


def main(argv=None):
    ap = argparse.ArgumentParser(description=__doc__, formatter_class=argparse.RawDescriptionHelpFormatter)
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=30)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", choices=["ours", "reference"], default="ours")
    ap.add_argument("--config", default="C5", choices=["C1", "C2", "C3", "C4", "C5"])
    ap.add_argument("--policy", default="auto", choices=["auto", "threshold", "binary", "none"])
    ap.add_argument("--nb", type=int, default=1, help="image batch for C3")
    ap.add_argument("--seed", type=int, default=0)
    ap.add_argument("--e2e-steps", type=int, default=3)
    ap.add_argument("--e2e-chunks", type=int, default=8)
    ap.add_argument("--cpu-seconds", type=float, default=10.0)
    ap.add_argument("--ref-step-seconds", type=float, default=1.0)
    ap.add_argument("--no-aux", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    args = ap.parse_args(argv)
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        return spawn_ranks(args.gpus, sys.argv[1:] if argv is None else list(argv))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    if world != args.gpus and args.impl == "ours":
        print(f"warning: --gpus {args.gpus} but WORLD_SIZE={world}; using WORLD_SIZE", file=sys.stderr)
    if args.impl == "reference":
        return main_reference(args)
    return main_ours(args)


if __name__ == "__main__":
    sys.exit(main())
