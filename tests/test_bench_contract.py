"""The bench.py contract on CPU: the reference arm (the fp64 oracle timed on the host) prints one
JSON line with the keys the driver reads, for a small config, and ranks other than 0 exit
without output.  The GPU arm is exercised by the driver on a B200."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _run(args, env=None):
    e = dict(os.environ)
    e.update(env or {})
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py")] + args, capture_output=True, text=True,
                         timeout=300, env=e, cwd=ROOT)
    assert out.returncode == 0, out.stderr[-2000:]
    return out.stdout


def test_reference_arm_json_line():
    out = _run(["--impl", "reference", "--config", "C1", "--steps", "2", "--warmup", "0", "--ref-step-seconds", "0.2"])
    lines = [l for l in out.splitlines() if l.startswith("{")]
    assert len(lines) == 1
    d = json.loads(lines[0])
    for k in ("metric", "value", "unit", "impl", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better",
              "scaling", "vs_baseline", "dtype", "data", "config", "cpu_baseline", "e2e", "gpu_launches"):
        assert k in d, k
    assert d["impl"] == "reference" and d["value"] > 0 and d["higher_is_better"] is True
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] >= 1
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["e2e"]["value"] == d["value"]
    assert d["config"]["workload"].startswith("C1")


def test_reference_arm_non_zero_rank_is_silent():
    out = _run(["--impl", "reference", "--config", "C1", "--steps", "1", "--warmup", "0"],
               env={"RANK": "1", "WORLD_SIZE": "2", "LOCAL_RANK": "1"})
    assert not [l for l in out.splitlines() if l.startswith("{")]


def test_reference_arm_spawns_its_own_ranks():
    """`bench.py --impl reference --gpus 2` with no launcher starts 2 ranks itself (torch
    distributed run on 127.0.0.1); rank 0 alone prints one line with n_gpus = 2."""
    env = {k: v for k, v in os.environ.items() if k not in ("WORLD_SIZE", "RANK", "LOCAL_RANK")}
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--gpus", "2",
                          "--config", "C1", "--steps", "1", "--warmup", "0", "--ref-step-seconds", "0.2"],
                         capture_output=True, text=True, timeout=300, env=env, cwd=ROOT)
    assert out.returncode == 0, out.stderr[-2000:]
    lines = [l for l in out.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["impl"] == "reference"


def test_aggregate_roofline_is_the_slowest_rank():
    sys.path.insert(0, ROOT)
    import bench
    peaks = {"hbm_gbs": 1000.0, "bf16_tflops": 1000.0, "bf16_tflops_sustained": 900.0, "sm_max_mhz": 1965.0}
    # two ranks, 1e9 and 1.2e9 bytes (HBM-bound), makespan 1.5 ms
    r = bench.aggregate_roofline("bf16", 1e9, 2.2e9, 1.5e-3, 1.2e3, 2, peaks)
    assert r["bound"] == "hbm" and abs(r["peak"] - 2000.0) < 1e-9
    assert abs(r["achieved"] - 2.2e9 / 1.5e-3 / 1e9) < 1e-6
    assert abs(r["frac"] - r["achieved"] / r["peak"]) < 1e-12
    assert abs(r["frac_makespan"] - 1.2e-3 / 1.5e-3) < 1e-12
