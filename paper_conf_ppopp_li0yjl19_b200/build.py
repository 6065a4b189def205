"""Build libvbgemm.so in-tree: nvcc for sm_100a (-gencode arch=compute_100a,code=sm_100a).

The CUDA runtime is linked statically and the driver API (cuTensorMapEncodeTiled) is
reached through cudaGetDriverEntryPoint, so the library loads on a GPU-less host (the
planner and the C-ABI symbols are usable there; compute calls need a B200).
"""
from __future__ import annotations

import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
CSRC = os.path.join(HERE, "csrc")
LIB = os.path.join(HERE, "libvbgemm.so")
TRACE_LIB = os.path.join(HERE, "libvbgemm_trace.so")
SOURCES = ["capi.cu", "planner.cpp", "forest.cpp", "kernel_f32.cu", "kernel_tc.cu", "fill.cu", "plan_dev.cu"]
HEADERS = ["tables.h", "planner.h", "plan_types.h", "sm100.cuh", "forest.h", "forest_b200.h"]
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
FLAGS = ["-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-lineinfo", "-std=c++17",
         "-Xcompiler", "-fPIC", "-Xcompiler", "-O3", "--expt-relaxed-constexpr",
         "-I", os.path.join(ROOT, "include"), "-I", CSRC]


def _stale() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    deps = [os.path.join(CSRC, f) for f in SOURCES + HEADERS] + [os.path.join(ROOT, "include", "vbgemm.h"),
                                                                   os.path.abspath(__file__)]
    return any(os.path.getmtime(d) > t for d in deps)


def build(force: bool = False, verbose: bool = False, trace: bool = False, defines=(), out: str = "") -> str:
    """trace=True builds libvbgemm_trace.so with -DVB_TRACE (per-role wait-cycle accounting);
    defines/out build an experiment variant (e.g. VB_PAGES=22) into another .so name."""
    lib = os.path.join(HERE, out) if out else (TRACE_LIB if trace else LIB)
    if not force and not trace and not out and not _stale():
        return LIB
    objdir = os.path.join(HERE, "build_" + (out.replace(".so", "") if out else ("trace" if trace else "main")))
    os.makedirs(objdir, exist_ok=True)
    objs = []
    procs = []
    for src in SOURCES:
        obj = os.path.join(objdir, src + ".o")
        cmd = [NVCC] + FLAGS + (["-DVB_TRACE"] if trace else []) + ["-D" + d for d in defines] + \
            ["-c", os.path.join(CSRC, src), "-o", obj]
        if src.endswith(".cu") and verbose:
            cmd += ["-Xptxas", "-v"]
        procs.append((src, subprocess.Popen(cmd, stdout=subprocess.PIPE, stderr=subprocess.STDOUT)))
        objs.append(obj)
    failed = []
    for src, pr in procs:
        out, _ = pr.communicate()
        if verbose or pr.returncode:
            sys.stderr.write(out.decode(errors="replace"))
        if pr.returncode:
            failed.append(src)
    if failed:
        raise RuntimeError(f"nvcc failed for {failed}")
    tmp = lib + f".tmp{os.getpid()}"
    subprocess.check_call([NVCC, "-gencode", "arch=compute_100a,code=sm_100a", "-shared", "-o", tmp] + objs)
    os.replace(tmp, lib)
    return lib


COV_LIB = os.path.join(HERE, "libvbgemm_cov.so")


def build_coverage(force: bool = False) -> str:
    """libvbgemm_cov.so: the same library with -DVB_COVERAGE (debug coverage counters, tests only)."""
    if not force and os.path.exists(COV_LIB) and not _stale() and os.path.getmtime(COV_LIB) >= os.path.getmtime(LIB):
        return COV_LIB
    return build(defines=("VB_COVERAGE",), out="libvbgemm_cov.so")


if __name__ == "__main__":
    defs = [a[2:] for a in sys.argv[1:] if a.startswith("-D")]
    outs = [a[6:] for a in sys.argv[1:] if a.startswith("--out=")]
    print(build(force="--force" in sys.argv, verbose="-v" in sys.argv, trace="--trace" in sys.argv, defines=defs,
                out=outs[0] if outs else ""))
