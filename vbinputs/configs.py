"""Workload recipes (sizes only) for the five BASELINE.json configs.

Recipes (readings C-20/C-21 in DESIGN.md):

* C1  8 fp32 GEMMs, ``default_rng(0).integers(16, 129, (8, 3))`` -> columns (M, N, K)
* C2  256 fp32 GEMMs, ``default_rng(0).integers(32, 513, (256, 3))``
* C3  GoogleNet inception conv-as-GEMM (PAPER.md P45: M = #filters, N = H*W*nb, K = Cin*kh*kw),
      all 54 branch convolutions of the 9 inception modules, bf16, alpha=1, beta=0
* C4  4096 bf16 GEMMs, ``integers([16,16,16], [1025,1025,4097], (4096, 3))``
* C5  65536 bf16 GEMMs, M, N, K each ``floor(exp(U(ln 16, ln 1025)))`` (log-uniform on [16, 1024])
"""
from __future__ import annotations

import numpy as np

DTYPES = ("f32", "bf16", "f16")


def elem_size(dtype: str) -> int:
    return {"f32": 4, "bf16": 2, "f16": 2}[dtype]


def padded_ld(cols, dtype: str, extra: int = 0):
    """Leading dimension (elements) rounded up to a 16-byte multiple, plus ``extra`` 16-B units."""
    q = 16 // elem_size(dtype)
    cols = np.asarray(cols, dtype=np.int64)
    return ((np.maximum(cols, 1) + q - 1) // q) * q + extra * q


# GoogLeNet (Szegedy et al. 2014, PAPER.md ref [25]) inception modules:
# name, input channels, spatial size, #1x1, #3x3reduce, #3x3, #5x5reduce, #5x5, pool_proj
_INCEPTION = [
    ("3a", 192, 28, 64, 96, 128, 16, 32, 32),
    ("3b", 256, 28, 128, 128, 192, 32, 96, 64),
    ("4a", 480, 14, 192, 96, 208, 16, 48, 64),
    ("4b", 512, 14, 160, 112, 224, 24, 64, 64),
    ("4c", 512, 14, 128, 128, 256, 24, 64, 64),
    ("4d", 512, 14, 112, 144, 288, 32, 64, 64),
    ("4e", 528, 14, 256, 160, 320, 32, 128, 128),
    ("5a", 832, 7, 256, 160, 320, 32, 128, 128),
    ("5b", 832, 7, 384, 192, 384, 48, 128, 128),
]


def googlenet_shapes(nb: int = 1, first_stage_only: bool = False, module: str | None = None):
    """List of (name, M, N, K) conv-as-GEMM shapes, N = H*W*nb.

    Branch order per module: 1x1, 3x3_reduce, 3x3, 5x5_reduce, 5x5, pool_proj.
    ``first_stage_only`` keeps the four GEMMs the paper batches per module (P350):
    1x1, 3x3_reduce, 5x5_reduce, pool_proj.
    """
    out = []
    for name, cin, hw, c1, r3, c3, r5, c5, pp in _INCEPTION:
        if module is not None and name != module:
            continue
        n = hw * hw * nb
        branches = [("1x1", c1, cin), ("3x3_reduce", r3, cin), ("3x3", c3, 9 * r3),
                    ("5x5_reduce", r5, cin), ("5x5", c5, 25 * r5), ("pool_proj", pp, cin)]
        for bname, m, k in branches:
            if first_stage_only and bname in ("3x3", "5x5"):
                continue
            out.append((f"{name}/{bname}", m, n, k))
    return out


def googlenet_convs(nb: int = 1, first_stage_only: bool = False, module: str | None = None):
    """The same inception-branch convolutions as dicts for the implicit-GEMM path (NEXT-3):
    name, nb, H, W, Cin, Cout, KH, KW, pad (stride 1, "same" padding).  pool_proj is the 1x1
    convolution applied to the (max-pooled) module input; the pooling itself is not part of
    the GEMM path."""
    out = []
    for name, cin, hw, c1, r3, c3, r5, c5, pp in _INCEPTION:
        if module is not None and name != module:
            continue
        branches = [("1x1", cin, c1, 1), ("3x3_reduce", cin, r3, 1), ("3x3", r3, c3, 3),
                    ("5x5_reduce", cin, r5, 1), ("5x5", r5, c5, 5), ("pool_proj", cin, pp, 1)]
        for bname, ci, co, k in branches:
            if first_stage_only and bname in ("3x3", "5x5"):
                continue
            out.append(dict(name=f"{name}/{bname}", nb=nb, H=hw, W=hw, Cin=ci, Cout=co, KH=k, KW=k, pad=(k - 1) // 2))
    return out


CONFIGS = {
    "C1": dict(dtype="f32", desc="8 fp32 GEMMs, M/N/K uniform random in [16,128], seed 0", ab="random"),
    "C2": dict(dtype="f32", desc="256 fp32 GEMMs, M/N/K uniform random in [32,512]", ab="random"),
    "C3": dict(dtype="bf16", desc="GoogleNet Inception conv-as-GEMM batch (54 branch convs), bf16", ab="conv"),
    "C4": dict(dtype="bf16", desc="4096 bf16 GEMMs, M,N in [16,1024], K in [16,4096]", ab="random"),
    "C5": dict(dtype="bf16", desc="65536 mixed-size bf16 GEMMs, M,N,K log-uniform [16,1024]", ab="random"),
}


def config_sizes(name: str, nb: int = 1):
    """(M, N, K) int64 arrays for a named config."""
    if name == "C1":
        r = np.random.default_rng(0).integers(16, 129, (8, 3))
    elif name == "C2":
        r = np.random.default_rng(0).integers(32, 513, (256, 3))
    elif name == "C3":
        r = np.array([[m, n, k] for _, m, n, k in googlenet_shapes(nb)], dtype=np.int64)
    elif name == "C4":
        r = np.random.default_rng(0).integers([16, 16, 16], [1025, 1025, 4097], (4096, 3))
    elif name == "C5":
        u = np.random.default_rng(0).uniform(np.log(16.0), np.log(1025.0), (65536, 3))
        r = np.clip(np.floor(np.exp(u)), 16, 1024).astype(np.int64)
    else:
        raise KeyError(name)
    r = np.asarray(r, dtype=np.int64)
    return r[:, 0].copy(), r[:, 1].copy(), r[:, 2].copy()
