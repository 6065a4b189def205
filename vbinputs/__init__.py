"""Seeded synthetic inputs for the variable-size batched GEMM (shared by tests, oracle and bench).

This module holds NO GEMM arithmetic: it only draws numbers.  It is the one module both
sides of the parity check may import (the oracle under ``oracle/`` and the CUDA path's
harness).  The device-side fill kernel (``vb_fill_uniform`` in the product library)
implements the *same* counter-based generator; ``tests/test_gpu_*`` check the two agree
bit for bit, so an oracle never consumes a value that came from the CUDA path.

Generator (PAPER.md P444 only says "random matrix size and batch size"):

* per-matrix key   ``mkey = splitmix64(splitmix64(seed + SEED_SALT) ^ ((gemm << 3) | operand))``
* element value    ``h = splitmix64(mkey + idx)``, ``idx = i*cols + j`` (LOGICAL index, so the
  leading-dimension padding never changes a value)
* matrix entries   ``u = (h >> 40) * 2^-23 - 1``  -> uniform on [-1, 1), exact in fp32
* alpha            ``0.5 + (h >> 41) * 2^-23``      -> [0.5, 1.5)   (operand 3, idx 0)
* beta             ``(h >> 40) * 2^-23 - 1``        -> [-1, 1)      (operand 4, idx 0)
* bf16 / fp16 inputs are the fp32 draw rounded to nearest-even.
"""
from __future__ import annotations

import numpy as np

from .configs import (CONFIGS, googlenet_shapes, googlenet_convs, config_sizes, padded_ld,  # noqa: F401
                      elem_size, DTYPES)

MASK64 = (1 << 64) - 1
SEED_SALT = 0x632BE59BD9B4E019
OP_A, OP_B, OP_C, OP_ALPHA, OP_BETA = 0, 1, 2, 3, 4

_G = np.uint64(0x9E3779B97F4A7C15)
_M1 = np.uint64(0xBF58476D1CE4E5B9)
_M2 = np.uint64(0x94D049BB133111EB)


def splitmix64(x):
    """Vectorised splitmix64 finaliser over uint64 (wrapping arithmetic)."""
    with np.errstate(over="ignore"):
        z = np.asarray(x, dtype=np.uint64) + _G
        z = (z ^ (z >> np.uint64(30))) * _M1
        z = (z ^ (z >> np.uint64(27))) * _M2
        return z ^ (z >> np.uint64(31))


def splitmix64_int(x: int) -> int:
    """Scalar reference of the same function on Python ints (used to pin the vector one)."""
    z = (x + 0x9E3779B97F4A7C15) & MASK64
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & MASK64
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & MASK64
    return z ^ (z >> 31)


def matrix_key(seed: int, gemm: int, operand: int) -> int:
    inner = splitmix64_int((seed + SEED_SALT) & MASK64)
    return splitmix64_int(inner ^ (((gemm << 3) | operand) & MASK64))


def _u24(seed, gemm, operand, idx):
    key = np.uint64(matrix_key(seed, gemm, operand))
    with np.errstate(over="ignore"):
        h = splitmix64(key + np.asarray(idx, dtype=np.uint64))
    return (h >> np.uint64(40)).astype(np.int64)


def uniform_f32(seed: int, gemm: int, operand: int, rows: int, cols: int) -> np.ndarray:
    """rows x cols fp32 matrix, entries uniform on [-1, 1) (logical, unpadded)."""
    idx = np.arange(rows * cols, dtype=np.uint64)
    u = _u24(seed, gemm, operand, idx).astype(np.float64) * (2.0 ** -23) - 1.0
    return u.astype(np.float32).reshape(rows, cols)


def uniform_at(seed: int, gemm: int, operand: int, cols: int, rows_idx, cols_idx) -> np.ndarray:
    """Random access: fp32 entries at (rows_idx[t], cols_idx[t]) of a matrix with ``cols`` columns."""
    idx = np.asarray(rows_idx, dtype=np.uint64) * np.uint64(cols) + np.asarray(cols_idx, dtype=np.uint64)
    u = _u24(seed, gemm, operand, idx).astype(np.float64) * (2.0 ** -23) - 1.0
    return u.astype(np.float32)


def f32_to_bf16_bits(x: np.ndarray) -> np.ndarray:
    """Round-to-nearest-even fp32 -> bf16, returned as uint16 bit patterns (no NaN/Inf inputs)."""
    b = np.ascontiguousarray(x, dtype=np.float32).view(np.uint32).astype(np.uint64)
    rounded = (b + np.uint64(0x7FFF) + ((b >> np.uint64(16)) & np.uint64(1))) >> np.uint64(16)
    return rounded.astype(np.uint16)


def bf16_bits_to_f64(bits: np.ndarray) -> np.ndarray:
    return (np.asarray(bits, dtype=np.uint32) << np.uint32(16)).view(np.float32).astype(np.float64)


def quantize(x_f32: np.ndarray, dtype: str):
    """Return (storage array, exact fp64 values) for dtype in {'f32','bf16','f16'}."""
    if dtype == "f32":
        s = np.ascontiguousarray(x_f32, dtype=np.float32)
        return s, s.astype(np.float64)
    if dtype == "bf16":
        s = f32_to_bf16_bits(x_f32)
        return s, bf16_bits_to_f64(s)
    if dtype == "f16":
        s = np.ascontiguousarray(x_f32, dtype=np.float32).astype(np.float16)
        return s, s.astype(np.float64)
    raise ValueError(dtype)


def matrix(seed: int, gemm: int, operand: int, rows: int, cols: int, dtype: str):
    """(storage, fp64 exact) for one operand matrix of one GEMM."""
    return quantize(uniform_f32(seed, gemm, operand, rows, cols), dtype)


_gen_lib = None


def _gen():
    """ctypes handle of the C implementation of the same generator (built on first use)."""
    global _gen_lib
    if _gen_lib is None:
        import ctypes
        import os
        import subprocess
        here = os.path.dirname(os.path.abspath(__file__))
        src, so = os.path.join(here, "_gen.c"), os.path.join(here, "_gen.so")
        if not os.path.exists(so) or os.path.getmtime(so) < os.path.getmtime(src):
            tmp = so + f".tmp{os.getpid()}"
            subprocess.check_call(["gcc", "-O2", "-fopenmp", "-ffp-contract=off", "-fPIC", "-shared", "-o", tmp, src])
            os.replace(tmp, so)
        lib = ctypes.CDLL(so)
        lib.vbgen_fill_f64.argtypes = [ctypes.c_uint64, ctypes.c_int64, ctypes.c_int64, ctypes.c_int, ctypes.c_void_p]
        lib.vbgen_fill_f64.restype = None
        _gen_lib = lib
    return _gen_lib


def matrix_f64_fast(seed: int, gemm: int, operand: int, rows: int, cols: int, dtype: str) -> np.ndarray:
    """Exact fp64 values of ``matrix(...)[1]`` from the C generator (multi-threaded)."""
    out = np.empty((rows, cols), np.float64)
    if out.size:
        _gen().vbgen_fill_f64(matrix_key(seed, gemm, operand), rows, cols, {"f32": 0, "bf16": 1, "f16": 2}[dtype],
                              out.ctypes.data)
    return out


def alpha_beta(seed: int, gemms, mode: str = "random"):
    """Per-GEMM fp32 alpha/beta. mode 'random' (alpha in [0.5,1.5), beta in [-1,1)) or 'conv' (1, 0)."""
    gemms = np.asarray(gemms, dtype=np.int64)
    if mode == "conv":
        return np.ones(len(gemms), np.float32), np.zeros(len(gemms), np.float32)
    al = np.empty(len(gemms), np.float32)
    be = np.empty(len(gemms), np.float32)
    for t, g in enumerate(gemms):
        al[t] = np.float32(0.5 + float(_u24(seed, int(g), OP_ALPHA, [0])[0] >> 1) * 2.0 ** -23)
        be[t] = np.float32(float(_u24(seed, int(g), OP_BETA, [0])[0]) * 2.0 ** -23 - 1.0)
    return al, be
