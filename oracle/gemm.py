"""ORACLE (test infrastructure only): Python front-end of the fp64 C triple loop.

Definition followed: PAPER.md P31 (§1) / P133 (§2.2), ``C = alpha*A x B + beta*C``.
See ``gemm_ref.c`` for the loop and the BLAS beta == 0 rule (C-16).
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "gemm_ref.c")
_LIB = os.path.join(_HERE, "_gemm_ref.so")
_lib = None


def build(force: bool = False) -> str:
    """Compile gemm_ref.c with gcc -O2 -fopenmp (no BLAS, no fast-math)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-ffp-contract=off", "-fPIC", "-shared", "-std=c99",
                               "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB)
        P = ctypes.POINTER
        lib.vbref_gemm.restype = ctypes.c_int
        lib.vbref_gemm.argtypes = [ctypes.c_int64, P(ctypes.c_int64), P(ctypes.c_int64), P(ctypes.c_int64),
                                   P(ctypes.c_void_p), P(ctypes.c_int64),
                                   P(ctypes.c_void_p), P(ctypes.c_int64),
                                   P(ctypes.c_void_p), P(ctypes.c_int64),
                                   P(ctypes.c_double), P(ctypes.c_double), ctypes.c_int]
        lib.vbref_max_threads.restype = ctypes.c_int
        _lib = lib
    return _lib


def max_threads() -> int:
    return int(_load().vbref_max_threads())


def _ld(x) -> int:
    if x.size == 0:
        return max(x.shape[1], 1)
    return x.strides[0] // 8 if x.shape[0] > 1 else x.shape[1]


def gemm_batch(As, Bs, Cs, alphas, betas, nthreads: int = 0):
    """In place: Cs[g] <- alpha[g] * As[g] @ Bs[g] + beta[g] * Cs[g], all fp64 2-D arrays.

    ``As[g]`` is M x K, ``Bs[g]`` K x N, ``Cs[g]`` M x N (row-major, C-contiguous rows; the
    leading dimension is taken from the array strides, so views with padded rows work).
    """
    lib = _load()
    n = len(As)
    if not (len(Bs) == len(Cs) == n == len(alphas) == len(betas)):
        raise ValueError("batch length mismatch")
    M = np.zeros(n, np.int64); N = np.zeros(n, np.int64); K = np.zeros(n, np.int64)
    lda = np.ones(n, np.int64); ldb = np.ones(n, np.int64); ldc = np.ones(n, np.int64)
    pa = (ctypes.c_void_p * max(n, 1))(); pb = (ctypes.c_void_p * max(n, 1))(); pc = (ctypes.c_void_p * max(n, 1))()
    keep = []
    for g in range(n):
        a, b, c = As[g], Bs[g], Cs[g]
        for x in (a, b, c):
            if x.dtype != np.float64 or x.ndim != 2 or (x.size and x.shape[1] > 1 and x.strides[1] != 8):
                raise ValueError("oracle wants fp64 2-D arrays with unit column stride")
        if c.flags.writeable is False:
            raise ValueError("C must be writeable")
        M[g], K[g] = a.shape
        if b.shape[0] != K[g] or c.shape != (M[g], b.shape[1]):
            raise ValueError(f"shape mismatch in GEMM {g}: {a.shape} {b.shape} {c.shape}")
        N[g] = b.shape[1]
        lda[g], ldb[g], ldc[g] = _ld(a), _ld(b), _ld(c)
        pa[g] = a.ctypes.data if a.size else None
        pb[g] = b.ctypes.data if b.size else None
        pc[g] = c.ctypes.data if c.size else None
        keep.append((a, b, c))
    al = np.ascontiguousarray(alphas, dtype=np.float64)
    be = np.ascontiguousarray(betas, dtype=np.float64)
    P64 = ctypes.POINTER(ctypes.c_int64)
    PD = ctypes.POINTER(ctypes.c_double)
    rc = lib.vbref_gemm(n, M.ctypes.data_as(P64), N.ctypes.data_as(P64), K.ctypes.data_as(P64),
                        pa, lda.ctypes.data_as(P64), pb, ldb.ctypes.data_as(P64),
                        pc, ldc.ctypes.data_as(P64), al.ctypes.data_as(PD), be.ctypes.data_as(PD),
                        int(nthreads))
    if rc != 0:
        raise RuntimeError(f"vbref_gemm failed: {rc}")
    return Cs


def gemm(A, B, C, alpha: float, beta: float):
    """Single GEMM convenience wrapper; returns a new array (C is not modified)."""
    out = np.array(C, dtype=np.float64, copy=True)
    gemm_batch([np.ascontiguousarray(A, np.float64)], [np.ascontiguousarray(B, np.float64)], [out],
               [alpha], [beta])
    return out
