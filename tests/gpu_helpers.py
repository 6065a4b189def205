"""Shared helpers for the -m gpu tests: run a batch through the C-ABI and compare every
(or a sample of) GEMM with the fp64 oracle on inputs regenerated on the HOST by vbinputs."""
from __future__ import annotations

import numpy as np
import torch

import vbinputs
from oracle import gemm as og
from oracle.checks import TOL, normwise_error, significant_rel_error

# achieved errors per named case, written by tests/conftest.py at session end to
# $VB_PARITY_OUT (default gpurun_out/parity.json) when any test recorded one
RECORD: dict = {}


def to_f64(t: torch.Tensor) -> np.ndarray:
    return t.detach().to("cpu", torch.float64).numpy()


def host_inputs(seed, gid, M, N, K, dtype):
    a = vbinputs.matrix(seed, gid, vbinputs.OP_A, M, K, dtype)[1]
    b = vbinputs.matrix(seed, gid, vbinputs.OP_B, K, N, dtype)[1]
    c = vbinputs.matrix(seed, gid, vbinputs.OP_C, M, N, dtype)[1]
    return a, b, c


def oracle_for(db, idx, seed, ab_mode, c_old=None):
    """fp64 oracle results for GEMMs idx of DeviceBatch db (inputs regenerated on host)."""
    As, Bs, Cs = [], [], []
    for t, g in enumerate(idx):
        a, b, c = host_inputs(seed, int(db.gemm_ids[g]), int(db.M[g]), int(db.N[g]), int(db.K[g]), db.dtype)
        if c_old is not None:
            c = c_old[t]
        As.append(a); Bs.append(b); Cs.append(np.array(c, dtype=np.float64))
    al, be = vbinputs.alpha_beta(seed, db.gemm_ids[list(idx)], ab_mode)
    og.gemm_batch(As, Bs, Cs, al.astype(np.float64), be.astype(np.float64))
    return Cs


def check_batch(db, idx, seed, ab_mode, c_old=None, tol=None):
    tol = TOL[db.dtype] if tol is None else tol
    refs = oracle_for(db, idx, seed, ab_mode, c_old)
    worst = 0.0
    for g, ref in zip(idx, refs):
        got = to_f64(db.c(g))
        err = normwise_error(got, ref)
        worst = max(worst, err)
        assert err <= tol, f"GEMM {g} (M,N,K)=({db.M[g]},{db.N[g]},{db.K[g]}): normwise error {err:.3e} > {tol}"
    return worst


U_OUT = {"f32": 2.0 ** -24, "bf16": 2.0 ** -8, "f16": 2.0 ** -11}


def check_bound(db, idx, seed, ab_mode, c_old=None):
    """Elementwise forward-error bound (Higham, Accuracy and Stability, Thm 3.5 style):
    |C_gpu - C_ref| <= (K+2) u32 (|alpha| |A||B| + |beta| |C_old|) + u_out |C_ref| + tiny,
    with fp32 accumulation (u32 = 2^-24) and rounding to the output type (u_out)."""
    refs = oracle_for(db, idx, seed, ab_mode, c_old)
    al, be = vbinputs.alpha_beta(seed, db.gemm_ids[list(idx)], ab_mode)
    for t, (g, ref) in enumerate(zip(idx, refs)):
        m, n, k = int(db.M[g]), int(db.N[g]), int(db.K[g])
        a, b, c = host_inputs(seed, int(db.gemm_ids[g]), m, n, k, db.dtype)
        if c_old is not None:
            c = np.asarray(c_old[t], np.float64)
        mag = [np.abs(c).copy()]
        og.gemm_batch([np.abs(a)], [np.abs(b)], mag, [abs(float(al[t]))], [abs(float(be[t]))])
        bound = (k + 2) * 2.0 ** -24 * mag[0] + U_OUT[db.dtype] * np.abs(ref) + 2.0 ** -24
        err = np.abs(to_f64(db.c(g)) - ref)
        bad = err > bound
        assert not bad.any(), (f"GEMM {g} (M,N,K)=({m},{n},{k}): {int(bad.sum())} elements outside the error "
                               f"bound, worst excess {float((err - bound).max()):.3e}")


def check_recorded(name, db, idx, seed, ab_mode, c_old=None):
    """Normwise tolerance AND the elementwise bound on GEMMs idx, and record the achieved
    errors under `name`: worst normwise error, worst err/bound ratio, worst significant
    elementwise relative error (C-18), and how many GEMMs / elements were checked."""
    refs = oracle_for(db, idx, seed, ab_mode, c_old)
    al, be = vbinputs.alpha_beta(seed, db.gemm_ids[list(idx)], ab_mode)
    tol = TOL[db.dtype]
    worst_nw = worst_ratio = worst_sig = 0.0
    n_el = 0
    for t, (g, ref) in enumerate(zip(idx, refs)):
        m, n, k = int(db.M[g]), int(db.N[g]), int(db.K[g])
        got = to_f64(db.c(g))
        nw = normwise_error(got, ref)
        assert nw <= tol, f"{name}: GEMM {g} (M,N,K)=({m},{n},{k}): normwise error {nw:.3e} > {tol}"
        a, b, c = host_inputs(seed, int(db.gemm_ids[g]), m, n, k, db.dtype)
        if c_old is not None:
            c = np.asarray(c_old[t], np.float64)
        mag = [np.abs(c).copy()]
        og.gemm_batch([np.abs(a)], [np.abs(b)], mag, [abs(float(al[t]))], [abs(float(be[t]))])
        bound = (k + 2) * 2.0 ** -24 * mag[0] + U_OUT[db.dtype] * np.abs(ref) + 2.0 ** -24
        err = np.abs(got - ref)
        ratio = float((err / bound).max()) if err.size else 0.0
        assert ratio <= 1.0, f"{name}: GEMM {g} (M,N,K)=({m},{n},{k}): {int((err > bound).sum())} elements outside the bound"
        worst_nw, worst_ratio = max(worst_nw, nw), max(worst_ratio, ratio)
        worst_sig = max(worst_sig, significant_rel_error(got, ref))
        n_el += err.size
    RECORD[name] = {"dtype": db.dtype, "gemms_checked": len(list(idx)), "elements_checked": int(n_el),
                    "normwise_max": worst_nw, "tolerance": tol, "bound_ratio_max": worst_ratio,
                    "significant_rel_max": worst_sig}
    return RECORD[name]
