"""Pins for the fp64 GEMM oracle (oracle/gemm_ref.c) against things other than itself.

Definition: PAPER.md P31 (§1), C = alpha*A x B + beta*C.  Pins: brute force on tiny
sizes against hand-written loops, closed forms (identity / zero / alpha=0 / beta=0 with
NaN-poisoned C / K=0), numpy's fp64 matmul (a library routine), ld-padded views, and
thread-count invariance.
"""
import itertools

import numpy as np
import pytest

from oracle import gemm as og


def _brute(A, B, C, al, be):
    M, K = A.shape
    N = B.shape[1]
    out = [[0.0] * N for _ in range(M)]
    for i in range(M):
        for j in range(N):
            s = 0.0
            for p in range(K):
                s += float(A[i, p]) * float(B[p, j])
            out[i][j] = al * s + be * float(C[i, j]) if be != 0.0 else al * s
    return np.array(out, dtype=np.float64).reshape(M, N)


def test_brute_force_tiny_exact():
    rng = np.random.default_rng(1)
    cases = list(itertools.product([1, 2, 3, 5], [1, 2, 4, 7], [0, 1, 3, 8]))
    As, Bs, Cs, ref, al, be = [], [], [], [], [], []
    for (m, n, k) in cases:
        A = rng.standard_normal((m, k)); B = rng.standard_normal((k, n)); C = rng.standard_normal((m, n))
        a, b = float(rng.uniform(-2, 2)), float(rng.uniform(-2, 2))
        ref.append(_brute(A, B, C, a, b))
        As.append(A); Bs.append(B); Cs.append(C.copy()); al.append(a); be.append(b)
    og.gemm_batch(As, Bs, Cs, al, be)
    for c, r in zip(Cs, ref):
        assert np.array_equal(c, r)   # same summation order in fp64 -> bit-exact


def test_not_transposed_and_sign():
    # A non-square, non-symmetric: a transposed operand or a sign slip changes the answer
    A = np.array([[1.0, 2.0, 3.0], [4.0, 5.0, 6.0]])          # 2x3
    B = np.array([[1.0, 0.0], [0.0, -1.0], [2.0, 1.0]])         # 3x2
    C = np.array([[1.0, 1.0], [1.0, 1.0]])
    out = og.gemm(A, B, C, 2.0, -3.0)
    # A@B = [[7, 1], [16, 1]] -> 2*AB - 3 = [[11, -1], [29, -1]]
    assert np.array_equal(out, np.array([[11.0, -1.0], [29.0, -1.0]]))


@pytest.mark.parametrize("m,n", [(1, 1), (5, 9), (33, 17)])
def test_identity_closed_form(m, n):
    rng = np.random.default_rng(2)
    B = rng.standard_normal((m, n)); C = rng.standard_normal((m, n))
    out = og.gemm(np.eye(m), B, C, 1.25, -0.5)
    assert np.array_equal(out, 1.25 * B + -0.5 * C)


def test_zero_matrix_and_alpha_zero():
    rng = np.random.default_rng(3)
    A = rng.standard_normal((7, 5)); B = rng.standard_normal((5, 6)); C = rng.standard_normal((7, 6))
    assert np.array_equal(og.gemm(np.zeros((7, 5)), B, C, 0.7, 0.3), 0.3 * C)
    assert np.array_equal(og.gemm(A, B, C, 0.0, 0.3), 0.3 * C)


def test_beta_zero_does_not_read_c():
    rng = np.random.default_rng(4)
    A = rng.standard_normal((4, 3)); B = rng.standard_normal((3, 5))
    C = np.full((4, 5), np.nan)
    out = og.gemm(A, B, C, 1.5, 0.0)
    assert np.all(np.isfinite(out))
    assert np.allclose(out, 1.5 * (A @ B), rtol=1e-14, atol=1e-14)


def test_k_zero_scales_c_and_empty_is_noop():
    C = np.arange(12.0).reshape(3, 4)
    out = og.gemm(np.zeros((3, 0)), np.zeros((0, 4)), C, 2.0, 0.5)
    assert np.array_equal(out, 0.5 * C)
    Cs = [np.zeros((0, 4)), np.zeros((3, 0))]
    og.gemm_batch([np.zeros((0, 2)), np.zeros((3, 2))], [np.zeros((2, 4)), np.zeros((2, 0))], Cs, [1.0, 1.0], [1.0, 1.0])


def test_against_numpy_fp64_matmul():
    rng = np.random.default_rng(5)
    As, Bs, Cs, al, be, ref = [], [], [], [], [], []
    for _ in range(40):
        m, n, k = rng.integers(1, 160, 3)
        A = rng.uniform(-1, 1, (m, k)); B = rng.uniform(-1, 1, (k, n)); C = rng.uniform(-1, 1, (m, n))
        a, b = float(rng.uniform(0.5, 1.5)), float(rng.uniform(-1, 1))
        ref.append(a * (A @ B) + b * C)
        As.append(A); Bs.append(B); Cs.append(C.copy()); al.append(a); be.append(b)
    og.gemm_batch(As, Bs, Cs, al, be)
    for c, r in zip(Cs, ref):
        assert np.max(np.abs(c - r)) <= 1e-12 * max(1.0, np.max(np.abs(r)))


def test_padded_leading_dimensions():
    rng = np.random.default_rng(6)
    Ab = rng.standard_normal((6, 11)); Bb = rng.standard_normal((4, 13)); Cb = rng.standard_normal((6, 9))
    A, B, C = Ab[:, :4], Bb[:, :7], Cb[:, :7]        # strided row views: lda=11, ldb=13, ldc=9
    pad_before = Cb[:, 7:].copy()
    ref = _brute(A, B, C, 0.5, 2.0)
    og.gemm_batch([A], [B], [C], [0.5], [2.0])
    assert np.array_equal(Cb[:, :7], ref)
    assert np.array_equal(Cb[:, 7:], pad_before)      # padding untouched


def test_thread_count_invariance():
    rng = np.random.default_rng(7)
    A = rng.standard_normal((300, 70)); B = rng.standard_normal((70, 90)); C = rng.standard_normal((300, 90))
    c1 = [C.copy()]; c8 = [C.copy()]
    og.gemm_batch([A], [B], c1, [1.0], [1.0], nthreads=1)
    og.gemm_batch([A], [B], c8, [1.0], [1.0], nthreads=8)
    assert np.array_equal(c1[0], c8[0])
