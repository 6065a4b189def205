"""Pins for the convolution oracle (oracle/conv_ref.py, NEXT-3) against things other than itself.

Definition: stride-1 zero-padded convolution, NHWC x HWIO (include/vbgemm.h vb_plan_conv;
P45: "GEMM is the core of convolution").  Pins: a pure-Python 7-loop brute force, the fp64
C GEMM oracle for 1x1 convolutions (conv == GEMM), closed forms that fix the tap orientation
and the zero border (a shift filter, all-ones counts at corners / edges / interior),
scipy.signal.correlate2d (a library routine) per channel pair, the output size rule, and
the alpha / beta (beta == 0 never reads C) rule.
"""
import numpy as np
import pytest
from scipy import signal

from oracle import conv_ref as cr
from oracle import gemm as og


def _brute(x, wt, pad):
    nb, H, W, Cin = x.shape
    KH, KW, _, Cout = wt.shape
    Ho, Wo = H + 2 * pad - KH + 1, W + 2 * pad - KW + 1
    y = np.zeros((nb, Ho, Wo, Cout))
    for n in range(nb):
        for h in range(Ho):
            for w in range(Wo):
                for co in range(Cout):
                    s = 0.0
                    for kh in range(KH):
                        for kw in range(KW):
                            ih, iw = h + kh - pad, w + kw - pad
                            if 0 <= ih < H and 0 <= iw < W:
                                for ci in range(Cin):
                                    s += float(x[n, ih, iw, ci]) * float(wt[kh, kw, ci, co])
                    y[n, h, w, co] = s
    return y


@pytest.mark.parametrize("shape", [(2, 3, 4, 2, 3, 3, 1), (1, 5, 5, 3, 2, 5, 2), (1, 4, 3, 2, 2, 3, 0),
                                   (1, 3, 3, 1, 1, 1, 0), (2, 2, 2, 3, 2, 3, 1)])
def test_brute_force_tiny(shape):
    nb, H, W, Cin, Cout, k, pad = shape
    rng = np.random.default_rng(sum(shape))
    x = rng.uniform(-1, 1, (nb, H, W, Cin))
    wt = rng.uniform(-1, 1, (k, k, Cin, Cout))
    got = cr.conv2d_nhwc(x, wt, pad)
    ref = _brute(x, wt, pad)
    assert got.shape == ref.shape
    assert np.max(np.abs(got - ref)) <= 1e-12


def test_one_by_one_is_the_gemm_oracle():
    rng = np.random.default_rng(3)
    x = rng.uniform(-1, 1, (2, 7, 5, 24))
    wt = rng.uniform(-1, 1, (1, 1, 24, 16))
    c = rng.uniform(-1, 1, (2 * 7 * 5, 16))
    got = cr.conv_gemm(x, wt, c, 1.25, -0.5, 0)
    ref = og.gemm(x.reshape(-1, 24), wt[0, 0], c, 1.25, -0.5)
    assert np.max(np.abs(got - ref)) <= 1e-12


def test_shift_filter_fixes_tap_orientation_and_border():
    # wt[kh=0, kw=0, ci, co] = [ci == co]: y[h, w] = x[h - 1, w - 1], zero on the top/left border
    rng = np.random.default_rng(4)
    x = rng.uniform(-1, 1, (1, 6, 5, 3))
    wt = np.zeros((3, 3, 3, 3))
    wt[0, 0] = np.eye(3)
    y = cr.conv2d_nhwc(x, wt, 1)
    assert np.all(y[:, 0, :, :] == 0) and np.all(y[:, :, 0, :] == 0)
    assert np.array_equal(y[:, 1:, 1:, :], x[:, :-1, :-1, :])
    # the opposite corner tap shifts the other way
    wt2 = np.zeros((3, 3, 3, 3))
    wt2[2, 2] = np.eye(3)
    y2 = cr.conv2d_nhwc(x, wt2, 1)
    assert np.array_equal(y2[:, :-1, :-1, :], x[:, 1:, 1:, :])
    assert np.all(y2[:, -1, :, :] == 0) and np.all(y2[:, :, -1, :] == 0)
    # a tap off the centre row only (kh = 0, kw = 1): pure vertical shift
    wt3 = np.zeros((3, 3, 3, 3))
    wt3[0, 1] = np.eye(3)
    y3 = cr.conv2d_nhwc(x, wt3, 1)
    assert np.array_equal(y3[:, 1:, :, :], x[:, :-1, :, :])


@pytest.mark.parametrize("k,pad", [(3, 1), (5, 2)])
def test_all_ones_counts_valid_taps(k, pad):
    H = W = 7
    Cin = 4
    y = cr.conv2d_nhwc(np.ones((1, H, W, Cin)), np.ones((k, k, Cin, 2)), pad)
    for h in range(H):
        for w in range(W):
            rows = sum(1 for kh in range(k) if 0 <= h + kh - pad < H)
            cols = sum(1 for kw in range(k) if 0 <= w + kw - pad < W)
            assert y[0, h, w, 0] == Cin * rows * cols
    assert y[0, 0, 0, 0] == Cin * (k - pad) ** 2           # corner
    assert y[0, 3, 3, 1] == Cin * k * k                     # interior


def test_matches_scipy_correlate_per_channel_pair():
    rng = np.random.default_rng(5)
    x = rng.uniform(-1, 1, (1, 9, 8, 2))
    wt = rng.uniform(-1, 1, (3, 3, 2, 3))
    y = cr.conv2d_nhwc(x, wt, 1)
    for co in range(3):
        ref = sum(signal.correlate2d(x[0, :, :, ci], wt[:, :, ci, co], mode="same") for ci in range(2))
        assert np.max(np.abs(y[0, :, :, co] - ref)) <= 1e-12


def test_valid_padding_output_size():
    assert cr.out_size(28, 28, 3, 3, 1) == (28, 28)
    assert cr.out_size(14, 14, 5, 5, 2) == (14, 14)
    assert cr.out_size(7, 9, 3, 3, 0) == (5, 7)
    y = cr.conv2d_nhwc(np.ones((1, 7, 9, 1)), np.ones((3, 3, 1, 1)), 0)
    assert y.shape == (1, 5, 7, 1) and np.all(y == 9)


def test_beta_zero_never_reads_c():
    rng = np.random.default_rng(6)
    x = rng.uniform(-1, 1, (1, 4, 4, 2))
    wt = rng.uniform(-1, 1, (3, 3, 2, 2))
    c = np.full((16, 2), np.nan)
    out = cr.conv_gemm(x, wt, c, 2.0, 0.0, 1)
    assert np.all(np.isfinite(out))
    assert np.allclose(out, 2.0 * cr.conv2d_nhwc(x, wt, 1).reshape(16, 2), rtol=0, atol=0)
