"""ORACLE (test infrastructure only): 2-D convolution, the second workload of SURVEY.md §8(f)
NEXT-3 ("GEMM is the core of convolution", PAPER.md P45; the GoogleNet inception layers of
§7.3, P338-352).

Definition followed (the plain definition of a stride-1 convolution with zero padding, in the
NHWC / HWIO orientation of include/vbgemm.h vb_plan_conv):

    y[n, h, w, co] = sum_{kh, kw, ci} x[n, h + kh - pad, w + kw - pad, ci] * wt[kh, kw, ci, co]

with x read as 0 outside the image, h < Hout = H + 2*pad - KH + 1, w < Wout likewise; then
C = alpha * y + beta * C_old (C_old not read when beta == 0, reading C-16).  Computed in fp64
on inputs converted exactly to fp64.  The sum over taps is a loop over (kh, kw) in the
definition's order; the sum over ci is a library matmul (numpy fp64) as one step.  Nothing
here is blocked, fused or reordered beyond that, and nothing is shared with the CUDA path.
"""
from __future__ import annotations

import numpy as np


def out_size(H: int, W: int, KH: int, KW: int, pad: int):
    return H + 2 * pad - KH + 1, W + 2 * pad - KW + 1


def conv2d_nhwc(x: np.ndarray, wt: np.ndarray, pad: int) -> np.ndarray:
    """x (nb, H, W, Cin), wt (KH, KW, Cin, Cout) -> y (nb, Hout, Wout, Cout), all fp64."""
    x = np.asarray(x, np.float64)
    wt = np.asarray(wt, np.float64)
    nb, H, W, Cin = x.shape
    KH, KW, Cin2, Cout = wt.shape
    assert Cin == Cin2
    Ho, Wo = out_size(H, W, KH, KW, pad)
    xp = np.zeros((nb, H + 2 * pad, W + 2 * pad, Cin), np.float64)   # x with its zero border
    xp[:, pad:pad + H, pad:pad + W, :] = x
    y = np.zeros((nb, Ho, Wo, Cout), np.float64)
    for kh in range(KH):
        for kw in range(KW):
            # y[n,h,w,:] += x[n, h+kh-pad, w+kw-pad, :] @ wt[kh, kw]  (padded index h+kh)
            y += xp[:, kh:kh + Ho, kw:kw + Wo, :] @ wt[kh, kw]
    return y


def conv_gemm(x, wt, c_old, alpha: float, beta: float, pad: int) -> np.ndarray:
    """C = alpha * conv(x, wt) + beta * C_old as the (nb*Hout*Wout) x Cout matrix (NHWC rows)."""
    y = conv2d_nhwc(x, wt, pad)
    y = y.reshape(-1, y.shape[-1])
    if beta == 0.0:
        return alpha * y
    return alpha * y + beta * np.asarray(c_old, np.float64)
