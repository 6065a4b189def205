"""Device-memory plumbing for a variable-size batch (PyTorch allocates; the library computes).

A batch lives in three arenas (A, B, C), each matrix at a 256-byte aligned offset with a
16-byte padded leading dimension, plus DEVICE arrays of pointers / sizes / GEMM ids and
fp32 alpha / beta — exactly the arguments of vb_exec_vbatched.  Inputs are drawn on the
device by the library's fill kernel (vb_fill_uniform_batch), keyed by the GLOBAL GEMM id,
so any subset (e.g. one rank's shard) reproduces the same numbers as the whole batch.
"""
from __future__ import annotations

import numpy as np
import torch

import vbinputs
from . import _native as nv

TORCH_DTYPE = {"f32": torch.float32, "bf16": torch.bfloat16, "f16": torch.float16}


def _layout(rows, cols, ld, es, align=256):
    """Element offsets of each matrix in an arena (256-byte aligned), and the arena size."""
    sizes = np.where((rows > 0) & (cols > 0), (np.maximum(rows, 1) - 1) * ld + cols, 0).astype(np.int64)
    q = align // es
    padded = (sizes + q - 1) // q * q
    offs = np.zeros(len(rows), np.int64)
    if len(rows):
        offs[1:] = np.cumsum(padded)[:-1]
    total = int(padded.sum()) + q
    return offs, total


class DeviceBatch:
    """All buffers of one batch on one device."""

    def __init__(self, M, N, K, dtype: str, device="cuda:0", gemm_ids=None, ld_extra: int = 0):
        self.M = np.asarray(M, np.int64)
        self.N = np.asarray(N, np.int64)
        self.K = np.asarray(K, np.int64)
        self.batch = len(self.M)
        self.dtype = dtype
        self.es = vbinputs.elem_size(dtype)
        self.device = torch.device(device)
        self.gemm_ids = np.arange(self.batch, dtype=np.int64) if gemm_ids is None else np.asarray(gemm_ids, np.int64)
        self.lda = vbinputs.padded_ld(self.K, dtype, ld_extra)
        self.ldb = vbinputs.padded_ld(self.N, dtype, ld_extra)
        self.ldc = vbinputs.padded_ld(self.N, dtype, ld_extra)
        td = TORCH_DTYPE[dtype]
        self.offA, nA = _layout(self.M, self.K, self.lda, self.es)
        self.offB, nB = _layout(self.K, self.N, self.ldb, self.es)
        self.offC, nC = _layout(self.M, self.N, self.ldc, self.es)
        self.A = torch.empty(nA, dtype=td, device=self.device)
        self.B = torch.empty(nB, dtype=td, device=self.device)
        self.C = torch.empty(nC, dtype=td, device=self.device)
        es = self.es

        def ptrs(arena, offs):
            return torch.from_numpy(arena.data_ptr() + offs * es).to(self.device)

        self.pA, self.pB, self.pC = ptrs(self.A, self.offA), ptrs(self.B, self.offB), ptrs(self.C, self.offC)
        self.alpha = torch.ones(max(self.batch, 1), dtype=torch.float32, device=self.device)
        self.beta = torch.zeros(max(self.batch, 1), dtype=torch.float32, device=self.device)
        self.d_gemm_ids = torch.from_numpy(self.gemm_ids).to(self.device)
        self._dims = {}

    # --------------------------------------------------------------------- bytes / flops
    def flops(self) -> int:
        return int((2 * self.M * self.N * self.K).sum())

    def algorithmic_bytes(self, beta_nonzero=True) -> int:
        """Compulsory bytes: s*(M*K + K*N) + s*M*N*(1 + [beta != 0])."""
        bn = np.ones(self.batch, bool) if beta_nonzero is True else np.asarray(beta_nonzero, bool)
        mn = self.M * self.N
        live = mn > 0
        return int((self.es * (self.M * self.K + self.K * self.N) * live + self.es * mn * (1 + bn)).sum())

    def arena_bytes(self) -> int:
        return (self.A.numel() + self.B.numel() + self.C.numel()) * self.es

    # --------------------------------------------------------------------- fill
    def _dim_arrays(self, which):
        if which not in self._dims:
            rows, cols, ld = {"A": (self.M, self.K, self.lda), "B": (self.K, self.N, self.ldb),
                              "C": (self.M, self.N, self.ldc)}[which]
            t = lambda a: torch.from_numpy(np.ascontiguousarray(a, np.int32)).to(self.device)  # noqa: E731
            self._dims[which] = (t(rows), t(cols), t(ld), int((rows * cols).sum()))
        return self._dims[which]

    def fill(self, seed: int = 0, ab_mode: str = "random", fill_c: bool = True, stream: int = 0) -> None:
        """Draw A, B, C (operands 0, 1, 2) and alpha/beta on the device (vbinputs recipe)."""
        for which, op, ptrs in (("A", vbinputs.OP_A, self.pA), ("B", vbinputs.OP_B, self.pB),
                                ("C", vbinputs.OP_C, self.pC)):
            if which == "C" and not fill_c:
                continue
            r, c, ld, tot = self._dim_arrays(which)
            nv.fill_uniform_batch(self.dtype, r.data_ptr(), c.data_ptr(), ld.data_ptr(), ptrs.data_ptr(),
                                  self.d_gemm_ids.data_ptr(), self.batch, seed, op, tot, stream)
        if ab_mode == "conv":
            self.alpha.fill_(1.0)
            self.beta.fill_(0.0)
        else:
            nv.fill_alpha_beta(self.batch, self.d_gemm_ids.data_ptr(), seed, self.alpha.data_ptr(),
                               self.beta.data_ptr(), stream)

    # --------------------------------------------------------------------- views
    def _view(self, arena, off, rows, cols, ld):
        if rows == 0 or cols == 0:
            return arena.new_empty((rows, cols))
        return torch.as_strided(arena, (int(rows), int(cols)), (int(ld), 1), int(off))

    def a(self, g):
        return self._view(self.A, self.offA[g], self.M[g], self.K[g], self.lda[g])

    def b(self, g):
        return self._view(self.B, self.offB[g], self.K[g], self.N[g], self.ldb[g])

    def c(self, g):
        return self._view(self.C, self.offC[g], self.M[g], self.N[g], self.ldc[g])

    # --------------------------------------------------------------------- plan / exec
    def plan(self, policy=nv.VB_BATCH_THRESHOLD, table_id=0, tlp_threshold=0, theta=0) -> nv.Plan:
        return nv.plan_vbatched(self.M, self.N, self.K, self.lda, self.ldb, self.ldc, self.dtype, policy,
                                device=self.device.index or 0, table_id=table_id, tlp_threshold=tlp_threshold,
                                theta=theta)

    def plan_tune(self, reps: int = 3, stream=None, **tuning):
        """vb_plan_tune on this batch's buffers (C is overwritten): (plan, [ms_threshold, ms_binary])."""
        s = torch.cuda.current_stream(self.device) if stream is None else stream
        return nv.plan_tune(self.M, self.N, self.K, self.lda, self.ldb, self.ldc, self.pA.data_ptr(),
                            self.pB.data_ptr(), self.pC.data_ptr(), self.alpha.data_ptr(), self.beta.data_ptr(),
                            self.dtype, device=self.device.index or 0, reps=reps, stream=s.cuda_stream, **tuning)

    def run(self, plan: nv.Plan, stream=None) -> None:
        """vb_exec_vbatched: bind this batch's pointers and run (two launches on the tc path)."""
        s = torch.cuda.current_stream(self.device) if stream is None else stream
        plan.exec(self.pA.data_ptr(), self.pB.data_ptr(), self.pC.data_ptr(), self.alpha.data_ptr(),
                  self.beta.data_ptr(), s.cuda_stream)

    def bind(self, plan: nv.Plan, stream=None) -> None:
        s = torch.cuda.current_stream(self.device) if stream is None else stream
        plan.bind(self.pA.data_ptr(), self.pB.data_ptr(), self.pC.data_ptr(), s.cuda_stream)

    def run_bound(self, plan: nv.Plan, stream=None) -> None:
        s = torch.cuda.current_stream(self.device) if stream is None else stream
        plan.exec_bound(self.alpha.data_ptr(), self.beta.data_ptr(), s.cuda_stream)


class ConvBatch(DeviceBatch):
    """A batch of convolutions for vb_plan_conv (implicit GEMM, NEXT-3): per convolution an
    NHWC input X (the exec call's A), HWIO weights (B, (KH*KW*Cin) x Cout, row stride ldb) and an
    NHWC output (C, (nb*Hout*Wout) x Cout, row stride ldc).  Inputs are drawn by the same device
    generator as GEMM batches: X is operand A with logical shape (nb*H*W) x Cin, the weights are
    operand B with shape K x Cout, the output operand C."""

    def __init__(self, convs, dtype: str = "bf16", device="cuda:0", gemm_ids=None):
        self.convs = [dict(c) for c in convs]
        for c in self.convs:
            c["Hout"] = c["H"] + 2 * c["pad"] - c["KH"] + 1
            c["Wout"] = c["W"] + 2 * c["pad"] - c["KW"] + 1
        cv = self.convs
        self.M = np.array([c["nb"] * c["Hout"] * c["Wout"] for c in cv], np.int64)
        self.N = np.array([c["Cout"] for c in cv], np.int64)
        self.K = np.array([c["KH"] * c["KW"] * c["Cin"] for c in cv], np.int64)
        self.P = np.array([c["nb"] * c["H"] * c["W"] for c in cv], np.int64)     # input pixels
        self.Cin = np.array([c["Cin"] for c in cv], np.int64)
        self.batch = len(cv)
        self.dtype = dtype
        self.es = vbinputs.elem_size(dtype)
        self.device = torch.device(device)
        self.gemm_ids = np.arange(self.batch, dtype=np.int64) if gemm_ids is None else np.asarray(gemm_ids, np.int64)
        self.lda = self.Cin.copy()                       # dense NHWC: pixel stride = Cin
        self.ldb = vbinputs.padded_ld(self.N, dtype)
        self.ldc = vbinputs.padded_ld(self.N, dtype)
        for c, b, l in zip(cv, self.ldb, self.ldc):
            c["ldb"], c["ldc"] = int(b), int(l)
        td = TORCH_DTYPE[dtype]
        self.offA, nA = _layout(self.P, self.Cin, self.lda, self.es)
        self.offB, nB = _layout(self.K, self.N, self.ldb, self.es)
        self.offC, nC = _layout(self.M, self.N, self.ldc, self.es)
        self.A = torch.empty(nA, dtype=td, device=self.device)
        self.B = torch.empty(nB, dtype=td, device=self.device)
        self.C = torch.empty(nC, dtype=td, device=self.device)
        es = self.es

        def ptrs(arena, offs):
            return torch.from_numpy(arena.data_ptr() + offs * es).to(self.device)

        self.pA, self.pB, self.pC = ptrs(self.A, self.offA), ptrs(self.B, self.offB), ptrs(self.C, self.offC)
        self.alpha = torch.ones(max(self.batch, 1), dtype=torch.float32, device=self.device)
        self.beta = torch.zeros(max(self.batch, 1), dtype=torch.float32, device=self.device)
        self.d_gemm_ids = torch.from_numpy(self.gemm_ids).to(self.device)
        self._dims = {}

    def algorithmic_bytes(self, beta_nonzero=True) -> int:
        """Compulsory bytes of the convolutions: input + weights + output (+ old output if beta != 0);
        the im2col matrix is never materialised."""
        bn = np.ones(self.batch, bool) if beta_nonzero is True else np.asarray(beta_nonzero, bool)
        mn = self.M * self.N
        return int((self.es * (self.P * self.Cin + self.K * self.N) + self.es * mn * (1 + bn)).sum())

    def _dim_arrays(self, which):
        if which not in self._dims:
            rows, cols, ld = {"A": (self.P, self.Cin, self.lda), "B": (self.K, self.N, self.ldb),
                              "C": (self.M, self.N, self.ldc)}[which]
            t = lambda a: torch.from_numpy(np.ascontiguousarray(a, np.int32)).to(self.device)  # noqa: E731
            self._dims[which] = (t(rows), t(cols), t(ld), int((rows * cols).sum()))
        return self._dims[which]

    def a(self, g):
        return self._view(self.A, self.offA[g], self.P[g], self.Cin[g], self.lda[g])

    def plan(self, policy=nv.VB_BATCH_THRESHOLD, table_id=0, tlp_threshold=0, theta=0) -> nv.Plan:
        return nv.plan_conv(self.convs, self.dtype, policy, device=self.device.index or 0, table_id=table_id,
                            tlp_threshold=tlp_threshold, theta=theta)
