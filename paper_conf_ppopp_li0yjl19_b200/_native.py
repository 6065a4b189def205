"""ctypes binding of include/vbgemm.h — argument marshalling only.

Every computation happens in libvbgemm.so (C++ planner + sm_100a kernels).  There is no
Python or CPU fallback: if the library is missing, importing this module raises.
"""
from __future__ import annotations

import ctypes
import os
import re

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
# VB_LIB selects an alternative build of the same library (e.g. libvbgemm_trace.so).
LIB_PATH = os.environ.get("VB_LIB") or os.path.join(HERE, "libvbgemm.so")
HEADER = os.path.join(os.path.dirname(HERE), "include", "vbgemm.h")

VB_OK, VB_ERR_INVALID_ARG, VB_ERR_ALIGNMENT, VB_ERR_UNSUPPORTED, VB_ERR_OOM, VB_ERR_CUDA, VB_ERR_INTERNAL = range(7)
VB_F32, VB_BF16, VB_F16 = 0, 1, 2
VB_BATCH_THRESHOLD, VB_BATCH_BINARY, VB_BATCH_NONE, VB_BATCH_AUTO = 0, 1, 2, 3
VB_TABLE_DEFAULT, VB_TABLE_V100, VB_TABLE_B200_FFMA, VB_TABLE_B200_TC = 0, 1, 2, 3
DTYPE_CODE = {"f32": VB_F32, "bf16": VB_BF16, "f16": VB_F16}


class VbError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{_status_name(status)}: {msg}")
        self.status = status


class vb_tuning(ctypes.Structure):
    _fields_ = [("table_id", ctypes.c_int32), ("tlp_threshold", ctypes.c_int64), ("theta", ctypes.c_int32)]


class vb_conv_desc(ctypes.Structure):
    _fields_ = [(n, ctypes.c_int32) for n in ("nb", "H", "W", "Cin", "Cout", "KH", "KW", "pad", "ldb", "ldc")]


if not os.path.exists(LIB_PATH):
    raise ImportError(f"{LIB_PATH} is missing: run `python paper_conf_ppopp_li0yjl19_b200/build.py` "
                      "(or __graft_entry__.build()) first; there is no fallback path")
lib = ctypes.CDLL(LIB_PATH)

_P = ctypes.POINTER
_i32p = _P(ctypes.c_int32)
_i64p = _P(ctypes.c_int64)
_vp = ctypes.c_void_p

lib.vb_status_str.restype = ctypes.c_char_p
lib.vb_status_str.argtypes = [ctypes.c_int]
lib.vb_last_error.restype = ctypes.c_char_p
lib.vb_version.restype = ctypes.c_char_p
lib.vb_plan_vbatched.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.c_int32] + [_i32p] * 6 + \
    [ctypes.c_int, _P(vb_tuning), _P(_vp)]
lib.vb_plan_from_schedule.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.c_int32] + [_i32p] * 6 + \
    [ctypes.c_int32, _i32p, ctypes.c_int32, ctypes.c_int32, _i32p, _i32p, _i32p, _i32p, _P(_vp)]
lib.vb_plan_conv.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.c_int32, _P(vb_conv_desc), ctypes.c_int,
                             _P(vb_tuning), _P(_vp)]
lib.vb_exec_vbatched.argtypes = [_vp, _vp, _vp, _vp, _vp, _vp, _vp]
lib.vb_plan_bind.argtypes = [_vp, _vp, _vp, _vp, _vp]
lib.vb_exec_bound.argtypes = [_vp, _vp, _vp, _vp]
lib.vb_plan_info.argtypes = [_vp, _i64p, _i64p, _i64p, _i32p, _i32p]
lib.vb_plan_export.argtypes = [_vp, _i32p, _i32p, _i32p, _i32p, _i32p]
lib.vb_plan_tiler_trace.argtypes = [_vp, ctypes.c_int32, _i64p, _i32p, _i32p]
lib.vb_plan_destroy.argtypes = [_vp]
lib.vb_plan_debug_tmaps.argtypes = [_vp, _vp, ctypes.c_int64, _i64p]
lib.vb_debug_set_coverage.argtypes = [ctypes.c_int, _vp, _vp, ctypes.c_int32]
lib.vb_plan_policy.argtypes = [_vp, _i32p]
lib.vb_plan_tune.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.c_int32] + [_i32p] * 6 + \
    [_P(vb_tuning), _vp, _vp, _vp, _vp, _vp, ctypes.c_int32, _vp, _P(_vp), _P(ctypes.c_float)]
lib.vb_shard_lpt.argtypes = [ctypes.c_int32, _i32p, _i32p, _i32p, ctypes.c_int32, _i32p]
lib.vb_fill_uniform_batch.argtypes = [ctypes.c_int, ctypes.c_int32, _vp, _vp, _vp, _vp, _vp, ctypes.c_uint64,
                                      ctypes.c_int32, ctypes.c_int64, _vp]
lib.vb_fill_alpha_beta.argtypes = [ctypes.c_int32, _vp, ctypes.c_uint64, _vp, _vp, _vp]
lib.vb_device_info.argtypes = [ctypes.c_int, _i32p, _i32p, _i32p]
for _f in ("vb_plan_vbatched", "vb_plan_from_schedule", "vb_exec_vbatched", "vb_plan_bind", "vb_exec_bound", "vb_plan_info", "vb_plan_export",
           "vb_plan_tiler_trace", "vb_plan_destroy", "vb_plan_policy", "vb_plan_tune", "vb_shard_lpt", "vb_fill_uniform_batch", "vb_fill_alpha_beta",
           "vb_device_info", "vb_plan_debug_tmaps", "vb_debug_set_coverage"):
    getattr(lib, _f).restype = ctypes.c_int


def _status_name(s: int) -> str:
    return lib.vb_status_str(int(s)).decode()


def check(status: int) -> None:
    if status != VB_OK:
        raise VbError(status, lib.vb_last_error().decode())


def header_symbols() -> list:
    """Every function name declared in include/vbgemm.h."""
    with open(HEADER) as f:
        txt = f.read()
    return sorted(set(re.findall(r"\b(vb_[a-z0-9_]+)\s*\(", txt)))


def _i32(a) -> np.ndarray:
    v = np.asarray(a, dtype=np.int64)
    if v.size and (v.min() < -2**31 or v.max() >= 2**31):
        raise ValueError("value outside the int32 range of the C-ABI")
    return np.ascontiguousarray(v.astype(np.int32))


def _ptr(a: np.ndarray, ty):
    return a.ctypes.data_as(ty)


class Plan:
    """Owning handle of a vb_plan_t."""

    def __init__(self, handle: int, batch: int, dtype: str):
        self.handle = ctypes.c_void_p(handle)
        self.batch = batch
        self.dtype = dtype

    def __del__(self):
        try:
            self.destroy()
        except Exception:
            pass

    def destroy(self):
        if self.handle and self.handle.value:
            lib.vb_plan_destroy(self.handle)
            self.handle = ctypes.c_void_p(0)

    # ---------------------------------------------------------------- queries
    def info(self) -> dict:
        nt, nb, ws = ctypes.c_int64(), ctypes.c_int64(), ctypes.c_int64()
        vt, nl = ctypes.c_int32(), ctypes.c_int32()
        check(lib.vb_plan_info(self.handle, ctypes.byref(nt), ctypes.byref(nb), ctypes.byref(ws),
                               ctypes.byref(vt), ctypes.byref(nl)))
        return dict(n_tiles=nt.value, n_blocks=nb.value, workspace_bytes=ws.value, version_T=vt.value,
                    launches_per_exec=nl.value)

    def policy(self) -> int:
        """The batching policy the plan was built with (AUTO resolved; -1 for a user schedule)."""
        v = ctypes.c_int32()
        check(lib.vb_plan_policy(self.handle, ctypes.byref(v)))
        return v.value

    def export(self) -> dict:
        inf = self.info()
        bp = np.zeros(inf["n_blocks"] + 1, np.int32)
        n = inf["n_tiles"]
        tg, ty, tx = (np.zeros(max(n, 1), np.int32) for _ in range(3))
        gs = np.zeros(max(self.batch, 1), np.int32)
        check(lib.vb_plan_export(self.handle, _ptr(bp, _i32p), _ptr(tg, _i32p), _ptr(ty, _i32p), _ptr(tx, _i32p),
                                 _ptr(gs, _i32p)))
        return dict(block_ptr=bp, tile_gemm=tg[:n], tile_y=ty[:n], tile_x=tx[:n], gemm_strategy=gs[:self.batch],
                    version_T=inf["version_T"])

    def debug_tmaps(self) -> np.ndarray:
        """The plan's tensor maps (device copy) as raw bytes [batch, maps, 128] (diagnostic)."""
        n = ctypes.c_int64()
        check(lib.vb_plan_debug_tmaps(self.handle, None, 0, ctypes.byref(n)))
        out = np.zeros(n.value, np.uint8)
        if n.value:
            check(lib.vb_plan_debug_tmaps(self.handle, out.ctypes.data, n.value, ctypes.byref(n)))
        return out.reshape(self.batch, -1, 128) if n.value else out

    def tiler_trace(self):
        n = ctypes.c_int32()
        check(lib.vb_plan_tiler_trace(self.handle, 0, None, None, ctypes.byref(n)))
        tl = np.zeros(max(n.value, 1), np.int64)
        vt = np.zeros(max(n.value, 1), np.int32)
        check(lib.vb_plan_tiler_trace(self.handle, n.value, _ptr(tl, _i64p), _ptr(vt, _i32p), ctypes.byref(n)))
        return [(int(a), int(b)) for a, b in zip(tl[:n.value], vt[:n.value])]

    # ---------------------------------------------------------------- exec
    def exec(self, A_ptrs: int, B_ptrs: int, C_ptrs: int, alpha: int, beta: int, stream: int = 0) -> None:
        """All arguments are raw DEVICE addresses (ints); stream is a cudaStream_t as int."""
        check(lib.vb_exec_vbatched(self.handle, _vp(A_ptrs), _vp(B_ptrs), _vp(C_ptrs), _vp(alpha), _vp(beta),
                                   _vp(stream)))

    def bind(self, A_ptrs: int, B_ptrs: int, C_ptrs: int, stream: int = 0) -> None:
        check(lib.vb_plan_bind(self.handle, _vp(A_ptrs), _vp(B_ptrs), _vp(C_ptrs), _vp(stream)))

    def exec_bound(self, alpha: int, beta: int, stream: int = 0) -> None:
        check(lib.vb_exec_bound(self.handle, _vp(alpha), _vp(beta), _vp(stream)))


def plan_vbatched(M, N, K, lda, ldb, ldc, dtype: str = "bf16", policy: int = VB_BATCH_THRESHOLD,
                  device: int = 0, table_id: int = 0, tlp_threshold: int = 0, theta: int = 0) -> Plan:
    arrs = [_i32(a) for a in (M, N, K, lda, ldb, ldc)]
    batch = len(arrs[0])
    tun = vb_tuning(table_id, tlp_threshold, theta)
    h = ctypes.c_void_p()
    check(lib.vb_plan_vbatched(int(device), DTYPE_CODE[dtype], batch, *[_ptr(a, _i32p) for a in arrs], int(policy),
                               ctypes.byref(tun), ctypes.byref(h)))
    return Plan(h.value, batch, dtype)


def plan_conv(convs, dtype: str = "bf16", policy: int = VB_BATCH_THRESHOLD, device: int = 0, table_id: int = 0,
              tlp_threshold: int = 0, theta: int = 0) -> Plan:
    """vb_plan_conv: convs = sequence of dicts with keys nb, H, W, Cin, Cout, KH, KW, pad, ldb, ldc."""
    arr = (vb_conv_desc * max(len(convs), 1))()
    for i, c in enumerate(convs):
        for k, _ in vb_conv_desc._fields_:
            setattr(arr[i], k, int(c[k]))
    tun = vb_tuning(table_id, tlp_threshold, theta)
    h = ctypes.c_void_p()
    check(lib.vb_plan_conv(int(device), DTYPE_CODE[dtype], len(convs), arr, int(policy), ctypes.byref(tun),
                           ctypes.byref(h)))
    return Plan(h.value, len(convs), dtype)


def plan_tune(M, N, K, lda, ldb, ldc, A_ptrs: int, B_ptrs: int, C_ptrs: int, alpha: int, beta: int,
              dtype: str = "bf16", device: int = 0, reps: int = 3, stream: int = 0, table_id: int = 0,
              tlp_threshold: int = 0, theta: int = 0):
    """vb_plan_tune: time THRESHOLD and BINARY on the given DEVICE buffers and keep the faster
    (P272).  Synchronises the stream; C is overwritten.  Returns (plan, [ms_threshold, ms_binary])."""
    arrs = [_i32(a) for a in (M, N, K, lda, ldb, ldc)]
    batch = len(arrs[0])
    tun = vb_tuning(table_id, tlp_threshold, theta)
    h = ctypes.c_void_p()
    ms = (ctypes.c_float * 2)()
    check(lib.vb_plan_tune(int(device), DTYPE_CODE[dtype], batch, *[_ptr(a, _i32p) for a in arrs], ctypes.byref(tun),
                           _vp(A_ptrs), _vp(B_ptrs), _vp(C_ptrs), _vp(alpha), _vp(beta), int(reps), _vp(stream),
                           ctypes.byref(h), ms))
    return Plan(h.value, batch, dtype), [ms[0], ms[1]]


def plan_from_schedule(M, N, K, lda, ldb, ldc, gemm_row, version_T, block_ptr, tile_gemm, tile_y, tile_x,
                       dtype: str = "bf16", device: int = 0, table_id: int = 0) -> Plan:
    arrs = [_i32(a) for a in (M, N, K, lda, ldb, ldc)]
    batch = len(arrs[0])
    gr, bp = _i32(gemm_row), _i32(block_ptr)
    tg, ty, tx = _i32(tile_gemm), _i32(tile_y), _i32(tile_x)
    h = ctypes.c_void_p()
    check(lib.vb_plan_from_schedule(int(device), DTYPE_CODE[dtype], batch, *[_ptr(a, _i32p) for a in arrs],
                                    int(table_id), _ptr(gr, _i32p), int(version_T), len(bp) - 1, _ptr(bp, _i32p),
                                    _ptr(tg, _i32p), _ptr(ty, _i32p), _ptr(tx, _i32p), ctypes.byref(h)))
    return Plan(h.value, batch, dtype)


def debug_set_coverage(device: int, counts_ptr: int, c_base_ptr: int, elem_bytes: int) -> None:
    """Coverage-counter build only (VB_LIB=.../libvbgemm_cov.so): count every stored C element."""
    check(lib.vb_debug_set_coverage(int(device), _vp(counts_ptr), _vp(c_base_ptr), int(elem_bytes)))


def shard_lpt(M, N, K, n_ranks: int) -> np.ndarray:
    m, n, k = _i32(M), _i32(N), _i32(K)
    out = np.zeros(max(len(m), 1), np.int32)
    check(lib.vb_shard_lpt(len(m), _ptr(m, _i32p), _ptr(n, _i32p), _ptr(k, _i32p), int(n_ranks), _ptr(out, _i32p)))
    return out[:len(m)]


def fill_uniform_batch(dtype: str, rows_d: int, cols_d: int, ld_d: int, ptrs_d: int, gemm_id_d: int, batch: int,
                       seed: int, operand: int, total_elems: int, stream: int = 0) -> None:
    check(lib.vb_fill_uniform_batch(DTYPE_CODE[dtype], int(batch), _vp(rows_d), _vp(cols_d), _vp(ld_d), _vp(ptrs_d),
                                    _vp(gemm_id_d), ctypes.c_uint64(seed), int(operand), int(total_elems),
                                    _vp(stream)))


def fill_alpha_beta(batch: int, gemm_id_d: int, seed: int, alpha_d: int, beta_d: int, stream: int = 0) -> None:
    check(lib.vb_fill_alpha_beta(int(batch), _vp(gemm_id_d), ctypes.c_uint64(seed), _vp(alpha_d), _vp(beta_d),
                                 _vp(stream)))


def device_info(device: int = 0) -> dict:
    s, a, b = ctypes.c_int32(), ctypes.c_int32(), ctypes.c_int32()
    check(lib.vb_device_info(int(device), ctypes.byref(s), ctypes.byref(a), ctypes.byref(b)))
    return dict(sm_count=s.value, cc=(a.value, b.value))


def version() -> str:
    return lib.vb_version().decode()
