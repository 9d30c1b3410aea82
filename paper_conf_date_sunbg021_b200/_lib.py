"""ctypes binding of include/bted.h (libbted.so).  Argument marshalling only:
every step of TED/BTED runs in the library's CUDA kernels.  There is no CPU
fallback -- if libbted.so is missing or no sm_100 device is usable, calls
raise."""
from __future__ import annotations

import ctypes
import os

import numpy as np

from .build import LIB

BTED_KERNEL_RBF = 0
BTED_KERNEL_LINEAR = 1
BTED_FLAG_NO_GRAPH = 1
BTED_FLAG_TIMING = 2
BTED_FLAG_DENSE = 4
BTED_FLAG_NO_SMALL = 8
BTED_FLAG_TMA = 16
BTED_FLAG_IMPLICIT = 32
BTED_FLAG_LITERAL = 64
BTED_FLAG_NO_REFINE = 128
BTED_FLAG_PERSISTENT_LOOP = 256
BTED_FLAG_LOOPBACK = 512
BTED_FLAG_NCCL = 1024
BTED_FLAG_NO_TC_GRAM = 2048
BTED_FLAG_RECOMPUTE = 4096
STATUS = {0: "BTED_OK", 1: "BTED_EINVAL", 2: "BTED_ENOMEM", 3: "BTED_ECUDA", 4: "BTED_ENCCL",
          5: "BTED_ENUMERIC", 6: "BTED_ESTATE"}


class BtedError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{STATUS.get(status, status)}: {msg}")
        self.status = status


class bted_params(ctypes.Structure):
    _fields_ = [
        ("gamma", ctypes.c_float),
        ("device", ctypes.c_int32),
        ("num_batches", ctypes.c_int32),
        ("seed", ctypes.c_uint64),
        ("x_on_device", ctypes.c_int32),
        ("flags", ctypes.c_uint32),
        ("stream", ctypes.c_size_t),
        ("num_devices", ctypes.c_int32),
        ("norm_mode", ctypes.c_int32),
    ]


class bted_stats(ctypes.Structure):
    _fields_ = [("teds", ctypes.c_uint64), ("k2_launches", ctypes.c_uint64),
                ("k1_ms", ctypes.c_double), ("k2_ms", ctypes.c_double),
                ("small_teds", ctypes.c_uint64), ("small_ms", ctypes.c_double),
                ("refined_steps", ctypes.c_uint64), ("corrected_steps", ctypes.c_uint64),
                ("full_refined_steps", ctypes.c_uint64)]


_lib = None
_vp, _i64, _i32, _u64, _f32 = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int32, ctypes.c_uint64, ctypes.c_float
_SIGS = {
    "bted_default_params": (None, [ctypes.POINTER(bted_params)]),
    "bted_create": (ctypes.c_int, [_vp, _i64, _i32, ctypes.c_int, ctypes.POINTER(bted_params), ctypes.POINTER(_vp)]),
    "bted_select": (ctypes.c_int, [_vp, _i32, _f32, _vp, _vp]),
    "bted_run_batches": (ctypes.c_int, [_vp, _i64, _i32, _f32, _vp, _vp, _vp]),
    "bted_batch_teds": (ctypes.c_int, [_vp, _i64, _i32, _f32, _i32, _i32, _vp, _i32]),
    "bted_merge": (ctypes.c_int, [_vp, _vp, _i64, _i32, _i32, _f32, _vp, _vp]),
    "bted_sample_batches": (ctypes.c_int, [_i64, _i64, _i32, _u64, _vp]),
    "bted_shard_create": (ctypes.c_int, [_vp, _i64, _i32, ctypes.c_int, _i64, _i64, ctypes.POINTER(bted_params),
                                         ctypes.POINTER(_vp)]),
    "bted_shard_gram": (ctypes.c_int, [_vp, _f32, _vp]),
    "bted_shard_step": (ctypes.c_int, [_vp, _i32, _f32, _vp, _vp]),
    "bted_shard_pivot_column": (ctypes.c_int, [_vp, _i32, _vp, _vp]),
    "bted_shard_colnorm": (ctypes.c_int, [_vp, _i32, _f32, _vp, _vp, _vp]),
    "bted_shard_scores": (ctypes.c_int, [_vp, _i32, _f32, _vp, _vp]),
    "bted_shard_ld": (_i64, [_vp]),
    "bted_shard_nearties": (ctypes.c_int, [_vp, _i32, _vp, _vp, _vp]),
    "bted_shard_refine": (ctypes.c_int, [_vp, _i32, _f32, _vp, _vp, _vp, _i32, _vp, ctypes.POINTER(_i32)]),
    "bted_ishard_create": (ctypes.c_int, [_vp, _i64, _i32, ctypes.c_int, _i32, _i32, ctypes.POINTER(bted_params),
                                          ctypes.POINTER(_vp)]),
    "bted_ishard_head": (ctypes.c_int, [_vp, _i32, _f32, _vp]),
    "bted_ishard_step": (ctypes.c_int, [_vp, _i32, _f32, _vp, _vp]),
    "bted_ishard_fin": (ctypes.c_int, [_vp, _i32, _f32, _vp, _vp]),
    "bted_ishard_qlen": (_i64, [_vp]),
    "bted_ishard_refine": (ctypes.c_int, [_vp, _i32, _f32, _vp, _vp, ctypes.POINTER(_i32)]),
    "bted_shard_check": (ctypes.c_int, [_vp]),
    "bted_destroy": (None, [_vp]),
    "bted_status_string": (ctypes.c_char_p, [ctypes.c_int]),
    "bted_last_error": (ctypes.c_char_p, []),
    "bted_kernel_launches": (_u64, []),
    "bted_debug_copy_K": (ctypes.c_int, [_vp, _i32, _vp, ctypes.POINTER(_i64)]),
    "bted_update": (ctypes.c_int, [_vp, _vp, _i32]),
    "bted_get_stats": (ctypes.c_int, [_vp, ctypes.POINTER(bted_stats)]),
    "bted_reset_stats": (ctypes.c_int, [_vp]),
    "bted_host_alloc": (ctypes.c_int, [ctypes.c_size_t, ctypes.POINTER(_vp)]),
    "bted_host_free": (None, [_vp]),
}
EXPORTS = tuple(_SIGS)


def lib():
    """Load libbted.so (built by __graft_entry__.build()); raise if absent."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB):
            raise RuntimeError(f"{LIB} is not built: run `python -c 'import __graft_entry__ as g; g.build()'` "
                               "(there is no CPU fallback)")
        L = ctypes.CDLL(LIB)
        for name, (res, args) in _SIGS.items():
            f = getattr(L, name)
            f.restype = res
            f.argtypes = args
        _lib = L
    return _lib


def check(status: int):
    if status != 0:
        raise BtedError(status, lib().bted_last_error().decode(errors="replace"))


def _ptr(a: np.ndarray) -> int:
    return a.ctypes.data


def default_params(gamma=1.0, device=-1, num_batches=1, seed=0, x_on_device=0, flags=0, stream=0,
                   num_devices=1, norm_mode=0) -> bted_params:
    p = bted_params()
    lib().bted_default_params(ctypes.byref(p))
    p.gamma, p.device, p.num_batches, p.seed = float(gamma), int(device), int(num_batches), int(seed)
    p.x_on_device, p.flags, p.stream = int(x_on_device), int(flags), int(stream)
    p.num_devices, p.norm_mode = int(num_devices), int(norm_mode)
    return p


# -------------------------------------------------------------- C-ABI names
def bted_create(X, N: int, d: int, kernel: int, params: bted_params) -> int:
    """X: host np.float32 [N, d] C-contiguous, or an int device pointer with
    params.x_on_device = 1.  Returns the opaque ctx handle."""
    out = _vp()
    xh = None if isinstance(X, int) else np.ascontiguousarray(X, dtype=np.float32)
    xp = X if xh is None else _ptr(xh)         # xh stays referenced across the call
    check(lib().bted_create(xp, int(N), int(d), int(kernel), ctypes.byref(params), ctypes.byref(out)))
    return out.value


def bted_shard_create(X, N: int, d: int, kernel: int, row0: int, row1: int, params: bted_params) -> int:
    out = _vp()
    xh = None if isinstance(X, int) else np.ascontiguousarray(X, dtype=np.float32)
    xp = X if xh is None else _ptr(xh)
    check(lib().bted_shard_create(xp, int(N), int(d), int(kernel), int(row0), int(row1), ctypes.byref(params),
                                  ctypes.byref(out)))
    return out.value


def bted_select(ctx: int, m: int, mu: float):
    idx = np.empty(int(m), dtype=np.int64)
    score = np.empty(int(m), dtype=np.float32)
    check(lib().bted_select(ctx, int(m), float(mu), _ptr(idx), _ptr(score)))
    return idx, score


def bted_run_batches(ctx: int, M: int, m: int, mu: float, num_batches: int, want_batches: bool = True):
    idx = np.empty(int(m), dtype=np.int64)
    count = ctypes.c_int32(0)
    bidx = np.empty((int(num_batches), int(m)), dtype=np.int64) if want_batches else None
    check(lib().bted_run_batches(ctx, int(M), int(m), float(mu), _ptr(idx), ctypes.addressof(count),
                                 _ptr(bidx) if bidx is not None else None))
    return idx[: count.value], bidx


def bted_batch_teds(ctx: int, M: int, m: int, mu: float, b_begin: int, b_step: int, out_winners,
                    winners_on_device: bool = False):
    """out_winners: host np.int64 array, or an int device pointer."""
    ptr = out_winners if isinstance(out_winners, int) else _ptr(out_winners)
    check(lib().bted_batch_teds(ctx, int(M), int(m), float(mu), int(b_begin), int(b_step), ptr,
                                1 if winners_on_device else 0))


def bted_merge(ctx: int, winners, n: int, m: int, mu: float, winners_on_device: bool = False):
    wh = None if isinstance(winners, int) else np.ascontiguousarray(winners, dtype=np.int64)
    ptr = winners if wh is None else _ptr(wh)
    idx = np.empty(int(m), dtype=np.int64)
    count = ctypes.c_int32(0)
    check(lib().bted_merge(ctx, ptr, int(n), 1 if winners_on_device else 0, int(m), float(mu), _ptr(idx),
                           ctypes.addressof(count)))
    return idx[: count.value]


def bted_sample_batches(P: int, M: int, B: int, seed: int) -> np.ndarray:
    out = np.empty((int(B), int(M)), dtype=np.int64)
    check(lib().bted_sample_batches(int(P), int(M), int(B), int(seed), _ptr(out)))
    return out


def bted_ishard_create(X, N: int, d: int, kernel: int, rank: int, nranks: int, params: bted_params) -> int:
    out = _vp()
    xh = None if isinstance(X, int) else np.ascontiguousarray(X, dtype=np.float32)
    xp = X if xh is None else _ptr(xh)
    check(lib().bted_ishard_create(xp, int(N), int(d), int(kernel), int(rank), int(nranks), ctypes.byref(params),
                                   ctypes.byref(out)))
    return out.value


def bted_ishard_head(ctx: int, m: int, mu: float, q_dev: int):
    check(lib().bted_ishard_head(ctx, int(m), float(mu), q_dev))


def bted_ishard_step(ctx: int, t: int, mu: float, keys_dev: int, q_dev: int):
    check(lib().bted_ishard_step(ctx, int(t), float(mu), keys_dev, q_dev))


def bted_ishard_fin(ctx: int, t: int, mu: float, q_dev: int, keys_dev: int):
    check(lib().bted_ishard_fin(ctx, int(t), float(mu), q_dev, keys_dev))


def bted_ishard_refine(ctx: int, m: int, mu: float, keys_dev: int) -> np.ndarray:
    """K4 for the tile-sharded engine: [] if the selection stands, else the keys to preset (u64)."""
    forced = np.zeros(int(m), dtype=np.uint64)
    n = _i32(0)
    check(lib().bted_ishard_refine(ctx, int(m), float(mu), keys_dev, _ptr(forced), ctypes.byref(n)))
    return forced[: n.value]


def bted_ishard_qlen(ctx: int) -> int:
    return int(lib().bted_ishard_qlen(ctx))


def bted_shard_gram(ctx: int, mu: float, keys_dev: int):
    check(lib().bted_shard_gram(ctx, float(mu), keys_dev))


def bted_shard_step(ctx: int, t: int, mu: float, pivot_dev: int, keys_dev: int):
    check(lib().bted_shard_step(ctx, int(t), float(mu), pivot_dev, keys_dev))


def bted_shard_pivot_column(ctx: int, t: int, keys_dev: int, col_dev: int):
    check(lib().bted_shard_pivot_column(ctx, int(t), keys_dev, col_dev))


def bted_shard_colnorm(ctx: int, t: int, mu: float, pivot_dev, keys_dev, colnorm_dev: int):
    check(lib().bted_shard_colnorm(ctx, int(t), float(mu), pivot_dev or None, keys_dev or None, colnorm_dev))


def bted_shard_scores(ctx: int, t: int, mu: float, colnorm_dev: int, keys_dev: int):
    check(lib().bted_shard_scores(ctx, int(t), float(mu), colnorm_dev, keys_dev))


def bted_shard_nearties(ctx: int, m: int, keys_dev: int, cand_dev: int, ncand_dev: int):
    check(lib().bted_shard_nearties(ctx, int(m), keys_dev, cand_dev, ncand_dev))


def bted_shard_refine(ctx: int, m: int, mu: float, keys_dev: int, cand_all: np.ndarray, ncand_all: np.ndarray,
                      nranks: int) -> np.ndarray:
    """K4 for the row-sharded TED: [] if the selection stands, else the keys to preset (u64)."""
    cand_all = np.ascontiguousarray(cand_all, dtype=np.uint32)
    ncand_all = np.ascontiguousarray(ncand_all, dtype=np.int32)
    forced = np.zeros(int(m), dtype=np.uint64)
    n = _i32(0)
    check(lib().bted_shard_refine(ctx, int(m), float(mu), keys_dev, _ptr(cand_all), _ptr(ncand_all), int(nranks),
                                  _ptr(forced), ctypes.byref(n)))
    return forced[: n.value]


def bted_shard_ld(ctx: int) -> int:
    return int(lib().bted_shard_ld(ctx))


def bted_shard_check(ctx: int):
    check(lib().bted_shard_check(ctx))


def bted_destroy(ctx: int):
    if ctx:
        lib().bted_destroy(ctx)


def bted_kernel_launches() -> int:
    return int(lib().bted_kernel_launches())


def bted_debug_copy_K(ctx: int, which: int, rows: int, ld: int) -> np.ndarray:
    out = np.empty((int(rows), int(ld)), dtype=np.float32)
    ldo = _i64(0)
    check(lib().bted_debug_copy_K(ctx, int(which), _ptr(out), ctypes.byref(ldo)))
    assert ldo.value == ld
    return out


_UPDATE_KEEP: dict = {}


def bted_update(ctx: int, X, x_on_device: bool = False, shape=None):
    """X: int pointer (host pinned or device; the caller guarantees N x d fp32),
    or a host array, which must be N x d (shape = the ctx's (N, d), checked when
    given) and is converted to C-contiguous fp32.  The H2D copy is asynchronous:
    the converted array is kept referenced until the next update of this ctx."""
    if isinstance(X, int):
        ptr = X
    else:
        A = np.ascontiguousarray(X, dtype=np.float32)
        if A.ndim != 2 or (shape is not None and tuple(A.shape) != tuple(shape)):
            raise ValueError(f"bted_update: X has shape {A.shape}, the context holds {shape}")
        _UPDATE_KEEP[ctx] = A            # alive until the copy has run (next update / call)
        ptr = _ptr(A)
    check(lib().bted_update(ctx, ptr, 1 if x_on_device else 0))


class PinnedArray:
    """A numpy view of page-locked memory from bted_host_alloc (freed on close/del)."""

    def __init__(self, shape, dtype=np.float32):
        dtype = np.dtype(dtype)
        n = int(np.prod(shape)) * dtype.itemsize
        p = _vp()
        check(lib().bted_host_alloc(n, ctypes.byref(p)))
        self.ptr = p.value
        buf = (ctypes.c_char * n).from_address(self.ptr)
        self.array = np.frombuffer(buf, dtype=dtype).reshape(shape)

    def close(self):
        if getattr(self, "ptr", None):
            self.array = None
            lib().bted_host_free(self.ptr)
            self.ptr = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def bted_get_stats(ctx: int) -> dict:
    st = bted_stats()
    check(lib().bted_get_stats(ctx, ctypes.byref(st)))
    return dict(teds=st.teds, k2_launches=st.k2_launches, k1_ms=st.k1_ms, k2_ms=st.k2_ms,
                small_teds=st.small_teds, small_ms=st.small_ms, refined_steps=st.refined_steps,
                corrected_steps=st.corrected_steps, full_refined_steps=st.full_refined_steps)


def bted_reset_stats(ctx: int):
    check(lib().bted_reset_stats(ctx))


def decode_keys(keys: np.ndarray):
    """Packed keys (u64) -> (index, fp32 score).  See include/bted.h."""
    keys = np.asarray(keys, dtype=np.uint64) & np.uint64(0x7FFFFFFFFFFFFFFF)   # K4's forced-pick flag
    idx = (np.uint64(0xFFFFFFFF) - (keys & np.uint64(0xFFFFFFFF))).astype(np.int64)
    bits = ((keys >> np.uint64(32)) - np.uint64(1)).astype(np.uint32)
    return idx, bits.view(np.float32)
