"""ctypes loader for oracle/ted_matfree.c (O2) -- TEST INFRASTRUCTURE ONLY.

Builds oracle/libted_matfree.so with gcc (plain C + OpenMP, fp64, no
-ffast-math, no FP contraction) on first use.  O2 runs Algorithm 1
 with K^(S) in its closed form K - L L^T (pin C2) and rows
of K recomputed from the features: O(N m) memory, so it reaches N = 65536
and beyond where the dense oracle (8 N^2 bytes) cannot.  Pinned against the
literal oracle (every score of every step) and a hand-computed example in
tests/test_oracle_pins.py.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

from .literal import TedTrace

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "ted_matfree.c")
_LIB = os.path.join(_HERE, "libted_matfree.so")
_lib = None


def build(force: bool = False) -> str:
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-ffp-contract=off", "-fPIC",
                               "-shared", _SRC, "-o", _LIB, "-lm"])
    return _LIB


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB)
        vp = ctypes.c_void_p
        lib.matfree_ted.argtypes = [vp, ctypes.c_int64, ctypes.c_int32, ctypes.c_double, ctypes.c_int32,
                                    ctypes.c_double, ctypes.c_int32, vp, vp, vp, vp, vp, vp, vp, ctypes.c_int64]
        lib.matfree_ted.restype = ctypes.c_int
        lib.matfree_num_threads.restype = ctypes.c_int
        _lib = lib
    return _lib


def num_threads() -> int:
    return int(_load().matfree_num_threads())


def cache_budget() -> int:
    """Bytes of host RAM the oracle may use to keep the N^2 kernel values
    (BTED_ORACLE_CACHE_GB overrides; default half of the available memory)."""
    env = os.environ.get("BTED_ORACLE_CACHE_GB")
    if env is not None:
        return int(float(env) * (1 << 30))
    try:
        avail = os.sysconf("SC_AVPHYS_PAGES") * os.sysconf("SC_PAGE_SIZE")
    except (ValueError, OSError):
        return 0
    return int(avail * 0.5)


def ted(X: np.ndarray, gamma: float, mu: float, m: int, forced=None, linear: bool = False,
        keep_scores: bool = False, cache_bytes: int | None = None) -> TedTrace:
    """TED(V, mu, m) (Alg. 1), matrix-free fp64.  keep_scores: the full masked
    score vector of every step in tr.scores (m x N).  cache_bytes: RAM granted
    for keeping the N^2 kernel values (same result, fewer recomputations);
    default cache_budget()."""
    X = np.ascontiguousarray(X, dtype=np.float32)
    N, d = X.shape
    idx = np.empty(m, np.int64); sc = np.empty(m); am = np.empty(m, np.int64)
    mx = np.empty(m); gp = np.empty(m)
    fptr = None
    if forced is not None:
        forced = np.ascontiguousarray(np.asarray(forced, dtype=np.int64)[:m])
        fptr = forced.ctypes.data
    allsc = np.empty((m, N)) if keep_scores else None
    rc = _load().matfree_ted(X.ctypes.data, N, d, float(gamma), 1 if linear else 0, float(mu), int(m), fptr,
                             idx.ctypes.data, sc.ctypes.data, am.ctypes.data, mx.ctypes.data, gp.ctypes.data,
                             allsc.ctypes.data if allsc is not None else None,
                             int(cache_budget() if cache_bytes is None else cache_bytes))
    if rc != 0:
        raise ValueError("matfree_ted: invalid input, allocation failure or forced index selected twice")
    tr = TedTrace()
    tr.idx, tr.score, tr.argmax = idx.tolist(), sc.tolist(), am.tolist()
    tr.max_score, tr.gap = mx.tolist(), gp.tolist()
    if allsc is not None:
        tr.scores = list(allsc)
    return tr
