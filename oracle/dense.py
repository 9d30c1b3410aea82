"""ctypes loader for oracle/ted_dense.c -- TEST INFRASTRUCTURE ONLY.

Builds oracle/libted_oracle.so with gcc (plain C + OpenMP, fp64, no
-ffast-math, no FP contraction) on first use if it is missing.  The same
literal Algorithm 1 as oracle/ted.py; tests pin the two
against each other and against the mathematical pins.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

from .literal import TedTrace

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "ted_dense.c")
_LIB = os.path.join(_HERE, "libted_oracle.so")
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
        i64p = ctypes.POINTER(ctypes.c_int64)
        f64p = ctypes.POINTER(ctypes.c_double)
        lib.oracle_gram.argtypes = [ctypes.c_void_p, ctypes.c_int64, ctypes.c_int32,
                                    ctypes.c_double, ctypes.c_void_p]
        lib.oracle_gram.restype = None
        lib.oracle_ted_on_matrix.argtypes = [ctypes.c_void_p, ctypes.c_int64, ctypes.c_double,
                                             ctypes.c_int32, ctypes.c_void_p, i64p, f64p,
                                             i64p, f64p, f64p]
        lib.oracle_ted_on_matrix.restype = ctypes.c_int
        lib.oracle_num_threads.restype = ctypes.c_int
        _lib = lib
    return _lib


def num_threads() -> int:
    return int(_load().oracle_num_threads())


def gram(X: np.ndarray, gamma: float) -> np.ndarray:
    X = np.ascontiguousarray(X, dtype=np.float32)
    N, d = X.shape
    K = np.empty((N, N), dtype=np.float64)
    _load().oracle_gram(X.ctypes.data, N, d, float(gamma), K.ctypes.data)
    return K


def ted_on_matrix(K: np.ndarray, mu: float, m: int, forced=None) -> TedTrace:
    """Alg. 1 l.2-7 on K (K is CONSUMED: deflated in place)."""
    assert K.dtype == np.float64 and K.flags.c_contiguous
    N = K.shape[0]
    lib = _load()
    idx = np.empty(m, np.int64); sc = np.empty(m); am = np.empty(m, np.int64)
    mx = np.empty(m); gp = np.empty(m)
    fptr = None
    if forced is not None:
        forced = np.ascontiguousarray(np.asarray(forced, dtype=np.int64)[:m])
        fptr = forced.ctypes.data
    rc = lib.oracle_ted_on_matrix(
        K.ctypes.data, N, float(mu), int(m), fptr,
        idx.ctypes.data_as(ctypes.POINTER(ctypes.c_int64)),
        sc.ctypes.data_as(ctypes.POINTER(ctypes.c_double)),
        am.ctypes.data_as(ctypes.POINTER(ctypes.c_int64)),
        mx.ctypes.data_as(ctypes.POINTER(ctypes.c_double)),
        gp.ctypes.data_as(ctypes.POINTER(ctypes.c_double)))
    if rc != 0:
        raise ValueError("oracle_ted_on_matrix: invalid input or forced index selected twice")
    tr = TedTrace()
    tr.idx, tr.score, tr.argmax = idx.tolist(), sc.tolist(), am.tolist()
    tr.max_score, tr.gap = mx.tolist(), gp.tolist()
    return tr


def ted(X: np.ndarray, gamma: float, mu: float, m: int, forced=None) -> TedTrace:
    """TED(V, mu, m) (Alg. 1) in C/OpenMP fp64; memory 8 N^2 bytes."""
    return ted_on_matrix(gram(X, gamma), mu, m, forced=forced)
