"""ctypes loader for oracle/c/oracle_ref.c — TEST INFRASTRUCTURE ONLY.

Built by ``__graft_entry__.build()`` (building the checker is not using it);
only tests and bench.py's cpu_baseline / reference legs call it.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
SRC = os.path.join(_HERE, "c", "oracle_ref.c")
LIB = os.path.join(_HERE, "c", "liboracle_ref.so")
_lib = None


def build(force=False):
    if force or not os.path.exists(LIB) or os.path.getmtime(LIB) < os.path.getmtime(SRC):
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-fPIC", "-shared", SRC, "-o", LIB])
    return LIB


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(LIB)
        P = ctypes.c_void_p
        L.oracle_spmv_f64.argtypes = [ctypes.c_int64, P, P, P, P, P, ctypes.c_int]
        L.oracle_gemm_f64.argtypes = [ctypes.c_int64] * 3 + [ctypes.c_double, P, P,
                                                            ctypes.c_double, P, P, ctypes.c_int]
        L.oracle_max_threads.restype = ctypes.c_int
        _lib = L
    return _lib


def _p(a):
    return a.ctypes.data_as(ctypes.c_void_p)


def spmv_f64(row_ptr, col, val, x, nthreads=1):
    rp = np.ascontiguousarray(row_ptr, np.int32)
    n = rp.shape[0] - 1
    y = np.empty(n, np.float64)
    c = np.ascontiguousarray(col, np.int32)
    v = np.ascontiguousarray(val, np.float32)
    xx = np.ascontiguousarray(x, np.float32)
    lib().oracle_spmv_f64(n, _p(rp), _p(c), _p(v), _p(xx), _p(y), int(nthreads))
    return y


def gemm_f64(A, B, C0, alpha, beta, nthreads=1):
    A = np.ascontiguousarray(A, np.float32)
    B = np.ascontiguousarray(B, np.float32)
    C0 = np.ascontiguousarray(C0, np.float32)
    M, K = A.shape
    N = B.shape[1]
    C = np.empty((M, N), np.float64)
    lib().oracle_gemm_f64(M, N, K, float(alpha), _p(A), _p(B), float(beta), _p(C0), _p(C), int(nthreads))
    return C


def max_threads():
    return int(lib().oracle_max_threads())
