"""Oracle for the Sweet KNN join -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py`` (its
``cpu_baseline`` leg and ``--impl reference`` arm) may import this package.
The product path (``paper_conf_icde_chends17_b200``) never imports it, and this
package never imports the product path; the two share no code.

Contents
--------
* ``knn_join``      -- plain C brute force (``oracle_knn.c``), fp64, the exact
                       definition of the KNN join.
* ``ti``            -- the paper's triangle-inequality bounds and its TI-based
                       KNN (Fig. 4, Alg. 1, Alg. 2) written out step by step in
                       fp64 numpy/Python, used to pin our reading of the paper.
* ``config``        -- the paper's adaptive-scheme arithmetic (Fig. 8, §IV-D).
* ``ref_numpy``     -- an independent tiny numpy lexsort brute force used to
                       cross-check the C oracle.

Parity status per function is listed in DESIGN.md §3 ("Oracle and pins").
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle_knn.c")
_LIB = os.path.join(_HERE, "liboracle_knn.so")
_lock = threading.Lock()
_lib = None


def build(force: bool = False) -> str:
    """Compile oracle_knn.c into liboracle_knn.so (gcc, OpenMP, no fast-math)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + ".tmp.%d" % os.getpid()
        cmd = ["gcc", "-O2", "-fopenmp", "-ffp-contract=off", "-fno-fast-math",
               "-shared", "-fPIC", _SRC, "-o", tmp, "-lm"]
        subprocess.check_call(cmd)
        os.replace(tmp, _LIB)
    return _LIB


def _load():
    global _lib
    with _lock:
        if _lib is None:
            build()
            lib = ctypes.CDLL(_LIB)
            lib.oracle_knn_join.restype = ctypes.c_int
            lib.oracle_knn_join.argtypes = [
                ctypes.c_void_p, ctypes.c_int64, ctypes.c_void_p, ctypes.c_int64,
                ctypes.c_int, ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p,
                ctypes.c_void_p, ctypes.c_int]
            lib.oracle_num_threads.restype = ctypes.c_int
            _lib = lib
    return _lib


def num_threads() -> int:
    return int(_load().oracle_num_threads())


def knn_join(Q, T, k: int, nthreads: int = 0, return_d2: bool = False):
    """Exact KNN join by brute force (fp64 accumulation, ties -> lowest index).

    Q: [nq, d] float32, T: [nt, d] float32 (host arrays).
    Returns (idx int32 [nq, k], dist float32 [nq, k]) and optionally the fp64
    squared distances.
    """
    Q = np.ascontiguousarray(Q, dtype=np.float32)
    T = np.ascontiguousarray(T, dtype=np.float32)
    if Q.ndim != 2 or T.ndim != 2 or Q.shape[1] != T.shape[1]:
        raise ValueError("Q and T must be [n, d] with equal d")
    nq, d = Q.shape
    nt = T.shape[0]
    idx = np.empty((nq, k), dtype=np.int32)
    dist = np.empty((nq, k), dtype=np.float32)
    d2 = np.empty((nq, k), dtype=np.float64) if return_d2 else None
    rc = _load().oracle_knn_join(
        Q.ctypes.data, nq, T.ctypes.data, nt, d, int(k), idx.ctypes.data,
        dist.ctypes.data, d2.ctypes.data if d2 is not None else None, int(nthreads))
    if rc != 0:
        raise ValueError("oracle_knn_join failed (rc=%d): check k <= nt, d > 0" % rc)
    return (idx, dist, d2) if return_d2 else (idx, dist)
