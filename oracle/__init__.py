"""ScalFrag oracle -- TEST INFRASTRUCTURE ONLY.

Plain, slow, obviously-correct CPU implementations of what the hot path
computes, written from PAPER.md.  Only ``tests/``, ``__graft_entry__.smoke()``
and ``bench.py``'s cpu_baseline / ``--impl reference`` leg may import this
package.  It shares no code with ``paper_conf_cluster_linwds24_b200`` (the
CUDA path) and neither imports the other.

* ``mttkrp`` / ``mttkrp_rows`` -- oracle.c, the elementwise definition of
  Eq. (4) in fp64, single thread, input order.
* ``plan.py``  -- the integer preprocessing the CUDA path must reproduce
  bit-exactly: stable mode orders, tiles, fragments, features (PAPER.md L189,
  L195, L205) and nnz-balanced shard cuts.
* ``cpals.py`` -- CP-ALS, Algorithm 1, the consumer.

Pins: tests/test_oracle.py, tests/test_oracle_plan.py.  Nothing here is
"parity unpinned" except where DESIGN.md §Readings says so.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "liboracle.so")
_SRC = os.path.join(_HERE, "oracle.c")
_lock = threading.Lock()
_lib = None


def build(force: bool = False) -> str:
    """Compile liboracle.so (plain C, gcc -O2, single thread, no fast-math)."""
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(_SRC):
        tmp = _SO + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-fno-fast-math", "-ffp-contract=off", "-shared",
                               "-fPIC", "-std=c11", "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _SO)
    return _SO


def lib():
    global _lib
    with _lock:
        if _lib is None:
            build()
            L = ctypes.CDLL(_SO)
            P = ctypes.c_void_p
            L.or_mttkrp.argtypes = [ctypes.c_int, P, ctypes.c_uint64, P, P, P, ctypes.c_int,
                                    ctypes.c_int, P, P]
            L.or_mttkrp.restype = ctypes.c_int
            L.or_mttkrp_rows.argtypes = [ctypes.c_int, P, ctypes.c_uint64, P, P, P, ctypes.c_int,
                                         ctypes.c_int, P, ctypes.c_int64, P, P]
            L.or_mttkrp_rows.restype = ctypes.c_int
            _lib = L
    return _lib


def _prep(dims, inds, vals, factors, rank):
    N = len(dims)
    d = np.ascontiguousarray(dims, dtype=np.uint64)
    inds = [np.ascontiguousarray(a, dtype=np.uint32) for a in inds]
    vals = np.ascontiguousarray(vals, dtype=np.float32)
    fac = []
    for m in range(N):
        f = factors[m]
        if f is None:
            f = np.zeros((1, rank), np.float32)
        fac.append(np.ascontiguousarray(f, dtype=np.float32))
    ip = (ctypes.c_void_p * N)(*[a.ctypes.data for a in inds])
    fp = (ctypes.c_void_p * N)(*[f.ctypes.data for f in fac])
    keep = (d, inds, vals, fac)
    return d, ip, fp, vals, keep


def mttkrp(dims, inds, vals, factors, rank, mode, with_scale=True):
    """Mode-`mode` MTTKRP, Eq. (4) elementwise (oracle.c).  Returns (Y, S) fp64 (I_n x R)."""
    d, ip, fp, v, keep = _prep(dims, inds, vals, factors, rank)
    In = int(dims[mode])
    Y = np.empty((In, rank), np.float64)
    S = np.empty((In, rank), np.float64) if with_scale else None
    rc = lib().or_mttkrp(len(dims), d.ctypes.data, len(v), ip, v.ctypes.data, fp, rank, mode,
                         Y.ctypes.data, S.ctypes.data if S is not None else None)
    if rc != 0:
        raise ValueError(f"or_mttkrp failed rc={rc}")
    return Y, S


def mttkrp_rows(dims, inds, vals, factors, rank, mode, rows):
    """Eq. (4) for the listed output rows only (one pass over all nonzeros)."""
    rows = np.asarray(rows, dtype=np.int64)
    d, ip, fp, v, keep = _prep(dims, inds, vals, factors, rank)
    slot = np.full(int(dims[mode]), -1, np.int32)
    slot[rows] = np.arange(len(rows), dtype=np.int32)
    Y = np.empty((len(rows), rank), np.float64)
    S = np.empty((len(rows), rank), np.float64)
    rc = lib().or_mttkrp_rows(len(dims), d.ctypes.data, len(v), ip, v.ctypes.data, fp, rank, mode,
                              slot.ctypes.data, len(rows), Y.ctypes.data, S.ctypes.data)
    if rc != 0:
        raise ValueError(f"or_mttkrp_rows failed rc={rc}")
    return Y, S


def max_rel_err(Y_test, Y, S):
    """Acceptance metric (reading R8): max |Y_test - Y| / S over S > 0,
    plus the max |Y_test| where S == 0 (must be exactly 0)."""
    Y_test = np.asarray(Y_test, dtype=np.float64)
    diff = np.abs(Y_test - Y)
    pos = S > 0
    rel = float(np.max(diff[pos] / S[pos])) if np.any(pos) else 0.0
    zero_violation = float(np.max(np.abs(Y_test[~pos]))) if np.any(~pos) else 0.0
    return rel, zero_violation
