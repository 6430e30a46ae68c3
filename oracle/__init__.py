"""CPU oracle for batched k-selection / brute-force k-NN -- TEST INFRASTRUCTURE.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py`` (its
``cpu_baseline`` leg and ``--impl reference``) may import this package.  The
product path (``paper_conf_ipps_tang0emg15_b200``) never imports it and shares
no code with it; the two meet only through the seeded input generators in
``synth/`` (which hold none of the method's arithmetic).

The arithmetic lives in ``ksel_oracle.c`` (plain C, qsort + a double-precision
triple loop); this module only compiles it with gcc and marshals numpy arrays
through ctypes.  Each function cites the passage it follows:

* :func:`select`   -- PAPER.md L11 (k smallest of an unordered list), L19
  (Algorithm 1: strict ``<`` in index order => ties keep the lower index),
  L637 (sorted output).  Definition: sort (value, index) pairs, truncate.
* :func:`merge`    -- PAPER.md L243 (divide-and-merge, ref. [18]): the k
  smallest of the union of S candidate lists.
* :func:`knn_dist` -- PAPER.md L13 (Euclidean distance phase); reading R9:
  squared L2 accumulated in double, one rounding to fp32.
* :func:`knn`      -- knn_dist followed by select.
* :func:`knn_graph` -- PAPER.md L635-L639 (k-NN graph construction, the target of
  QMS [9]): per point, the k nearest other points (self excluded).

Pins (tests/test_oracle_pins.py): brute-force rank counting, numpy stable
argsort, the north-star invariants, the paper's worked examples
(tests/golden/), closed forms and exact-integer cases for the distance.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "ksel_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None


def build(force: bool = False) -> str:
    """Compile ksel_oracle.c -> liboracle.so (gcc, no fast-math, no FMA contraction)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + ".tmp%d" % os.getpid()
        subprocess.check_call(
            ["gcc", "-O2", "-std=c11", "-fPIC", "-shared", "-ffp-contract=off",
             "-fno-fast-math", "-Wall", "-o", tmp, _SRC, "-lpthread", "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB)
        i64, i32 = ctypes.c_int64, ctypes.c_int
        p = ctypes.c_void_p
        lib.oracle_select.argtypes = [p, i64, i64, i64, p, p, i32]
        lib.oracle_merge.argtypes = [p, p, i64, i64, i64, i64, p, p]
        lib.oracle_knn_dist.argtypes = [p, p, i64, i64, i64, p, i32]
        lib.oracle_knn.argtypes = [p, p, i64, i64, i64, i64, i64, p, p, p, i32]
        lib.oracle_knn_graph.argtypes = [p, i64, i64, i64, p, p, p, i32]
        for f in (lib.oracle_select, lib.oracle_merge, lib.oracle_knn_dist, lib.oracle_knn,
                  lib.oracle_knn_graph):
            f.restype = ctypes.c_int
        _lib = lib
    return _lib


def default_threads() -> int:
    return max(1, len(os.sched_getaffinity(0)))


def _ptr(a: np.ndarray) -> int:
    return a.ctypes.data


def select(dist, k: int, nthreads: int | None = None):
    """(values, indices) of the k smallest (dist[q][j], j) per row, ascending.

    ``dist``: 2-D float32 array-like (Q x N).  Returns float32 (Q x k) holding the
    input bits and int32 (Q x k) 0-based column indices.
    """
    d = np.ascontiguousarray(dist, dtype=np.float32)
    if d.ndim != 2:
        raise ValueError("dist must be 2-D")
    Q, N = d.shape
    ov = np.empty((Q, k), np.float32)
    oi = np.empty((Q, k), np.int32)
    rc = _load().oracle_select(_ptr(d), Q, N, k, _ptr(ov), _ptr(oi),
                               nthreads or default_threads())
    if rc:
        raise ValueError("oracle_select failed (%d)" % rc)
    return ov, oi


def merge(cand_val, cand_idx, k: int):
    """Top-k of the union of S sorted candidate lists; inputs are [S][Q][kin]."""
    v = np.ascontiguousarray(cand_val, dtype=np.float32)
    i = np.ascontiguousarray(cand_idx, dtype=np.int32)
    if v.ndim != 3 or v.shape != i.shape:
        raise ValueError("cand_val/cand_idx must be [S][Q][kin] and equal shapes")
    S, Q, kin = v.shape
    ov = np.empty((Q, k), np.float32)
    oi = np.empty((Q, k), np.int32)
    rc = _load().oracle_merge(_ptr(v), _ptr(i), Q, S, kin, k, _ptr(ov), _ptr(oi))
    if rc:
        raise ValueError("oracle_merge failed (%d)" % rc)
    return ov, oi


def knn_dist(ref, query, nthreads: int | None = None):
    """Q x N squared-L2 distances, double accumulation, one rounding to fp32."""
    r = np.ascontiguousarray(ref, dtype=np.float32)
    q = np.ascontiguousarray(query, dtype=np.float32)
    if r.ndim != 2 or q.ndim != 2 or r.shape[1] != q.shape[1]:
        raise ValueError("ref (N x D) and query (Q x D) must share D")
    N, D = r.shape
    Q = q.shape[0]
    out = np.empty((Q, N), np.float32)
    rc = _load().oracle_knn_dist(_ptr(r), _ptr(q), N, Q, D, _ptr(out),
                                 nthreads or default_threads())
    if rc:
        raise ValueError("oracle_knn_dist failed (%d)" % rc)
    return out


def knn(ref, query, k: int, idx_offset: int = 0, nthreads: int | None = None):
    """(squared distances, global indices) of the k nearest references per query."""
    r = np.ascontiguousarray(ref, dtype=np.float32)
    q = np.ascontiguousarray(query, dtype=np.float32)
    N, D = r.shape
    Q = q.shape[0]
    scratch = np.empty((Q, N), np.float32)
    ov = np.empty((Q, k), np.float32)
    oi = np.empty((Q, k), np.int32)
    rc = _load().oracle_knn(_ptr(r), _ptr(q), N, Q, D, k, idx_offset, _ptr(scratch),
                            _ptr(ov), _ptr(oi), nthreads or default_threads())
    if rc:
        raise ValueError("oracle_knn failed (%d)" % rc)
    return ov, oi


def knn_graph(points, k: int, nthreads: int | None = None):
    """(squared distances, indices) of the k nearest OTHER points of every point."""
    x = np.ascontiguousarray(points, dtype=np.float32)
    if x.ndim != 2:
        raise ValueError("points must be N x D")
    N, D = x.shape
    scratch = np.empty((N, N), np.float32)
    ov = np.empty((N, k), np.float32)
    oi = np.empty((N, k), np.int32)
    rc = _load().oracle_knn_graph(_ptr(x), N, D, k, _ptr(scratch), _ptr(ov), _ptr(oi),
                                  nthreads or default_threads())
    if rc:
        raise ValueError("oracle_knn_graph failed (%d)" % rc)
    return ov, oi
