"""CPU oracle for the blocked Floyd–Warshall APSP hot path — TEST INFRASTRUCTURE.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` legs may import this package. It is a
ctypes wrapper over ``apsp_oracle.c`` (plain C, compiled with gcc) and shares
nothing with the CUDA path in ``paper_conf_ipps_xia0ar22_b200``.

Every function cites the passage of ``PAPER.md`` it follows (see the header of
``apsp_oracle.c``):

* :func:`init_i64` / :func:`init_f64` — PAPER.md:60 (§II-A), dist := weights,
  infinity where no edge.
* :func:`fw_i64` / :func:`fw_f64` — PAPER.md:60 (§II-A) plain Floyd–Warshall,
  optionally stopped after ``k_iters`` outer iterations.
* :func:`dijkstra_rows_i64` / :func:`dijkstra_rows_f64` — PAPER.md:66 (§II-B).
* :func:`bellman_ford_row_i64` — PAPER.md:68 (§II-B).

Integers are computed in int64, reals in float64 (fp64). "No path" is
``INF_I64`` (= int64 max) or ``+inf``.

Pins: ``tests/test_oracle.py`` (closed forms, brute force, cross-checks).
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "apsp_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")

INF_I64 = np.iinfo(np.int64).max

_lib = None


def build(force: bool = False) -> str:
    """Compile apsp_oracle.c -> liboracle.so with gcc -O2 -fopenmp."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + ".tmp%d" % os.getpid()
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-fPIC", "-shared", "-std=c11",
                               "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB)
        P = ctypes.c_void_p
        I64 = ctypes.c_int64
        for name, args in [
            ("oracle_init_i64", [I64, P, P, P, P]),
            ("oracle_init_f64", [I64, P, P, P, P]),
            ("oracle_fw_i64", [I64, P, I64, I64]),
            ("oracle_fw_f64", [I64, P, I64, I64]),
            ("oracle_dijkstra_rows_i64", [I64, P, P, P, I64, P, P]),
            ("oracle_dijkstra_rows_f64", [I64, P, P, P, I64, P, P]),
            ("oracle_bellman_ford_row_i64", [I64, P, P, P, I64, P]),
        ]:
            f = getattr(lib, name)
            f.argtypes = args
            f.restype = ctypes.c_int
        lib.oracle_certify_rows_i32.argtypes = [I64, P, P, P, I64, I64, P, I64, ctypes.c_int32, P]
        lib.oracle_certify_rows_i32.restype = I64
        lib.oracle_omp_max_threads.restype = ctypes.c_int
        lib.oracle_omp_max_threads.argtypes = []
        _lib = lib
    return _lib


def _p(a: np.ndarray):
    return a.ctypes.data_as(ctypes.c_void_p)


def _csr(row_ptr, col, w, wdtype):
    row_ptr = np.ascontiguousarray(row_ptr, dtype=np.int64)
    col = np.ascontiguousarray(col, dtype=np.int32)
    w = np.ascontiguousarray(w, dtype=wdtype)
    n = row_ptr.shape[0] - 1
    assert col.shape[0] == row_ptr[n] and w.shape[0] == row_ptr[n]
    return n, row_ptr, col, w


def threads() -> int:
    """OpenMP threads the oracle's parallel loops use."""
    return int(_load().oracle_omp_max_threads())


def init_i64(row_ptr, col, w) -> np.ndarray:
    """PAPER.md:60 initial dist for integer weights (int64, INF_I64 = no edge)."""
    n, row_ptr, col, w = _csr(row_ptr, col, w, np.int64)
    d = np.empty((n, n), dtype=np.int64)
    _load().oracle_init_i64(n, _p(row_ptr), _p(col), _p(w), _p(d))
    return d


def init_f64(row_ptr, col, w) -> np.ndarray:
    """PAPER.md:60 initial dist for real weights (float64, +inf = no edge)."""
    n, row_ptr, col, w = _csr(row_ptr, col, w, np.float64)
    d = np.empty((n, n), dtype=np.float64)
    _load().oracle_init_f64(n, _p(row_ptr), _p(col), _p(w), _p(d))
    return d


def fw_dense_i64(d: np.ndarray, k_iters: int | None = None, k_begin: int = 0):
    """Plain FW in place on an int64 matrix, outer iterations
    k_begin .. k_iters-1 (default: all); returns the negative-cycle flag."""
    assert d.dtype == np.int64 and d.flags.c_contiguous and d.shape[0] == d.shape[1]
    n = d.shape[0]
    k = n if k_iters is None else int(k_iters)
    return bool(_load().oracle_fw_i64(n, _p(d), int(k_begin), k))


def fw_dense_f64(d: np.ndarray, k_iters: int | None = None, k_begin: int = 0):
    assert d.dtype == np.float64 and d.flags.c_contiguous and d.shape[0] == d.shape[1]
    n = d.shape[0]
    k = n if k_iters is None else int(k_iters)
    return bool(_load().oracle_fw_f64(n, _p(d), int(k_begin), k))


def fw_i64(row_ptr, col, w, k_iters: int | None = None):
    """APSP by plain FW on integer weights. Returns (dist int64 n x n, negcycle)."""
    d = init_i64(row_ptr, col, w)
    neg = fw_dense_i64(d, k_iters)
    return d, neg


def fw_f64(row_ptr, col, w, k_iters: int | None = None):
    """APSP by plain FW on real weights in fp64. Returns (dist float64, negcycle)."""
    d = init_f64(row_ptr, col, w)
    neg = fw_dense_f64(d, k_iters)
    return d, neg


def dijkstra_rows_i64(row_ptr, col, w, srcs) -> np.ndarray:
    """Rows dist[s, :] for s in srcs by Dijkstra; weights >= 0."""
    n, row_ptr, col, w = _csr(row_ptr, col, w, np.int64)
    srcs = np.ascontiguousarray(srcs, dtype=np.int64)
    out = np.empty((srcs.shape[0], n), dtype=np.int64)
    rc = _load().oracle_dijkstra_rows_i64(n, _p(row_ptr), _p(col), _p(w), srcs.shape[0],
                                           _p(srcs), _p(out))
    if rc != 0:
        raise ValueError("dijkstra: negative weight or out of memory")
    return out


def dijkstra_rows_f64(row_ptr, col, w, srcs) -> np.ndarray:
    n, row_ptr, col, w = _csr(row_ptr, col, w, np.float64)
    srcs = np.ascontiguousarray(srcs, dtype=np.int64)
    out = np.empty((srcs.shape[0], n), dtype=np.float64)
    rc = _load().oracle_dijkstra_rows_f64(n, _p(row_ptr), _p(col), _p(w), srcs.shape[0],
                                           _p(srcs), _p(out))
    if rc != 0:
        raise ValueError("dijkstra: negative weight or out of memory")
    return out


def bellman_ford_row_i64(row_ptr, col, w, src: int):
    """Row dist[src, :] by Bellman–Ford. Returns (row, negcycle)."""
    n, row_ptr, col, w = _csr(row_ptr, col, w, np.int64)
    out = np.empty(n, dtype=np.int64)
    neg = _load().oracle_bellman_ford_row_i64(n, _p(row_ptr), _p(col), _p(w), int(src), _p(out))
    return out, bool(neg)


def certify_rows_i32(row_ptr, col, w, r0: int, rows: np.ndarray, inf: int):
    """Optimality certificate (apsp_oracle.c: oracle_certify_rows_i32) for claimed
    int32 distance rows dist[r0 .. r0+len(rows)) of a graph with weights > 0.
    `rows` may be a strided 2-D view (C-contiguous rows). Returns (n_bad, first_bad_source)."""
    n, row_ptr, col, w = _csr(row_ptr, col, w, np.int64)
    assert rows.dtype == np.int32 and rows.ndim == 2 and rows.strides[1] == 4
    assert rows.shape[1] >= n
    ld = rows.strides[0] // 4
    first = np.zeros(1, dtype=np.int64)
    bad = _load().oracle_certify_rows_i32(n, _p(row_ptr), _p(col), _p(w), int(r0), rows.shape[0],
                                          rows.ctypes.data_as(ctypes.c_void_p), ld, int(inf), _p(first))
    if bad < 0:
        raise ValueError("certificate needs strictly positive weights")
    return int(bad), int(first[0])
