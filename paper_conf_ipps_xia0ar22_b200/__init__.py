"""B200-native blocked Floyd–Warshall APSP — thin Python binding over ``libapsp.so``.

The C ABI is declared in ``include/apsp.h``; every step of the hot path runs in
the library's sm_100a kernels. This module only marshals arguments (ctypes):
the functions keep the C names (``apsp_init_from_csr``, ``apsp_fw_blocked``,
``apsp_get_dist`` ...) and raise :class:`ApspError` on a non-OK status.

There is no CPU fallback: importing this package fails loudly if the library
has not been built (``python -c "import __graft_entry__ as g; g.build()"``),
and ``apsp_init_from_csr`` fails with ``APSP_ECUDA`` when no GPU is visible.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libapsp.so")

if not os.path.exists(LIB_PATH):
    raise ImportError(
        "libapsp.so is not built at %s — run __graft_entry__.build() (nvcc, sm_100a). "
        "There is no CPU fallback." % LIB_PATH)

_lib = ctypes.CDLL(LIB_PATH)

# ----------------------------------------------------------------- constants
APSP_I32, APSP_F32 = 0, 1
APSP_OK, APSP_EINVAL, APSP_ERANGE, APSP_ENOMEM, APSP_ECUDA, APSP_ENCCL, APSP_ENEGCYCLE, APSP_ESTATE = range(8)
STATUS_NAMES = ["APSP_OK", "APSP_EINVAL", "APSP_ERANGE", "APSP_ENOMEM", "APSP_ECUDA", "APSP_ENCCL",
                "APSP_ENEGCYCLE", "APSP_ESTATE"]
APSP_INF_I32 = 0x3FFFFFFF
APSP_MODE_INCORE, APSP_MODE_OUT_OF_CORE, APSP_MODE_BOUNDARY, APSP_MODE_JOHNSON = 0, 1, 2, 3
TILE = 128
APSP_SCHED_AUTO, APSP_SCHED_PER_PHASE, APSP_SCHED_DATAFLOW, APSP_SCHED_SMALL = 0, 1, 2, 3


class apsp_config(ctypes.Structure):
    _fields_ = [
        ("struct_size", ctypes.c_int32),
        ("device", ctypes.c_int32),
        ("world_size", ctypes.c_int32),
        ("rank", ctypes.c_int32),
        ("nccl_unique_id", ctypes.c_void_p),
        ("virtual_ranks", ctypes.c_int32),
        ("tile", ctypes.c_int32),
        ("stream", ctypes.c_void_p),
        ("dist_device", ctypes.c_void_p),
        ("dist_device_bytes", ctypes.c_int64),
        ("device_budget_bytes", ctypes.c_int64),
        ("ooc_block", ctypes.c_int32),
        ("timing", ctypes.c_int32),
        ("force_out_of_core", ctypes.c_int32),
        ("packed16", ctypes.c_int32),
        ("schedule", ctypes.c_int32),
        ("no_lookahead", ctypes.c_int32),
        ("ooc_stream_all", ctypes.c_int32),
        ("force_nccl", ctypes.c_int32),
        ("minplus_variant", ctypes.c_int32),
        ("dataflow_delay", ctypes.c_int32),
        ("exact_f32", ctypes.c_int32),
        ("reserved", ctypes.c_int32 * 3),
    ]


class apsp_info(ctypes.Structure):
    _fields_ = [
        ("n", ctypes.c_int64), ("n_pad", ctypes.c_int64),
        ("tile", ctypes.c_int32), ("dtype", ctypes.c_int32), ("world_size", ctypes.c_int32),
        ("rank", ctypes.c_int32), ("mode", ctypes.c_int32), ("ooc_block", ctypes.c_int32),
        ("rounds", ctypes.c_int64), ("device_bytes", ctypes.c_int64), ("host_bytes", ctypes.c_int64),
        ("dist_device", ctypes.c_void_p), ("ld", ctypes.c_int64),
        ("arith", ctypes.c_int32), ("packed16_eligible", ctypes.c_int32),
        ("boundary_nodes", ctypes.c_int64),
        ("edges_scanned", ctypes.c_int64),
        ("kernel", ctypes.c_int32), ("exact_f32_eligible", ctypes.c_int32),
    ]


APSP_ARITH_I32, APSP_ARITH_S16X2, APSP_ARITH_F32, APSP_ARITH_F32_EXACT = 0, 1, 2, 3
(APSP_KERNEL_PER_PHASE, APSP_KERNEL_DATAFLOW, APSP_KERNEL_DATAFLOW_PAIR, APSP_KERNEL_SMALL, APSP_KERNEL_DATAFLOW16,
 APSP_KERNEL_SHARDED, APSP_KERNEL_OUT_OF_CORE) = range(1, 8)
KERNEL_NAMES = {0: "none", 1: "per_phase", 2: "dataflow", 3: "dataflow_pair", 4: "small64", 5: "dataflow16",
                6: "sharded_dataflow", 7: "out_of_core"}
ARITH_NAMES = {0: "i32", 1: "s16x2", 2: "f32", 3: "f32_exact"}


class apsp_selection(ctypes.Structure):
    _fields_ = [("method", ctypes.c_int32), ("candidates", ctypes.c_int32), ("density", ctypes.c_double),
                ("est_seconds", ctypes.c_double * 4), ("boundary_nodes", ctypes.c_int64)]


class apsp_phase_stats(ctypes.Structure):
    _fields_ = [("ms", ctypes.c_double * 4), ("launches", ctypes.c_int64 * 4), ("relax", ctypes.c_double * 4)]


_H = ctypes.c_void_p
_P = ctypes.c_void_p
_I64 = ctypes.c_int64
_I32 = ctypes.c_int32
_sig = {
    "apsp_config_default": (None, [ctypes.POINTER(apsp_config)]),
    "apsp_init_from_csr": (ctypes.c_int, [ctypes.POINTER(_H), _I64, _P, _P, _P, ctypes.c_int,
                                          ctypes.POINTER(apsp_config)]),
    "apsp_fw_blocked": (ctypes.c_int, [_H]),
    "apsp_init_boundary": (ctypes.c_int, [ctypes.POINTER(_H), _I64, _P, _P, _P, ctypes.c_int, _P, _I32,
                                          ctypes.POINTER(apsp_config)]),
    "apsp_init_johnson": (ctypes.c_int, [ctypes.POINTER(_H), _I64, _P, _P, _P, ctypes.c_int, ctypes.c_double,
                                         _I64, ctypes.POINTER(apsp_config)]),
    "apsp_select": (ctypes.c_int, [_I64, _P, _P, _P, ctypes.c_int, _P, _I32, ctypes.POINTER(apsp_config),
                                   ctypes.POINTER(apsp_selection)]),
    "apsp_checkpoint": (ctypes.c_int, [_H, ctypes.c_char_p]),
    "apsp_restore": (ctypes.c_int, [_H, ctypes.c_char_p]),
    "apsp_solve": (ctypes.c_int, [_H]),
    "apsp_reinit": (ctypes.c_int, [_H]),
    "apsp_fw_rounds": (ctypes.c_int, [_H, _I64, _I64]),
    "apsp_get_dist": (ctypes.c_int, [_H, _I64, _I64, _P, _I64]),
    "apsp_fw_blocked_async": (ctypes.c_int, [_H]),
    "apsp_get_dist_async": (ctypes.c_int, [_H, _I64, _I64, _P, _I64]),
    "apsp_synchronize": (ctypes.c_int, [_H]),
    "apsp_load_csr": (ctypes.c_int, [_H, _P, _P, _P]),
    "apsp_debug_queue": (ctypes.c_int64, [_I32, _I32, _I32, _I64, _P, _I64]),
    "apsp_local_rows": (ctypes.c_int, [_H, ctypes.POINTER(_I64), ctypes.POINTER(_I64)]),
    "apsp_partition": (ctypes.c_int, [_I64, _I32, _I32, _I32, ctypes.POINTER(_I64), ctypes.POINTER(_I64),
                                      ctypes.POINTER(_I64)]),
    "apsp_dist_device_bytes": (ctypes.c_int, [_I64, _I32, _I32, _I32, ctypes.POINTER(_I64)]),
    "apsp_get_info": (ctypes.c_int, [_H, ctypes.POINTER(apsp_info)]),
    "apsp_get_phase_stats": (ctypes.c_int, [_H, ctypes.POINTER(apsp_phase_stats)]),
    "apsp_nccl_unique_id": (ctypes.c_int, [_P]),
    "apsp_destroy": (None, [_H]),
    "apsp_trim_memory": (ctypes.c_int, [_I32]),
    "apsp_last_error": (ctypes.c_char_p, [_H]),
    "apsp_version": (ctypes.c_char_p, []),
}
for _name, (_res, _args) in _sig.items():
    _f = getattr(_lib, _name)
    _f.restype = _res
    _f.argtypes = _args

EXPORTED_SYMBOLS = tuple(_sig)


class ApspError(RuntimeError):
    def __init__(self, status: int, msg: str):
        self.status = status
        super().__init__("%s: %s" % (STATUS_NAMES[status] if 0 <= status < 8 else status, msg))


class NegativeCycleError(ApspError):
    pass


def _check(st: int, h=None):
    if st != APSP_OK:
        msg = _lib.apsp_last_error(h).decode(errors="replace")
        if st == APSP_ENEGCYCLE:
            raise NegativeCycleError(st, msg)
        raise ApspError(st, msg)


def _ptr(a: np.ndarray):
    return a.ctypes.data_as(ctypes.c_void_p)


# ------------------------------------------------------------- C-ABI mirror

def apsp_version() -> str:
    return _lib.apsp_version().decode()


def apsp_config_default(**kw) -> apsp_config:
    cfg = apsp_config()
    _lib.apsp_config_default(ctypes.byref(cfg))
    for k, v in kw.items():
        setattr(cfg, k, v)
    return cfg


def apsp_nccl_unique_id() -> bytes:
    buf = ctypes.create_string_buffer(128)
    _check(_lib.apsp_nccl_unique_id(buf))
    return buf.raw


def apsp_partition(n: int, world_size: int, rank: int, tile: int = 0):
    np_, rb, rc = _I64(), _I64(), _I64()
    _check(_lib.apsp_partition(n, tile, world_size, rank, ctypes.byref(np_), ctypes.byref(rb), ctypes.byref(rc)))
    return np_.value, rb.value, rc.value


def apsp_dist_device_bytes(n: int, world_size: int = 1, virtual_ranks: int = 0, tile: int = 0) -> int:
    """Bytes a caller-owned apsp_config.dist_device buffer needs (host arithmetic)."""
    b = _I64()
    _check(_lib.apsp_dist_device_bytes(n, tile, world_size, virtual_ranks, ctypes.byref(b)))
    return b.value


class Handle:
    """Owns an ``apsp_handle*``; released by :meth:`close` / context exit."""

    def __init__(self, raw: ctypes.c_void_p, dtype: int, n: int, keep=()):
        self.raw = raw
        self.dtype = dtype
        self.n = n
        self._keep = keep

    def close(self):
        if self.raw:
            _lib.apsp_destroy(self.raw)
            self.raw = None

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    @property
    def np_dtype(self):
        return np.int32 if self.dtype == APSP_I32 else np.float32


def _csr_args(n: int, row_ptr, col_idx, weights, dtype: int | None):
    """Marshal a CSR graph for the C ABI: contiguous int64 row_ptr[n+1], int32 col_idx and
    int32/float32 weights with at least row_ptr[n] entries each (the C side reads exactly
    row_ptr[n] arcs, so shorter arrays are refused here with APSP_EINVAL)."""
    row_ptr = np.ascontiguousarray(row_ptr, dtype=np.int64)
    col_idx = np.ascontiguousarray(col_idx, dtype=np.int32)
    w = np.asarray(weights)
    if dtype is None:
        dtype = APSP_F32 if w.dtype.kind == "f" else APSP_I32
    w = np.ascontiguousarray(w, dtype=np.int32 if dtype == APSP_I32 else np.float32)
    if row_ptr.ndim != 1 or row_ptr.shape[0] != n + 1:
        raise ApspError(APSP_EINVAL, "row_ptr must have n+1 entries")
    m = int(row_ptr[-1]) if n >= 0 else 0
    if m < 0 or col_idx.shape[0] < m or w.shape[0] < m:
        raise ApspError(APSP_EINVAL, "col_idx and weights need row_ptr[n] = %d entries (got %d, %d)"
                        % (m, col_idx.shape[0], w.shape[0]))
    return row_ptr, col_idx, w, dtype


def apsp_init_from_csr(n: int, row_ptr, col_idx, weights, dtype: int | None = None,
                       cfg: apsp_config | None = None) -> Handle:
    row_ptr, col_idx, w, dtype = _csr_args(n, row_ptr, col_idx, weights, dtype)
    if cfg is None:
        cfg = apsp_config_default()
    raw = ctypes.c_void_p()
    _check(_lib.apsp_init_from_csr(ctypes.byref(raw), n, _ptr(row_ptr), _ptr(col_idx), _ptr(w), dtype,
                                   ctypes.byref(cfg)))
    keep = (cfg,)
    return Handle(raw, dtype, n, keep)


def apsp_fw_blocked(h: Handle) -> None:
    _check(_lib.apsp_fw_blocked(h.raw), h.raw)


def apsp_init_boundary(n: int, row_ptr, col_idx, weights, comp, k: int, dtype: int | None = None,
                       cfg: apsp_config | None = None) -> Handle:
    """Boundary algorithm with the caller's partition comp[v] in [0, k)."""
    row_ptr, col_idx, w, dtype = _csr_args(n, row_ptr, col_idx, weights, dtype)
    comp = np.ascontiguousarray(comp, dtype=np.int32)
    if comp.shape[0] != n:
        raise ApspError(APSP_EINVAL, "comp must have n entries")
    if cfg is None:
        cfg = apsp_config_default()
    raw = ctypes.c_void_p()
    _check(_lib.apsp_init_boundary(ctypes.byref(raw), n, _ptr(row_ptr), _ptr(col_idx), _ptr(w), dtype, _ptr(comp),
                                   k, ctypes.byref(cfg)))
    return Handle(raw, dtype, n, (cfg,))


def apsp_init_johnson(n: int, row_ptr, col_idx, weights, dtype: int | None = None, delta: float = 0.0,
                      batch: int = 0, cfg: apsp_config | None = None) -> Handle:
    """Johnson's algorithm with batched Near-Far SSSP (Algorithm 2)."""
    row_ptr, col_idx, w, dtype = _csr_args(n, row_ptr, col_idx, weights, dtype)
    if cfg is None:
        cfg = apsp_config_default()
    raw = ctypes.c_void_p()
    _check(_lib.apsp_init_johnson(ctypes.byref(raw), n, _ptr(row_ptr), _ptr(col_idx), _ptr(w), dtype,
                                  float(delta), int(batch), ctypes.byref(cfg)))
    return Handle(raw, dtype, n, (cfg,))


def apsp_select(n: int, row_ptr, col_idx, weights, comp=None, k: int = 0, dtype: int | None = None,
                cfg: apsp_config | None = None) -> apsp_selection:
    """The paper's method selection (§IV): density filter + device-calibrated cost models."""
    row_ptr, col_idx, w, dtype = _csr_args(n, row_ptr, col_idx, weights, dtype)
    cp = None
    if comp is not None:
        cp = np.ascontiguousarray(comp, dtype=np.int32)
        if cp.shape[0] != n:
            raise ApspError(APSP_EINVAL, "comp must have n entries")
    if cfg is None:
        cfg = apsp_config_default()
    sel = apsp_selection()
    _check(_lib.apsp_select(n, _ptr(row_ptr), _ptr(col_idx), _ptr(w), dtype,
                            _ptr(cp) if cp is not None else None, int(k), ctypes.byref(cfg), ctypes.byref(sel)))
    return sel


def apsp_checkpoint(h: Handle, path: str) -> None:
    """Save the blocked-FW state (this rank's rows + next round) to path."""
    _check(_lib.apsp_checkpoint(h.raw, os.fsencode(path)), h.raw)


def apsp_restore(h: Handle, path: str) -> None:
    """Load a checkpoint into a handle made for the same graph / placement."""
    _check(_lib.apsp_restore(h.raw, os.fsencode(path)), h.raw)


def apsp_solve(h: Handle) -> None:
    _check(_lib.apsp_solve(h.raw), h.raw)


def apsp_reinit(h: Handle) -> None:
    _check(_lib.apsp_reinit(h.raw), h.raw)


def apsp_fw_rounds(h: Handle, k_begin: int, k_end: int) -> None:
    _check(_lib.apsp_fw_rounds(h.raw, k_begin, k_end), h.raw)


def apsp_get_dist(h: Handle, row_begin: int = 0, row_count: int | None = None, out: np.ndarray | None = None):
    """Rows [row_begin, row_begin+row_count) of dist as a (row_count, n) array (or into ``out``)."""
    if row_count is None:
        row_count = h.n - row_begin
    if out is None:
        out = np.empty((row_count, h.n), dtype=h.np_dtype)
    assert out.dtype == h.np_dtype and out.ndim == 2 and out.shape[0] >= row_count and out.flags.c_contiguous
    _check(_lib.apsp_get_dist(h.raw, row_begin, row_count, _ptr(out), out.shape[1]), h.raw)
    return out


def apsp_get_dist_ptr(h: Handle, row_begin: int, row_count: int, out_ptr: int, ld_out: int) -> None:
    """Raw-pointer form (e.g. a pinned torch tensor's data_ptr())."""
    _check(_lib.apsp_get_dist(h.raw, row_begin, row_count, ctypes.c_void_p(out_ptr), ld_out), h.raw)


def apsp_fw_blocked_async(h: Handle) -> None:
    """Enqueue the closure and return (in core); the status comes from apsp_synchronize."""
    _check(_lib.apsp_fw_blocked_async(h.raw), h.raw)


def apsp_get_dist_async(h: Handle, row_begin: int, row_count: int, out_ptr: int, ld_out: int) -> None:
    """Enqueue the D2H of rows into caller memory (pinned: e.g. a pinned tensor's data_ptr()),
    valid after apsp_synchronize."""
    _check(_lib.apsp_get_dist_async(h.raw, row_begin, row_count, ctypes.c_void_p(out_ptr), ld_out), h.raw)


def apsp_load_csr(h: Handle, row_ptr, col_idx, weights) -> None:
    """Next graph (same n and dtype) into an in-core handle; the init is enqueued. Arrays are
    numpy (converted like apsp_init_from_csr; pinned arrays copy fastest)."""
    row_ptr, col_idx, w, _ = _csr_args(h.n, row_ptr, col_idx, weights, h.dtype)
    _check(_lib.apsp_load_csr(h.raw, _ptr(row_ptr), _ptr(col_idx), _ptr(w)), h.raw)


def apsp_debug_queue(nb: int, P: int, q: int, delay: int) -> np.ndarray:
    """The dataflow kernel's task queue (host decoder): (total, 4) int32 rows (type, k, i, j)."""
    total = _lib.apsp_debug_queue(nb, P, q, delay, None, 0)
    if total < 0:
        raise ValueError("bad queue arguments")
    out = np.zeros((max(total, 1), 4), dtype=np.int32)
    _lib.apsp_debug_queue(nb, P, q, delay, _ptr(out), total)
    return out[:total]


def apsp_synchronize(h: Handle) -> None:
    _check(_lib.apsp_synchronize(h.raw), h.raw)


def apsp_local_rows(h: Handle):
    rb, rc = _I64(), _I64()
    _check(_lib.apsp_local_rows(h.raw, ctypes.byref(rb), ctypes.byref(rc)), h.raw)
    return rb.value, rc.value


def apsp_get_info(h: Handle) -> apsp_info:
    info = apsp_info()
    _check(_lib.apsp_get_info(h.raw, ctypes.byref(info)), h.raw)
    return info


def apsp_get_phase_stats(h: Handle) -> apsp_phase_stats:
    st = apsp_phase_stats()
    _check(_lib.apsp_get_phase_stats(h.raw, ctypes.byref(st)), h.raw)
    return st


def apsp_destroy(h: Handle) -> None:
    h.close()


def apsp_trim_memory(device: int = -1) -> None:
    _check(_lib.apsp_trim_memory(device))


def apsp_last_error(h: Handle | None = None) -> str:
    return _lib.apsp_last_error(h.raw if h is not None else None).decode(errors="replace")


# ------------------------------------------------------------- convenience

def solve(g, cfg: apsp_config | None = None, dtype: int | None = None) -> np.ndarray:
    """Full APSP of a ``graphgen.CSR``-like object (n, row_ptr, col, w) -> n x n host array."""
    with apsp_init_from_csr(g.n, g.row_ptr, g.col, g.w, dtype=dtype, cfg=cfg) as h:
        apsp_fw_blocked(h)
        return apsp_get_dist(h)


def solve_johnson(g, delta: float = 0.0, batch: int = 0, cfg: apsp_config | None = None) -> np.ndarray:
    """Full APSP by Johnson's algorithm (batched Near-Far SSSP)."""
    with apsp_init_johnson(g.n, g.row_ptr, g.col, g.w, delta=delta, batch=batch, cfg=cfg) as h:
        apsp_solve(h)
        return apsp_get_dist(h)


def solve_boundary(g, comp, k: int, cfg: apsp_config | None = None) -> np.ndarray:
    """Full APSP by the boundary algorithm with partition comp (k components)."""
    with apsp_init_boundary(g.n, g.row_ptr, g.col, g.w, comp, k, cfg=cfg) as h:
        apsp_solve(h)
        return apsp_get_dist(h)
