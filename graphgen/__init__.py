"""Seeded synthetic graph generators shared by the tests, the bench and the oracle checks.

This module holds NO shortest-path arithmetic: it only draws graphs (arc lists
and weights) and packs them as CSR, the input format of the C ABI
(``include/apsp.h``). Both the CUDA path and the CPU oracle consume its output;
neither is imported here.

Workload shapes follow the paper's graph classes (PAPER.md:335-338 and
Table III): small-separator road/mesh-like graphs (2-D grids),
random sparse graphs (Erdős–Rényi) and denser random graphs. The recipe for each
BASELINE.json config is :func:`baseline_config` (DESIGN.md §"Input recipe").

All randomness comes from ``numpy.random.default_rng(seed)`` (PCG64), so a
seed gives the same graph on every machine.
"""
from __future__ import annotations

from dataclasses import dataclass

import numpy as np


@dataclass
class CSR:
    """Directed weighted graph in CSR form: row = source vertex (PAPER.md:56 w[i][j])."""

    n: int
    row_ptr: np.ndarray  # int64 [n+1]
    col: np.ndarray  # int32 [m]
    w: np.ndarray  # int32 or float32 [m]
    name: str = ""
    meta: dict | None = None  # generator facts (grid: rows, cols, perm)

    @property
    def m(self) -> int:
        return int(self.row_ptr[-1])

    @property
    def density(self) -> float:
        """m / n^2, the density column of the paper's Table III."""
        return self.m / float(self.n) ** 2

    def arcs(self):
        """(src, dst, w) arrays."""
        src = np.repeat(np.arange(self.n, dtype=np.int64), np.diff(self.row_ptr))
        return src, self.col.astype(np.int64), self.w


def csr_from_arcs(n: int, src, dst, w, name: str = "") -> CSR:
    """Pack an arc list into CSR (stable sort by source; duplicates are kept)."""
    src = np.asarray(src, dtype=np.int64)
    dst = np.asarray(dst, dtype=np.int64)
    w = np.asarray(w)
    assert src.shape == dst.shape == w.shape
    if src.size:
        assert src.min() >= 0 and src.max() < n and dst.min() >= 0 and dst.max() < n
    order = np.argsort(src, kind="stable")
    counts = np.bincount(src, minlength=n) if n > 0 else np.zeros(0, np.int64)
    row_ptr = np.zeros(n + 1, dtype=np.int64)
    np.cumsum(counts, out=row_ptr[1:])
    return CSR(n, row_ptr, dst[order].astype(np.int32), np.ascontiguousarray(w[order]), name)


def draw_weights(rng: np.random.Generator, m: int, dtype: str = "i32", lo=1, hi=100):
    """Integer weights uniform in {lo..hi} (int32) or real weights uniform in [lo, hi) (float32).

    ``dtype="f32int"`` draws integer values stored as float32 (exact in fp32)."""
    if dtype == "i32":
        return rng.integers(lo, hi + 1, size=m, dtype=np.int64).astype(np.int32)
    if dtype == "f32":
        return rng.uniform(lo, hi, size=m).astype(np.float32)
    if dtype == "f32int":
        return rng.integers(lo, hi + 1, size=m, dtype=np.int64).astype(np.float32)
    raise ValueError(dtype)


def erdos_renyi(n: int, m: int, seed: int, dtype: str = "i32", undirected: bool = False,
                lo=1, hi=100, name: str = "") -> CSR:
    """G(n, m): m distinct arcs (u != v) drawn uniformly; undirected doubles each edge."""
    rng = np.random.default_rng(seed)
    target = m // 2 if undirected else m
    max_pairs = n * (n - 1) // (2 if undirected else 1)
    target = min(target, max_pairs)
    keys = np.zeros(0, dtype=np.int64)
    while keys.size < target:
        need = target - keys.size
        u = rng.integers(0, n, size=int(need * 1.1) + 16, dtype=np.int64)
        v = rng.integers(0, n, size=u.size, dtype=np.int64)
        keep = u != v
        u, v = u[keep], v[keep]
        if undirected:
            u, v = np.minimum(u, v), np.maximum(u, v)
        keys = np.unique(np.concatenate([keys, u * n + v]))
    if keys.size > target:
        keys = rng.choice(keys, size=target, replace=False)
    u, v = keys // n, keys % n
    w = draw_weights(rng, u.size, dtype, lo, hi)
    if undirected:
        u, v, w = np.concatenate([u, v]), np.concatenate([v, u]), np.concatenate([w, w])
    return csr_from_arcs(n, u, v, w, name or f"er_n{n}_m{m}")


def grid_2d(rows: int, cols: int, seed: int, dtype: str = "i32", permute: bool = True,
            lo=1, hi=100, unit: bool = False, name: str = "") -> CSR:
    """Undirected 4-neighbour rows x cols grid (road/mesh-like, small separator).

    Vertex (r, c) has id r*cols + c before the optional random relabelling.
    ``unit=True`` gives every edge weight 1 (closed form: Manhattan distance)."""
    rng = np.random.default_rng(seed)
    r, c = np.meshgrid(np.arange(rows), np.arange(cols), indexing="ij")
    vid = (r * cols + c).astype(np.int64)
    hu, hv = vid[:, :-1].ravel(), vid[:, 1:].ravel()
    vu, vv = vid[:-1, :].ravel(), vid[1:, :].ravel()
    u = np.concatenate([hu, vu])
    v = np.concatenate([hv, vv])
    if unit:
        w = np.ones(u.size, dtype=np.float32 if dtype.startswith("f32") else np.int32)
    else:
        w = draw_weights(rng, u.size, dtype, lo, hi)
    n = rows * cols
    perm = np.arange(n, dtype=np.int64)
    if permute:
        perm = rng.permutation(n).astype(np.int64)
        u, v = perm[u], perm[v]
    g = csr_from_arcs(n, np.concatenate([u, v]), np.concatenate([v, u]),
                      np.concatenate([w, w]), name or f"grid_{rows}x{cols}")
    g.meta = {"rows": rows, "cols": cols, "perm": perm}  # vertex (r, c) has id perm[r*cols + c]
    return g


def grid_block_partition(g: CSR, block_rows: int, block_cols: int):
    """Geometric partition of a grid_2d graph into block_rows x block_cols rectangles of
    cells (the stand-in for the paper's METIS k-way partition, on mesh-like
    graphs). Returns (comp int32[n], k)."""
    rows, cols, perm = g.meta["rows"], g.meta["cols"], g.meta["perm"]
    old = np.empty(g.n, dtype=np.int64)
    old[perm] = np.arange(g.n)
    r, c = old // cols, old % cols
    bh = -(-rows // block_rows)
    bw = -(-cols // block_cols)
    comp = (r // bh) * block_cols + (c // bw)
    return comp.astype(np.int32), block_rows * block_cols


def random_partition(n: int, k: int, seed: int):
    """Balanced random partition (many boundary nodes: a stress case, not a small separator)."""
    rng = np.random.default_rng(seed)
    comp = np.arange(n) % k
    rng.shuffle(comp)
    return comp.astype(np.int32), k


def relabel(g: CSR, perm) -> CSR:
    """Vertex v becomes perm[v]."""
    perm = np.asarray(perm, dtype=np.int64)
    s, d, w = g.arcs()
    return csr_from_arcs(g.n, perm[s], perm[d], w, g.name + "_perm")


def reverse(g: CSR) -> CSR:
    """Every arc u->v becomes v->u."""
    s, d, w = g.arcs()
    return csr_from_arcs(g.n, d, s, w, g.name + "_rev")


def directed_ring(n: int, w: int = 1, dtype=np.int32) -> CSR:
    """Arcs i -> (i+1) mod n, all of weight w."""
    s = np.arange(n, dtype=np.int64)
    return csr_from_arcs(n, s, (s + 1) % n, np.full(n, w, dtype=dtype), f"ring{n}")


def weighted_path(weights, dtype=np.int32) -> CSR:
    """Undirected path 0 - 1 - ... - n-1 with edge i--(i+1) of weight weights[i]."""
    weights = np.asarray(weights, dtype=dtype)
    n = weights.size + 1
    s = np.arange(n - 1, dtype=np.int64)
    return csr_from_arcs(n, np.concatenate([s, s + 1]), np.concatenate([s + 1, s]),
                         np.concatenate([weights, weights]), f"path{n}")


def complete(n: int, w: int = 1, dtype=np.int32) -> CSR:
    """Complete directed graph, every arc weight w."""
    u, v = np.meshgrid(np.arange(n), np.arange(n), indexing="ij")
    keep = u != v
    return csr_from_arcs(n, u[keep], v[keep], np.full(int(keep.sum()), w, dtype=dtype), f"K{n}")


def disjoint_union(a: CSR, b: CSR) -> CSR:
    sa, da, wa = a.arcs()
    sb, db, wb = b.arcs()
    return csr_from_arcs(a.n + b.n, np.concatenate([sa, sb + a.n]), np.concatenate([da, db + a.n]),
                         np.concatenate([wa, wb]), a.name + "+" + b.name)


def empty(n: int, dtype=np.int32) -> CSR:
    return csr_from_arcs(n, np.zeros(0, np.int64), np.zeros(0, np.int64), np.zeros(0, dtype), f"empty{n}")


def with_arcs(g: CSR, src, dst, w) -> CSR:
    """g plus extra arcs (duplicates allowed)."""
    s, d, ww = g.arcs()
    return csr_from_arcs(g.n, np.concatenate([s, np.asarray(src, np.int64)]),
                         np.concatenate([d, np.asarray(dst, np.int64)]),
                         np.concatenate([ww, np.asarray(w, dtype=ww.dtype)]), g.name + "+arcs")


# ---------------------------------------------------------------------------
# BASELINE.json configs
# ---------------------------------------------------------------------------

BASELINE_CONFIGS = {
    # name: (description, builder)
    "cfg1_er1024": "n=1024 Erdos-Renyi, directed, avg out-degree 8, int32 U{1..100}, seed 1",
    "cfg2_grid16384": "n=16384 (128x128) 2-D grid, undirected, relabelled, int32 U{1..100}, seed 2",
    "cfg3_er65536": "n=65536 Erdos-Renyi, directed, avg out-degree 16, int32 U{1..100}, seed 3",
    "cfg4_er131072_f32": "n=131072 Erdos-Renyi, directed, avg out-degree 256, fp32 U[1,100), seed 4",
    "cfg5_grid262144": "n=262144 (512x512) 2-D grid, undirected, relabelled, int32 U{1..100}, seed 5",
}


def baseline_config(name: str) -> CSR:
    if name == "cfg1_er1024":
        return erdos_renyi(1024, 8 * 1024, seed=1, name=name)
    if name == "cfg2_grid16384":
        return grid_2d(128, 128, seed=2, name=name)
    if name == "cfg3_er65536":
        return erdos_renyi(65536, 16 * 65536, seed=3, name=name)
    if name == "cfg4_er131072_f32":
        return erdos_renyi(131072, 256 * 131072, seed=4, dtype="f32", name=name)
    if name == "cfg5_grid262144":
        return grid_2d(512, 512, seed=5, name=name)
    raise KeyError(name)
