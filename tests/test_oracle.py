"""Pins of the CPU oracle (oracle/) to things other than itself — CPU only.

Each test checks an oracle function against a closed form, a textbook worked
example, brute-force path enumeration, or an independent algorithm, so that a
plausible slip (a dropped term, a wrong sign or index, a transposed operand)
in oracle/apsp_oracle.c fails at least one of them.
"""
import itertools
import os

import numpy as np
import pytest

import graphgen as gg
import oracle

import golden_io

INF = oracle.INF_I64


# ----------------------------------------------------------- brute force --

def brute_force(n, arcs, allowed_mid=None):
    """Shortest i->j over SIMPLE paths by exhaustive enumeration (n <= 7).

    allowed_mid: set of vertices that may appear as intermediates (None = all).
    Returns (dist int64 with INF, has_negative_simple_cycle)."""
    best = {}
    for (u, v, w) in arcs:
        best[(u, v)] = min(best.get((u, v), 1 << 62), int(w))
    adj = {u: [] for u in range(n)}
    for (u, v), w in best.items():
        adj[u].append((v, w))
    d = np.full((n, n), INF, dtype=np.int64)
    neg_cycle = False
    for s in range(n):
        d[s, s] = 0
        stack = [(s, 0, {s})]
        while stack:
            u, acc, seen = stack.pop()
            for v, w in adj[u]:
                if v == s:
                    if acc + w < 0:
                        neg_cycle = True
                    continue
                if v in seen:
                    continue
                if acc + w < d[s, v]:
                    d[s, v] = acc + w
                if allowed_mid is None or v in allowed_mid:
                    stack.append((v, acc + w, seen | {v}))
    # a self-loop (u,u,w<0) is a negative cycle; the diagonal keeps min(0, w)
    for (u, v), w in best.items():
        if u == v and w < 0:
            neg_cycle = True
    return d, neg_cycle


def random_arcs(rng, n, m, lo, hi, self_loops=False):
    arcs = []
    for _ in range(m):
        u, v = int(rng.integers(n)), int(rng.integers(n))
        if u == v and not self_loops:
            continue
        arcs.append((u, v, int(rng.integers(lo, hi + 1))))
    return arcs


def csr_of(n, arcs, dtype=np.int32):
    if arcs:
        s, d, w = zip(*arcs)
    else:
        s, d, w = (), (), ()
    return gg.csr_from_arcs(n, np.array(s, np.int64), np.array(d, np.int64), np.array(w, dtype))


# ------------------------------------------------------------- closed forms

def test_unit_grid_is_manhattan():
    rows, cols = 7, 9
    g = gg.grid_2d(rows, cols, seed=0, permute=False, unit=True)
    d, neg = oracle.fw_i64(g.row_ptr, g.col, g.w)
    assert not neg
    r = np.arange(rows * cols) // cols
    c = np.arange(rows * cols) % cols
    expect = np.abs(r[:, None] - r[None, :]) + np.abs(c[:, None] - c[None, :])
    assert np.array_equal(d, expect)


def test_permuted_unit_grid_is_permuted_manhattan():
    rows, cols = 6, 5
    rng = np.random.default_rng(5)
    perm = rng.permutation(rows * cols)
    g = gg.relabel(gg.grid_2d(rows, cols, seed=0, permute=False, unit=True), perm)
    d, _ = oracle.fw_i64(g.row_ptr, g.col, g.w)
    r = np.arange(rows * cols) // cols
    c = np.arange(rows * cols) % cols
    man = np.abs(r[:, None] - r[None, :]) + np.abs(c[:, None] - c[None, :])
    assert np.array_equal(d[np.ix_(perm, perm)], man)


@pytest.mark.parametrize("n,w", [(1, 3), (2, 5), (17, 3), (40, 7)])
def test_directed_ring(n, w):
    g = gg.directed_ring(n, w)
    d, _ = oracle.fw_i64(g.row_ptr, g.col, g.w)
    i, j = np.meshgrid(np.arange(n), np.arange(n), indexing="ij")
    assert np.array_equal(d, w * ((j - i) % n))


def test_weighted_path_prefix_sums():
    rng = np.random.default_rng(3)
    wts = rng.integers(1, 100, size=30)
    g = gg.weighted_path(wts)
    d, _ = oracle.fw_i64(g.row_ptr, g.col, g.w)
    pre = np.concatenate([[0], np.cumsum(wts)])
    assert np.array_equal(d, np.abs(pre[:, None] - pre[None, :]))


def test_complete_graph_and_trivial_cases():
    g = gg.complete(9, 4)
    d, _ = oracle.fw_i64(g.row_ptr, g.col, g.w)
    assert np.array_equal(d, 4 * (1 - np.eye(9, dtype=np.int64)))
    e = gg.empty(6)
    d, _ = oracle.fw_i64(e.row_ptr, e.col, e.w)
    assert np.array_equal(np.diag(d), np.zeros(6)) and np.all(d[~np.eye(6, dtype=bool)] == INF)
    one = gg.empty(1)
    d, _ = oracle.fw_i64(one.row_ptr, one.col, one.w)
    assert d.tolist() == [[0]]


def test_disjoint_union_is_block_diagonal():
    a = gg.erdos_renyi(20, 80, seed=1)
    b = gg.grid_2d(3, 4, seed=2)
    u = gg.disjoint_union(a, b)
    d, _ = oracle.fw_i64(u.row_ptr, u.col, u.w)
    da, _ = oracle.fw_i64(a.row_ptr, a.col, a.w)
    db, _ = oracle.fw_i64(b.row_ptr, b.col, b.w)
    assert np.array_equal(d[:20, :20], da) and np.array_equal(d[20:, 20:], db)
    assert np.all(d[:20, 20:] == INF) and np.all(d[20:, :20] == INF)


def test_textbook_worked_example():
    """CLRS 3e Fig. 25.4 (Floyd–Warshall on a 5-vertex graph with negative arcs)."""
    arcs, _, expect = golden_io.load("clrs_fig25_4.txt", base=1)
    g = csr_of(5, arcs)
    d, neg = oracle.fw_i64(g.row_ptr, g.col, g.w)
    assert not neg
    assert d.tolist() == expect


def test_textbook_bellman_ford_example():
    """CLRS 3e Fig. 24.4 (negative arcs): FW row s and Bellman–Ford from s both
    equal the figure's final d[v]."""
    arcs, s, (expect,) = golden_io.load("clrs_fig24_4.txt")
    g = csr_of(5, arcs)
    d, neg = oracle.fw_i64(g.row_ptr, g.col, g.w)
    assert not neg
    assert d[s].tolist() == expect
    row, neg = oracle.bellman_ford_row_i64(g.row_ptr, g.col, g.w, s)
    assert not neg
    assert row.tolist() == expect


def test_textbook_dijkstra_example():
    """CLRS 3e Fig. 24.6: FW row s, Dijkstra from s and Bellman–Ford from s all
    equal the figure's final d[v]."""
    arcs, s, (expect,) = golden_io.load("clrs_fig24_6.txt")
    g = csr_of(5, arcs)
    d, neg = oracle.fw_i64(g.row_ptr, g.col, g.w)
    assert not neg
    assert d[s].tolist() == expect
    assert oracle.dijkstra_rows_i64(g.row_ptr, g.col, g.w, [s])[0].tolist() == expect
    assert oracle.bellman_ford_row_i64(g.row_ptr, g.col, g.w, s)[0].tolist() == expect
    df, _ = oracle.fw_f64(g.row_ptr, g.col, g.w.astype(np.float32))
    assert df[s].tolist() == [float(x) for x in expect]


# -------------------------------------------------------------- brute force

@pytest.mark.parametrize("seed", range(60))
def test_fw_equals_brute_force_small(seed):
    rng = np.random.default_rng(100 + seed)
    n = int(rng.integers(1, 8))
    arcs = random_arcs(rng, n, int(rng.integers(0, 3 * n + 1)), 1, 20, self_loops=True)
    g = csr_of(n, arcs)
    d, neg = oracle.fw_i64(g.row_ptr, g.col, g.w)
    bf, bneg = brute_force(n, arcs)
    assert not neg and not bneg
    assert np.array_equal(d, bf)


@pytest.mark.parametrize("seed", range(60))
def test_fw_negative_weights_and_cycles_brute_force(seed):
    """Negative arcs: the oracle must flag exactly the graphs that hold a negative cycle,
    and otherwise match brute force."""
    rng = np.random.default_rng(900 + seed)
    n = int(rng.integers(2, 7))
    arcs = random_arcs(rng, n, int(rng.integers(1, 2 * n + 2)), -6, 20, self_loops=seed % 5 == 0)
    g = csr_of(n, arcs)
    d, neg = oracle.fw_i64(g.row_ptr, g.col, g.w)
    bf, bneg = brute_force(n, arcs)
    assert neg == bneg
    if not neg:
        assert np.array_equal(d, bf)


@pytest.mark.parametrize("seed", range(30))
def test_partial_fw_restricted_intermediates(seed):
    """After K outer iterations dist[i][j] = shortest path with intermediates in {0..K-1}
    (the FW invariant behind per-round parity of the blocked GPU path)."""
    rng = np.random.default_rng(300 + seed)
    n = int(rng.integers(2, 8))
    arcs = random_arcs(rng, n, 3 * n, 1, 30)
    g = csr_of(n, arcs)
    for K in range(n + 1):
        d, _ = oracle.fw_i64(g.row_ptr, g.col, g.w, k_iters=K)
        bf, _ = brute_force(n, arcs, allowed_mid=set(range(K)))
        assert np.array_equal(d, bf), K
        # continuing from iteration K reaches the full result
        oracle.fw_dense_i64(d, n, k_begin=K)
        assert np.array_equal(d, brute_force(n, arcs)[0]), K


# --------------------------------------------------- independent algorithms

@pytest.mark.parametrize("seed", range(40))
def test_fw_equals_dijkstra(seed):
    rng = np.random.default_rng(seed)
    n = int(rng.integers(1, 90))
    if seed % 3 == 0:
        g = gg.grid_2d(max(1, n // 9), 9, seed=seed)
    else:
        g = gg.erdos_renyi(n, int(rng.integers(0, 4 * n + 1)), seed=seed, undirected=seed % 2 == 0)
    d, neg = oracle.fw_i64(g.row_ptr, g.col, g.w)
    rows = oracle.dijkstra_rows_i64(g.row_ptr, g.col, g.w, np.arange(g.n))
    assert not neg
    assert np.array_equal(d, rows)


def test_dijkstra_rejects_negative_weights():
    g = csr_of(3, [(0, 1, -1)])
    with pytest.raises(ValueError):
        oracle.dijkstra_rows_i64(g.row_ptr, g.col, g.w, [0])


@pytest.mark.parametrize("seed", range(20))
def test_potential_reweighting(seed):
    """w'(u,v) = w(u,v) + p(u) - p(v) keeps shortest paths: D' = D + p(i) - p(j)
    (Johnson's reweighting identity). Negative arcs appear; no negative cycles do.
    Also cross-checks FW against Bellman–Ford on negative weights."""
    rng = np.random.default_rng(50 + seed)
    g = gg.erdos_renyi(40, 200, seed=seed)
    p = rng.integers(-300, 300, size=g.n)
    s, t, w = g.arcs()
    g2 = gg.csr_from_arcs(g.n, s, t, (w.astype(np.int64) + p[s] - p[t]).astype(np.int32))
    assert (g2.w < 0).any()
    d, _ = oracle.fw_i64(g.row_ptr, g.col, g.w)
    d2, neg = oracle.fw_i64(g2.row_ptr, g2.col, g2.w)
    assert not neg
    fin = d != INF
    assert np.array_equal((d2 != INF), fin)
    assert np.array_equal(d2[fin], (d + p[:, None] - p[None, :])[fin])
    for src in (0, 7, 39):
        row, bneg = oracle.bellman_ford_row_i64(g2.row_ptr, g2.col, g2.w, src)
        assert not bneg and np.array_equal(row, d2[src])


def test_bellman_ford_detects_planted_cycle():
    g = gg.erdos_renyi(30, 120, seed=9)
    g = gg.with_arcs(g, [3, 11, 20], [11, 20, 3], [-50, -50, -50])
    _, neg_bf = oracle.bellman_ford_row_i64(g.row_ptr, g.col, g.w, 3)
    _, neg_fw = oracle.fw_i64(g.row_ptr, g.col, g.w)
    assert neg_bf and neg_fw


# --------------------------------------------------------------- invariants

@pytest.mark.parametrize("seed", range(8))
def test_invariants(seed):
    undirected = seed % 2 == 0
    g = gg.erdos_renyi(120, 700, seed=seed, undirected=undirected)
    d, _ = oracle.fw_i64(g.row_ptr, g.col, g.w)
    n = g.n
    assert np.all(np.diag(d) == 0)
    # D[u][v] <= w(u,v) for every arc
    s, t, w = g.arcs()
    assert np.all(d[s, t] <= w)
    # triangle inequality over all triples (INF-aware)
    df = np.where(d == INF, np.inf, d.astype(np.float64))
    for k in range(n):
        assert np.all(df <= df[:, k:k + 1] + df[k:k + 1, :])
    if undirected:
        assert np.array_equal(d, d.T)
    # adding an arc never increases any distance
    g2 = gg.with_arcs(g, [1], [2], [1])
    d2, _ = oracle.fw_i64(g2.row_ptr, g2.col, g2.w)
    assert np.all(d2 <= d)


def test_duplicates_and_self_loops():
    g = csr_of(3, [(0, 1, 9), (0, 1, 4), (0, 1, 7), (1, 1, 5), (1, 2, 2)])
    d, _ = oracle.fw_i64(g.row_ptr, g.col, g.w)
    assert d.tolist() == [[0, 4, 6], [INF, 0, 2], [INF, INF, 0]]
    g = csr_of(2, [(1, 1, -1)])
    _, neg = oracle.fw_i64(g.row_ptr, g.col, g.w)
    assert neg


def test_metamorphic_reverse_and_scale():
    g = gg.erdos_renyi(60, 300, seed=4)
    d, _ = oracle.fw_i64(g.row_ptr, g.col, g.w)
    r = gg.reverse(g)
    dr, _ = oracle.fw_i64(r.row_ptr, r.col, r.w)
    assert np.array_equal(dr, d.T)
    s, t, w = g.arcs()
    g3 = gg.csr_from_arcs(g.n, s, t, (3 * w).astype(np.int32))
    d3, _ = oracle.fw_i64(g3.row_ptr, g3.col, g3.w)
    fin = d != INF
    assert np.array_equal(d3[fin], 3 * d[fin]) and np.all(d3[~fin] == INF)


# ---------------------------------------------------------------------- fp64

@pytest.mark.parametrize("seed", range(10))
def test_f64_fw_equals_dijkstra(seed):
    g = gg.erdos_renyi(70, 400, seed=seed, dtype="f32")
    d, neg = oracle.fw_f64(g.row_ptr, g.col, g.w)
    rows = oracle.dijkstra_rows_f64(g.row_ptr, g.col, g.w, np.arange(g.n))
    assert not neg
    fin = np.isfinite(rows)
    assert np.array_equal(np.isfinite(d), fin)
    np.testing.assert_allclose(d[fin], rows[fin], rtol=1e-12)


def test_f64_integer_weights_equal_int_oracle():
    g = gg.erdos_renyi(80, 500, seed=7, dtype="f32int")
    d, _ = oracle.fw_f64(g.row_ptr, g.col, g.w)
    gi = gg.csr_from_arcs(g.n, *g.arcs()[:2], g.w.astype(np.int32))
    di, _ = oracle.fw_i64(gi.row_ptr, gi.col, gi.w)
    fin = di != INF
    assert np.array_equal(d[fin], di[fin].astype(np.float64)) and np.all(np.isinf(d[~fin]))


def test_unit_grid_f64_manhattan():
    g = gg.grid_2d(5, 6, seed=0, permute=False, unit=True, dtype="f32")
    d, _ = oracle.fw_f64(g.row_ptr, g.col, g.w)
    r = np.arange(30) // 6
    c = np.arange(30) % 6
    assert np.array_equal(d, (np.abs(r[:, None] - r[None, :]) + np.abs(c[:, None] - c[None, :])).astype(float))


# ----------------------------------------------------------------- graphgen

def test_graphgen_shapes():
    g = gg.grid_2d(128, 128, seed=2)
    assert g.n == 16384 and g.m == 65024
    e = gg.erdos_renyi(1024, 8192, seed=1)
    assert e.m == 8192
    s, t, _ = e.arcs()
    assert np.all(s != t) and np.unique(s * 1024 + t).size == 8192
    assert abs(e.density - 8192 / 1024 ** 2) < 1e-15
    g1 = gg.erdos_renyi(500, 3000, seed=11)
    g2 = gg.erdos_renyi(500, 3000, seed=11)
    assert np.array_equal(g1.col, g2.col) and np.array_equal(g1.w, g2.w)


# ------------------------------------------------- optimality certificate

INF32 = 0x3FFFFFFF  # the int32 output's "no path" value (include/apsp.h, R1)


def _as_i32(d):
    return np.where(d == oracle.INF_I64, INF32, d).astype(np.int32)


@pytest.mark.parametrize("seed", range(6))
def test_certificate_accepts_apsp_and_rejects_every_single_perturbation(seed):
    """The certificate (Bellman optimality conditions) accepts the true APSP rows
    (brute force on tiny graphs) and rejects ANY single-entry change: +1, -1, a
    finite entry made unreachable, an unreachable one made finite."""
    rng = np.random.default_rng(100 + seed)
    n = 7
    arcs = random_arcs(rng, n, 12, 1, 9)
    bf, _ = brute_force(n, arcs)
    g = csr_of(n, arcs)
    d = _as_i32(bf)
    assert oracle.certify_rows_i32(g.row_ptr, g.col, g.w, 0, d, INF32) == (0, -1)
    for s in range(n):
        for v in range(n):
            for new in (d[s, v] + 1, d[s, v] - 1, INF32, 5):
                if new == d[s, v]:
                    continue
                e = d.copy()
                e[s, v] = new
                bad, first = oracle.certify_rows_i32(g.row_ptr, g.col, g.w, 0, e, INF32)
                assert bad == 1 and first == s, (s, v, new)


def test_certificate_on_row_slices_and_strided_rows():
    g = gg.grid_2d(20, 30, seed=7)
    d, _ = oracle.fw_i64(g.row_ptr, g.col, g.w)
    d32 = _as_i32(d)
    wide = np.full((g.n, g.n + 40), -7, dtype=np.int32)
    wide[:, :g.n] = d32
    assert oracle.certify_rows_i32(g.row_ptr, g.col, g.w, 100, wide[100:300], INF32) == (0, -1)
    wide[250, 3] += 1
    assert oracle.certify_rows_i32(g.row_ptr, g.col, g.w, 100, wide[100:300], INF32) == (1, 250)
    # a row certified against the wrong source fails (d[s][s] != 0)
    assert oracle.certify_rows_i32(g.row_ptr, g.col, g.w, 101, wide[100:101], INF32)[0] == 1


def test_certificate_disconnected_and_rejects_zero_weights():
    a = gg.grid_2d(4, 4, seed=1)
    arcs = list(zip(*[x.tolist() for x in a.arcs()]))
    arcs += [(16 + u, 16 + v, w) for (u, v, w) in arcs]
    g = csr_of(32, arcs)
    d, _ = oracle.fw_i64(g.row_ptr, g.col, g.w)
    d32 = _as_i32(d)
    assert oracle.certify_rows_i32(g.row_ptr, g.col, g.w, 0, d32, INF32) == (0, -1)
    e = d32.copy()
    e[0, 20] = 1000  # finite entry for an unreachable vertex: no tight arc can support it
    assert oracle.certify_rows_i32(g.row_ptr, g.col, g.w, 0, e, INF32)[0] == 1
    z = csr_of(3, [(0, 1, 0), (1, 2, 4)])
    with pytest.raises(ValueError):
        oracle.certify_rows_i32(z.row_ptr, z.col, z.w, 0, np.zeros((3, 3), np.int32), INF32)


def test_duplicates_and_self_loops_f64():
    """R2/R3 for the fp64 oracle (init_f64 + fw_f64): duplicate arcs keep the minimum weight, a
    positive self-loop leaves the diagonal at 0, a negative one is a negative cycle; values the
    worked-out closure below fixes by hand."""
    g = csr_of(3, [(0, 1, 9.5), (0, 1, 4.25), (0, 1, 7.0), (1, 1, 5.0), (1, 2, 2.5), (2, 2, 0.5)], np.float32)
    d0 = oracle.init_f64(g.row_ptr, g.col, g.w)
    assert d0.tolist() == [[0.0, 4.25, np.inf], [np.inf, 0.0, 2.5], [np.inf, np.inf, 0.0]]
    d, neg = oracle.fw_f64(g.row_ptr, g.col, g.w)
    assert not neg
    assert d.tolist() == [[0.0, 4.25, 6.75], [np.inf, 0.0, 2.5], [np.inf, np.inf, 0.0]]
    g = csr_of(2, [(0, 1, 1.0), (1, 1, -0.5)], np.float32)
    d0 = oracle.init_f64(g.row_ptr, g.col, g.w)
    assert d0[1, 1] == -0.5  # min(0, w) on the diagonal
    _, neg = oracle.fw_f64(g.row_ptr, g.col, g.w)
    assert neg
