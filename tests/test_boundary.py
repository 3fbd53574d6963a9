"""Boundary algorithm (Djidjev et al.; eq. (1); Algorithm 3).

CPU part: the decomposition itself — dist2 per component, dist3 on the boundary graph
with virtual edges, dist4 by eq. (1) — computed here with the CPU oracle's FW and numpy
min-plus products reproduces the oracle's plain FW on the whole graph (a check of the
reading of eq. (1), including same-component pairs, not of the kernels).
GPU part: apsp_init_boundary + apsp_solve, bit-exact against the oracle.
"""
import numpy as np
import pytest

import graphgen as gg
import oracle

INF32 = 0x3FFFFFFF
BIG = oracle.INF_I64


def fw_dense(d):
    d = d.copy()
    oracle.fw_dense_i64(d)
    return d


def minplus(a, b):
    """(a (x) b)[i][j] = min_k a[i][k] + b[k][j] with INF_I64 as infinity."""
    out = np.full((a.shape[0], b.shape[1]), BIG, dtype=np.int64)
    for kk in range(a.shape[1]):
        col = a[:, kk:kk + 1]
        row = b[kk:kk + 1, :]
        ok = (col != BIG) & (row != BIG)
        cand = np.where(ok, col + np.where(row == BIG, 0, row), BIG)
        out = np.minimum(out, cand)
    return out


def boundary_reference(g, comp, k):
    """eq. (1) with the oracle's FW as the per-component / boundary-graph solver."""
    n = g.n
    d0 = oracle.init_i64(g.row_ptr, g.col, g.w)
    s, t, _ = g.arcs()
    isb = np.zeros(n, bool)
    cross = comp[s] != comp[t]
    isb[s[cross]] = True
    isb[t[cross]] = True
    comps = [np.flatnonzero(comp == c) for c in range(k)]
    bnd = [cv[isb[cv]] for cv in comps]
    # step 2: dist2 inside every component (arcs between components removed)
    dist2 = {}
    for c in range(k):
        cv = comps[c]
        dist2[c] = fw_dense(np.ascontiguousarray(d0[np.ix_(cv, cv)]))
    # step 3: boundary graph with virtual edges, dist3
    B = np.concatenate(bnd) if k else np.zeros(0, int)
    pos = {v: i for i, v in enumerate(B)}
    bound = np.ascontiguousarray(d0[np.ix_(B, B)])
    for c in range(k):
        idx = np.array([pos[v] for v in bnd[c]], dtype=np.int64)
        loc = np.searchsorted(comps[c], bnd[c])
        bound[np.ix_(idx, idx)] = np.minimum(bound[np.ix_(idx, idx)], dist2[c][np.ix_(loc, loc)])
    dist3 = fw_dense(bound)
    # step 4: dist4(v_i, v_j) = min(dist2(v_i,b_i) + dist3(b_i,b_j) + dist2(b_j,v_j)); same component: min with dist2
    out = np.full((n, n), BIG, dtype=np.int64)
    for i in range(k):
        li = np.searchsorted(comps[i], bnd[i])
        c2b = dist2[i][:, li]
        bi = np.array([pos[v] for v in bnd[i]], dtype=np.int64)
        for j in range(k):
            lj = np.searchsorted(comps[j], bnd[j])
            b2c = dist2[j][lj, :]
            bj = np.array([pos[v] for v in bnd[j]], dtype=np.int64)
            blk = minplus(minplus(c2b, dist3[np.ix_(bi, bj)]), b2c) if len(bi) and len(bj) else \
                np.full((len(comps[i]), len(comps[j])), BIG, dtype=np.int64)
            if i == j:
                blk = np.minimum(blk, dist2[i])
            out[np.ix_(comps[i], comps[j])] = blk
    return out


@pytest.mark.parametrize("case", ["grid", "grid_neg", "er_random", "disjoint", "single"])
def test_boundary_decomposition_matches_fw(case):
    if case.startswith("grid"):
        g = gg.grid_2d(9, 12, seed=3)
        if case == "grid_neg":
            rng = np.random.default_rng(1)
            p = rng.integers(-40, 40, size=g.n)
            s, t, w = g.arcs()
            g2 = gg.csr_from_arcs(g.n, s, t, (w.astype(np.int64) + p[s] - p[t]).astype(np.int32))
            g2.meta = g.meta
            g = g2
        comp, k = gg.grid_block_partition(g, 3, 2)
    elif case == "er_random":
        g = gg.erdos_renyi(70, 250, seed=5)
        comp, k = gg.random_partition(g.n, 4, seed=2)
    elif case == "disjoint":
        g = gg.disjoint_union(gg.erdos_renyi(30, 90, seed=1), gg.directed_ring(25, 3))
        comp = np.r_[np.zeros(30), np.ones(25)].astype(np.int32)
        k = 2
    else:
        g = gg.erdos_renyi(40, 160, seed=6)
        comp, k = np.zeros(40, np.int32), 1
    want, neg = oracle.fw_i64(g.row_ptr, g.col, g.w)
    assert not neg
    assert np.array_equal(boundary_reference(g, comp, k), want)


def test_grid_block_partition_shape():
    g = gg.grid_2d(128, 128, seed=2)
    comp, k = gg.grid_block_partition(g, 4, 8)
    assert k == 32 and np.all(np.bincount(comp, minlength=k) == 512)
    s, t, _ = g.arcs()
    isb = np.zeros(g.n, bool)
    cross = comp[s] != comp[t]
    isb[s[cross]] = True
    # 4x8 blocks of 32x16 cells: boundary ~ perimeter cells
    assert 2000 < isb.sum() < 3500


# ----------------------------------------------------------------------------- GPU


def oracle_i32(g):
    d, _ = oracle.fw_i64(g.row_ptr, g.col, g.w)
    return np.where(d == BIG, INF32, d)


@pytest.mark.gpu
@pytest.mark.parametrize("shape,blocks", [((20, 30), (2, 3)), ((33, 17), (3, 1)), ((40, 40), (4, 4)),
                                          ((12, 11), (1, 1))])
def test_boundary_gpu_grid(lib, shape, blocks):
    g = gg.grid_2d(*shape, seed=shape[0])
    comp, k = gg.grid_block_partition(g, *blocks)
    got = lib.solve_boundary(g, comp, k, cfg=lib.apsp_config_default(device=0))
    assert np.array_equal(got.astype(np.int64), oracle_i32(g))


@pytest.mark.gpu
def test_boundary_gpu_random_partition_and_disjoint(lib):
    g = gg.erdos_renyi(500, 2000, seed=4)
    comp, k = gg.random_partition(g.n, 5, seed=1)
    assert np.array_equal(lib.solve_boundary(g, comp, k).astype(np.int64), oracle_i32(g))
    g2 = gg.disjoint_union(gg.grid_2d(10, 20, seed=1), gg.erdos_renyi(150, 600, seed=2))
    comp2 = np.r_[np.zeros(200), np.ones(150)].astype(np.int32)
    assert np.array_equal(lib.solve_boundary(g2, comp2, 2).astype(np.int64), oracle_i32(g2))


@pytest.mark.gpu
def test_boundary_gpu_negative_weights_and_cycle(lib):
    g = gg.grid_2d(24, 24, seed=7)
    rng = np.random.default_rng(3)
    p = rng.integers(-300, 300, size=g.n)
    s, t, w = g.arcs()
    gn = gg.csr_from_arcs(g.n, s, t, (w.astype(np.int64) + p[s] - p[t]).astype(np.int32))
    gn.meta = g.meta
    comp, k = gg.grid_block_partition(gn, 3, 3)
    assert np.array_equal(lib.solve_boundary(gn, comp, k).astype(np.int64), oracle_i32(gn))
    gc = gg.with_arcs(g, [3, 500], [500, 3], [-900, 100])
    gc.meta = g.meta
    with lib.apsp_init_boundary(gc.n, gc.row_ptr, gc.col, gc.w, comp, k) as h:
        with pytest.raises(lib.NegativeCycleError):
            lib.apsp_solve(h)


@pytest.mark.gpu
def test_boundary_gpu_f32(lib):
    g = gg.grid_2d(25, 30, seed=2, dtype="f32")
    comp, k = gg.grid_block_partition(g, 2, 3)
    got = lib.solve_boundary(g, comp, k)
    want, _ = oracle.fw_f64(g.row_ptr, g.col, g.w)
    assert np.all(np.abs(got - want) <= 1e-5 * np.abs(want))


@pytest.mark.gpu
def test_boundary_gpu_config2_size(lib):
    """BASELINE config 2's grid (n=16384) with k = sqrt(n)/4 = 32 components:
    sampled rows vs the oracle's Dijkstra, row ranges, reinit + second solve."""
    g = gg.baseline_config("cfg2_grid16384")
    comp, k = gg.grid_block_partition(g, 4, 8)
    cfg = lib.apsp_config_default(device=0, timing=1)
    with lib.apsp_init_boundary(g.n, g.row_ptr, g.col, g.w, comp, k, cfg=cfg) as h:
        info = lib.apsp_get_info(h)
        assert info.mode == lib.APSP_MODE_BOUNDARY and 2000 < info.boundary_nodes < 3500
        lib.apsp_solve(h)
        lib.apsp_reinit(h)
        lib.apsp_solve(h)
        srcs = np.array([0, 1, 777, 8191, 16383])
        want = oracle.dijkstra_rows_i64(g.row_ptr, g.col, g.w, srcs)
        for i, s in enumerate(srcs):
            assert np.array_equal(lib.apsp_get_dist(h, int(s), 1)[0].astype(np.int64), want[i])
        blk = lib.apsp_get_dist(h, 100, 300)
        assert np.array_equal(blk[:, srcs].T.astype(np.int64), want[:, 100:400])


# --------------------------------------------------- out of core (Alg. 3 l.20)


def bnd_cfg(lib, budget=0, force=1):
    return lib.apsp_config_default(device=0, timing=1, force_out_of_core=force, device_budget_bytes=budget)


@pytest.mark.gpu
@pytest.mark.parametrize("shape,blocks", [((20, 30), (2, 3)), ((40, 40), (4, 4)), ((33, 17), (3, 1)),
                                          ((64, 48), (8, 6))])
def test_boundary_out_of_core_forced(lib, shape, blocks):
    """Every block row streams through the two device buffers into pinned host memory
    (force_out_of_core), then apsp_get_dist gathers from the host matrix: bit-exact."""
    g = gg.grid_2d(*shape, seed=shape[1])
    comp, k = gg.grid_block_partition(g, *blocks)
    with lib.apsp_init_boundary(g.n, g.row_ptr, g.col, g.w, comp, k, cfg=bnd_cfg(lib)) as h:
        info = lib.apsp_get_info(h)
        assert info.mode == lib.APSP_MODE_BOUNDARY and info.ooc_block > 0 and info.host_bytes > 0
        lib.apsp_solve(h)
        got = lib.apsp_get_dist(h)
        st = lib.apsp_get_phase_stats(h)
        assert st.launches[3] > 0  # the D2H transfers are inside the solve
        lib.apsp_reinit(h)
        lib.apsp_solve(h)
        assert np.array_equal(lib.apsp_get_dist(h, 3, 50), got[3:53])
    assert np.array_equal(got.astype(np.int64), oracle_i32(g))


@pytest.mark.gpu
def test_boundary_out_of_core_budget_many_groups_and_residency(lib):
    """A device budget (L of P:186) small enough that each buffer holds one or two block rows
    (N_row), so many groups alternate between the two buffers / streams; a larger budget keeps
    the last block rows resident in HBM (R21) while the rest stream: both bit-exact."""
    g = gg.grid_2d(96, 64, seed=9)  # n = 6144
    comp, k = gg.grid_block_partition(g, 6, 4)  # 24 components of 256 vertices
    want = oracle_i32(g)
    seen = set()
    for budget in (40 << 20, 64 << 20, 120 << 20):
        with lib.apsp_init_boundary(g.n, g.row_ptr, g.col, g.w, comp, k, cfg=bnd_cfg(lib, budget, 0)) as h:
            info = lib.apsp_get_info(h)
            assert info.ooc_block > 0, "the result (%d B) must not fit %d B" % (info.n_pad ** 2 * 4, budget)
            seen.add((info.host_bytes < info.n_pad ** 2 * 4, info.ooc_block))
            lib.apsp_solve(h)
            assert np.array_equal(lib.apsp_get_dist(h).astype(np.int64), want), budget
    assert any(part for part, _ in seen), "no budget left block rows resident"


@pytest.mark.gpu
def test_boundary_out_of_core_disjoint_negative_f32(lib):
    # components without boundary nodes (their rows / columns stay +inf but for dist2)
    g2 = gg.disjoint_union(gg.grid_2d(10, 20, seed=1), gg.erdos_renyi(150, 600, seed=2))
    comp2 = np.r_[np.zeros(200), np.ones(150)].astype(np.int32)
    with lib.apsp_init_boundary(g2.n, g2.row_ptr, g2.col, g2.w, comp2, 2, cfg=bnd_cfg(lib)) as h:
        lib.apsp_solve(h)
        assert np.array_equal(lib.apsp_get_dist(h).astype(np.int64), oracle_i32(g2))
    g = gg.grid_2d(24, 24, seed=7)
    p = np.random.default_rng(3).integers(-300, 300, size=g.n)
    s, t, w = g.arcs()
    gn = gg.csr_from_arcs(g.n, s, t, (w.astype(np.int64) + p[s] - p[t]).astype(np.int32))
    gn.meta = g.meta
    comp, k = gg.grid_block_partition(gn, 3, 3)
    with lib.apsp_init_boundary(gn.n, gn.row_ptr, gn.col, gn.w, comp, k, cfg=bnd_cfg(lib)) as h:
        lib.apsp_solve(h)
        assert np.array_equal(lib.apsp_get_dist(h).astype(np.int64), oracle_i32(gn))
    gf = gg.grid_2d(25, 30, seed=2, dtype="f32")
    comp, k = gg.grid_block_partition(gf, 2, 3)
    with lib.apsp_init_boundary(gf.n, gf.row_ptr, gf.col, gf.w, comp, k, cfg=bnd_cfg(lib)) as h:
        lib.apsp_solve(h)
        got = lib.apsp_get_dist(h)
    want, _ = oracle.fw_f64(gf.row_ptr, gf.col, gf.w)
    assert np.all(np.abs(got - want) <= 1e-5 * np.abs(want))


@pytest.mark.gpu
def test_boundary_out_of_core_config2_certified(lib):
    """Config 2's grid, k = sqrt(n)/4 = 32 components, forced out of core with a
    budget: EVERY row proven by the oracle's optimality certificate."""
    g = gg.baseline_config("cfg2_grid16384")
    comp, k = gg.grid_block_partition(g, 4, 8)
    with lib.apsp_init_boundary(g.n, g.row_ptr, g.col, g.w, comp, k, cfg=bnd_cfg(lib, 600 << 20, 0)) as h:
        info = lib.apsp_get_info(h)
        assert info.ooc_block > 0 and info.host_bytes > 0
        lib.apsp_solve(h)
        for r0 in range(0, g.n, 4096):
            rows = lib.apsp_get_dist(h, r0, 4096)
            assert oracle.certify_rows_i32(g.row_ptr, g.col, g.w, r0, rows, INF32) == (0, -1), r0


@pytest.mark.gpu
@pytest.mark.slow
def test_boundary_out_of_core_config5_certified(lib):
    """Config 5 (n = 262144, the 275 GB result exceeds the device) with k = sqrt(n)/4 = 128 grid
    components: the out-of-core boundary algorithm streams the block rows that do not fit
    (P:184-197), and EVERY row is proven exact by the oracle's optimality certificate."""
    g = gg.baseline_config("cfg5_grid262144")
    comp, k = gg.grid_block_partition(g, 16, 8)
    assert k == 128
    with lib.apsp_init_boundary(g.n, g.row_ptr, g.col, g.w, comp, k, cfg=lib.apsp_config_default(device=0)) as h:
        info = lib.apsp_get_info(h)
        assert info.ooc_block > 0 and info.host_bytes > 0  # out of core, some block rows streamed
        lib.apsp_solve(h)
        for r0 in range(0, g.n, 8192):
            rows = lib.apsp_get_dist(h, r0, 8192)
            assert oracle.certify_rows_i32(g.row_ptr, g.col, g.w, r0, rows, INF32) == (0, -1), r0
