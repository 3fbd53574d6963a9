"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py times
(default config, one handle, apsp_reinit + apsp_fw_blocked), on outputs the oracle
computes one by one: sampled full rows by the oracle's Dijkstra compared
bit-exactly, plus properties that hold at any size (zero diagonal, symmetry of an
undirected graph, D[u][v] <= w(u,v)), and EVERY row checked by the oracle's optimality
certificate (oracle.certify_rows_i32, exact for strictly positive weights)."""
import numpy as np
import pytest

import graphgen as gg
import oracle

pytestmark = pytest.mark.gpu

INF32 = 0x3FFFFFFF


def run_like_bench(lib, g, **kw):
    cfg = lib.apsp_config_default(device=0, timing=1)
    for k, v in kw.items():
        setattr(cfg, k, v)
    h = lib.apsp_init_from_csr(g.n, g.row_ptr, g.col, g.w, cfg=cfg)
    lib.apsp_fw_blocked(h)
    lib.apsp_reinit(h)          # bench steps re-initialise from the HBM-resident CSR
    lib.apsp_fw_blocked(h)
    return h


def check_sampled_rows(lib, h, g, n_rows=48, seed=0):
    rng = np.random.default_rng(seed)
    srcs = np.unique(np.concatenate([[0, g.n - 1], rng.choice(g.n, size=n_rows, replace=False)]))
    want = oracle.dijkstra_rows_i64(g.row_ptr, g.col, g.w, srcs)
    want = np.where(want == oracle.INF_I64, INF32, want)
    for i, s in enumerate(srcs):
        got = lib.apsp_get_dist(h, int(s), 1)[0].astype(np.int64)
        assert got[s] == 0
        assert np.array_equal(got, want[i]), "row %d differs at %d places" % (s, int((got != want[i]).sum()))


def test_config2_grid16384_full_size(lib):
    g = gg.baseline_config("cfg2_grid16384")
    h = run_like_bench(lib, g)
    try:
        check_sampled_rows(lib, h, g)
        d = lib.apsp_get_dist(h)
        assert np.all(np.diag(d) == 0)
        # undirected grid -> symmetric distances (checked on a strided sample of blocks)
        for r0 in range(0, g.n, 4096):
            blk = d[r0:r0 + 512]
            assert np.array_equal(blk, d[:, r0:r0 + 512].T)
        s, t, w = g.arcs()
        assert np.all(d[s, t] <= w)
        assert np.all(d < INF32)  # connected grid
        assert oracle.certify_rows_i32(g.row_ptr, g.col, g.w, 0, d, INF32) == (0, -1)
    finally:
        h.close()


def test_config3_er65536_full_size(lib):
    g = gg.baseline_config("cfg3_er65536")
    h = run_like_bench(lib, g)
    try:
        check_sampled_rows(lib, h, g, n_rows=24, seed=3)
        for r0 in range(0, g.n, 8192):  # whole 17 GB result, 2 GB at a time
            rows = lib.apsp_get_dist(h, r0, 8192)
            assert oracle.certify_rows_i32(g.row_ptr, g.col, g.w, r0, rows, INF32) == (0, -1)
    finally:
        h.close()


def test_config4_shape_f32_scaled_down(lib):
    """Config 4's graph class (ER, avg degree 256, fp32 U[1,100)) at n=4096 vs the fp64 oracle
    Dijkstra, within the north-star 1e-5 relative tolerance."""
    g = gg.erdos_renyi(4096, 256 * 4096, seed=4, dtype="f32")
    h = run_like_bench(lib, g)
    try:
        srcs = np.arange(0, g.n, 97)
        want = oracle.dijkstra_rows_f64(g.row_ptr, g.col, g.w, srcs)
        for i, s in enumerate(srcs):
            got = lib.apsp_get_dist(h, int(s), 1)[0].astype(np.float64)
            fin = np.isfinite(want[i])
            assert np.array_equal(np.isfinite(got), fin)
            assert np.all(np.abs(got[fin] - want[i][fin]) <= 1e-5 * np.abs(want[i][fin]))
    finally:
        h.close()
