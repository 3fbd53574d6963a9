"""Johnson's algorithm with batched Near-Far SSSP (Algorithm 2,
P:113-135) through the C ABI (apsp_init_johnson + apsp_solve), bit-exact against the
CPU oracle for int32 (FW on small graphs, Dijkstra rows and the optimality certificate
at config sizes) and within the north-star 1e-5 relative tolerance for fp32."""
import numpy as np
import pytest

import graphgen as gg
import oracle

pytestmark = pytest.mark.gpu

INF32 = 0x3FFFFFFF


def oracle_i32(g):
    d, neg = oracle.fw_i64(g.row_ptr, g.col, g.w)
    assert not neg
    return np.where(d == oracle.INF_I64, INF32, d)


def solve(lib, g, **kw):
    cfg = kw.pop("cfg", None) or lib.apsp_config_default(device=0, timing=1)
    with lib.apsp_init_johnson(g.n, g.row_ptr, g.col, g.w, cfg=cfg, **kw) as h:
        info = lib.apsp_get_info(h)
        assert info.mode == lib.APSP_MODE_JOHNSON
        lib.apsp_solve(h)
        assert lib.apsp_get_info(h).edges_scanned >= g.m or g.n == 1
        return lib.apsp_get_dist(h), lib.apsp_get_info(h)


@pytest.mark.parametrize("kind,n", [("er", 300), ("er", 1000), ("grid", 31 * 17), ("grid", 1024),
                                    ("er_dense", 700), ("ring", 257)])
def test_johnson_int32_bit_exact(lib, kind, n):
    if kind == "er":
        g = gg.erdos_renyi(n, 6 * n, seed=n)
    elif kind == "er_dense":
        g = gg.erdos_renyi(n, 200 * n, seed=n)  # degree 200: 32 lanes per vertex
    elif kind == "ring":
        s = np.arange(n)
        g = gg.csr_from_arcs(n, s, (s + 1) % n, np.full(n, 7, np.int32))
    else:
        g = gg.grid_2d(31, n // 31, seed=n)
    got, info = solve(lib, g)
    assert np.array_equal(got.astype(np.int64), oracle_i32(g))


@pytest.mark.parametrize("delta", [1, 3, 50, 1000, 10 ** 7])
def test_johnson_any_delta_same_result(lib, delta):
    """Delta only changes the schedule, never the distances."""
    g = gg.grid_2d(20, 40, seed=5)
    got, _ = solve(lib, g, delta=delta)
    assert np.array_equal(got.astype(np.int64), oracle_i32(g))


def test_johnson_trivial_and_disconnected(lib):
    g1 = gg.csr_from_arcs(1, np.zeros(0, np.int64), np.zeros(0, np.int64), np.zeros(0, np.int32))
    got, _ = solve(lib, g1)
    assert got.tolist() == [[0]]
    g0 = gg.csr_from_arcs(5, np.zeros(0, np.int64), np.zeros(0, np.int64), np.zeros(0, np.int32))
    got, _ = solve(lib, g0)
    assert np.array_equal(got, np.where(np.eye(5, dtype=bool), 0, INF32))
    g2 = gg.disjoint_union(gg.grid_2d(10, 20, seed=1), gg.erdos_renyi(150, 600, seed=2))
    got, _ = solve(lib, g2)
    assert np.array_equal(got.astype(np.int64), oracle_i32(g2))


def test_johnson_duplicates_and_self_loops(lib):
    g = gg.csr_from_arcs(4, np.array([0, 0, 1, 2, 2, 3]), np.array([1, 1, 2, 2, 3, 0]),
                         np.array([9, 4, 3, 5, 1, 2], np.int32))
    got, _ = solve(lib, g)
    assert np.array_equal(got.astype(np.int64), oracle_i32(g))


def test_johnson_negative_weights_reweighted(lib):
    """Negative arcs without negative cycles (potential reweighting of a grid):
    Johnson's Bellman-Ford potentials give the exact int32 APSP."""
    g = gg.grid_2d(24, 30, seed=7)
    rng = np.random.default_rng(3)
    p = rng.integers(-300, 300, size=g.n)
    s, t, w = g.arcs()
    gn = gg.csr_from_arcs(g.n, s, t, (w.astype(np.int64) + p[s] - p[t]).astype(np.int32))
    assert (gn.w < 0).any()
    got, _ = solve(lib, gn)
    assert np.array_equal(got.astype(np.int64), oracle_i32(gn))


@pytest.mark.parametrize("where", ["interior", "self_loop", "last"])
def test_johnson_negative_cycle(lib, where):
    g = gg.grid_2d(12, 12, seed=3)
    if where == "interior":
        gc = gg.with_arcs(g, [3, 50], [50, 3], [-900, 100])
    elif where == "self_loop":
        gc = gg.with_arcs(g, [77], [77], [-1])
    else:
        gc = gg.with_arcs(g, [g.n - 1, g.n - 2], [g.n - 2, g.n - 1], [-200, 150])
    with lib.apsp_init_johnson(gc.n, gc.row_ptr, gc.col, gc.w) as h:
        with pytest.raises(lib.NegativeCycleError):
            lib.apsp_solve(h)


def test_johnson_f32_tolerance(lib):
    g = gg.erdos_renyi(900, 16 * 900, seed=4, dtype="f32")
    got, _ = solve(lib, g)
    want, _ = oracle.fw_f64(g.row_ptr, g.col, g.w)
    fin = np.isfinite(want)
    assert np.array_equal(np.isfinite(got), fin)
    assert np.all(np.abs(got[fin] - want[fin]) <= 1e-5 * np.abs(want[fin]))
    gi = gg.grid_2d(20, 30, seed=2)
    gf = gg.csr_from_arcs(gi.n, *gi.arcs()[:2], gi.w.astype(np.float32))
    got, _ = solve(lib, gf)  # integer-valued fp32 weights: exact
    assert np.array_equal(got.astype(np.int64), oracle_i32(gi))


def test_johnson_f32_negative_rejected(lib):
    g = gg.csr_from_arcs(3, np.array([0, 1]), np.array([1, 2]), np.array([1.0, -2.0], np.float32))
    with pytest.raises(lib.ApspError):
        lib.apsp_init_johnson(g.n, g.row_ptr, g.col, g.w)


@pytest.mark.parametrize("batch", [37, 256, 0])
def test_johnson_out_of_core_batches(lib, batch):
    """Algorithm 2: batches of `bat` sources copied back to a pinned host matrix while
    the next batch runs; ragged last batch."""
    g = gg.erdos_renyi(1000, 8000, seed=9)
    cfg = lib.apsp_config_default(device=0, timing=1, force_out_of_core=1)
    with lib.apsp_init_johnson(g.n, g.row_ptr, g.col, g.w, batch=batch, cfg=cfg) as h:
        info = lib.apsp_get_info(h)
        assert info.host_bytes == g.n * g.n * 4
        lib.apsp_solve(h)
        got = lib.apsp_get_dist(h)
        part = lib.apsp_get_dist(h, 123, 77)
        st = lib.apsp_get_phase_stats(h)
    want = oracle_i32(g)
    assert np.array_equal(got.astype(np.int64), want)
    assert np.array_equal(part.astype(np.int64), want[123:200])
    if batch:
        assert st.launches[2] == -(-g.n // batch) and st.launches[3] == st.launches[2]


def test_johnson_global_bitmaps(lib, monkeypatch):
    """The queue flags live in global memory when 2 x n/8 bytes exceed shared memory
    (n > ~393K); the test hook forces that layout at small n."""
    monkeypatch.setenv("APSP_TEST_JN_GLOBAL_BITS", "1")
    g = gg.grid_2d(30, 40, seed=11)
    got, _ = solve(lib, g)
    assert np.array_equal(got.astype(np.int64), oracle_i32(g))


@pytest.mark.parametrize("env", [{"APSP_JN_THREADS": "256"}, {"APSP_JN_THREADS": "1024"},
                                 {"APSP_JN_CTAS_PER_SM": "1"}, {"APSP_JN_THREADS": "1024", "APSP_JN_CTAS_PER_SM": "1"}])
def test_johnson_kernel_variants_same_result(lib, monkeypatch, env):
    """256/1024 threads per block, grid caps: schedule-only choices, identical distances
    (int32 with negatives, and fp32)."""
    for k, v in env.items():
        monkeypatch.setenv(k, v)
    g = gg.grid_2d(30, 37, seed=12)
    rng = np.random.default_rng(5)
    p = rng.integers(-50, 50, size=g.n)
    s, t, w = g.arcs()
    gn = gg.csr_from_arcs(g.n, s, t, (w.astype(np.int64) + p[s] - p[t]).astype(np.int32))
    got, _ = solve(lib, gn)
    assert np.array_equal(got.astype(np.int64), oracle_i32(gn))
    gf = gg.erdos_renyi(600, 40 * 600, seed=6, dtype="f32")
    got, _ = solve(lib, gf)
    want, _ = oracle.fw_f64(gf.row_ptr, gf.col, gf.w)
    fin = np.isfinite(want)
    assert np.array_equal(np.isfinite(got), fin)
    assert np.all(np.abs(got[fin] - want[fin]) <= 1e-5 * np.abs(want[fin]))


def test_johnson_reinit_and_second_solve(lib):
    g = gg.erdos_renyi(500, 3000, seed=13)
    with lib.apsp_init_johnson(g.n, g.row_ptr, g.col, g.w) as h:
        lib.apsp_solve(h)
        a = lib.apsp_get_dist(h)
        with pytest.raises(lib.ApspError):
            lib.apsp_solve(h)
        lib.apsp_reinit(h)
        lib.apsp_solve(h)
        b = lib.apsp_get_dist(h)
    assert np.array_equal(a, b)
    assert np.array_equal(a.astype(np.int64), oracle_i32(g))


def test_johnson_config2_grid_every_row_certified(lib):
    """BASELINE config 2 (n=16384 road-like grid): every row by the oracle's optimality
    certificate, sampled rows by its Dijkstra."""
    g = gg.baseline_config("cfg2_grid16384")
    got, info = solve(lib, g)
    assert oracle.certify_rows_i32(g.row_ptr, g.col, g.w, 0, got, INF32) == (0, -1)
    srcs = np.array([0, 5, 4097, 16383])
    want = oracle.dijkstra_rows_i64(g.row_ptr, g.col, g.w, srcs)
    assert np.array_equal(got[srcs].astype(np.int64), want)


def test_johnson_config3_er65536_every_row_certified(lib):
    """BASELINE config 3 (n=65536 ER, degree 16; 17 GB result in core)."""
    g = gg.baseline_config("cfg3_er65536")
    with lib.apsp_init_johnson(g.n, g.row_ptr, g.col, g.w) as h:
        lib.apsp_solve(h)
        for r0 in range(0, g.n, 8192):
            rows = lib.apsp_get_dist(h, r0, 8192)
            assert oracle.certify_rows_i32(g.row_ptr, g.col, g.w, r0, rows, INF32) == (0, -1)
        srcs = np.array([1, 30000, 65535])
        want = oracle.dijkstra_rows_i64(g.row_ptr, g.col, g.w, srcs)
        for i, s in enumerate(srcs):
            assert np.array_equal(lib.apsp_get_dist(h, int(s), 1)[0].astype(np.int64), want[i])


@pytest.mark.parametrize("world,ooc", [(2, 0), (3, 0), (3, 1)])
def test_johnson_sharded_by_source(lib, world, ooc):
    """world_size > 1: rank r computes the rows of its block of sources (no communicator:
    the SSSP instances are independent); the ranks' rows together equal the oracle.
    All ranks run here as separate handles on one GPU."""
    g = gg.erdos_renyi(700, 700 * 5, seed=31)
    want = oracle_i32(g)
    got = np.full((g.n, g.n), -1, dtype=np.int64)
    covered = 0
    for r in range(world):
        cfg = lib.apsp_config_default(device=0, world_size=world, rank=r, force_out_of_core=ooc)
        with lib.apsp_init_johnson(g.n, g.row_ptr, g.col, g.w, cfg=cfg, batch=50 if ooc else 0) as h:
            rb, rc = lib.apsp_local_rows(h)
            assert rb == r * (-(-g.n // world)) and rc > 0
            lib.apsp_solve(h)
            got[rb:rb + rc] = lib.apsp_get_dist(h, rb, rc)
            covered += rc
            with pytest.raises(lib.ApspError):
                lib.apsp_get_dist(h, (rb + rc) % g.n, 1)
    assert covered == g.n
    assert np.array_equal(got, want)
