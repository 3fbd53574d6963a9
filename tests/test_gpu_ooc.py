"""Out-of-core path (Algorithm 1) at small n, forced by a device
budget / force_out_of_core, bit-exact against the oracle (and vs the in-core path)."""
import numpy as np
import pytest

import graphgen as gg
import oracle

pytestmark = pytest.mark.gpu

INF32 = 0x3FFFFFFF


def ooc_cfg(lib, block, budget_mb=0, stream_all=True):
    c = lib.apsp_config_default(device=0, force_out_of_core=1, ooc_block=block, timing=1)
    if budget_mb:
        c.device_budget_bytes = int(budget_mb * 2 ** 20)
    if stream_all:
        c.ooc_stream_all = 1
    return c


def oracle_i32(g):
    d, neg = oracle.fw_i64(g.row_ptr, g.col, g.w)
    return np.where(d == oracle.INF_I64, INF32, d), neg


@pytest.mark.parametrize("n,block", [(1000, 256), (700, 128), (1536, 512), (300, 128)])
def test_ooc_int32_bit_exact(lib, n, block):
    g = gg.grid_2d(max(2, n // 25), 25, seed=n) if n % 2 == 0 else gg.erdos_renyi(n, 4 * n, seed=n)
    with lib.apsp_init_from_csr(g.n, g.row_ptr, g.col, g.w, cfg=ooc_cfg(lib, block)) as h:
        info = lib.apsp_get_info(h)
        assert info.mode == lib.APSP_MODE_OUT_OF_CORE and info.ooc_block == block
        assert info.host_bytes > 0
        lib.apsp_fw_blocked(h)
        got = lib.apsp_get_dist(h)
        st = lib.apsp_get_phase_stats(h)
    want, _ = oracle_i32(g)
    assert np.array_equal(got.astype(np.int64), want)
    assert st.launches[3] > 0  # host transfers happened
    assert abs(sum(st.relax[:3]) - float(info.n_pad) ** 3) < 1


def test_ooc_with_resident_bands(lib):
    g = gg.erdos_renyi(1024, 6000, seed=3)
    # n_pad=1024, B=256: band = 1 MiB; working set = 3 pivot buffers + 3 ring slots + 2 B x B
    # scratches (6.5 MiB) + CSR; the budget leaves room for 2 resident bands
    with lib.apsp_init_from_csr(g.n, g.row_ptr, g.col, g.w,
                                cfg=ooc_cfg(lib, 256, budget_mb=8.7, stream_all=False)) as h:
        info = lib.apsp_get_info(h)
        assert info.mode == lib.APSP_MODE_OUT_OF_CORE
        assert 0 < info.host_bytes < 1024 * 1024 * 4
        lib.apsp_fw_blocked(h)
        got = lib.apsp_get_dist(h)
        part = lib.apsp_get_dist(h, 200, 300)
    want, _ = oracle_i32(g)
    assert np.array_equal(got.astype(np.int64), want)
    assert np.array_equal(part.astype(np.int64), want[200:500])


def test_ooc_negative_weights_and_cycle(lib):
    rng = np.random.default_rng(0)
    g0 = gg.erdos_renyi(640, 3000, seed=1)
    p = rng.integers(-300, 300, size=g0.n)
    s, t, w = g0.arcs()
    g = gg.csr_from_arcs(g0.n, s, t, (w.astype(np.int64) + p[s] - p[t]).astype(np.int32))
    with lib.apsp_init_from_csr(g.n, g.row_ptr, g.col, g.w, cfg=ooc_cfg(lib, 128)) as h:
        lib.apsp_fw_blocked(h)
        got = lib.apsp_get_dist(h)
    want, _ = oracle_i32(g)
    assert np.array_equal(got.astype(np.int64), want)
    gc = gg.with_arcs(g0, [500, 20], [20, 500], [-200, 50])
    with lib.apsp_init_from_csr(gc.n, gc.row_ptr, gc.col, gc.w, cfg=ooc_cfg(lib, 128)) as h:
        with pytest.raises(lib.NegativeCycleError):
            lib.apsp_fw_blocked(h)


def test_ooc_config2_size_mixed_residency(lib):
    """BASELINE config 2's graph (n=16384) through the out-of-core scheduler with
    B=2048 (8 bands) and a budget that keeps 3 bands resident and streams 5 through
    pinned host memory; sampled rows vs the oracle's Dijkstra, bit-exact."""
    g = gg.baseline_config("cfg2_grid16384")
    bb = 2048 * 16384 * 4
    c = ooc_cfg(lib, 2048, stream_all=False)
    c.device_budget_bytes = 6 * bb + 2 * 2048 * 2048 * 4 + 3 * bb + (2 << 20)  # working set + 3 bands
    with lib.apsp_init_from_csr(g.n, g.row_ptr, g.col, g.w, cfg=c) as h:
        info = lib.apsp_get_info(h)
        assert info.mode == lib.APSP_MODE_OUT_OF_CORE and info.host_bytes == 5 * bb
        lib.apsp_fw_blocked(h)
        srcs = np.array([0, 1, 2047, 2048, 5000, 8191, 12000, 16383])
        want = oracle.dijkstra_rows_i64(g.row_ptr, g.col, g.w, srcs)
        for i, s in enumerate(srcs):
            got = lib.apsp_get_dist(h, int(s), 1)[0]
            assert np.array_equal(got.astype(np.int64), want[i]), s


def test_ooc_f32_and_reinit(lib):
    g = gg.erdos_renyi(800, 8000, seed=5, dtype="f32")
    with lib.apsp_init_from_csr(g.n, g.row_ptr, g.col, g.w, cfg=ooc_cfg(lib, 256)) as h:
        lib.apsp_fw_blocked(h)
        a = lib.apsp_get_dist(h)
        lib.apsp_reinit(h)
        lib.apsp_fw_blocked(h)
        b = lib.apsp_get_dist(h)
    assert np.array_equal(a, b)
    want, _ = oracle.fw_f64(g.row_ptr, g.col, g.w)
    fin = np.isfinite(want)
    assert np.array_equal(np.isfinite(a), fin)
    assert np.all(np.abs(a[fin] - want[fin]) <= 1e-5 * np.abs(want[fin]))


# ------------------------------------- out of core x P ranks (SURVEY §8(e) last bullet, NEXT-3)


@pytest.mark.parametrize("world,n,block", [(2, 1000, 128), (3, 700, 128), (4, 1536, 128), (2, 2048, 256),
                                           (8, 1024, 128)])
def test_ooc_virtual_ranks_bit_exact(lib, world, n, block):
    """Rank r owns bands [r nd/P, (r+1) nd/P) in its own pinned memory; the owner of band K
    closes it and broadcasts the finished pivot band (here a device copy between virtual
    ranks, the non-root receive path of the NCCL broadcast); every rank updates its bands."""
    g = gg.grid_2d(max(2, n // 25), 25, seed=n + world) if world % 2 == 0 else gg.erdos_renyi(n, 4 * n, seed=n)
    c = ooc_cfg(lib, block)
    c.world_size = world
    c.virtual_ranks = 1
    with lib.apsp_init_from_csr(g.n, g.row_ptr, g.col, g.w, cfg=c) as h:
        info = lib.apsp_get_info(h)
        assert info.mode == lib.APSP_MODE_OUT_OF_CORE and info.ooc_block == block
        assert info.n_pad % (block * world) == 0 and info.host_bytes == info.n_pad ** 2 * 4
        lib.apsp_fw_blocked(h)
        got = lib.apsp_get_dist(h)
        st = lib.apsp_get_phase_stats(h)
    want, _ = oracle_i32(g)
    assert np.array_equal(got.astype(np.int64), want)
    assert abs(sum(st.relax[:3]) - float(info.n_pad) ** 3) < 1


def test_ooc_virtual_ranks_resident_negative_f32(lib):
    # resident bands on every rank (a budget shared by the virtual ranks), negative weights
    rng = np.random.default_rng(4)
    g0 = gg.erdos_renyi(1024, 6000, seed=6)
    p = rng.integers(-300, 300, size=g0.n)
    s, t, w = g0.arcs()
    g = gg.csr_from_arcs(g0.n, s, t, (w.astype(np.int64) + p[s] - p[t]).astype(np.int32))
    c = ooc_cfg(lib, 128, budget_mb=8.6, stream_all=False)  # 2 of each rank's 4 bands resident
    c.world_size = 2
    c.virtual_ranks = 1
    with lib.apsp_init_from_csr(g.n, g.row_ptr, g.col, g.w, cfg=c) as h:
        info = lib.apsp_get_info(h)
        assert 0 < info.host_bytes < info.n_pad ** 2 * 4
        lib.apsp_fw_blocked(h)
        got = lib.apsp_get_dist(h)
    want, _ = oracle_i32(g)
    assert np.array_equal(got.astype(np.int64), want)
    gc = gg.with_arcs(g0, [900, 30], [30, 900], [-200, 50])
    c2 = ooc_cfg(lib, 128)
    c2.world_size, c2.virtual_ranks = 4, 1
    with lib.apsp_init_from_csr(gc.n, gc.row_ptr, gc.col, gc.w, cfg=c2) as h:
        with pytest.raises(lib.NegativeCycleError):
            lib.apsp_fw_blocked(h)
    gf = gg.erdos_renyi(900, 9000, seed=7, dtype="f32")
    c3 = ooc_cfg(lib, 128)
    c3.world_size, c3.virtual_ranks = 3, 1
    a = lib.solve(gf, cfg=c3)
    b = lib.solve(gf, cfg=lib.apsp_config_default(device=0, schedule=1))
    assert np.array_equal(a.view(np.int32), b.view(np.int32))  # same relaxations, same RN adds


def test_ooc_virtual_ranks_partial_rounds(lib):
    """apsp_fw_rounds in whole super-rounds over 2 virtual ranks: the state after super-round
    K is the FW state with intermediates {0 .. (K+1)B - 1}."""
    g = gg.erdos_renyi(1024, 5000, seed=12)
    c = ooc_cfg(lib, 256)
    c.world_size, c.virtual_ranks = 2, 1
    with lib.apsp_init_from_csr(g.n, g.row_ptr, g.col, g.w, cfg=c) as h:
        lib.apsp_fw_rounds(h, 0, 4)  # super-rounds 0 and 1 (B = 256 = 2 rounds of 128)
        d, _ = oracle.fw_i64(g.row_ptr, g.col, g.w, k_iters=512)
        assert np.array_equal(lib.apsp_get_dist(h).astype(np.int64), np.where(d == oracle.INF_I64, INF32, d))
        lib.apsp_fw_blocked(h)
        want, _ = oracle_i32(g)
        assert np.array_equal(lib.apsp_get_dist(h).astype(np.int64), want)
