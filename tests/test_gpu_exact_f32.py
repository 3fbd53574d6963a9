"""R25 (apsp_config.exact_f32): int32 inputs closed by the fp32 engine (FADD2 + FMNMX3) when
every candidate sum of the blocked FW is an integer of magnitude <= 2^24
(weights in [0, W], 2 (n - 1) W <= 2^24; R25). The int32 output must be
bit-identical to the oracle's and to the int32 engine's; graphs outside the
bound, negative weights and the small-n kernel fall back to int32 arithmetic (arith says
which ran); a serving handle re-decides per loaded graph; config 3 at full size is
certified row by row, as the bench runs it."""
import numpy as np
import pytest

import graphgen as gg
import oracle

from test_gpu_fullsize import check_sampled_rows

pytestmark = pytest.mark.gpu

INF32 = 0x3FFFFFFF
B24 = 1 << 24


def want_i32(g):
    d, neg = oracle.fw_i64(g.row_ptr, g.col, g.w)
    assert not neg
    return np.where(d == oracle.INF_I64, INF32, d)


def solve(lib, g, exact_f32, **kw):
    cfg = lib.apsp_config_default(device=0, exact_f32=exact_f32, **kw)
    with lib.apsp_init_from_csr(g.n, g.row_ptr, g.col, g.w, cfg=cfg) as h:
        lib.apsp_fw_blocked(h)
        info = lib.apsp_get_info(h)
        return lib.apsp_get_dist(h), info


def with_weights(g, lo, hi, seed):
    s, t, _ = g.arcs()
    w = np.random.default_rng(seed).integers(lo, hi + 1, size=s.size).astype(np.int32)
    w[0] = hi  # the bound is reached by at least one arc
    return gg.csr_from_arcs(g.n, s, t, w)


@pytest.mark.parametrize("n", [2049, 2500, 3000, 4096])
def test_exact_f32_bit_exact(lib, n):
    g = gg.erdos_renyi(n, 6 * n, seed=n)  # weights 1..100
    got, info = solve(lib, g, 1)
    assert info.arith == lib.APSP_ARITH_F32_EXACT and info.exact_f32_eligible == 1
    assert info.kernel == lib.APSP_KERNEL_DATAFLOW
    assert np.array_equal(got.astype(np.int64), want_i32(g))
    ref, info0 = solve(lib, g, 0)
    assert info0.arith == lib.APSP_ARITH_I32 and np.array_equal(got, ref)


def test_exact_f32_at_the_bound_and_past_it(lib):
    """W = floor(2^24 / (2 (n - 1))) is eligible; W + 1 is not (int32 arithmetic), both exact.
    A directed ring with 3 random chords (weights in [W/2, W]) keeps shortest paths long, so
    candidate sums near 2 (n - 1) W ~ 2^24 really occur."""
    n = 2500
    W = B24 // (2 * (n - 1))
    rng = np.random.default_rng(7)
    s = np.concatenate([np.arange(n), rng.integers(0, n, 3)])
    t = np.concatenate([(np.arange(n) + 1) % n, rng.integers(0, n, 3)])
    for w_max, eligible in ((W, True), (W + 1, False)):
        w = np.random.default_rng(w_max).integers(w_max // 2, w_max + 1, size=s.size).astype(np.int32)
        w[0] = w_max
        g = gg.csr_from_arcs(n, s, t, w)
        got, info = solve(lib, g, 1)
        assert info.exact_f32_eligible == int(eligible)
        assert info.arith == (lib.APSP_ARITH_F32_EXACT if eligible else lib.APSP_ARITH_I32)
        want = want_i32(g)
        assert want[want < INF32].max() > B24 // 4  # large distances really occur
        assert np.array_equal(got.astype(np.int64), want)


def test_exact_f32_not_applied(lib):
    """Negative weights, the small-n kernel (n_pad <= 2048) and the launch-per-phase schedule
    keep int32 arithmetic."""
    g = gg.erdos_renyi(2600, 2600 * 4, seed=5)
    s, t, w = g.arcs()
    p = np.random.default_rng(1).integers(-50, 50, size=g.n)
    gn = gg.csr_from_arcs(g.n, s, t, (w.astype(np.int64) + p[s] - p[t]).astype(np.int32))
    for graph, kw in ((gn, {}), (gg.erdos_renyi(1500, 6000, seed=2), {}), (g, {"schedule": 1})):
        got, info = solve(lib, graph, 1, **kw)
        assert info.arith == lib.APSP_ARITH_I32 and info.exact_f32_eligible == 0
        assert np.array_equal(got.astype(np.int64), want_i32(graph))


def test_exact_f32_serving_handle_redecides_per_graph(lib):
    n = 3000
    a = gg.erdos_renyi(n, 5 * n, seed=21)
    b = with_weights(a, 1, 4000, seed=3)  # 2 (n - 1) 4000 > 2^24: int32
    cfg = lib.apsp_config_default(device=0, exact_f32=1)
    with lib.apsp_init_from_csr(a.n, a.row_ptr, a.col, a.w, cfg=cfg) as h:
        for g, arith in ((a, lib.APSP_ARITH_F32_EXACT), (b, lib.APSP_ARITH_I32), (a, lib.APSP_ARITH_F32_EXACT)):
            lib.apsp_load_csr(h, g.row_ptr, g.col, g.w)
            lib.apsp_fw_blocked(h)
            assert lib.apsp_get_info(h).arith == arith
            assert np.array_equal(lib.apsp_get_dist(h).astype(np.int64), want_i32(g))


def test_exact_f32_config3_full_size(lib):
    """Config 3 (n = 65536 ER, weights 1..100: 2 (n - 1) 100 = 13.1M <= 2^24) as bench.py's
    exact_f32 leg runs it: sampled rows against the oracle's Dijkstra, every row certified."""
    g = gg.baseline_config("cfg3_er65536")
    cfg = lib.apsp_config_default(device=0, timing=1, exact_f32=1)
    h = lib.apsp_init_from_csr(g.n, g.row_ptr, g.col, g.w, cfg=cfg)
    try:
        lib.apsp_fw_blocked(h)
        lib.apsp_reinit(h)
        lib.apsp_fw_blocked(h)
        assert lib.apsp_get_info(h).arith == lib.APSP_ARITH_F32_EXACT
        check_sampled_rows(lib, h, g, n_rows=16, seed=5)
        for r0 in range(0, g.n, 8192):
            rows = lib.apsp_get_dist(h, r0, 8192)
            assert oracle.certify_rows_i32(g.row_ptr, g.col, g.w, r0, rows, INF32) == (0, -1)
    finally:
        h.close()
