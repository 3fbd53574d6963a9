"""Packed int16 path (apsp_config.packed16 = 1; VIADDMNMX.S16x2, two relaxations per DPX
instruction): bit-exact against the int32 oracle, with the exactness check and the int32
redo exercised (reading R16). Both schedules: the persistent dataflow kernel
(fw_dataflow16_kernel, the default) and the launch-per-phase kernels (schedule = APSP_SCHED_PER_PHASE)."""
import numpy as np
import pytest

import graphgen as gg
import oracle

pytestmark = pytest.mark.gpu

INF32 = 0x3FFFFFFF


def want_i32(g):
    d, _ = oracle.fw_i64(g.row_ptr, g.col, g.w)
    return np.where(d == oracle.INF_I64, INF32, d)


def run16(lib, g, legacy=False, delay=0):
    c = lib.apsp_config_default(device=0, packed16=1, timing=1)
    c.schedule = 1 if legacy else 0
    c.dataflow_delay = delay
    with lib.apsp_init_from_csr(g.n, g.row_ptr, g.col, g.w, cfg=c) as h:
        eligible = lib.apsp_get_info(h).packed16_eligible
        lib.apsp_fw_blocked(h)
        arith = lib.apsp_get_info(h).arith
        d = lib.apsp_get_dist(h)
        part = lib.apsp_get_dist(h, g.n // 3, max(1, g.n // 4))
    return d, part, eligible, arith


@pytest.mark.parametrize("legacy", [False, True], ids=["dataflow", "per_phase"])
@pytest.mark.parametrize("n", [1, 2, 5, 127, 128, 129, 300, 640, 1000])
def test_packed16_bit_exact(lib, n, legacy):
    gens = [gg.erdos_renyi(n, 4 * n, seed=n), gg.erdos_renyi(n, 3 * n, seed=n + 1, undirected=True)]
    if n >= 16:
        gens.append(gg.grid_2d(max(1, n // 16), 16, seed=n))
        gens.append(gg.disjoint_union(gg.erdos_renyi(n // 2, 2 * n, seed=3), gg.directed_ring(n - n // 2, 7)))
    for g in gens:
        d, part, eligible, arith = run16(lib, g, legacy)
        w = want_i32(g)
        assert eligible == 1
        assert np.array_equal(d.astype(np.int64), w)
        r0, cnt = g.n // 3, max(1, g.n // 4)
        assert np.array_equal(part.astype(np.int64), w[r0:r0 + cnt])
        if w[w < INF32].max(initial=0) < 8192:
            assert arith == lib.APSP_ARITH_S16X2


def test_packed16_falls_back_to_int32_for_long_distances(lib):
    # a weighted path: the far ends are > 8192 apart, so the int16 result cannot be used
    g = gg.weighted_path(np.full(299, 100))
    d, _, eligible, arith = run16(lib, g)
    assert eligible == 1 and arith == lib.APSP_ARITH_I32
    assert np.array_equal(d.astype(np.int64), want_i32(g))
    # the boundary: 8191 is the largest distance the int16 path may return
    g2 = gg.weighted_path([8191, 1])
    d2, _, _, arith2 = run16(lib, g2)
    assert np.array_equal(d2.astype(np.int64), want_i32(g2)) and arith2 == lib.APSP_ARITH_I32
    g3 = gg.weighted_path([8190, 1])
    d3, _, _, arith3 = run16(lib, g3)
    assert np.array_equal(d3.astype(np.int64), want_i32(g3)) and arith3 == lib.APSP_ARITH_S16X2


def test_packed16_not_eligible(lib):
    g = gg.erdos_renyi(200, 800, seed=1)
    s, t, w = g.arcs()
    w = w.copy()
    w[0] = 8192  # weight above the int16 bound
    g2 = gg.csr_from_arcs(g.n, s, t, w)
    d, _, eligible, arith = run16(lib, g2)
    assert eligible == 0 and arith == lib.APSP_ARITH_I32
    assert np.array_equal(d.astype(np.int64), want_i32(g2))
    w[0] = -1  # negative weights are never packed
    g3 = gg.csr_from_arcs(g.n, s, t, w)
    d, _, eligible, _ = run16(lib, g3)
    assert eligible == 0 and np.array_equal(d.astype(np.int64), want_i32(g3))


def test_packed16_reinit_and_rounds(lib):
    g = gg.grid_2d(20, 32, seed=4)
    c = lib.apsp_config_default(device=0, packed16=1)
    with lib.apsp_init_from_csr(g.n, g.row_ptr, g.col, g.w, cfg=c) as h:
        with pytest.raises(lib.ApspError):
            lib.apsp_fw_rounds(h, 0, 1)
        lib.apsp_fw_blocked(h)
        a = lib.apsp_get_dist(h)
        lib.apsp_reinit(h)
        lib.apsp_fw_blocked(h)
        b = lib.apsp_get_dist(h)
    assert np.array_equal(a, b) and np.array_equal(a.astype(np.int64), want_i32(g))
    # a graph that needs int32: the second run goes straight to int32 and stays exact
    gp = gg.weighted_path(np.full(150, 90))
    with lib.apsp_init_from_csr(gp.n, gp.row_ptr, gp.col, gp.w, cfg=c) as h:
        lib.apsp_fw_blocked(h)
        lib.apsp_reinit(h)
        lib.apsp_fw_blocked(h)
        assert lib.apsp_get_info(h).arith == lib.APSP_ARITH_I32
        assert np.array_equal(lib.apsp_get_dist(h).astype(np.int64), want_i32(gp))


def test_packed16_config1(lib):
    g = gg.baseline_config("cfg1_er1024")
    d, _, eligible, arith = run16(lib, g)
    assert eligible == 1 and arith == lib.APSP_ARITH_S16X2
    assert np.array_equal(d.astype(np.int64), want_i32(g))


@pytest.mark.parametrize("delay", [1, 7, 1000000])
def test_packed16_dataflow_queue_delays(lib, delay):
    """Panel tasks right behind the diagonal (1), a few phase-3 tiles ahead (7), or after the
    whole previous phase 3 (huge): every order is dependency-safe and gives the same result."""
    g = gg.erdos_renyi(1280, 1280 * 6, seed=11)
    d, _, _, arith = run16(lib, g, delay=delay)
    assert arith == lib.APSP_ARITH_S16X2
    assert np.array_equal(d.astype(np.int64), want_i32(g))


def test_packed16_dataflow_matches_per_phase_grid(lib):
    """A relabelled grid (long unique shortest paths cross every tile boundary) at n = 2560
    (20 rounds): dataflow and launch-per-phase schedules agree bit for bit, and a sample of rows
    equals the oracle's Dijkstra."""
    g = gg.grid_2d(40, 64, seed=12, hi=60)  # max distance < 8192: stays in int16
    a, _, _, arith_a = run16(lib, g)
    b, _, _, arith_b = run16(lib, g, legacy=True)
    assert arith_a == arith_b == lib.APSP_ARITH_S16X2
    assert np.array_equal(a, b)
    rows = np.arange(0, g.n, 97)
    want = oracle.dijkstra_rows_i64(g.row_ptr, g.col, g.w, rows)
    want = np.where(want == oracle.INF_I64, INF32, want)
    assert np.array_equal(a[rows].astype(np.int64), want)


@pytest.mark.parametrize("pair", ["0", "1"])
def test_packed16_pair_and_one_round_queues(lib, monkeypatch, pair):
    """fw_dataflow16_kernel on the two-round queue (decode2: rounds k, k+1 of a bulk tile in one
    depth-256 task, 4 panel-copy parities; the default) and on the one-round queue
    (APSP_DF16_PAIR=0): bit-exact at odd and even round counts (a last single round), a ragged
    tail, and the 8191/8192 fallback boundary's int16 side."""
    monkeypatch.setenv("APSP_DF16_PAIR", pair)
    for n, seed in ((129, 1), (640, 2), (1000, 3), (1300, 4)):
        g = gg.erdos_renyi(n, 5 * n, seed=seed)
        d, _, _, arith = run16(lib, g)
        assert arith == lib.APSP_ARITH_S16X2
        assert np.array_equal(d.astype(np.int64), want_i32(g)), n
    g = gg.grid_2d(40, 64, seed=12, hi=60)
    d, _, _, _ = run16(lib, g)
    assert np.array_equal(d.astype(np.int64), want_i32(g))
