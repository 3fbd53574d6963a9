"""The small-n kernel (csrc/apsp_fw_small.cu): the blocked FW with 64x64
tiles, all rounds in one persistent launch (APSP_SCHED_SMALL; the default for n_pad <=
2048). Bit-exact against the oracle at every tile count around the 64/128 boundaries,
negative weights and planted negative cycles (R6: first step of the cycle's largest
vertex), fp32 against the fp64 oracle, the queue delay, forced at a larger n, and equal
to the 128-tile dataflow kernel and the launch-per-phase schedule."""
import numpy as np
import pytest

import graphgen as gg
import oracle

pytestmark = pytest.mark.gpu

INF32 = 0x3FFFFFFF


def want_i32(g):
    d, neg = oracle.fw_i64(g.row_ptr, g.col, g.w)
    assert not neg
    return np.where(d == oracle.INF_I64, INF32, d)


def run(lib, g, schedule=3, **kw):
    c = lib.apsp_config_default(device=0, schedule=schedule, **kw)
    return lib.solve(g, cfg=c)


@pytest.mark.parametrize("n", [1, 2, 63, 64, 65, 127, 128, 129, 191, 192, 255, 256, 300, 640, 1000, 1024, 1500,
                               2048])
def test_small_bit_exact_every_tile_count(lib, n):
    gens = [gg.erdos_renyi(n, 4 * n, seed=n + 3)]
    if n >= 32:
        gens.append(gg.grid_2d(max(1, n // 32), 32, seed=n))
    for g in gens:
        assert np.array_equal(run(lib, g).astype(np.int64), want_i32(g)), n


def test_small_is_the_default_for_small_n(lib):
    g = gg.baseline_config("cfg1_er1024")
    c = lib.apsp_config_default(device=0, timing=1)
    with lib.apsp_init_from_csr(g.n, g.row_ptr, g.col, g.w, cfg=c) as h:
        lib.apsp_fw_blocked(h)
        st = lib.apsp_get_phase_stats(h)
        assert st.launches[2] == 1 and st.launches[0] == 0 and st.relax[2] == 1024.0 ** 3
        got = lib.apsp_get_dist(h)
    assert np.array_equal(got.astype(np.int64), want_i32(g))


@pytest.mark.parametrize("delay", [1, 7, 100, 1 << 30])
def test_small_queue_delays(lib, delay):
    g = gg.grid_2d(30, 40, seed=delay % 13)
    assert np.array_equal(run(lib, g, dataflow_delay=delay).astype(np.int64), want_i32(g))


def test_small_negative_weights_and_cycles(lib):
    g = gg.grid_2d(24, 30, seed=4)
    p = np.random.default_rng(2).integers(-400, 400, size=g.n)
    s, t, w = g.arcs()
    gn = gg.csr_from_arcs(g.n, s, t, (w.astype(np.int64) + p[s] - p[t]).astype(np.int32))
    assert np.array_equal(run(lib, gn).astype(np.int64), want_i32(gn))
    base = gg.erdos_renyi(700, 2800, seed=5)
    # a cycle inside a 64-tile, one across the 64 boundary, one through the last vertex
    for u, v in ((10, 40), (60, 70), (5, 699)):
        gc = gg.with_arcs(base, [u, v], [v, u], [-300, 100])
        _, neg = oracle.fw_i64(gc.row_ptr, gc.col, gc.w)
        assert neg
        with pytest.raises(lib.NegativeCycleError):
            run(lib, gc)


def test_small_f32(lib):
    g = gg.erdos_renyi(1100, 1100 * 64, seed=9, dtype="f32")
    got = run(lib, g).astype(np.float64)
    want, _ = oracle.fw_f64(g.row_ptr, g.col, g.w)
    fin = np.isfinite(want)
    assert np.array_equal(np.isfinite(got), fin)
    assert np.all(np.abs(got[fin] - want[fin]) <= 1e-5 * np.abs(want[fin]))
    # deterministic (each candidate sum is one RN add of operands fixed by the schedule); a
    # different round depth b (the 128-tile kernels) rounds other partial paths, so across b
    # the results agree within the tolerance only (R13)
    assert np.array_equal(run(lib, g).view(np.int32), got.astype(np.float32).view(np.int32))
    other = run(lib, g, schedule=1).astype(np.float64)
    assert np.all(np.abs(other[fin] - got[fin]) <= 2e-5 * np.abs(want[fin]))


def test_small_forced_at_larger_n_equals_other_schedules(lib):
    g = gg.erdos_renyi(3000, 3000 * 5, seed=21)
    a = run(lib, g)
    assert np.array_equal(a.astype(np.int64), want_i32(g))
    assert np.array_equal(a, run(lib, g, schedule=2))
    assert np.array_equal(a, run(lib, g, schedule=1))


def test_small_repeated_runs_and_reinit(lib):
    g = gg.erdos_renyi(900, 4500, seed=8)
    want = want_i32(g)
    with lib.apsp_init_from_csr(g.n, g.row_ptr, g.col, g.w, cfg=lib.apsp_config_default(device=0)) as h:
        for _ in range(3):
            lib.apsp_fw_blocked(h)
            assert np.array_equal(lib.apsp_get_dist(h).astype(np.int64), want)
            lib.apsp_reinit(h)


@pytest.mark.parametrize("split", [1, 2, 4, 8, 16])
def test_small_split_chain_tiles(lib, monkeypatch, split):
    """The chain panel tiles P2R(k; k,k+1) / P2C(k; k+1,k) run as `split` parts (column / row ranges,
    counted into their own flags): bit-exact at several tile counts, with negative weights, a
    negative cycle next to the diagonal, and fp32 bit-identical to whole tasks (same sums)."""
    monkeypatch.setenv("APSP_SMALL_SPLIT", str(split))
    for n in (64, 65, 200, 1024, 1999):
        g = gg.erdos_renyi(n, 6 * n, seed=n + split)
        assert np.array_equal(run(lib, g).astype(np.int64), want_i32(g)), n
    g = gg.grid_2d(20, 50, seed=3)
    p = np.random.default_rng(5).integers(-300, 300, size=g.n)
    s, t, w = g.arcs()
    gn = gg.csr_from_arcs(g.n, s, t, (w.astype(np.int64) + p[s] - p[t]).astype(np.int32))
    assert np.array_equal(run(lib, gn).astype(np.int64), want_i32(gn))
    gc = gg.with_arcs(gg.erdos_renyi(500, 2000, seed=6), [100, 130], [130, 100], [-200, 50])  # tiles 1 / 2
    with pytest.raises(lib.NegativeCycleError):
        run(lib, gc)
    gf = gg.erdos_renyi(700, 700 * 16, seed=10, dtype="f32")
    got = run(lib, gf)
    monkeypatch.setenv("APSP_SMALL_SPLIT", "1")
    assert np.array_equal(got.view(np.int32), run(lib, gf).view(np.int32))


def test_small_queue_rebuilt_when_its_configuration_changes(lib, monkeypatch):
    """One handle, the split switched between runs: the queue in the work buffer is rebuilt for the
    new configuration (its key), and every run stays exact; repeated runs reuse it (flags re-zeroed
    by the previous launch's last CTA)."""
    g = gg.erdos_renyi(1000, 5000, seed=12)
    want = want_i32(g)
    with lib.apsp_init_from_csr(g.n, g.row_ptr, g.col, g.w, cfg=lib.apsp_config_default(device=0)) as h:
        for split in ("8", "8", "1", "2", "2", "16", "4"):
            monkeypatch.setenv("APSP_SMALL_SPLIT", split)
            lib.apsp_reinit(h)
            lib.apsp_fw_blocked(h)
            assert np.array_equal(lib.apsp_get_dist(h).astype(np.int64), want), split
