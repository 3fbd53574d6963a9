"""GPU parity: the CUDA path (through the C ABI) vs the CPU oracle, element by element.

int32: bit-exact (BASELINE.json north_star). fp32: |gpu - oracle| <= 1e-5 * |oracle|
against the fp64 oracle, INF where the oracle has INF, exact 0 on the diagonal.
"""
import numpy as np
import pytest

import graphgen as gg
import oracle

pytestmark = pytest.mark.gpu

INF32 = 0x3FFFFFFF
RTOL = 1e-5


def oracle_i32(g, k_iters=None):
    d, neg = oracle.fw_i64(g.row_ptr, g.col, g.w, k_iters=k_iters)
    return np.where(d == oracle.INF_I64, INF32, d), neg


def assert_i32_equal(got, want):
    got = got.astype(np.int64)
    if not np.array_equal(got, want):
        bad = np.argwhere(got != want)
        i, j = bad[0]
        raise AssertionError("%d mismatches; first at (%d,%d): gpu %d oracle %d" %
                             (len(bad), i, j, got[i, j], want[i, j]))


def assert_f32_close(got, want):
    fin = np.isfinite(want)
    assert np.array_equal(np.isfinite(got), fin), "INF pattern differs"
    err = np.abs(got[fin].astype(np.float64) - want[fin])
    tol = RTOL * np.abs(want[fin])
    assert np.all(err <= tol), "max rel err %.3g" % np.max(err / np.maximum(np.abs(want[fin]), 1e-30))
    assert np.all(np.diag(got) == 0)


def cfg(lib, **kw):
    c = lib.apsp_config_default(device=0)
    for k, v in kw.items():
        setattr(c, k, v)
    return c


# -------------------------------------------------------------------- init --

@pytest.mark.parametrize("n", [1, 5, 128, 300])
def test_init_matches_oracle(lib, n):
    g = gg.erdos_renyi(n, 4 * n, seed=n)
    g = gg.with_arcs(g, [0, 0, n - 1], [n - 1, n - 1, n - 1], [50, 7, 3])  # duplicates + self loop
    with lib.apsp_init_from_csr(g.n, g.row_ptr, g.col, g.w, cfg=cfg(lib)) as h:
        got = lib.apsp_get_dist(h)
    want = oracle.init_i64(g.row_ptr, g.col, g.w)
    assert_i32_equal(got, np.where(want == oracle.INF_I64, INF32, want))


# ---------------------------------------------------------------- full FW --

SIZES = [1, 2, 3, 5, 31, 127, 128, 129, 255, 256, 257, 300, 640]


def graphs_for(n, seed):
    yield "er_dir", gg.erdos_renyi(n, 3 * n, seed=seed)
    yield "er_und", gg.erdos_renyi(n, 4 * n, seed=seed + 1, undirected=True)
    if n >= 4:
        r = max(1, int(np.sqrt(n)))
        yield "grid_perm", gg.grid_2d(r, n // r, seed=seed + 2)
        half = n // 2
        yield "disjoint", gg.disjoint_union(gg.erdos_renyi(half, 3 * half, seed=seed + 3),
                                            gg.directed_ring(n - half, 5))


@pytest.mark.parametrize("n", SIZES)
def test_fw_int32_bit_exact(lib, n):
    for name, g in graphs_for(n, seed=10 * n):
        got = lib.solve(g, cfg=cfg(lib))
        want, neg = oracle_i32(g)
        assert not neg
        assert_i32_equal(got, want)


@pytest.mark.parametrize("variant", [1, 2])
@pytest.mark.parametrize("n", [129, 640, 1000])
def test_fw_minplus_variants(lib, n, variant):
    """minplus_variant selects the min-plus kernel: 1 = cp.async + one CTA barrier per chunk,
    2 = TMA + mbarrier persistent (0, the cp.async + mbarrier pipeline, is the default)."""
    for name, g in graphs_for(n, seed=n + 3):
        c = cfg(lib)
        c.minplus_variant = variant
        c.schedule = 1  # launch-per-phase schedule (the min-plus launches take the variant)
        got = lib.solve(g, cfg=c)
        want, _ = oracle_i32(g)
        assert_i32_equal(got, want)
    gf = gg.erdos_renyi(n, 6 * n, seed=n, dtype="f32")
    c = cfg(lib)
    c.minplus_variant = variant
    c.schedule = 1
    assert_f32_close(lib.solve(gf, cfg=c), oracle.fw_f64(gf.row_ptr, gf.col, gf.w)[0])


@pytest.mark.parametrize("n", [384, 640, 1000])
def test_fw_without_lookahead(lib, n):
    """no_lookahead = 1 runs phases 1-3 strictly in order on one stream (no split phase 3)."""
    for name, g in graphs_for(n, seed=n + 7):
        c = cfg(lib)
        c.no_lookahead = 1
        c.schedule = 1
        got = lib.solve(g, cfg=c)
        want, _ = oracle_i32(g)
        assert_i32_equal(got, want)


@pytest.mark.parametrize("seed", [0, 1, 2])
def test_fw_negative_weights_reweighted(lib, seed):
    """Potential-reweighted arcs are negative but no cycle is; INF must stay canonical."""
    rng = np.random.default_rng(seed)
    g0 = gg.disjoint_union(gg.erdos_renyi(200, 900, seed=seed), gg.grid_2d(10, 13, seed=seed))
    p = rng.integers(-500, 500, size=g0.n)
    s, t, w = g0.arcs()
    g = gg.csr_from_arcs(g0.n, s, t, (w.astype(np.int64) + p[s] - p[t]).astype(np.int32))
    assert (g.w < 0).any()
    got = lib.solve(g, cfg=cfg(lib))
    want, neg = oracle_i32(g)
    assert not neg
    assert_i32_equal(got, want)


@pytest.mark.parametrize("where", [(3, 9, 77), (120, 127, 128), (250, 256, 299), (0, 1, 383), (382, 383, 5)])
def test_negative_cycle_detected(lib, where):
    g = gg.erdos_renyi(384, 384 * 3, seed=4)
    a, b, c = where
    g = gg.with_arcs(g, [a, b, c], [b, c, a], [-400, 100, 100])
    _, neg = oracle.fw_i64(g.row_ptr, g.col, g.w)
    assert neg
    with lib.apsp_init_from_csr(g.n, g.row_ptr, g.col, g.w, cfg=cfg(lib)) as h:
        with pytest.raises(lib.NegativeCycleError):
            lib.apsp_fw_blocked(h)


def test_negative_self_loop_is_a_cycle(lib):
    g = gg.with_arcs(gg.erdos_renyi(200, 800, seed=1), [150], [150], [-1])
    with lib.apsp_init_from_csr(g.n, g.row_ptr, g.col, g.w, cfg=cfg(lib)) as h:
        with pytest.raises(lib.NegativeCycleError):
            lib.apsp_fw_blocked(h)


def test_per_round_state_equals_partial_fw(lib):
    """After K rounds of b=128 the matrix equals plain FW after K*128 iterations
    (PAPER.md:60 invariant): catches phase-ordering bugs round by round."""
    g = gg.grid_2d(20, 30, seed=3)  # n = 600 -> 5 rounds, long shortest paths
    with lib.apsp_init_from_csr(g.n, g.row_ptr, g.col, g.w, cfg=cfg(lib)) as h:
        info = lib.apsp_get_info(h)
        assert info.rounds == 5
        for K in range(1, 6):
            lib.apsp_fw_rounds(h, K - 1, K)
            got = lib.apsp_get_dist(h)
            want, _ = oracle_i32(g, k_iters=min(K * 128, g.n))
            assert_i32_equal(got, want)


def test_metamorphic_permutation(lib):
    g = gg.grid_2d(16, 25, seed=9, permute=False)
    perm = np.random.default_rng(1).permutation(g.n)
    d = lib.solve(g, cfg=cfg(lib))
    dp = lib.solve(gg.relabel(g, perm), cfg=cfg(lib))
    assert np.array_equal(dp[np.ix_(perm, perm)], d)


def test_config1_er1024(lib):
    g = gg.baseline_config("cfg1_er1024")
    got = lib.solve(g, cfg=cfg(lib))
    want, _ = oracle_i32(g)
    assert_i32_equal(got, want)


def test_get_dist_row_ranges(lib):
    g = gg.erdos_renyi(500, 2500, seed=5)
    want, _ = oracle_i32(g)
    with lib.apsp_init_from_csr(g.n, g.row_ptr, g.col, g.w, cfg=cfg(lib)) as h:
        lib.apsp_fw_blocked(h)
        for r0, cnt in [(0, 1), (499, 1), (100, 157), (0, 500)]:
            out = np.full((cnt, 640), -7, dtype=np.int32)
            lib.apsp_get_dist(h, r0, cnt, out)
            assert_i32_equal(out[:, :500], want[r0:r0 + cnt])
            assert np.all(out[:, 500:] == -7)
        with pytest.raises(lib.ApspError):
            lib.apsp_fw_blocked(h)  # already ran -> ESTATE
        with pytest.raises(lib.ApspError):
            lib.apsp_get_dist(h, 400, 101)


# ---------------------------------------------------------------- fp32 -----

@pytest.mark.parametrize("sched", [0, 1], ids=["dataflow", "per_phase"])
@pytest.mark.parametrize("n", [7, 128, 300, 515])
def test_fw_f32_integer_weights_bit_exact(lib, n, sched):
    g = gg.erdos_renyi(n, 5 * n, seed=n, dtype="f32int")
    c = cfg(lib)
    c.schedule = sched
    got = lib.solve(g, cfg=c)
    gi = gg.csr_from_arcs(g.n, *g.arcs()[:2], g.w.astype(np.int32))
    want, _ = oracle.fw_i64(gi.row_ptr, gi.col, gi.w)
    fin = want != oracle.INF_I64
    assert np.array_equal(got[fin].astype(np.int64), want[fin]) and np.all(np.isinf(got[~fin]))


@pytest.mark.parametrize("sched", [0, 1], ids=["dataflow", "per_phase"])
@pytest.mark.parametrize("n", [100, 256, 700])
def test_fw_f32_real_weights(lib, n, sched):
    g = gg.erdos_renyi(n, 8 * n, seed=n + 1, dtype="f32")
    c = cfg(lib)
    c.schedule = sched
    got = lib.solve(g, cfg=c)
    want, _ = oracle.fw_f64(g.row_ptr, g.col, g.w)
    assert_f32_close(got, want)


def test_fw_f32_negative_weights(lib):
    rng = np.random.default_rng(2)
    g0 = gg.erdos_renyi(260, 1500, seed=3, dtype="f32")
    p = rng.uniform(-20, 20, size=g0.n)
    s, t, w = g0.arcs()
    g = gg.csr_from_arcs(g0.n, s, t, (w + p[s] - p[t]).astype(np.float32))
    got = lib.solve(g, cfg=cfg(lib))
    want, _ = oracle.fw_f64(g.row_ptr, g.col, g.w)
    fin = np.isfinite(want)
    assert np.array_equal(np.isfinite(got), fin)
    # reweighted distances can be near 0: bound the error by the path's absolute scale
    scale = np.abs(want[fin]) + np.abs(p[:, None] - p[None, :])[fin] + 100.0
    assert np.all(np.abs(got[fin] - want[fin]) <= RTOL * scale)


# --------------------------------------------------- virtual ranks (1 GPU) --

@pytest.mark.parametrize("world", [2, 3, 4])
def test_virtual_ranks_match_oracle(lib, world):
    """The 1-D block-row sharded schedule (owner phase 1 + row panel, band broadcast,
    local column panel + phase 3) run as `world` shards on one GPU."""
    for g in [gg.grid_2d(20, 33, seed=world), gg.erdos_renyi(900, 3000, seed=world)]:
        got = lib.solve(g, cfg=cfg(lib, world_size=world, virtual_ranks=1))
        want, _ = oracle_i32(g)
        assert_i32_equal(got, want)


@pytest.mark.parametrize("world", [2, 4])
def test_virtual_ranks_without_lookahead(lib, world):
    """no_lookahead = 1: the sharded schedule round by round on one stream (no pivot lookahead)."""
    for g in [gg.grid_2d(20, 33, seed=world + 7), gg.erdos_renyi(1100, 4000, seed=world + 7)]:
        c = cfg(lib, world_size=world, virtual_ranks=1)
        c.no_lookahead = 1
        c.schedule = 1  # launch-per-phase sharded schedule (the dataflow kernel ignores no_lookahead)
        assert_i32_equal(lib.solve(g, cfg=c), oracle_i32(g)[0])


def test_virtual_ranks_f32(lib):
    g = gg.erdos_renyi(800, 6400, seed=8, dtype="f32")
    got = lib.solve(g, cfg=cfg(lib, world_size=3, virtual_ranks=1))
    assert_f32_close(got, oracle.fw_f64(g.row_ptr, g.col, g.w)[0])


@pytest.mark.parametrize("sched", [2, 0], ids=["sharded_dataflow", "per_phase_bcast"])
def test_nccl_path_single_rank(lib, sched):
    """force_nccl = 1: the sharded schedules with a real 1-rank NCCL communicator: the
    sharded dataflow kernel (schedule = APSP_SCHED_DATAFLOW; barrier + status all-reduce through NCCL) or the
    launch-per-phase schedule (default: ncclBroadcast of the pivot band every round)."""
    for g in [gg.grid_2d(17, 31, seed=1), gg.erdos_renyi(700, 2800, seed=2)]:
        c = cfg(lib)
        c.force_nccl = 1
        c.schedule = sched
        got = lib.solve(g, cfg=c)
        want, _ = oracle_i32(g)
        assert_i32_equal(got, want)
    g = gg.with_arcs(gg.erdos_renyi(300, 900, seed=3), [10, 290], [290, 10], [-100, 20])
    c = cfg(lib)
    c.force_nccl = 1
    c.schedule = sched
    with lib.apsp_init_from_csr(g.n, g.row_ptr, g.col, g.w, cfg=c) as h:
        with pytest.raises(lib.NegativeCycleError):
            lib.apsp_fw_blocked(h)


def test_virtual_ranks_negative_cycle(lib):
    g = gg.with_arcs(gg.erdos_renyi(700, 2500, seed=5), [600, 650], [650, 600], [-300, 100])
    with lib.apsp_init_from_csr(g.n, g.row_ptr, g.col, g.w, cfg=cfg(lib, world_size=4, virtual_ranks=1)) as h:
        with pytest.raises(lib.NegativeCycleError):
            lib.apsp_fw_blocked(h)


# ---------------------------------------------------------- phase stats ----

def test_phase_stats_count_all_relaxations(lib):
    g = gg.erdos_renyi(1000, 5000, seed=1)
    c = cfg(lib, timing=1)
    c.schedule = 1  # launch-per-phase schedule
    with lib.apsp_init_from_csr(g.n, g.row_ptr, g.col, g.w, cfg=c) as h:
        lib.apsp_fw_blocked(h)
        st = lib.apsp_get_phase_stats(h)
        n_pad = lib.apsp_get_info(h).n_pad
    assert sum(st.relax[:3]) == float(n_pad) ** 3
    nb = n_pad // 128
    # phase 3 = one launch in the last round, two (3A + 3B, lookahead split) before it
    assert st.launches[0] == nb and st.launches[2] == 2 * (nb - 1) + 1 and st.ms[2] > 0
