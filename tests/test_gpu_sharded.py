"""The sharded dataflow kernel (launch_fw_dataflow_sharded): a 1-D block-row shard over P
ranks in which the owner of each round stores the closed diagonal block and the row panel
straight into every rank's panel buffer and raises their flags (peer stores; no collective
between rounds). Run here as P virtual ranks in ONE launch on one GPU (CTA b serves rank
b % P), which exercises the same queue decoding, flag protocol and peer stores as P GPUs;
bit-exact against the oracle and against the launch-per-phase sharded schedule. Selected
with apsp_config.schedule = 2 (sharded placements default to the launch-per-phase
schedule with NCCL broadcasts)."""
import numpy as np
import pytest

import graphgen as gg
import oracle

pytestmark = pytest.mark.gpu

INF32 = 0x3FFFFFFF


def want_i32(g):
    d, _ = oracle.fw_i64(g.row_ptr, g.col, g.w)
    return np.where(d == oracle.INF_I64, INF32, d)


def solve(lib, g, world, sched=2, delay=0, **kw):
    c = lib.apsp_config_default(device=0, world_size=world, virtual_ranks=1, **kw)
    c.schedule = sched
    c.dataflow_delay = delay
    return lib.solve(g, cfg=c)


@pytest.mark.parametrize("world", [2, 3, 4, 5, 8])
def test_sharded_dataflow_matches_oracle(lib, world):
    # n_pad = 128 * world * m: one, two and three tile rows per rank, ragged tails
    for n in (128 * world - 7, 256 * world - 100, 384 * world):
        g = gg.erdos_renyi(n, 5 * n, seed=n + world)
        assert np.array_equal(solve(lib, g, world).astype(np.int64), want_i32(g)), (world, n)


@pytest.mark.parametrize("world", [2, 4])
def test_sharded_dataflow_grids_and_unions(lib, world):
    """Long unique shortest paths across every rank boundary (relabelled grid), and
    disconnected components (INF blocks)."""
    gs = [gg.grid_2d(24, 40, seed=world), gg.disjoint_union(gg.erdos_renyi(500, 2000, seed=1),
                                                           gg.directed_ring(430, 9))]
    for g in gs:
        assert np.array_equal(solve(lib, g, world).astype(np.int64), want_i32(g))


@pytest.mark.parametrize("delay", [1, 5, 1000000])
def test_sharded_dataflow_queue_delays(lib, delay):
    g = gg.erdos_renyi(1500, 7000, seed=delay % 97)
    assert np.array_equal(solve(lib, g, 3, delay=delay).astype(np.int64), want_i32(g))


def test_sharded_dataflow_equals_per_phase_and_repeats(lib):
    g = gg.grid_2d(30, 50, seed=3)
    a = solve(lib, g, 4)
    b = solve(lib, g, 4, sched=1)
    assert np.array_equal(a, b)
    c = lib.apsp_config_default(device=0, world_size=4, virtual_ranks=1)
    c.schedule = 2
    with lib.apsp_init_from_csr(g.n, g.row_ptr, g.col, g.w, cfg=c) as h:
        for _ in range(3):  # flags are zeroed per run; the shard buffers are reused
            lib.apsp_reinit(h)
            lib.apsp_fw_blocked(h)
            assert np.array_equal(lib.apsp_get_dist(h), a)


def test_sharded_dataflow_f32(lib):
    g = gg.erdos_renyi(1000, 8000, seed=8, dtype="f32")
    want, _ = oracle.fw_f64(g.row_ptr, g.col, g.w)
    got = solve(lib, g, 4)
    fin = np.isfinite(want)
    assert np.array_equal(np.isfinite(got), fin)
    assert np.all(np.abs(got[fin] - want[fin]) <= 1e-5 * np.abs(want[fin]))


@pytest.mark.parametrize("where", ["first_rank", "rank_boundary", "last_rank"])
def test_sharded_dataflow_negative_cycle(lib, where):
    n = 1024  # 4 ranks x 2 tile rows
    u, v = {"first_rank": (3, 40), "rank_boundary": (255, 256), "last_rank": (1000, 1020)}[where]
    g = gg.with_arcs(gg.erdos_renyi(n, 4 * n, seed=6), [u, v], [v, u], [-250, 100])
    c = lib.apsp_config_default(device=0, world_size=4, virtual_ranks=1)
    c.schedule = 2
    with lib.apsp_init_from_csr(g.n, g.row_ptr, g.col, g.w, cfg=c) as h:
        with pytest.raises(lib.NegativeCycleError):
            lib.apsp_fw_blocked(h)


def test_sharded_dataflow_negative_weights(lib):
    g = gg.erdos_renyi(900, 5000, seed=12)
    p = np.random.default_rng(12).integers(0, 60, g.n)
    s, t, w = g.arcs()
    g2 = gg.csr_from_arcs(g.n, s, t, (w + p[s] - p[t]).astype(np.int32))
    assert np.array_equal(solve(lib, g2, 3).astype(np.int64), want_i32(g2))
