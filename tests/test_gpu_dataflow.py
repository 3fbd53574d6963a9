"""The persistent dataflow kernel (csrc/apsp_fw_dataflow.cu): every round and phase of the
blocked FW in one launch, tasks ordered by a global queue and synchronised
by per-tile flags. It is the default single-GPU in-core path, so every test in
test_gpu_parity.py that does not set schedule already runs it; this file stresses the
parts specific to it: the queue order at every tile count (segment boundaries, nb = 1, 2,
3), the queue delay of the panel tasks (dataflow_delay: 1 = panels right behind the
diagonal, huge = panels after the whole previous phase 3), deep round overlap on small
matrices, and agreement with the launch-per-phase schedule (schedule = APSP_SCHED_PER_PHASE).
"""
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


def run(lib, g, delay=0, legacy=False, timing=0):
    c = lib.apsp_config_default(device=0, timing=timing)
    c.schedule = 1 if legacy else 2  # 2 = the dataflow kernel (the single-GPU default for both dtypes)
    c.dataflow_delay = delay
    return lib.solve(g, cfg=c)


@pytest.mark.parametrize("n", [1, 100, 128, 129, 256, 257, 384, 385, 512, 1000, 1537, 2048])
def test_dataflow_bit_exact_every_tile_count(lib, n):
    g = gg.erdos_renyi(n, 4 * n, seed=n + 1)
    got = run(lib, g).astype(np.int64)
    assert np.array_equal(got, want_i32(g))


@pytest.mark.parametrize("delay", [1, 5, 64, 1 << 30])
@pytest.mark.parametrize("n", [640, 1500])
def test_dataflow_queue_delays(lib, n, delay):
    r = int(np.sqrt(n))
    for g in (gg.grid_2d(r, n // r, seed=n + delay % 97), gg.erdos_renyi(n, 3 * n, seed=delay % 89)):
        assert np.array_equal(run(lib, g, delay=delay).astype(np.int64), want_i32(g))


def test_dataflow_long_paths(lib):
    """A relabelled ring: every distance needs information from all earlier rounds."""
    n = 2000
    g = gg.directed_ring(n, 3)
    perm = np.random.default_rng(5).permutation(n)
    g = gg.relabel(g, perm) if hasattr(gg, "relabel") else g
    assert np.array_equal(run(lib, g).astype(np.int64), want_i32(g))


def test_dataflow_equals_launch_per_phase(lib):
    g = gg.erdos_renyi(3000, 3000 * 6, seed=11)
    a = run(lib, g)
    b = run(lib, g, legacy=True)
    assert np.array_equal(a, b)
    gf = gg.erdos_renyi(2000, 2000 * 6, seed=12, dtype="f32")
    af = run(lib, gf)
    bf = run(lib, gf, legacy=True)
    # fp32: both take the minimum over the same candidate sums; min is exact, and every
    # candidate sum is rounded the same way (one add of two identical stored values)
    assert np.array_equal(af, bf)


def test_dataflow_repeated_runs_are_identical(lib):
    g = gg.erdos_renyi(2500, 2500 * 5, seed=13)
    want = want_i32(g)
    with lib.apsp_init_from_csr(g.n, g.row_ptr, g.col, g.w, cfg=lib.apsp_config_default(device=0)) as h:
        for _ in range(5):
            lib.apsp_reinit(h)
            lib.apsp_solve(h)
            assert np.array_equal(lib.apsp_get_dist(h).astype(np.int64), want)


def test_dataflow_negative_cycle(lib):
    g = gg.erdos_renyi(700, 2800, seed=3)
    g = gg.with_arcs(g, [300, 301], [301, 300], [-5, 2])
    with pytest.raises(lib.ApspError) as e:
        run(lib, g)
    assert e.value.status == lib.APSP_ENEGCYCLE


def test_dataflow_phase_stats(lib):
    g = gg.erdos_renyi(1000, 5000, seed=1)
    c = lib.apsp_config_default(device=0, timing=1)
    with lib.apsp_init_from_csr(g.n, g.row_ptr, g.col, g.w, cfg=c) as h:
        lib.apsp_fw_blocked(h)
        st = lib.apsp_get_phase_stats(h)
        n_pad = lib.apsp_get_info(h).n_pad
    assert sum(st.relax[:3]) == float(n_pad) ** 3
    assert st.launches[2] == 1 and st.launches[0] == 0 and st.ms[2] > 0


def test_dataflow_banded_phase3_order_partial_band(lib):
    """nb = 70 tile rows: the round's bulk phase 3 runs in 64-column bands plus a partial
    band; dataflow == launch-per-phase bit for bit, sampled rows == the oracle's Dijkstra."""
    g = gg.erdos_renyi(128 * 70 - 3, (128 * 70 - 3) * 4, seed=17)
    a = run(lib, g)
    b = run(lib, g, legacy=True)
    assert np.array_equal(a, b)
    srcs = np.array([0, 4500, g.n - 1])
    want = oracle.dijkstra_rows_i64(g.row_ptr, g.col, g.w, srcs)
    assert np.array_equal(a[srcs].astype(np.int64), np.where(want == oracle.INF_I64, INF32, want))


@pytest.mark.parametrize("n", [300, 512, 640, 1000, 1152, 2560, 8960])
def test_pair_schedule_equals_single_round_schedule(lib, monkeypatch, n):
    """The two-round (pair) queue (decode2: rounds k, k+1 of a tile in one depth-256 task, panel
    copies kept for 4 rounds; the single-GPU default) against the one-round queue: bit-identical
    for int32 and fp32 (every candidate sum is the same RN add of the same panel operands; min is
    exact), and int32 equal to the oracle. Odd and even tile counts, nb >= 67 (multi-band)."""
    g = gg.erdos_renyi(n, 5 * n, seed=n + 2)
    gf = gg.erdos_renyi(n, 5 * n, seed=n + 3, dtype="f32")
    out = {}
    for pair in ("0", "1"):
        monkeypatch.setenv("APSP_DF_PAIR", pair)
        out[pair] = (run(lib, g), run(lib, gf))
    assert np.array_equal(out["1"][0], out["0"][0])
    assert np.array_equal(out["1"][1].view(np.int32), out["0"][1].view(np.int32))
    if n <= 2560:
        assert np.array_equal(out["1"][0].astype(np.int64), want_i32(g))


def test_kernel_reported_per_placement(lib, monkeypatch):
    """apsp_info.kernel names what ran the closure (the bench's roofline reads it): the small-n
    kernel at n <= 2048, the one-round dataflow kernel above, the pair kernel when selected,
    launch-per-phase, packed16, the sharded kernel, out of core."""
    def kernel_of(g, **kw):
        with lib.apsp_init_from_csr(g.n, g.row_ptr, g.col, g.w, cfg=lib.apsp_config_default(device=0, **kw)) as h:
            lib.apsp_fw_blocked(h)
            return lib.KERNEL_NAMES[lib.apsp_get_info(h).kernel]
    small, big = gg.erdos_renyi(1000, 5000, seed=1), gg.erdos_renyi(3000, 15000, seed=2)
    assert kernel_of(small) == "small64"
    assert kernel_of(big) == "dataflow"
    monkeypatch.setenv("APSP_DF_PAIR", "1")
    assert kernel_of(big) == "dataflow_pair"
    monkeypatch.delenv("APSP_DF_PAIR")
    assert kernel_of(big, schedule=1) == "per_phase"
    assert kernel_of(big, packed16=1) == "dataflow16"
    assert kernel_of(big, world_size=2, virtual_ranks=1, schedule=2) == "sharded_dataflow"
    assert kernel_of(small, force_out_of_core=1, ooc_block=256) == "out_of_core"
