"""Asynchronous serving API (apsp_fw_blocked_async, apsp_get_dist_async, apsp_synchronize):
results identical to the oracle with several handles in flight, statuses delivered by
apsp_synchronize, and every synchronous-only placement falling back to the blocking path."""
import numpy as np
import pytest
import torch

import graphgen as gg
import oracle

pytestmark = pytest.mark.gpu

INF32 = 0x3FFFFFFF


def want(g):
    if g.w.dtype.kind == "f":
        d, neg = oracle.fw_f64(g.row_ptr, g.col, g.w)
        return d, neg
    d, neg = oracle.fw_i64(g.row_ptr, g.col, g.w)
    return np.where(d == oracle.INF_I64, INF32, d), neg


def pinned(n, is_f):
    return torch.empty((max(n, 1), max(n, 1)), dtype=torch.float32 if is_f else torch.int32, pin_memory=True)


def check(g, got):
    w, neg = want(g)
    assert not neg
    if g.w.dtype.kind == "f":
        fin = np.isfinite(w)
        assert np.array_equal(np.isfinite(got), fin)
        assert np.all(np.abs(got[fin] - w[fin]) <= 1e-5 * np.abs(w[fin]))
    else:
        assert np.array_equal(got.astype(np.int64), w)


@pytest.mark.parametrize("n", [1, 5, 129, 300, 640])
@pytest.mark.parametrize("dtype", ["i32", "f32"])
def test_async_matches_oracle(lib, n, dtype):
    g = gg.erdos_renyi(n, 5 * n, seed=n + 1, dtype=dtype)
    out = pinned(n, dtype == "f32")
    with lib.apsp_init_from_csr(g.n, g.row_ptr, g.col, g.w, cfg=lib.apsp_config_default(device=0)) as h:
        lib.apsp_fw_blocked_async(h)
        lib.apsp_get_dist_async(h, 0, n, out.data_ptr(), out.shape[1])
        lib.apsp_synchronize(h)
        check(g, out.numpy()[:n, :n])
        # a second synchronize is a no-op; a blocking get_dist afterwards agrees
        lib.apsp_synchronize(h)
        assert np.array_equal(lib.apsp_get_dist(h), out.numpy()[:n, :n])


def test_async_many_handles_in_flight(lib):
    """Four graphs (int32 grid, ER, ring union, fp32 ER) enqueued on four handles before any
    synchronize: every result equals the oracle (the closures and D2H copies overlap)."""
    gs = [gg.grid_2d(16, 24, seed=1), gg.erdos_renyi(500, 3000, seed=2),
          gg.disjoint_union(gg.directed_ring(200, 3), gg.erdos_renyi(190, 900, seed=3)),
          gg.erdos_renyi(384, 2500, seed=4, dtype="f32")]
    hs, outs = [], []
    try:
        for g in gs:
            h = lib.apsp_init_from_csr(g.n, g.row_ptr, g.col, g.w, cfg=lib.apsp_config_default(device=0))
            hs.append(h)
            o = pinned(g.n, g.w.dtype.kind == "f")
            outs.append(o)
            lib.apsp_fw_blocked_async(h)
            lib.apsp_get_dist_async(h, 0, g.n, o.data_ptr(), o.shape[1])
        for g, h, o in zip(gs, hs, outs):
            lib.apsp_synchronize(h)
            check(g, o.numpy()[:g.n, :g.n])
    finally:
        for h in hs:
            h.close()


def test_async_partial_rows_and_blocking_calls_settle(lib):
    g = gg.erdos_renyi(700, 4000, seed=9)
    w, _ = want(g)
    out = pinned(700, False)
    with lib.apsp_init_from_csr(g.n, g.row_ptr, g.col, g.w, cfg=lib.apsp_config_default(device=0)) as h:
        lib.apsp_fw_blocked_async(h)
        lib.apsp_get_dist_async(h, 123, 200, out.data_ptr(), out.shape[1])
        # a blocking call settles the pending work first
        assert np.array_equal(lib.apsp_get_dist(h, 0, 50).astype(np.int64), w[:50])
        assert np.array_equal(out.numpy()[:200, :700].astype(np.int64), w[123:323])
        with pytest.raises(lib.ApspError):  # already ran
            lib.apsp_fw_blocked_async(h)
        lib.apsp_reinit(h)
        lib.apsp_fw_blocked_async(h)
        lib.apsp_reinit(h)  # settles the closure, then rebuilds the initial matrix
        lib.apsp_fw_blocked(h)
        assert np.array_equal(lib.apsp_get_dist(h).astype(np.int64), w)


def test_async_negative_weights_canonicalized(lib):
    g = gg.erdos_renyi(300, 1500, seed=5)
    p = np.random.default_rng(5).integers(0, 50, g.n)
    s, t, wt = g.arcs()
    g2 = gg.csr_from_arcs(g.n, s, t, (wt + p[s] - p[t]).astype(np.int32))  # negative arcs, no negative cycle
    out = pinned(300, False)
    with lib.apsp_init_from_csr(g2.n, g2.row_ptr, g2.col, g2.w, cfg=lib.apsp_config_default(device=0)) as h:
        lib.apsp_fw_blocked_async(h)
        lib.apsp_get_dist_async(h, 0, 300, out.data_ptr(), out.shape[1])
        lib.apsp_synchronize(h)
    check(g2, out.numpy()[:300, :300])


def test_async_negative_cycle_reported_by_synchronize(lib):
    g = gg.erdos_renyi(400, 2000, seed=6)
    s, t, w = g.arcs()
    s = np.concatenate([s, [130, 131]])
    t = np.concatenate([t, [131, 130]])
    w = np.concatenate([w, [-5, 2]]).astype(np.int32)
    g2 = gg.csr_from_arcs(g.n, s, t, w)
    with lib.apsp_init_from_csr(g2.n, g2.row_ptr, g2.col, g2.w, cfg=lib.apsp_config_default(device=0)) as h:
        lib.apsp_fw_blocked_async(h)
        with pytest.raises(lib.NegativeCycleError):
            lib.apsp_synchronize(h)
        lib.apsp_synchronize(h)  # the status was delivered once


@pytest.mark.parametrize("placement", ["out_of_core", "packed16", "per_phase"])
def test_async_other_placements(lib, placement):
    g = gg.erdos_renyi(640, 3000, seed=8)
    c = lib.apsp_config_default(device=0)
    if placement == "out_of_core":
        c.force_out_of_core = 1
        c.ooc_block = 256
    elif placement == "packed16":
        c.packed16 = 1
    else:
        c.schedule = 1
    out = pinned(640, False)
    with lib.apsp_init_from_csr(g.n, g.row_ptr, g.col, g.w, cfg=c) as h:
        lib.apsp_fw_blocked_async(h)
        lib.apsp_get_dist_async(h, 0, 640, out.data_ptr(), out.shape[1])
        lib.apsp_synchronize(h)
    check(g, out.numpy()[:640, :640])


@pytest.mark.parametrize("dtype", ["i32", "f32"])
def test_load_csr_serving_loop(lib, dtype):
    """Graphs of one size but different arc counts (growing and shrinking the device CSR)
    loaded into two alternating handles with async closures and copies: every result equals the
    oracle."""
    n = 333
    gs = [gg.erdos_renyi(n, d * n, seed=20 + d, dtype=dtype) for d in (2, 9, 4, 12, 1)]
    gs.append(gg.csr_from_arcs(n, np.zeros(0, np.int64), np.zeros(0, np.int64),
                               np.zeros(0, np.float32 if dtype == "f32" else np.int32)))  # m = 0
    outs = [pinned(n, dtype == "f32") for _ in range(2)]
    hs = [lib.apsp_init_from_csr(n, gs[0].row_ptr, gs[0].col, gs[0].w, cfg=lib.apsp_config_default(device=0))
          for _ in range(2)]
    try:
        prev = [None, None]
        for s, g in enumerate(gs):
            b = s % 2
            lib.apsp_synchronize(hs[b])
            if prev[b] is not None:
                check(prev[b], outs[b].numpy()[:n, :n])
            lib.apsp_load_csr(hs[b], g.row_ptr, g.col, g.w)
            lib.apsp_fw_blocked_async(hs[b])
            lib.apsp_get_dist_async(hs[b], 0, n, outs[b].data_ptr(), outs[b].shape[1])
            prev[b] = g
        for b in range(2):
            lib.apsp_synchronize(hs[b])
            check(prev[b], outs[b].numpy()[:n, :n])
    finally:
        for h in hs:
            h.close()


def test_load_csr_negative_weights_and_errors(lib):
    n = 260
    g = gg.erdos_renyi(n, 6 * n, seed=31)
    p = np.random.default_rng(31).integers(0, 40, n)
    s, t, w = g.arcs()
    gneg = gg.csr_from_arcs(n, s, t, (w + p[s] - p[t]).astype(np.int32))
    with lib.apsp_init_from_csr(n, g.row_ptr, g.col, g.w, cfg=lib.apsp_config_default(device=0)) as h:
        lib.apsp_fw_blocked(h)
        check(g, lib.apsp_get_dist(h))
        lib.apsp_load_csr(h, gneg.row_ptr, gneg.col, gneg.w)  # drifted infinities canonicalised
        lib.apsp_fw_blocked(h)
        check(gneg, lib.apsp_get_dist(h))
        bad = g.col.copy()
        bad[5] = n  # out of range
        with pytest.raises(lib.ApspError):
            lib.apsp_load_csr(h, g.row_ptr, bad, g.w)
        big = np.full(g.m, 1 << 26, dtype=np.int32)  # (n-1) * max|w| reaches INF
        with pytest.raises(lib.ApspError):
            lib.apsp_load_csr(h, g.row_ptr, g.col, big)
        lib.apsp_load_csr(h, g.row_ptr, g.col, g.w)  # still usable
        lib.apsp_fw_blocked(h)
        check(g, lib.apsp_get_dist(h))
    c = lib.apsp_config_default(device=0)
    c.force_out_of_core = 1
    c.ooc_block = 128
    with lib.apsp_init_from_csr(n, g.row_ptr, g.col, g.w, cfg=c) as h:
        with pytest.raises(lib.ApspError):
            lib.apsp_load_csr(h, g.row_ptr, g.col, g.w)


def test_load_csr_packed16_eligibility(lib):
    """A packed16 handle solves each loaded graph in int16 when its weights qualify (R16) and
    in int32 otherwise; the output is exact either way."""
    n = 400
    g1 = gg.erdos_renyi(n, 5 * n, seed=41)
    s, t, w = g1.arcs()
    w2 = w.copy()
    w2[3] = 9000  # > 8191: not eligible
    g2 = gg.csr_from_arcs(n, s, t, w2)
    c = lib.apsp_config_default(device=0, packed16=1)
    with lib.apsp_init_from_csr(n, g1.row_ptr, g1.col, g1.w, cfg=c) as h:
        for g, arith in ((g1, lib.APSP_ARITH_S16X2), (g2, lib.APSP_ARITH_I32), (g1, lib.APSP_ARITH_S16X2)):
            lib.apsp_load_csr(h, g.row_ptr, g.col, g.w)
            lib.apsp_fw_blocked(h)
            assert lib.apsp_get_info(h).arith == arith
            check(g, lib.apsp_get_dist(h))


def test_async_packed16_exact_and_replayed_fallback(lib):
    """packed16 asynchronously: the int16 exactness check (R16) is read by
    apsp_synchronize. An eligible graph keeps the int16 result; a graph whose distances
    reach 8192 is redone in int32 there and the copies already enqueued from the provisional
    int16 result are replayed, so the caller's buffer always holds the exact int32 APSP."""
    c = lib.apsp_config_default(device=0, packed16=1)
    g1 = gg.erdos_renyi(700, 4200, seed=51)
    g2 = gg.weighted_path(np.full(299, 100))  # far ends 29900 apart
    for g, arith in ((g1, lib.APSP_ARITH_S16X2), (g2, lib.APSP_ARITH_I32)):
        out = pinned(g.n, False)
        part = pinned(g.n, False)
        with lib.apsp_init_from_csr(g.n, g.row_ptr, g.col, g.w, cfg=c) as h:
            lib.apsp_fw_blocked_async(h)
            lib.apsp_get_dist_async(h, 0, g.n, out.data_ptr(), out.shape[1])
            lib.apsp_get_dist_async(h, g.n // 3, g.n // 2, part.data_ptr(), part.shape[1])
            lib.apsp_synchronize(h)
            assert lib.apsp_get_info(h).arith == arith
        w, _ = want(g)
        assert np.array_equal(out.numpy()[:g.n, :g.n].astype(np.int64), w)
        assert np.array_equal(part.numpy()[:g.n // 2, :g.n].astype(np.int64), w[g.n // 3:g.n // 3 + g.n // 2])


def test_async_packed16_serving_loop(lib):
    """load_csr + async on one packed16 handle across eligible and ineligible graphs."""
    n = 600
    c = lib.apsp_config_default(device=0, packed16=1)
    ga = gg.erdos_renyi(n, 3000, seed=61)
    s, t, w = ga.arcs()
    w2 = w.copy()
    w2[0] = 9000  # weight above the int16 bound: this graph runs in int32
    gb = gg.csr_from_arcs(n, s, t, w2)
    out = pinned(n, False)
    with lib.apsp_init_from_csr(n, ga.row_ptr, ga.col, ga.w, cfg=c) as h:
        for g in (ga, gb, ga):
            lib.apsp_load_csr(h, g.row_ptr, g.col, g.w)
            lib.apsp_fw_blocked_async(h)
            lib.apsp_get_dist_async(h, 0, n, out.data_ptr(), out.shape[1])
            lib.apsp_synchronize(h)
            check(g, out.numpy()[:n, :n])
