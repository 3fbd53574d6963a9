"""Parity at the sizes where the benchmarked code paths diverge from the small-n ones
(VERDICT r1 weak #1). Phase 3 of the dataflow kernels runs in 64-column bands once
nb - 3 >= 64 (apsp_df_common.cuh), and the fp32 engine has a cross-task chunk prefetch
(kXpref) that only the multi-band queue order exercises at scale; the benchmarked
configurations run at nb = 128 (config 2), 512 (config 3) and 1024 (config 4).

* fp32 dataflow at n = 16384 (nb = 128) and n = 20000 (nb = 157, ragged): sampled rows
  against the oracle's fp64 Dijkstra within the north-star 1e-5 relative
  tolerance (R13), +inf exactly, and bit-identical to the launch-per-phase schedule
  (both evaluate every relaxation as one RN add of the same operands and an exact min).
* fp32 at config 4's full size (n = 131072, 33.5M arcs, 68.7 GB): 32 sampled rows.
* packed16 (R16) on config 2 at full size: the int16 arithmetic is kept and every row
  is proven exact by the oracle's optimality certificate.
* the sharded dataflow kernel and the launch-per-phase sharded schedule as 2 and 8 virtual
  ranks at n = 16384 (nb = 128): every row certified.
"""
import numpy as np
import pytest

import graphgen as gg
import oracle

pytestmark = pytest.mark.gpu

INF32 = 0x3FFFFFFF


def check_f32_rows(lib, h, g, srcs):
    want = oracle.dijkstra_rows_f64(g.row_ptr, g.col, g.w, srcs)
    for i, s in enumerate(srcs):
        got = lib.apsp_get_dist(h, int(s), 1)[0].astype(np.float64)
        fin = np.isfinite(want[i])
        assert np.array_equal(np.isfinite(got), fin), "row %d: +inf pattern differs" % s
        assert got[s] == 0.0
        err = np.abs(got[fin] - want[i][fin])
        assert np.all(err <= 1e-5 * np.abs(want[i][fin])), "row %d: max rel err %.3g" % (
            s, float(np.max(err / np.maximum(np.abs(want[i][fin]), 1e-30))))


def f32_handle(lib, g, sched):
    c = lib.apsp_config_default(device=0, timing=1)
    c.schedule = sched  # 0 auto (dataflow for fp32), 1 launch-per-phase
    h = lib.apsp_init_from_csr(g.n, g.row_ptr, g.col, g.w, cfg=c)
    lib.apsp_fw_blocked(h)
    lib.apsp_reinit(h)  # as bench.py: re-initialise from the HBM-resident CSR, run again
    lib.apsp_fw_blocked(h)
    return h


@pytest.mark.parametrize("n,deg", [(16384, 64), (20000, 32)])
def test_f32_dataflow_multiband(lib, n, deg):
    g = gg.erdos_renyi(n, deg * n, seed=n + 4, dtype="f32")
    s, t, w = g.arcs()  # add duplicate arcs (R3: the minimum is kept) on a few sources
    rng = np.random.default_rng(n)
    dup = rng.choice(len(s), size=256, replace=False)
    g = gg.csr_from_arcs(n, np.concatenate([s, s[dup]]), np.concatenate([t, t[dup]]),
                         np.concatenate([w, (w[dup] * 0.5).astype(np.float32)]).astype(np.float32))
    rng = np.random.default_rng(1)
    srcs = np.unique(np.concatenate([[0, n - 1], rng.choice(n, 40, replace=False)]))
    with f32_handle(lib, g, 0) as h:
        info = lib.apsp_get_info(h)
        assert info.arith == lib.APSP_ARITH_F32
        st = lib.apsp_get_phase_stats(h)
        assert st.launches[0] == 0 and st.launches[2] == 1, "fp32 default must be the one-launch dataflow kernel"
        check_f32_rows(lib, h, g, srcs)
        a = lib.apsp_get_dist(h)
    with f32_handle(lib, g, 1) as h:
        b = lib.apsp_get_dist(h)
    assert np.array_equal(a.view(np.int32), b.view(np.int32)), "dataflow and launch-per-phase fp32 differ"


def test_f32_config4_full_size(lib):
    g = gg.baseline_config("cfg4_er131072_f32")
    rng = np.random.default_rng(4)
    srcs = np.unique(np.concatenate([[0, g.n - 1], rng.choice(g.n, 32, replace=False)]))
    c = lib.apsp_config_default(device=0, timing=1)
    with lib.apsp_init_from_csr(g.n, g.row_ptr, g.col, g.w, cfg=c) as h:
        lib.apsp_fw_blocked(h)
        st = lib.apsp_get_phase_stats(h)
        assert st.launches[2] == 1 and st.relax[2] == float(g.n) ** 3
        check_f32_rows(lib, h, g, srcs)


def certify_all(lib, g, get_rows, chunk=4096):
    for r0 in range(0, g.n, chunk):
        rows = np.ascontiguousarray(get_rows(r0, min(chunk, g.n - r0)))
        assert oracle.certify_rows_i32(g.row_ptr, g.col, g.w, r0, rows, INF32) == (0, -1), r0


def test_packed16_config2_full_size(lib):
    g = gg.baseline_config("cfg2_grid16384")
    c = lib.apsp_config_default(device=0, packed16=1, timing=1)
    with lib.apsp_init_from_csr(g.n, g.row_ptr, g.col, g.w, cfg=c) as h:
        lib.apsp_fw_blocked(h)
        lib.apsp_reinit(h)
        lib.apsp_fw_blocked(h)
        assert lib.apsp_get_info(h).arith == lib.APSP_ARITH_S16X2
        certify_all(lib, g, lambda r0, c_: lib.apsp_get_dist(h, r0, c_))


@pytest.mark.parametrize("world,sched", [(2, 2), (8, 2), (8, 1)], ids=["df-P2", "df-P8", "per_phase-P8"])
def test_sharded_virtual_ranks_n16384(lib, world, sched):
    g = gg.erdos_renyi(16384, 8 * 16384, seed=world * 10 + sched)
    c = lib.apsp_config_default(device=0, world_size=world, virtual_ranks=1)
    c.schedule = sched
    d = lib.solve(g, cfg=c)
    certify_all(lib, g, lambda r0, c_: d[r0:r0 + c_])
