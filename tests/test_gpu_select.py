"""Method selection (§IV) through apsp_select: the density filter
(§IV-C) decides the candidate set; the device-calibrated cost models (§IV-B)
pick among them. The estimates are checked against the methods' measured times."""
import time

import numpy as np
import pytest

import graphgen as gg

pytestmark = pytest.mark.gpu

FW, BND, JN = 0, 2, 3


def bits(*modes):
    return sum(1 << m for m in modes)


def test_select_middle_density_is_johnson(lib):
    """0.01 % <= density <= 1 %: always Johnson (config 2's grid: 0.024 %); the Johnson
    estimate from 5 sampled batches is within 2x of the measured solve."""
    g = gg.baseline_config("cfg2_grid16384")
    comp, k = gg.grid_block_partition(g, 4, 8)
    sel = lib.apsp_select(g.n, g.row_ptr, g.col, g.w, comp, k)
    assert abs(sel.density - g.m / g.n ** 2) < 1e-15
    assert sel.candidates == bits(JN) and sel.method == JN
    assert sel.est_seconds[FW] < 0 and sel.est_seconds[BND] < 0 and sel.est_seconds[JN] > 0
    assert 2000 < sel.boundary_nodes < 3500
    with lib.apsp_init_johnson(g.n, g.row_ptr, g.col, g.w) as h:
        lib.apsp_solve(h)
        lib.apsp_reinit(h)
        t0 = time.perf_counter()
        lib.apsp_solve(h)
        t = time.perf_counter() - t0
    assert 0.5 * t < sel.est_seconds[JN] < 2.0 * t, (sel.est_seconds[JN], t)


def test_select_dense_graph_fw_or_johnson(lib):
    """density > 1 %: blocked FW vs Johnson; FW estimate T0 (n/n0)^3 within 2x of its run."""
    n = 4096
    g = gg.erdos_renyi(n, int(0.05 * n * n), seed=21)
    sel = lib.apsp_select(g.n, g.row_ptr, g.col, g.w)
    assert sel.candidates == bits(FW, JN)
    assert sel.est_seconds[FW] > 0 and sel.est_seconds[JN] > 0
    assert sel.method == (FW if sel.est_seconds[FW] < sel.est_seconds[JN] else JN)
    with lib.apsp_init_from_csr(g.n, g.row_ptr, g.col, g.w) as h:
        lib.apsp_fw_blocked(h)
        lib.apsp_reinit(h)
        t0 = time.perf_counter()
        lib.apsp_fw_blocked(h)
        t = time.perf_counter() - t0
    assert 0.5 * t < sel.est_seconds[FW] < 2.0 * t, (sel.est_seconds[FW], t)


def test_select_sparse_small_separator_boundary_or_johnson(lib):
    """density < 0.01 % (a 256 x 256 grid, 0.006 %): Johnson vs the boundary algorithm;
    without a partition the boundary algorithm is not a candidate (the paper uses METIS)."""
    g = gg.grid_2d(256, 256, seed=8)
    comp, k = gg.grid_block_partition(g, 16, 16)
    sel = lib.apsp_select(g.n, g.row_ptr, g.col, g.w, comp, k)
    assert sel.candidates == bits(JN, BND)
    assert sel.est_seconds[BND] > 0 and sel.est_seconds[JN] > 0 and sel.est_seconds[FW] < 0
    assert sel.method in (JN, BND)
    sel2 = lib.apsp_select(g.n, g.row_ptr, g.col, g.w)
    assert sel2.candidates == bits(JN) and sel2.method == JN


def test_select_f32_negative_weights_is_fw(lib):
    g = gg.erdos_renyi(512, 4096, seed=3, dtype="f32")
    w = g.w.copy()
    w[::7] -= 2.0  # some negative arcs; Johnson takes fp32 weights >= 0 only (DESIGN R19)
    sel = lib.apsp_select(g.n, g.row_ptr, g.col, w)
    assert sel.candidates == bits(FW) and sel.method == FW


def test_select_rejects_bad_partition(lib):
    g = gg.grid_2d(8, 8, seed=1)
    with pytest.raises(lib.ApspError):
        lib.apsp_select(g.n, g.row_ptr, g.col, g.w, np.full(g.n, 5, np.int32), 2)
