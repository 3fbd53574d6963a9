"""Caller-owned device memory (apsp_config.dist_device): torch allocates the
distance matrix and the library computes into it (north star: PyTorch supplies device
memory). The result is read both through apsp_get_dist and straight from the torch tensor
(row-major, ld = n_pad), bit-exact against the oracle; the buffer outlives the handle."""
import numpy as np
import pytest

import graphgen as gg
import oracle

pytestmark = pytest.mark.gpu

INF32 = 0x3FFFFFFF


def want_i32(g):
    d, _ = oracle.fw_i64(g.row_ptr, g.col, g.w)
    return np.where(d == oracle.INF_I64, INF32, d)


@pytest.mark.parametrize("packed16,sched", [(0, 0), (0, 1), (1, 0)], ids=["dataflow", "per_phase", "packed16"])
def test_torch_owned_matrix(lib, packed16, sched):
    import torch
    g = gg.erdos_renyi(700, 4200, seed=17)
    need = lib.apsp_dist_device_bytes(g.n)
    n_pad, _, _ = lib.apsp_partition(g.n, 1, 0)
    buf = torch.full((need // 4,), -7, dtype=torch.int32, device="cuda:0")
    cfg = lib.apsp_config_default(device=0, dist_device=buf.data_ptr(), dist_device_bytes=need,
                                  packed16=packed16, schedule=sched)
    with lib.apsp_init_from_csr(g.n, g.row_ptr, g.col, g.w, cfg=cfg) as h:
        info = lib.apsp_get_info(h)
        assert info.device_bytes < need  # the matrix is not the library's
        lib.apsp_fw_blocked(h)
        got = lib.apsp_get_dist(h)
        arith = lib.apsp_get_info(h).arith
    want = want_i32(g)
    assert np.array_equal(got.astype(np.int64), want)
    torch.cuda.synchronize()
    if arith == lib.APSP_ARITH_I32:  # the int32 matrix lives in the caller's buffer
        m = buf.view(n_pad, n_pad)[:g.n, :g.n].cpu().numpy()
        assert np.array_equal(m.astype(np.int64), want)
    else:  # packed16: int16 working matrix in the first half of the buffer (R16, INF16 = 16383)
        m = buf.view(torch.int16)[:n_pad * n_pad].view(n_pad, n_pad)[:g.n, :g.n].cpu().numpy().astype(np.int64)
        assert np.array_equal(np.where(m >= 16383, INF32, m), want)


def test_torch_owned_matrix_int32_fallback(lib):
    """packed16 with distances >= 8192: the int32 redo reuses the caller's whole buffer."""
    import torch
    g = gg.weighted_path(np.full(299, 100))
    need = lib.apsp_dist_device_bytes(g.n)
    buf = torch.zeros((need // 4,), dtype=torch.int32, device="cuda:0")
    cfg = lib.apsp_config_default(device=0, dist_device=buf.data_ptr(), dist_device_bytes=need, packed16=1)
    with lib.apsp_init_from_csr(g.n, g.row_ptr, g.col, g.w, cfg=cfg) as h:
        lib.apsp_fw_blocked(h)
        assert lib.apsp_get_info(h).arith == lib.APSP_ARITH_I32
        got = lib.apsp_get_dist(h)
    assert np.array_equal(got.astype(np.int64), want_i32(g))


def test_torch_owned_matrix_virtual_ranks(lib):
    import torch
    g = gg.grid_2d(20, 30, seed=5)
    need = lib.apsp_dist_device_bytes(g.n, 4, 1)
    buf = torch.zeros((need // 4,), dtype=torch.int32, device="cuda:0")
    cfg = lib.apsp_config_default(device=0, world_size=4, virtual_ranks=1, dist_device=buf.data_ptr(),
                                  dist_device_bytes=need)
    assert np.array_equal(lib.solve(g, cfg=cfg).astype(np.int64), want_i32(g))
