"""Checkpoint / resume of the blocked FW: the state after round k is the
plain FW state with intermediates {0 .. k*b-1}; out of core, the host +
resident bands after a super-round (Algorithm 1). A run checkpointed part-way and resumed
in a fresh handle must equal the oracle bit for bit."""
import numpy as np
import pytest

import graphgen as gg
import oracle

pytestmark = pytest.mark.gpu

INF32 = 0x3FFFFFFF


def o32(d):
    return np.where(d == oracle.INF_I64, INF32, d)


def partial(g, k_iters):
    d, neg = oracle.fw_i64(g.row_ptr, g.col, g.w, k_iters=k_iters)
    assert not neg
    return o32(d)


def test_checkpoint_resume_in_core(lib, tmp_path):
    g = gg.erdos_renyi(1000, 5000, seed=41)
    path = str(tmp_path / "a.ckpt")
    with lib.apsp_init_from_csr(g.n, g.row_ptr, g.col, g.w, cfg=lib.apsp_config_default(device=0)) as h:
        lib.apsp_fw_rounds(h, 0, 3)
        lib.apsp_checkpoint(h, path)
    with lib.apsp_init_from_csr(g.n, g.row_ptr, g.col, g.w, cfg=lib.apsp_config_default(device=0)) as h:
        lib.apsp_restore(h, path)
        assert np.array_equal(lib.apsp_get_dist(h).astype(np.int64), partial(g, 3 * 128))
        lib.apsp_fw_blocked(h)  # the remaining rounds
        got = lib.apsp_get_dist(h)
    assert np.array_equal(got.astype(np.int64), partial(g, None))


def test_checkpoint_resume_out_of_core(lib, tmp_path):
    """Forced out of core, B = 256 (2 rounds per super-round), every band streamed."""
    g = gg.grid_2d(25, 40, seed=42)
    path = str(tmp_path / "o.ckpt")

    def cfg():
        c = lib.apsp_config_default(device=0, force_out_of_core=1, ooc_block=256)
        c.ooc_stream_all = 1
        return c
    with lib.apsp_init_from_csr(g.n, g.row_ptr, g.col, g.w, cfg=cfg()) as h:
        assert lib.apsp_get_info(h).mode == lib.APSP_MODE_OUT_OF_CORE
        with pytest.raises(lib.ApspError):
            lib.apsp_fw_rounds(h, 0, 1)  # not a super-round boundary
        lib.apsp_fw_rounds(h, 0, 4)       # super-rounds 0 and 1
        lib.apsp_checkpoint(h, path)
    with lib.apsp_init_from_csr(g.n, g.row_ptr, g.col, g.w, cfg=cfg()) as h:
        lib.apsp_restore(h, path)
        assert np.array_equal(lib.apsp_get_dist(h).astype(np.int64), partial(g, 512))
        lib.apsp_fw_blocked(h)
        got = lib.apsp_get_dist(h)
    assert np.array_equal(got.astype(np.int64), partial(g, None))


def test_checkpoint_out_of_core_resident_bands(lib, tmp_path):
    """Bands resident in HBM (a budget that keeps some) are saved and restored too."""
    g = gg.erdos_renyi(1536, 1536 * 6, seed=43)
    path = str(tmp_path / "r.ckpt")
    budget_mb = 18  # 6 bands of 256 rows x 1536 x 4 B = 1.5 MB each: some resident, some streamed

    def cfg():
        c = lib.apsp_config_default(device=0, force_out_of_core=1, ooc_block=256)
        c.device_budget_bytes = budget_mb << 20
        return c
    with lib.apsp_init_from_csr(g.n, g.row_ptr, g.col, g.w, cfg=cfg()) as h:
        info = lib.apsp_get_info(h)
        assert 0 < info.host_bytes < g.n * g.n * 4
        lib.apsp_fw_rounds(h, 0, 6)
        lib.apsp_checkpoint(h, path)
    with lib.apsp_init_from_csr(g.n, g.row_ptr, g.col, g.w, cfg=cfg()) as h:
        lib.apsp_restore(h, path)
        lib.apsp_fw_blocked(h)
        got = lib.apsp_get_dist(h)
    assert np.array_equal(got.astype(np.int64), partial(g, None))


def test_checkpoint_f32_and_negative_weights(lib, tmp_path):
    gf = gg.erdos_renyi(700, 700 * 8, seed=44, dtype="f32")
    # fp32 rounding depends on the round depth b: compare with an uninterrupted b = 128 run
    # (n = 700 would default to the 64-tile small-n kernel)
    straight = lib.solve(gf, cfg=lib.apsp_config_default(schedule=lib.APSP_SCHED_PER_PHASE))
    path = str(tmp_path / "f.ckpt")
    with lib.apsp_init_from_csr(gf.n, gf.row_ptr, gf.col, gf.w) as h:
        lib.apsp_fw_rounds(h, 0, 2)
        lib.apsp_checkpoint(h, path)
    with lib.apsp_init_from_csr(gf.n, gf.row_ptr, gf.col, gf.w) as h:
        lib.apsp_restore(h, path)
        lib.apsp_fw_blocked(h)
        assert np.array_equal(lib.apsp_get_dist(h), straight)
    g = gg.grid_2d(20, 30, seed=45)
    rng = np.random.default_rng(9)
    p = rng.integers(-200, 200, size=g.n)
    s, t, w = g.arcs()
    gn = gg.csr_from_arcs(g.n, s, t, (w.astype(np.int64) + p[s] - p[t]).astype(np.int32))
    with lib.apsp_init_from_csr(gn.n, gn.row_ptr, gn.col, gn.w) as h:
        lib.apsp_fw_rounds(h, 0, 1)
        lib.apsp_checkpoint(h, path)
    with lib.apsp_init_from_csr(gn.n, gn.row_ptr, gn.col, gn.w) as h:
        lib.apsp_restore(h, path)
        lib.apsp_fw_blocked(h)
        assert np.array_equal(lib.apsp_get_dist(h).astype(np.int64), partial(gn, None))


def test_restore_rejects_mismatch(lib, tmp_path):
    g = gg.erdos_renyi(300, 1500, seed=46)
    path = str(tmp_path / "m.ckpt")
    with lib.apsp_init_from_csr(g.n, g.row_ptr, g.col, g.w) as h:
        lib.apsp_checkpoint(h, path)
    g2 = gg.erdos_renyi(400, 1500, seed=46)
    with lib.apsp_init_from_csr(g2.n, g2.row_ptr, g2.col, g2.w) as h:
        with pytest.raises(lib.ApspError):
            lib.apsp_restore(h, path)
    junk = tmp_path / "junk.ckpt"
    junk.write_bytes(b"x" * 200)
    with lib.apsp_init_from_csr(g.n, g.row_ptr, g.col, g.w) as h:
        with pytest.raises(lib.ApspError):
            lib.apsp_restore(h, str(junk))
        with pytest.raises(lib.ApspError):
            lib.apsp_restore(h, str(tmp_path / "missing.ckpt"))


@pytest.mark.parametrize("ooc", [False, True])
def test_checkpoint_carries_negative_cycle_flag(lib, tmp_path, ooc):
    """A cycle inside tile 0 is flagged by phase 1 of round 0 only (R6: the round of its
    largest vertex); later rounds never look again. A run checkpointed after round 1 and
    resumed in a fresh handle must still report the cycle (the flag is saved)."""
    g0 = gg.erdos_renyi(400, 2400, seed=47)
    s, t, w = g0.arcs()
    s = np.concatenate([s, [3, 5]])
    t = np.concatenate([t, [5, 3]])
    w = np.concatenate([w, [-5, 2]]).astype(np.int32)
    g = gg.csr_from_arcs(g0.n, s, t, w)
    _, neg = oracle.fw_i64(g.row_ptr, g.col, g.w)
    assert neg
    path = str(tmp_path / "neg.ckpt")

    def cfg():
        c = lib.apsp_config_default(device=0)
        if ooc:
            c.force_out_of_core = 1
            c.ooc_block = 128
        return c

    with lib.apsp_init_from_csr(g.n, g.row_ptr, g.col, g.w, cfg=cfg()) as h:
        try:
            lib.apsp_fw_rounds(h, 0, 2)
        except lib.NegativeCycleError:
            pass
        lib.apsp_checkpoint(h, path)
    with lib.apsp_init_from_csr(g.n, g.row_ptr, g.col, g.w, cfg=cfg()) as h:
        lib.apsp_restore(h, path)
        with pytest.raises(lib.NegativeCycleError):
            lib.apsp_fw_blocked(h)
