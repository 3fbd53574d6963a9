#!/usr/bin/env python
"""Tiny runs of every kernel family through the C ABI, for compute-sanitizer
(memcheck / racecheck / synccheck / initcheck; tools/gpu_sanitize.sh). No oracle here
(tools/ do not import it): each case compares two product paths that must agree
bit for bit (dataflow vs launch-per-phase, async vs blocking, ...).

    compute-sanitizer --tool memcheck python tools/san_case.py
"""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import graphgen as gg  # noqa: E402
import paper_conf_ipps_xia0ar22_b200 as apsp  # noqa: E402


def run(g, **kw):
    c = apsp.apsp_config_default(device=0)
    for k, v in kw.items():
        setattr(c, k, v)
    with apsp.apsp_init_from_csr(g.n, g.row_ptr, g.col, g.w, cfg=c) as h:
        apsp.apsp_fw_blocked(h)
        return apsp.apsp_get_dist(h)


def same(a, b, what):
    assert np.array_equal(a, b), what
    print("ok", what, flush=True)


def main():
    n = int(os.environ.get("SAN_N", "300"))
    only = os.environ.get("SAN_CASES", "")  # comma-separated case names; empty = all
    want = lambda c: not only or c in only.split(",")  # noqa: E731
    g = gg.erdos_renyi(n, 5 * n, seed=1)
    gf = gg.erdos_renyi(n, 5 * n, seed=2, dtype="f32")
    gb = gg.erdos_renyi(512, 2500, seed=3)
    p = np.random.default_rng(4).integers(0, 30, n)
    s, t, w = g.arcs()
    gn = gg.csr_from_arcs(n, s, t, (w + p[s] - p[t]).astype(np.int32))
    if want("dataflow"):
        same(run(g), run(g, schedule=1), "int32 dataflow vs per-phase")
        same(run(gf, schedule=2), run(gf, schedule=1), "fp32 dataflow vs per-phase")
        same(run(g, packed16=1), run(g, packed16=1, schedule=1), "packed16 dataflow vs per-phase")
    if want("barrier"):  # per-phase kernels with CTA barriers only (minplus_variant = 1: no mbarriers)
        same(run(g, minplus_variant=1, schedule=1), run(g, minplus_variant=1, schedule=1, packed16=1), "int32 vs packed16, per-phase CTA-barrier kernels")
        same(run(gf, minplus_variant=1, schedule=1), run(gf, minplus_variant=1, schedule=1, world_size=2, virtual_ranks=1), "fp32 per-phase, 1 vs 2 virtual ranks")
        same(run(g, packed16=1, schedule=1), run(g, minplus_variant=1, schedule=1), "packed16 per-phase vs int32")
        same(run(gn, minplus_variant=1, schedule=1), run(gn, minplus_variant=1, schedule=1, world_size=2, virtual_ranks=1), "negative weights, 1 vs 2 virtual ranks")
    if want("ooc"):
        same(run(gb, force_out_of_core=1, ooc_block=256, minplus_variant=1), run(gb, minplus_variant=1, schedule=1), "out of core vs in core")
        same(run(gb, world_size=2, virtual_ranks=1, minplus_variant=1), run(gb, minplus_variant=1, schedule=1), "2 virtual ranks vs 1 GPU")
    if want("small"):  # 64-tile kernel: split chain panel tiles, flags re-zeroed by the last CTA between runs
        with apsp.apsp_init_from_csr(n, g.row_ptr, g.col, g.w, cfg=apsp.apsp_config_default(device=0)) as h:
            for _ in range(2):
                apsp.apsp_reinit(h)
                apsp.apsp_fw_blocked(h)
                same(apsp.apsp_get_dist(h), run(g, schedule=1), "small kernel (split parts), repeated run")
    if want("exact"):  # R25: int32 in fp32 arithmetic (128-tile dataflow kernel: n_pad > 2048)
        gx = gg.erdos_renyi(2100, 8400, seed=6)
        same(run(gx, exact_f32=1), run(gx, schedule=1), "exact_f32 vs int32 per-phase")
    if want("neg"):
        same(run(gn), run(gn, schedule=1), "negative weights (canonicalize)")
    if want("johnson"):
        with apsp.apsp_init_johnson(n, g.row_ptr, g.col, g.w) as h:
            apsp.apsp_solve(h)
            dj = apsp.apsp_get_dist(h)
        same(dj, run(g, minplus_variant=1, schedule=1), "Johnson vs blocked FW")
    if want("boundary"):
        gg2 = gg.grid_2d(16, 16, seed=5, permute=False)
        comp, k = gg.grid_block_partition(gg2, 2, 2)
        with apsp.apsp_init_boundary(gg2.n, gg2.row_ptr, gg2.col, gg2.w, comp, k) as h:
            apsp.apsp_solve(h)
            db = apsp.apsp_get_dist(h)
        same(db, run(gg2, minplus_variant=1, schedule=1), "boundary vs blocked FW")
    if want("async"):
        import torch
        out = torch.empty((n, n), dtype=torch.int32, pin_memory=True)
        with apsp.apsp_init_from_csr(n, g.row_ptr, g.col, g.w) as h:
            apsp.apsp_load_csr(h, gn.row_ptr, gn.col, gn.w)
            apsp.apsp_fw_blocked_async(h)
            apsp.apsp_get_dist_async(h, 0, n, out.data_ptr(), n)
            apsp.apsp_synchronize(h)
        same(out.numpy(), run(gn, schedule=1), "load_csr + async vs blocking")
    print("san_case done", flush=True)


if __name__ == "__main__":
    main()
