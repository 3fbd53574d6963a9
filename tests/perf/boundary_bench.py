#!/usr/bin/env python
"""Boundary algorithm vs blocked FW on a small-separator graph, plus the paper-style
multi-core CPU APSP comparator (BGL-Plus = parallel Dijkstra per source;
here the oracle's OpenMP Dijkstra rows, timed on a sample of sources and extrapolated,
the paper's own sampling method).

    python tests/perf/boundary_bench.py [--workload cfg2_grid16384] [--blocks 4 8] [--steps 5]
        [--force-ooc] [--budget-gb G] [--certify]

Out of core (the result does not fit the device budget, or --force-ooc): Algorithm 3's
batched, double-buffered D2H of N_row block rows is inside every timed solve
(P:531); the line then reports the host-link traffic and its fraction of the measured
pinned D2H rate (MEASURED_DPX.json host_link_gbs). --certify reads every row back through
apsp_get_dist and proves it with the oracle's optimality certificate.

Prints one JSON line. The boundary algorithm does far fewer than n^3 relaxations, so its
rate is reported as time (and as n^3/time "FW-equivalent" for comparison only).
"""
import argparse
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)

import graphgen as gg  # noqa: E402
import oracle  # noqa: E402
import paper_conf_ipps_xia0ar22_b200 as apsp  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="cfg2_grid16384")
    ap.add_argument("--blocks", type=int, nargs=2, default=[4, 8])
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--cpu-sources", type=int, default=512)
    ap.add_argument("--no-fw", action="store_true")
    ap.add_argument("--force-ooc", action="store_true")
    ap.add_argument("--budget-gb", type=float, default=0.0)
    ap.add_argument("--certify", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    a = ap.parse_args()
    import torch
    torch.cuda.set_device(0)
    stream = torch.cuda.current_stream()
    g = gg.baseline_config(a.workload)
    n = g.n
    comp, k = gg.grid_block_partition(g, *a.blocks)

    def timed(make, run, bnd=False, keep=False):
        cfg = apsp.apsp_config_default(device=0, timing=1)
        cfg.stream = stream.cuda_stream
        if bnd:
            cfg.force_out_of_core = int(a.force_ooc)
            cfg.device_budget_bytes = int(a.budget_gb * 2 ** 30)
        t_init = time.time()
        h = make(cfg)
        t_init = time.time() - t_init
        for _ in range(a.warmup):
            apsp.apsp_reinit(h)
            run(h)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for _ in range(a.steps):
            apsp.apsp_reinit(h)
            run(h)
        e1.record(stream)
        torch.cuda.synchronize()
        st = apsp.apsp_get_phase_stats(h)
        info = apsp.apsp_get_info(h)
        if keep:
            return e0.elapsed_time(e1) / a.steps, st, info, t_init, h
        apsp.apsp_destroy(h)
        return e0.elapsed_time(e1) / a.steps, st, info, t_init

    ms_b, st_b, info_b, init_b, hb = timed(
        lambda c: apsp.apsp_init_boundary(n, g.row_ptr, g.col, g.w, comp, k, cfg=c), apsp.apsp_solve, True, True)
    relax_b = sum(st_b.relax[:3])
    out = {"workload": a.workload, "n": n, "n_pad": info_b.n_pad, "k": k, "boundary_nodes": info_b.boundary_nodes,
           "steps": a.steps, "warmup": a.warmup,
           "boundary_ms": ms_b, "boundary_relaxations": relax_b,
           "boundary_relax_per_s": relax_b / (ms_b * 1e-3), "init_s": init_b,
           "boundary_phase_ms_last_run": list(st_b.ms), "fw_equivalent_n3_per_s": float(n) ** 3 / (ms_b * 1e-3),
           "out_of_core": info_b.ooc_block > 0, "device_bytes": info_b.device_bytes}
    if info_b.ooc_block > 0:
        link = info_b.host_bytes  # every streamed block row crosses the link once per solve
        dpx = json.load(open(os.path.join(ROOT, "MEASURED_DPX.json")))
        peak = dpx["host_link_gbs"]["d2h"]
        out["ooc"] = {"buffer_rows": info_b.ooc_block, "host_bytes_streamed_per_solve": link,
                      "resident_fraction": 1.0 - link / (float(info_b.n_pad) ** 2 * 4),
                      "link_gbs": link / (ms_b * 1e-3) / 1e9, "link_peak_gbs": peak,
                      "link_frac": link / (ms_b * 1e-3) / 1e9 / peak,
                      "link_peak_source": "MEASURED_DPX.json host_link_gbs.d2h (pinned, 1 GiB copies)",
                      "note": "Alg. 3 l.20 with P:184-197: two device buffers of N_row block rows on two streams "
                              "alternate into pinned host memory; block rows left over memory allows stay resident "
                              "(DESIGN.md R21)"}
    if a.certify:
        t0 = time.time()
        bad = 0
        for r0 in range(0, n, 4096):
            rows = apsp.apsp_get_dist(hb, r0, min(4096, n - r0))
            bad += oracle.certify_rows_i32(g.row_ptr, g.col, g.w, r0, rows, 0x3FFFFFFF)[0]
        out["certified_rows"] = n
        out["certificate_failures"] = bad
        out["certify_s"] = time.time() - t0
    apsp.apsp_destroy(hb)
    if a.workload == "cfg5_grid262144":
        try:
            r = json.load(open(os.path.join(ROOT, "profiles", "r01_cfg5_ooc_262144.json")))
            out["fw_out_of_core_s_r01"] = r["t_fw_s"]
            out["fw_out_of_core_source"] = ("profiles/r01_cfg5_ooc_262144.json (blocked FW out of core on the "
                                            "same graph, round 1, 40 of 64 bands resident)")
            out["boundary_speedup_vs_fw_out_of_core"] = r["t_fw_s"] / (ms_b * 1e-3)
        except Exception:
            pass
    if not a.no_fw:
        ms_f, _, _, _ = timed(lambda c: apsp.apsp_init_from_csr(n, g.row_ptr, g.col, g.w, cfg=c), apsp.apsp_fw_blocked)
        out["fw_ms"] = ms_f
        out["boundary_speedup_vs_fw"] = ms_f / ms_b
    if a.no_cpu:
        print(json.dumps(out), flush=True)
        return
    # paper-style multi-core CPU APSP (Dijkstra per source, all host cores), sampled
    rng = np.random.default_rng(0)
    srcs = rng.choice(n, size=min(n, a.cpu_sources), replace=False)
    t0 = time.time()
    oracle.dijkstra_rows_i64(g.row_ptr, g.col, g.w, srcs)
    t = time.time() - t0
    cpu_s = t * n / len(srcs)
    out["cpu_dijkstra_apsp_s_extrapolated"] = cpu_s
    out["cpu_cores"] = oracle.threads()
    out["cpu_sample"] = "%d random sources of %d, %.2f s" % (len(srcs), n, t)
    out["boundary_speedup_vs_cpu_dijkstra"] = cpu_s / (ms_b * 1e-3)
    out["paper_context"] = ("boundary algorithm vs BGL-Plus: 8.22-12.40x on 1x V100 vs 14-core Xeon E5-2680 "
                            "(PAPER.md:531; abstract P:25 says 8.82), transfers included")
    print(json.dumps(out), flush=True)


if __name__ == "__main__":
    main()
