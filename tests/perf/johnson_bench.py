#!/usr/bin/env python
"""Johnson's algorithm (batched Near-Far SSSP, Algorithm 2) vs the blocked
FW on the same graph, plus the paper-style multi-core CPU APSP comparator (PAPER.md:531:
parallel Dijkstra per source; here the oracle's OpenMP Dijkstra rows on a sample of sources,
extrapolated — the paper's own sampling method).

    python tests/perf/johnson_bench.py [--workload cfg2_grid16384] [--deltas 0 100 400] [--steps 3]

Prints one JSON line per workload. Johnson does O(n * m * re-expansions) work instead of n^3,
so its rate is reported as arcs relaxed per second (and n^3/time "FW-equivalent", for
comparison only). The paper reports 2.23-2.79x for its out-of-core Johnson over a multi-core
APSP on "other sparse" graphs (abstract) on a V100.
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
    ap.add_argument("--workload", nargs="+", default=["cfg2_grid16384"])
    ap.add_argument("--deltas", type=float, nargs="+", default=[0.0])
    ap.add_argument("--steps", type=int, default=3)
    ap.add_argument("--warmup", type=int, default=1)
    ap.add_argument("--cpu-sources", type=int, default=512)
    ap.add_argument("--fw", action="store_true", help="also time the blocked FW on the same graph")
    ap.add_argument("--ooc", action="store_true", help="force Algorithm 2's batches to pinned host memory")
    ap.add_argument("--env", nargs="+", default=[""],
                    help="kernel variants to sweep, e.g. 'APSP_JN_THREADS=512,APSP_JN_SMEM_DIST=0'")
    a = ap.parse_args()
    import torch
    torch.cuda.set_device(0)
    stream = torch.cuda.current_stream()
    for wl in a.workload:
        g = gg.baseline_config(wl)
        n = g.n

        def timed(make, run):
            cfg = apsp.apsp_config_default(device=0, timing=1, force_out_of_core=1 if a.ooc else 0)
            cfg.stream = stream.cuda_stream
            h = make(cfg)
            for _ in range(a.warmup):
                apsp.apsp_reinit(h)
                run(h)
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            t0 = time.perf_counter()
            e0.record(stream)
            for _ in range(a.steps):
                apsp.apsp_reinit(h)
                run(h)
            e1.record(stream)
            torch.cuda.synchronize()
            wall = (time.perf_counter() - t0) / a.steps
            st = apsp.apsp_get_phase_stats(h)
            info = apsp.apsp_get_info(h)
            apsp.apsp_destroy(h)
            return e0.elapsed_time(e1) / a.steps, wall * 1e3, st, info

        out = {"workload": wl, "n": n, "m": g.m, "runs": []}
        variants = [(d, e) for e in a.env for d in a.deltas]
        for d, env in variants:
            for k in ("APSP_JN_THREADS", "APSP_JN_SMEM_DIST", "APSP_JN_CTAS_PER_SM"):
                os.environ.pop(k, None)
            for kv in filter(None, env.split(",")):
                k, v = kv.split("=")
                os.environ[k] = v
            ms, wall_ms, st, info = timed(
                lambda c: apsp.apsp_init_johnson(n, g.row_ptr, g.col, g.w, delta=d, cfg=c), apsp.apsp_solve)
            # the library synchronises inside apsp_solve, so wall time is the honest one
            t = max(ms, wall_ms)
            out["runs"].append({"delta": d, "env": env, "ms": t, "kernel_ms": st.ms[2], "reweight_ms": st.ms[1],
                                "d2h_ms": st.ms[3], "edges_scanned": info.edges_scanned,
                                "edges_per_source": info.edges_scanned / n, "reexpansion": info.edges_scanned / n / g.m,
                                "arcs_per_s": info.edges_scanned / (t * 1e-3),
                                "fw_equivalent_n3_per_s": float(n) ** 3 / (t * 1e-3),
                                "result_bytes": n * n * 4, "host_bytes": info.host_bytes})
        for k in ("APSP_JN_THREADS", "APSP_JN_SMEM_DIST", "APSP_JN_CTAS_PER_SM"):
            os.environ.pop(k, None)
        best = min(out["runs"], key=lambda r: r["ms"])
        out["best"] = {"delta": best["delta"], "env": best["env"]}
        out["best_ms"] = best["ms"]
        if a.fw:
            ms_f, wall_f, _, _ = timed(lambda c: apsp.apsp_init_from_csr(n, g.row_ptr, g.col, g.w, cfg=c),
                                       apsp.apsp_fw_blocked)
            out["fw_ms"] = max(ms_f, wall_f)
            out["johnson_speedup_vs_fw"] = out["fw_ms"] / best["ms"]
        rng = np.random.default_rng(0)
        srcs = rng.choice(n, size=min(n, a.cpu_sources), replace=False)
        t0 = time.time()
        oracle.dijkstra_rows_i64(g.row_ptr, g.col, g.w, srcs)
        tc = time.time() - t0
        cpu_s = tc * n / len(srcs)
        out["cpu_dijkstra_apsp_s_extrapolated"] = cpu_s
        out["cpu_cores"] = oracle.threads()
        out["cpu_sample"] = "%d random sources of %d, %.2f s" % (len(srcs), n, tc)
        out["johnson_speedup_vs_cpu_dijkstra"] = cpu_s / (best["ms"] * 1e-3)
        out["paper_context"] = ("out-of-core Johnson vs a multi-core APSP: 2.23-2.79x on 1x V100 vs a 14-core "
                                "Xeon E5-2680 for 'other sparse' graphs (PAPER.md:25, :531)")
        print(json.dumps(out), flush=True)


if __name__ == "__main__":
    main()
