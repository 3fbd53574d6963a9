#!/usr/bin/env python
"""Throughput of the sharded dataflow kernel run as P virtual ranks on one GPU (one launch,
CTA b serves rank b % P) vs the single-GPU dataflow kernel and the launch-per-phase sharded
schedule, same graph: the cost of the shard protocol (peer stores of the pivot panels,
per-rank queues, system-scope flags) without NVLink.

    python tools/vr_bench.py --n 16384 --worlds 1 2 4 8
"""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import graphgen as gg  # noqa: E402
import paper_conf_ipps_xia0ar22_b200 as apsp  # noqa: E402


def timed(g, runs, **kw):
    c = apsp.apsp_config_default(device=0)
    for k, v in kw.items():
        setattr(c, k, v)
    with apsp.apsp_init_from_csr(g.n, g.row_ptr, g.col, g.w, cfg=c) as h:
        best = 1e30
        for r in range(runs + 1):
            apsp.apsp_reinit(h)
            t0 = time.perf_counter()
            apsp.apsp_fw_blocked(h)
            if r:
                best = min(best, time.perf_counter() - t0)
    return best


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=16384)
    ap.add_argument("--worlds", type=int, nargs="+", default=[1, 2, 4, 8])
    ap.add_argument("--runs", type=int, default=2)
    ap.add_argument("--delays", type=int, nargs="+", default=[0], help="queue delays (dataflow_delay; 0 = auto)")
    a = ap.parse_args()
    g = gg.erdos_renyi(a.n, 8 * a.n, seed=4)
    out = {"n": a.n}
    for w in a.worlds:
        if w == 1:
            t = timed(g, a.runs)
            out["single_gpu_dataflow"] = {"s": t, "relax_per_s": a.n ** 3 / t}
            continue
        tp = timed(g, a.runs, world_size=w, virtual_ranks=1, schedule=1)
        out["virtual_%d" % w] = {"per_phase_bcast_s": tp, "per_phase_relax_per_s": a.n ** 3 / tp}
        for d in a.delays:
            t = timed(g, a.runs, world_size=w, virtual_ranks=1, schedule=2, dataflow_delay=d)
            out["virtual_%d" % w]["sharded_dataflow_delay_%d" % d] = {"s": t, "relax_per_s": a.n ** 3 / t}
    print(json.dumps(out), flush=True)


if __name__ == "__main__":
    main()
