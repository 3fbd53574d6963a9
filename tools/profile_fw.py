#!/usr/bin/env python
"""One apsp_fw_blocked on a BASELINE workload, for ncu captures (no timing here).

    ncu --set full -k regex:fw_dataflow --launch-skip 1 -c 1 -o gpurun_out/df python tools/profile_fw.py
    python tools/profile_fw.py --workload cfg2_grid16384 --runs 2 [--legacy] [--packed16]
"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import graphgen as gg  # noqa: E402
import paper_conf_ipps_xia0ar22_b200 as apsp  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="cfg2_grid16384")
    ap.add_argument("--runs", type=int, default=2)
    ap.add_argument("--legacy", action="store_true")
    ap.add_argument("--packed16", action="store_true")
    ap.add_argument("--df-delay", type=int, default=0)
    ap.add_argument("--ooc-block", type=int, default=0, help="> 0: out-of-core path with this band height")
    ap.add_argument("--er", type=int, default=0, help="> 0: seeded ER graph with this n instead of --workload")
    ap.add_argument("--deg", type=int, default=16)
    ap.add_argument("--dtype", default="i32", choices=["i32", "f32"])
    ap.add_argument("--dataflow", action="store_true", help="force the dataflow kernel (fp32 default is per-phase)")
    a = ap.parse_args()
    g = gg.erdos_renyi(a.er, a.deg * a.er, seed=4, dtype=a.dtype) if a.er else gg.baseline_config(a.workload)
    cfg = apsp.apsp_config_default(device=0)
    cfg.schedule = 1 if a.legacy else (2 if a.dataflow else 0)
    cfg.dataflow_delay = a.df_delay
    cfg.packed16 = 1 if a.packed16 else 0
    if a.ooc_block:
        cfg.force_out_of_core = 1
        cfg.ooc_block = a.ooc_block
    with apsp.apsp_init_from_csr(g.n, g.row_ptr, g.col, g.w, cfg=cfg) as h:
        for _ in range(a.runs):
            apsp.apsp_reinit(h)
            apsp.apsp_fw_blocked(h)
    print("done", a.workload, a.runs)


if __name__ == "__main__":
    main()
