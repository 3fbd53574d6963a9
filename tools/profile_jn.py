#!/usr/bin/env python
"""One Johnson apsp_solve (batched Near-Far, Alg. 2) on a BASELINE workload, for
ncu captures (no timing here).

    ncu --set full -k regex:mssp --launch-skip 1 -c 1 -o gpurun_out/jn python tools/profile_jn.py
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
    a = ap.parse_args()
    g = gg.baseline_config(a.workload)
    with apsp.apsp_init_johnson(g.n, g.row_ptr, g.col, g.w, cfg=apsp.apsp_config_default(device=0)) as h:
        for r in range(a.runs):
            if r:
                apsp.apsp_reinit(h)
            apsp.apsp_solve(h)
        print("edges scanned per run", apsp.apsp_get_info(h).edges_scanned)


if __name__ == "__main__":
    main()
