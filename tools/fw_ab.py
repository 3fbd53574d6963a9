#!/usr/bin/env python
"""A/B of the in-core FW schedules on a seeded ER graph: the persistent dataflow kernel vs the
launch-per-phase schedule (apsp_config.schedule = 1), int32 or fp32.

    python tools/fw_ab.py --n 32768 --deg 256 --dtype f32 --runs 2
    python tools/fw_ab.py --n 1024 --deg 8 --dtype i32 --runs 20 --modes small dataflow per_phase
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


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=32768)
    ap.add_argument("--deg", type=int, default=256)
    ap.add_argument("--dtype", default="f32", choices=["i32", "f32"])
    ap.add_argument("--runs", type=int, default=2)
    ap.add_argument("--modes", nargs="+", default=["dataflow", "per_phase"])
    ap.add_argument("--packed16", action="store_true", help="int32 input solved on the packed int16 path")
    ap.add_argument("--exact-f32", action="store_true", help="int32 input closed by the fp32 engine (R25)")
    ap.add_argument("--delay", type=int, default=0, help="apsp_config.dataflow_delay (0 = auto)")
    a = ap.parse_args()
    g = gg.erdos_renyi(a.n, a.deg * a.n, seed=4, dtype=a.dtype)
    out = {"n": a.n, "deg": a.deg, "dtype": a.dtype, "packed16": a.packed16}
    for name, legacy in (("dataflow", 2), ("per_phase", 1), ("small", 3), ("auto", 0)):
        if name not in a.modes:
            continue
        cfg = apsp.apsp_config_default(device=0, timing=1, packed16=int(a.packed16), exact_f32=int(a.exact_f32))
        cfg.schedule = legacy
        cfg.dataflow_delay = a.delay
        with apsp.apsp_init_from_csr(g.n, g.row_ptr, g.col, g.w, cfg=cfg) as h:
            best, best_dev = 1e30, 1e30
            for r in range(a.runs + 1):
                apsp.apsp_reinit(h)
                t0 = time.perf_counter()
                apsp.apsp_fw_blocked(h)
                t = time.perf_counter() - t0
                st = apsp.apsp_get_phase_stats(h)
                if r:
                    best = min(best, t)
                    best_dev = min(best_dev, sum(st.ms[:4]) * 1e-3)
            arith = apsp.ARITH_NAMES[apsp.apsp_get_info(h).arith]
        out[name] = {"s": best, "relax_per_s": float(a.n) ** 3 / best, "device_s": best_dev,
                     "device_relax_per_s": float(a.n) ** 3 / best_dev,
                     "phase3_rate": st.relax[2] / (st.ms[2] * 1e-3) if st.ms[2] else None, "arith": arith}
    print(json.dumps(out), flush=True)


if __name__ == "__main__":
    main()
