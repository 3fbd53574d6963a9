#!/usr/bin/env python
"""Benchmark: blocked Floyd–Warshall APSP on B200 through the C ABI.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference] [--workload NAME]

Metric (BASELINE.json): APSP relaxations/s = n^3 / time (whole job, all ranks).
One step = one pass of the whole hot path over the workload's graph with the
CSR already resident in HBM: CSR->dense init (apsp_reinit) + all n/b rounds of
phases 1-3 (apsp_fw_blocked; with N>1 ranks also the NCCL pivot-band broadcast).

Default workload at EVERY N: cfg3_er65536 (BASELINE.json configs[2], the config the metric
"relaxations/s at 1/2/4/8 B200" is quoted on: n=65536, 17.2 GB, fits one GPU), sharded 1-D
block-row over N GPUs for N > 1: the total work is fixed, so scaling is "strong".
Inputs are larger than L2 (n^2*4 B = 17.2 GB > 126 MB), so no explicit flush.

Launch: `python bench.py --gpus N` without torchrun re-executes itself under
`python -m torch.distributed.run --nproc-per-node N --master-addr 127.0.0.1`; under
torchrun (WORLD_SIZE set) every rank runs directly.

Legs beside the headline on one GPU (each guarded; skip flags --no-packed16, --no-exact-f32-leg,
--no-ooc-leg, --no-boundary-leg, --no-johnson): packed16 (R16), exact_f32 (R25: the int32 graph
closed by the fp32 engine under the 2(n-1)W <= 2^24 bound), the same workload fully out of core
(N = 1; --ooc-leg-multi at N > 1),
the boundary algorithm on a grid of the same n, Johnson's algorithm.

`--impl reference` times the CPU oracle (oracle/, plain C + OpenMP) on a bounded
sample of the same workload (the reference arm of this paper-only tier).
"""
from __future__ import annotations

import argparse
import ctypes
import json
import os
import subprocess
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "APSP relaxations/s (n^3/time) at 1/2/4/8 B200; % of DPX min-plus peak"
UNIT = "relax/s"


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--workload", default=None)
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--force-ooc", action="store_true", help="use the out-of-core path (experiments)")
    ap.add_argument("--ooc-block", type=int, default=0, help="out-of-core band height B (0 = auto)")
    ap.add_argument("--stream-all", action="store_true", help="out-of-core: keep no band resident")
    ap.add_argument("--no-lookahead", action="store_true", help="in-core: no phase-3 split / overlap")
    ap.add_argument("--sharded-dataflow", action="store_true",
                    help="N > 1: the sharded dataflow kernel (owner stores the pivot panels into every GPU's "
                         "panel buffer over NVLink) instead of the launch-per-phase schedule with NCCL broadcasts")
    ap.add_argument("--legacy", action="store_true",
                    help="single GPU: launch-per-phase schedule instead of the persistent dataflow kernel")
    ap.add_argument("--df-delay", type=int, default=0, help="dataflow kernel queue delay (0 = auto)")
    ap.add_argument("--minplus-variant", type=int, default=0,
                    help="min-plus kernel for A/B: 0 cp.async + mbarrier pipeline (default), "
                         "1 cp.async + CTA barrier per chunk, 2 TMA persistent")
    ap.add_argument("--no-packed16", action="store_true", help="skip the packed-int16 alternative measurement")
    ap.add_argument("--no-johnson", action="store_true", help="skip the Johnson (Near-Far) alternative measurement")
    ap.add_argument("--no-exact-f32-leg", action="store_true",
                    help="skip the exact-fp32 leg (int32 closed by the fp32 engine under the R25 bound)")
    ap.add_argument("--packed16", action="store_true",
                    help="packed int16 arithmetic (VIADDMNMX.S16x2) when exact, int32 otherwise")
    ap.add_argument("--cpu-seconds", type=float, default=15.0, help="target oracle sample time")
    ap.add_argument("--e2e-steps", type=int, default=0,
                    help="serving-loop e2e steps (0 = auto: K when a step is short, else min(K, 5))")
    ap.add_argument("--e2e-serial", action="store_true",
                    help="also time the blocking init + fw + get_dist + destroy sequence (e2e.serial)")
    ap.add_argument("--packed16-e2e", action="store_true", help="also time the packed16 leg end to end")
    ap.add_argument("--ooc-leg-multi", action="store_true",
                    help="also run the out-of-core leg at N > 1 (out of core x P ranks over NCCL)")
    ap.add_argument("--no-ooc-leg", action="store_true",
                    help="skip the out-of-core leg (every band streamed from pinned host memory, B = 4096)")
    ap.add_argument("--no-boundary-leg", action="store_true",
                    help="skip the boundary-algorithm leg (2-D grid of the same n, k = sqrt(n)/4, out of core)")
    ap.add_argument("--rendezvous-only", action="store_true",
                    help="launcher check: init the process group (gloo), barrier, print the rank, exit")
    return ap.parse_args()


def dist_env():
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", str(rank)))
    return world, rank, local


def default_workload(n_gpus):
    """BASELINE.json's metric is quoted "at 1/2/4/8 B200" on configs[2] (n=65536, sharded over
    1/2/4/8 B200): the same workload at every N (strong scaling)."""
    return "cfg3_er65536"


def peaks():
    """Roofline denominators: measured DPX min-plus rate (MEASURED_DPX.json, committed, from
    build/dpx_peak) and the driver's MEASURED_PEAKS.json."""
    out = {}
    p = os.path.join(ROOT, "MEASURED_DPX.json")
    if os.path.exists(p):
        out["dpx"] = json.load(open(p))
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        out["driver"] = json.load(open(p))
    return out


class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled every 200 ms during the timed region."""

    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, device):
        self.device = device
        self.proc = None

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.device), "--query-gpu=" + self.Q,
                                          "--format=csv,noheader,nounits", "-lms", "200"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except Exception:
            self.proc = None

    def stop(self):
        if self.proc is None:
            return None
        self.proc.terminate()
        try:
            out = self.proc.communicate(timeout=5)[0]
        except Exception:
            self.proc.kill()
            out = ""
        sms, mx, reasons = [], None, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for line in out.strip().splitlines():
            f = [x.strip() for x in line.split(",")]
            if len(f) < 9:
                continue
            try:
                sms.append(float(f[1]))
                mx = float(f[2])
            except ValueError:
                continue
            for nm, v in zip(names, f[5:9]):
                if v.lower() == "active":
                    reasons.add(nm)
        if not sms:
            return None
        return {"sm_mhz": float(np.median(sms)), "sm_max_mhz": mx, "reasons": sorted(reasons),
                "samples": len(sms)}


def oracle_whole_run(g, steps):
    """One complete oracle plain-FW run split into `steps` timed parts of n/steps
    outer iterations: value = n^3 / (sum of part times) is the oracle's exact whole-run rate.
    Returns (relax_per_s, secs, per-part rates)."""
    import oracle
    n = g.n
    is_f = g.w.dtype.kind == "f"
    d = oracle.init_f64(g.row_ptr, g.col, g.w) if is_f else oracle.init_i64(g.row_ptr, g.col, g.w)
    fw = oracle.fw_dense_f64 if is_f else oracle.fw_dense_i64
    secs, rates = 0.0, []
    for i in range(steps):
        k0, k1 = i * n // steps, (i + 1) * n // steps
        ts = time.time()
        fw(d, k1, k_begin=k0)
        dt = time.time() - ts
        secs += dt
        rates.append((k1 - k0) * float(n) ** 2 / max(dt, 1e-9))
    return float(n) ** 3 / secs, secs, rates


def oracle_steady_rate(g, warm_s, step_s, steps):
    """The oracle's plain FW (oracle.fw_dense_i64 / _f64 as it stands, all host cores) timed
    at its steady-state cost per outer iteration on this workload's n x n matrix.

    The oracle skips row i at iteration k while D[i][k] is still infinite (PAPER.md:60's
    infinity), so a run's first iterations are far cheaper than the rest, and any sample taken
    from the start of a run overstates the rate (5.6x at cfg2). Here the
    workload's initial matrix has every infinite entry replaced by a finite
    weight (10^12, larger than any path): no row is ever skipped, every outer iteration
    performs all n^2 relaxations, exactly the cost of the run's bulk once its distances
    have become finite. After `warm_s` of discarded iterations, `steps` equal-time samples of
    ~`step_s` each continue the run; rate = iterations * n^2 / time. This is a LOWER bound
    of the whole-run rate n^3 / T_run (a real run is faster by the share of its cheap early
    iterations: ~2x on the cfg2 grid, whose labels percolate late, a few to ~15 % on the ER
    configs). Both bench arms use this function for n > FULL_RUN_MAX_N (the repo arm's
    cpu_baseline with a shorter budget), so they agree.
    Returns (relax_per_s, cores, sample, per-step rates, ms per step)."""
    import oracle
    n = g.n
    is_f = g.w.dtype.kind == "f"
    t0 = time.time()
    d = oracle.init_f64(g.row_ptr, g.col, g.w) if is_f else oracle.init_i64(g.row_ptr, g.col, g.w)
    big = 1e12
    if is_f:
        np.copyto(d, big, where=np.isinf(d))
    else:
        np.copyto(d, int(big), where=(d == oracle.INF_I64))
    t_init = time.time() - t0
    fw = oracle.fw_dense_f64 if is_f else oracle.fw_dense_i64
    k = 0

    def run_chunk(c):
        nonlocal k
        if k + c > n:  # wrap: restart the outer loop on the (still all-finite) matrix
            k = 0
        k1 = min(n, k + c)
        ts = time.time()
        fw(d, k1, k_begin=k)
        dt = time.time() - ts
        it = k1 - k
        k = k1
        return it, dt

    tw = time.time()
    chunk, per = 1, None
    while time.time() - tw < warm_s:
        it, dt = run_chunk(chunk)
        per = dt / it
        chunk = max(1, min(chunk * 2, int(0.25 / per)))
    t_warm = time.time() - tw
    rates, times, iters = [], [], []
    for _ in range(steps):
        c = max(1, int(step_s / per))
        it, dt = run_chunk(c)
        per = dt / it
        rates.append(it * float(n) ** 2 / dt)
        times.append(dt)
        iters.append(it)
    value = sum(iters) * float(n) ** 2 / sum(times)
    sample = ("oracle plain FW (%s, OpenMP over rows, %d threads) at its steady-state cost per outer iteration: "
              "n=%d initial matrix (PAPER.md:60) with infinite entries set to 1e12 so no row is skipped (every "
              "iteration does all n^2 relaxations, as the bulk of a real run does); %.1f s warm-up discarded, then "
              "%d timed samples of %d outer iterations in total (%.1f s, per-sample rates %.3g..%.3g relax/s); a "
              "lower bound of the whole-run rate (a real run's early iterations skip rows still at infinity); "
              "init %.1f s not counted" % ("fp64" if is_f else "int64", oracle.threads(), n, t_warm, len(times),
                                           sum(iters), sum(times), min(rates), max(rates), t_init))
    return value, oracle.threads(), sample, rates, float(np.mean(times)) * 1e3


FULL_RUN_MAX_N = 16384  # reference arm: whole oracle run when n <= this (cfg1, cfg2)
CPU_BASELINE_FULL_MAX_N = 4096  # repo arm's cpu_baseline: whole run only where it takes seconds


def run_reference(args):
    world, rank, _ = dist_env()
    if rank != 0:
        return 0
    import graphgen as gg
    wl = args.workload or default_workload(args.gpus)
    g = gg.baseline_config(wl)
    import oracle
    oracle.build()
    cores = oracle.threads()
    n = g.n
    if n <= FULL_RUN_MAX_N:
        # The K timed steps together are ONE complete oracle FW run (step i = outer
        # iterations [i*n/K, (i+1)*n/K)), so value = n^3 / (sum of step times) is the
        # oracle's exact whole-run rate -- no early-iteration (INF-skip) or steady-state
        # bias. cfg2 (n=16384): ~150 s on 16 cores. Warm-up: one discarded small run.
        for i in range(min(args.warmup, 1)):
            oracle_steady_rate(g, 0.2, 0.2, 1)
        t0 = time.time()
        value, secs, rates = oracle_whole_run(g, args.steps)
        wall = time.time() - t0
        ms_step = secs / args.steps * 1e3
        is_f = g.w.dtype.kind == "f"
        sample = "the whole workload: one complete oracle plain FW run (%s, OpenMP over rows, " \
            "n=%d, %.1f s, init not counted) split into %d timed steps of n/%d outer iterations " \
            "(per-step rates %.3g..%.3g relax/s)" % ("fp64" if is_f else "int64", n, secs,
                                                     args.steps, args.steps, min(rates), max(rates))
    else:
        # Too large for one run within minutes: the steady state of one run (warm-up
        # discarded), K equal-time steps; the same function as the repo arm's cpu_baseline.
        per_step = max(2.0, min(args.cpu_seconds, 120.0 / max(1, args.steps)))
        t0 = time.time()
        value, cores, sample, rates, ms_step = oracle_steady_rate(
            g, warm_s=max(3.0, per_step * min(args.warmup, 3) / 2), step_s=per_step, steps=args.steps)
        wall = time.time() - t0
    n = g.n
    line = {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": args.gpus, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms_step, "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None,
        "dtype": "f64" if g.w.dtype.kind == "f" else "int64", "data": "synthetic",
        "config": {"workload": wl, "n": n, "m": g.m, "desc": gg.BASELINE_CONFIGS[wl]},
        "impl": "reference",
        "cpu_baseline": {"value": value, "unit": UNIT, "cores": cores, "kind": "oracle", "sample": sample},
        "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
        "wall_s": wall, "ms_whole_workload": float(n) ** 3 / value * 1e3,
    }
    print(json.dumps(line), flush=True)
    return 0


def run_ours(args):
    import torch
    import torch.distributed as dist

    import graphgen as gg
    import paper_conf_ipps_xia0ar22_b200 as apsp

    world, rank, local = dist_env()
    if world != args.gpus:
        raise SystemExit("--gpus %d but WORLD_SIZE=%d" % (args.gpus, world))
    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    wl = args.workload or default_workload(args.gpus)
    g = gg.baseline_config(wl)
    n = g.n
    is_f = g.w.dtype.kind == "f"
    stream = torch.cuda.current_stream()

    def fresh_uid():
        """A new ncclUniqueId for every handle (a communicator per handle; an id serves one
        ncclCommInitRank): rank 0 draws it, every rank receives it (collective, SPMD order)."""
        obj = [apsp.apsp_nccl_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0)
        return obj[0]

    def make_cfg(timing, packed16, ooc=False, exact_f32=False):
        cfg = apsp.apsp_config_default(device=local, world_size=world, rank=rank, timing=timing)
        cfg.stream = stream.cuda_stream
        if args.force_ooc:
            cfg.force_out_of_core = 1
            cfg.ooc_block = args.ooc_block
            if args.stream_all:
                cfg.ooc_stream_all = 1
        if ooc:  # the out-of-core leg: the paper's setting, every band streamed
            cfg.force_out_of_core = 1
            cfg.ooc_block = args.ooc_block or 4096
            cfg.ooc_stream_all = 1
        if args.no_lookahead:
            cfg.no_lookahead = 1
        cfg.minplus_variant = args.minplus_variant
        if args.legacy:
            cfg.schedule = 1
        if args.sharded_dataflow:
            cfg.schedule = 2
        cfg.dataflow_delay = args.df_delay
        if packed16:
            cfg.packed16 = 1
        if exact_f32:
            cfg.exact_f32 = 1
        if world > 1:
            cfg._uid_buf = ctypes.create_string_buffer(fresh_uid(), 128)
            cfg.nccl_unique_id = ctypes.cast(cfg._uid_buf, ctypes.c_void_p)
        return cfg

    def barrier():
        if world > 1:
            dist.barrier(device_ids=[local])

    def max_over_ranks(x):
        if world == 1:
            return x
        t = torch.tensor([x], dtype=torch.float64, device="cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    pk = peaks()

    def device_timed(packed16, steps=None, warmup=None, ooc=False, exact_f32=False):
        """W warm-up + K timed steps (apsp_reinit + apsp_fw_blocked, CSR resident in HBM),
        CUDA events on the library's stream, max over ranks; roofline of phase 3."""
        steps = args.steps if steps is None else steps
        warmup = args.warmup if warmup is None else warmup
        cfg = make_cfg(1, packed16, ooc, exact_f32)
        ooc_mode = args.force_ooc or ooc
        dist_buf = None
        if not ooc_mode:  # torch owns the distance matrix (apsp_config.dist_device)
            need = apsp.apsp_dist_device_bytes(n, world)
            dist_buf = torch.empty(need // 4, dtype=torch.int32, device="cuda")
            cfg.dist_device, cfg.dist_device_bytes = dist_buf.data_ptr(), need
        h = apsp.apsp_init_from_csr(n, g.row_ptr, g.col, g.w, cfg=cfg)
        info = apsp.apsp_get_info(h)
        for _ in range(warmup):
            apsp.apsp_reinit(h)
            apsp.apsp_fw_blocked(h)
        torch.cuda.synchronize()
        st_acc = np.zeros((3, 4))
        clk = ClockSampler(local)
        barrier()
        torch.cuda.synchronize()
        clk.start()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for _ in range(steps):
            apsp.apsp_reinit(h)
            apsp.apsp_fw_blocked(h)
            s = apsp.apsp_get_phase_stats(h)
            st_acc[0] += np.array(s.ms[:])
            st_acc[1] += np.array(s.launches[:])
            st_acc[2] += np.array(s.relax[:])
        e1.record(stream)
        torch.cuda.synchronize()
        barrier()
        clocks = clk.stop()
        ms_step = max_over_ranks(e0.elapsed_time(e1)) / steps
        value = float(n) ** 3 / (ms_step * 1e-3)
        info_end = apsp.apsp_get_info(h)
        arith = apsp.ARITH_NAMES[info_end.arith]
        kernel_used = apsp.KERNEL_NAMES.get(info_end.kernel, "other")
        apsp.apsp_destroy(h)
        del dist_buf
        # roofline of the dominant kernel: phase-3 min-plus launches
        p3_ms = st_acc[0][2] / max(1, st_acc[1][2])
        p3_relax = st_acc[2][2] / max(1, st_acc[1][2])
        achieved = p3_relax / (p3_ms * 1e-3)
        dpx = pk.get("dpx", {})
        if is_f or arith == "f32_exact":
            peak = dpx.get("f32_relax_per_s")
            peak_src = "measured fp32 min-plus rate, FADD2 (broadcast) + FMNMX3 form (MEASURED_DPX.json)"
        elif arith == "s16x2":
            peak = dpx.get("s16x2_relax_per_s")
            peak_src = "measured VIADDMNMX.S16x2 rate, 2 relaxations/instruction (MEASURED_DPX.json)"
        else:
            peak = dpx.get("s32_relax_per_s")
            peak_src = "measured VIADDMNMX s32 rate (MEASURED_DPX.json)"
        if not peak:
            peak = 148 * 64 * 1.965e9 * (2 if arith == "s16x2" else 1)
            peak_src = "derived: 148 SMs x 64 lanes/clk x 1.965 GHz (no MEASURED_DPX.json)"
        dataflow = st_acc[1][0] == 0 and st_acc[1][2] == steps  # one launch per step, no phase-1 launches
        elem = 2 if arith == "s16x2" else 4
        traffic = None
        tp = os.path.join(ROOT, "profiles", "phase3_traffic.json")
        if os.path.exists(tp) and not ooc_mode:
            try:
                sched = kernel_used if kernel_used in ("dataflow_pair", "small64") else (
                    "dataflow" if dataflow else "legacy")
                for tj in json.load(open(tp)).get("captures", []):
                    if (tj.get("workload") == wl and tj.get("arith") == arith
                            and tj.get("schedule", "legacy") == sched):
                        # measured DRAM bytes per relaxation (ncu capture) x this run's relax per launch
                        traffic = tj["dram_bytes_per_relax"] * p3_relax
            except Exception:
                pass
        kname = ("%s: all rounds and phases 1-3 in one persistent launch (%s)"
                 % ("fw_dataflow16_kernel" if arith == "s16x2" else "fw_dataflow_kernel", arith) if dataflow
                 else "phase-3 min-plus (%s)" % arith)
        if kernel_used == "dataflow_pair":
            kname = ("fw_dataflow_kernel (two-round queue: rounds k, k+1 of each bulk tile in one depth-256 task): "
                     "all rounds and phases 1-3 in one persistent launch (%s)" % arith)
        elif kernel_used == "small64":
            kname = "fw_small_kernel (64x64 tiles): all rounds and phases in one persistent launch (%s)" % arith
        if dataflow and world > 1:
            kname = ("fw_dataflow_kernel<sharded>: this rank's tile rows, all rounds in one persistent launch, "
                     "pivot panels stored into every GPU by their owner (%s)" % arith)
        roofline = {"bound": "alu", "kernel": kname, "kernel_id": kernel_used, "achieved": achieved / 1e12,
                    "peak": peak / 1e12, "unit": "Trelax/s", "frac": achieved / peak, "traffic": traffic,
                    "traffic_unit": "bytes per launch (DRAM read+write)",
                    "algorithmic_bytes_per_launch": (p3_relax * 2 * 128 * 128 * elem / 128 ** 3
                                                     if not ooc_mode else None),
                    "peak_source": peak_src, "avg_launch_ms": p3_ms, "relax_per_launch": p3_relax,
                    "share_of_step": (st_acc[0][2] / steps) / ms_step}
        if info.mode == apsp.APSP_MODE_OUT_OF_CORE:
            # host link of the out-of-core step (transfers are part of the time):
            # every streamed band crosses the link once each way per super-round, plus the init's
            # D2H of every streamed band (apsp_reinit) -> bytes per direction per step
            nd = info.n_pad // info.ooc_block
            link_bytes = float(info.host_bytes) * (nd + 1)
            lk = pk.get("dpx", {}).get("host_link_gbs", {})
            lpeak = lk.get("duplex_each_dir") or 47.59
            roofline["link"] = {"bytes_each_direction_per_step": link_bytes,
                                "achieved_gbs": link_bytes / (ms_step * 1e-3) / 1e9, "peak_gbs": lpeak,
                                "link_frac": link_bytes / (ms_step * 1e-3) / 1e9 / lpeak,
                                "peak_source": "MEASURED_DPX.json host_link_gbs.duplex_each_dir (pinned H2D and "
                                               "D2H at once, 1 GiB copies)",
                                "bands": nd, "band_rows": int(info.ooc_block),
                                "streamed_bytes": int(info.host_bytes),
                                "resident_bands": int(nd - info.host_bytes // (info.ooc_block * info.n_pad * 4))}
        return {"value": value, "ms_per_step": ms_step, "arith": arith, "clocks": clocks, "roofline": roofline,
                "steps": steps, "warmup": warmup,
                "launches_per_step": int(round(st_acc[1][:3].sum() / steps)) + 1,  # + init kernel
                "relax_per_step_rank0": st_acc[2][:3].sum() / steps, "n_pad": int(info.n_pad),
                "phase_ms_per_step_rank0": {"phase1": st_acc[0][0] / steps,
                                            "phase2": st_acc[0][1] / steps,
                                            "phase3": st_acc[0][2] / steps,
                                            "comm": st_acc[0][3] / steps}}

    def end_to_end(packed16):
        """Same metric through the C ABI with host buffers, every step: apsp_init_from_csr (pinned
        host CSR, H2D inside) + the closure + the D2H of all of this rank's rows into pinned host
        memory + apsp_destroy. Reported value: a serving loop with two handles in flight
        (apsp_fw_blocked_async + apsp_get_dist_async; step s's D2H overlaps step s+1's closure,
        each step's copies inside the timed region). Beside it ("serial"): the blocking calls
        one after the other."""
        rb, rc = (0, n)
        if world > 1:
            _, rb, rc = apsp.apsp_partition(n, world, rank)
        odt = torch.float32 if is_f else torch.int32
        host_out = [torch.empty((max(rc, 1), n), dtype=odt, pin_memory=True) for _ in range(2)]
        rp = torch.from_numpy(g.row_ptr).pin_memory().numpy()
        cl = torch.from_numpy(g.col).pin_memory().numpy()
        ww = torch.from_numpy(g.w).pin_memory().numpy()
        h2d = rp.nbytes + cl.nbytes + ww.nbytes
        d2h = rc * n * host_out[0].element_size()
        k_e2e = max(1, min(args.steps, 3))
        serial = None
        if args.e2e_serial:
            barrier()
            torch.cuda.synchronize()
            parts = np.zeros(4)
            per_step = []
            t0 = time.perf_counter()
            for _ in range(k_e2e):
                ta = time.perf_counter()
                he = apsp.apsp_init_from_csr(n, rp, cl, ww, cfg=make_cfg(0, packed16))
                tb = time.perf_counter()
                apsp.apsp_fw_blocked(he)
                tc = time.perf_counter()
                if rc > 0:
                    apsp.apsp_get_dist_ptr(he, rb, rc, host_out[0].data_ptr(), n)
                td = time.perf_counter()
                apsp.apsp_destroy(he)
                per_step.append([tb - ta, tc - tb, td - tc, time.perf_counter() - td])
                parts += np.array(per_step[-1])
            torch.cuda.synchronize()
            el_serial = max_over_ranks(time.perf_counter() - t0)
            serial = {"value": float(n) ** 3 / (el_serial / k_e2e), "steps": k_e2e,
                      "ms_parts_each_step": (np.array(per_step) * 1e3).round(2).tolist(),
                      "ms_per_step_parts": dict(zip(["init", "fw", "get_dist", "destroy"],
                                                    (parts / k_e2e * 1e3).round(2).tolist())),
                      "note": "blocking calls one after the other: apsp_init_from_csr + apsp_fw_blocked + "
                              "apsp_get_dist + apsp_destroy"}

        # pipelined serving loop: two handles (created once, like a server's buffers), each step
        # loads its graph (H2D) into one of them while the other's closure / D2H are in flight
        if args.e2e_steps > 0:
            k_pipe = args.e2e_steps
        else:  # a whole-K serving loop when steps are short; bounded when a step takes seconds
            k_pipe = max(3, args.steps if main_run["ms_per_step"] < 2000 else min(args.steps, 5))
        hs = [apsp.apsp_init_from_csr(n, rp, cl, ww, cfg=make_cfg(0, packed16)) for _ in range(2)]
        barrier()
        torch.cuda.synchronize()
        pipe_parts = []
        t0 = time.perf_counter()
        for s_ in range(k_pipe):
            b = s_ % 2
            ta = time.perf_counter()
            apsp.apsp_synchronize(hs[b])  # step s-2 finished: its result is in host_out[b]
            tb = time.perf_counter()
            apsp.apsp_load_csr(hs[b], rp, cl, ww)  # this step's input, host -> device
            tc = time.perf_counter()
            if world > 1:
                # one communicator per handle: keep at most one of them with NCCL work in flight
                # (concurrent collectives on two communicators can deadlock across ranks)
                apsp.apsp_synchronize(hs[1 - b])
            apsp.apsp_fw_blocked_async(hs[b])
            if rc > 0:
                apsp.apsp_get_dist_async(hs[b], rb, rc, host_out[b].data_ptr(), n)
            pipe_parts.append([tb - ta, tc - tb, time.perf_counter() - tc])
        for b in range(2):
            apsp.apsp_synchronize(hs[b])
        torch.cuda.synchronize()
        el_pipe = max_over_ranks(time.perf_counter() - t0)
        for h_ in hs:
            apsp.apsp_destroy(h_)
        return {"value": float(n) ** 3 / (el_pipe / k_pipe), "unit": UNIT, "h2d_bytes_per_step": int(h2d),
                "d2h_bytes_per_step": int(d2h), "steps": k_pipe, "ms_per_step": el_pipe / k_pipe * 1e3,
                "note": "serving loop through the C ABI, host wall clock: per step apsp_load_csr (this step's "
                        "pinned host CSR -> device, init enqueued) + apsp_fw_blocked_async + apsp_get_dist_async "
                        "(all rows -> pinned host) + apsp_synchronize two steps later; two handles (created "
                        "before the timed region) alternate, so step s's D2H overlaps step s+1's closure",
                "ms_parts_each_step": {"sync_load_enqueue": (np.array(pipe_parts) * 1e3).round(2).tolist()},
                "serial": serial}

    def johnson_timed():
        # world > 1: every rank solves its block of sources (no communicator: the SSSP
        # instances are independent), timed as the max over ranks
        cfg = apsp.apsp_config_default(device=local, timing=1, world_size=world, rank=rank)
        cfg.stream = stream.cuda_stream
        h = apsp.apsp_init_johnson(n, g.row_ptr, g.col, g.w, cfg=cfg)
        for _ in range(args.warmup):
            apsp.apsp_reinit(h)
            apsp.apsp_solve(h)
        barrier()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        t0 = time.perf_counter()
        e0.record(stream)
        for _ in range(args.steps):
            apsp.apsp_reinit(h)
            apsp.apsp_solve(h)
        e1.record(stream)
        torch.cuda.synchronize()
        ms = max_over_ranks(max(e0.elapsed_time(e1), (time.perf_counter() - t0) * 1e3) / args.steps)
        edges = apsp.apsp_get_info(h).edges_scanned
        apsp.apsp_destroy(h)
        if world > 1:
            t = torch.tensor([float(edges)], dtype=torch.float64, device="cuda")
            dist.all_reduce(t)
            edges = int(t.item())
        return {"ms_per_apsp": ms, "speedup_vs_fw_step": main_run["ms_per_step"] / ms,
                "arcs_relaxed_per_apsp": edges, "arcs_per_s": edges / (ms * 1e-3),
                "fw_equivalent_relax_per_s": float(n) ** 3 / (ms * 1e-3), "n_gpus": world,
                "note": "apsp_init_johnson + apsp_solve (one block per source, Near-Far queues; PAPER.md:66, "
                        ":72, Alg. 2), same graph, result resident in HBM (rank r: its block of source rows); "
                        "bit-exact in tests/test_gpu_johnson.py"}

    main_run = device_timed(args.packed16)

    def guarded(fn, *a):  # an optional leg never takes the headline line down
        try:
            return fn(*a)
        except Exception as exc:
            return {"error": str(exc)[:300]}

    e2e = None if args.no_e2e else guarded(end_to_end, args.packed16)

    # the packed int16 alternative (exact, verified; R16), single GPU int32 inputs
    alt16 = None
    if world == 1 and not is_f and not args.packed16 and not args.no_packed16 and not args.force_ooc:
        long_steps = main_run["ms_per_step"] >= 2000  # bound the extra leg when a step takes seconds
        r16 = guarded(device_timed, True, min(args.steps, 5) if long_steps else args.steps,
                      min(args.warmup, 3) if long_steps else args.warmup)
        alt16 = r16 if "error" in r16 else {
            "value": r16["value"], "ms_per_step": r16["ms_per_step"], "dtype": r16["arith"],
            "steps": r16["steps"], "warmup": r16["warmup"], "roofline": r16["roofline"], "clocks": r16["clocks"],
            "e2e": guarded(end_to_end, True) if args.packed16_e2e and not args.no_e2e else None,
            "note": "same workload, apsp_config.packed16=1: VIADDMNMX.S16x2 (2 relaxations per DPX instruction) "
                    "with the exactness check of DESIGN.md R16; the result is the exact int32 APSP (bit-exact in "
                    "tests/test_gpu_packed16.py); falls back to int32 when distances reach 8192 (dtype then reads i32)"}

    # int32 distances closed by the fp32 engine when the a priori bound makes every sum exact
    # (apsp_config.exact_f32, R25; config 3: 2 (n - 1) 100 <= 2^24)
    alt_f32x = None
    if world == 1 and not is_f and not args.packed16 and not args.no_exact_f32_leg and not args.force_ooc:
        long_steps = main_run["ms_per_step"] >= 2000
        rx = guarded(device_timed, False, min(args.steps, 3) if long_steps else args.steps,
                     min(args.warmup, 1) if long_steps else args.warmup, False, True)
        alt_f32x = rx if "error" in rx else {
            "value": rx["value"], "ms_per_step": rx["ms_per_step"], "dtype": rx["arith"],
            "steps": rx["steps"], "warmup": rx["warmup"], "roofline": rx["roofline"], "clocks": rx["clocks"],
            "note": "same workload, apsp_config.exact_f32=1: the int32 matrix converted to fp32 in place, closed "
                    "by fw_dataflow_kernel<float> (FADD2 + FMNMX3, 1 instruction per relaxation on two pipes "
                    "instead of VIADDMNMX on one), converted back, all inside the timed step; exact because every "
                    "candidate sum is an integer <= 2 (n - 1) max w <= 2^24 (R25, checked before the run); "
                    "output bit-exact int32 (tests/test_gpu_exact_f32.py, config 3 certified); dtype f32_exact, "
                    "i32 when the graph is outside the bound"}

    # the out-of-core scheduler on the same workload with every band streamed through pinned host
    # memory (Algorithm 1, the paper's setting; transfers inside the step):
    # roofline.link = host-link bytes per step against the measured duplex rate
    alt_ooc = None
    # (N > 1: out of core x P ranks has run as virtual ranks only, never with a real multi-rank NCCL
    # communicator, so the scaling runs keep to the headline unless --ooc-leg-multi asks for it)
    if not args.force_ooc and not args.no_ooc_leg and (world == 1 or args.ooc_leg_multi):
        ro = guarded(device_timed, False, min(args.steps, 2), 1, True)
        alt_ooc = ro if "error" in ro else {
            "value": ro["value"], "ms_per_step": ro["ms_per_step"], "dtype": ro["arith"],
            "steps": ro["steps"], "warmup": ro["warmup"], "roofline": ro["roofline"], "clocks": ro["clocks"],
            "note": "same workload through the out-of-core scheduler (apsp_config.force_out_of_core, ooc_stream_all, "
                    "B = %d): the whole matrix in pinned host memory, every band streamed each super-round, pivot "
                    "lookahead; step = apsp_reinit (init + D2H of every band) + apsp_fw_blocked; bit-exact in "
                    "tests/test_gpu_ooc.py" % (args.ooc_block or 4096)}

    # the boundary algorithm (eq. (1), Alg. 3) out of core on a small-separator graph of
    # the same n: a sqrt(n) x sqrt(n) 2-D grid (cfg2/cfg5's recipe) split into the paper's
    # k = sqrt(n)/4 components, every block row of the result streamed to pinned host
    # memory through two N_row buffers (transfers inside the solve), beside the
    # blocked-FW out-of-core step of the same n (dense FW cost does not depend on the structure)
    def boundary_timed():
        side = int(round(n ** 0.5))
        if side * side != n:
            return {"skipped": "n=%d is not a square" % n}
        gb = gg.grid_2d(side, side, seed=3, name="grid%d" % n)
        blocks = max(1, int(round((side / 4) ** 0.5)))  # blocks x blocks components, k ~ sqrt(n)/4
        comp, k = gg.grid_block_partition(gb, blocks, blocks)
        cfg = apsp.apsp_config_default(device=local, timing=1)
        cfg.stream = stream.cuda_stream
        cfg.force_out_of_core = 1
        h = apsp.apsp_init_boundary(n, gb.row_ptr, gb.col, gb.w, comp, k, cfg=cfg)
        try:
            steps = min(args.steps, 5)
            for _ in range(min(args.warmup, 2)):
                apsp.apsp_reinit(h)
                apsp.apsp_solve(h)
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            for _ in range(steps):
                apsp.apsp_reinit(h)
                apsp.apsp_solve(h)
            e1.record(stream)
            torch.cuda.synchronize()
            ms = e0.elapsed_time(e1) / steps
            info = apsp.apsp_get_info(h)
            st = apsp.apsp_get_phase_stats(h)
        finally:
            apsp.apsp_destroy(h)
        link = float(info.host_bytes)
        lk = peaks().get("dpx", {}).get("host_link_gbs", {})
        d2h = lk.get("d2h") or 0.0
        out = {"workload": "grid %dx%d, seed 3, int32 U{1..100}, k = %d components (%dx%d blocks)" %
                           (side, side, k, blocks, blocks),
               "ms_per_solve": ms, "steps": steps, "boundary_nodes": int(info.boundary_nodes),
               "relaxations_per_solve": float(sum(st.relax[:3])),
               "out_of_core": bool(info.ooc_block > 0), "buffer_rows": int(info.ooc_block),
               "host_bytes_per_solve": int(link), "link_gbs": link / (ms * 1e-3) / 1e9,
               "link_frac_d2h": (link / (ms * 1e-3) / 1e9 / d2h) if d2h else None,
               "note": "apsp_init_boundary (force_out_of_core: nothing resident, every block row crosses the "
                       "link) + apsp_reinit + apsp_solve per step; bit-exact in tests/test_boundary.py"}
        if alt_ooc and "ms_per_step" in alt_ooc:
            out["fw_out_of_core_ms_per_step_same_n"] = alt_ooc["ms_per_step"]
            out["speedup_vs_fw_out_of_core"] = alt_ooc["ms_per_step"] / ms
        return out

    alt_bnd = None
    if world == 1 and not is_f and not args.force_ooc and not args.no_boundary_leg:
        alt_bnd = guarded(boundary_timed)

    # Johnson's algorithm on the same graph (batched Near-Far SSSP): the
    # paper's method for sparse graphs; a different algorithm (O(n m) work, not n^3), so it is
    # reported as time per APSP beside the FW step, not as the metric
    alt_jn = None
    if not args.no_johnson and not args.force_ooc and not (is_f and bool((g.w < 0).any())):
        alt_jn = guarded(johnson_timed)

    # ---------------- CPU oracle baseline (rank 0, N=1 only) ------------------
    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu:
        if n <= CPU_BASELINE_FULL_MAX_N:
            r, secs, _ = oracle_whole_run(g, 4)
            cores = __import__("oracle").threads()
            sample = ("the whole workload: one complete oracle plain FW run (OpenMP over rows, n=%d, %.2f s, "
                      "init not counted)" % (n, secs))
        else:
            r, cores, sample, _, _ = oracle_steady_rate(g, warm_s=2.0, step_s=args.cpu_seconds / 3, steps=3)
        cpu = {"value": r, "unit": UNIT, "cores": cores, "kind": "oracle", "sample": sample}

    if rank == 0:
        line = {
            "metric": METRIC, "value": main_run["value"], "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": main_run["ms_per_step"], "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None,
            "dtype": main_run["arith"], "data": "synthetic",
            "config": {"workload": wl, "n": n, "n_pad": main_run["n_pad"], "m": g.m, "tile": 128,
                       "desc": gg.BASELINE_CONFIGS[wl],
                       "parallelism": "1-D block-row x%d, NCCL pivot-band broadcast" % world if world > 1
                       else "single GPU",
                       "l2": "inputs larger than L2 (dist = %.2f GB per step >> 126 MB L2); no flush" %
                             (float(main_run["n_pad"]) ** 2 * (2 if main_run["arith"] == "s16x2" else 4) / 1e9),
                       "step": "apsp_reinit (CSR->dense, CSR resident in HBM) + apsp_fw_blocked",
                       "dist_memory": "torch-allocated device tensor passed as apsp_config.dist_device"},
            "clocks": main_run["clocks"],
            "e2e": e2e,
            "gpu_launches": main_run["launches_per_step"] * args.steps,
            "roofline": main_run["roofline"],
            "cpu_baseline": cpu,
            "packed16": alt16,
            "exact_f32": alt_f32x,
            "out_of_core": alt_ooc,
            "johnson": alt_jn,
            "boundary": alt_bnd,
            "relax_per_step_rank0": main_run["relax_per_step_rank0"],
            "phase_ms_per_step_rank0": main_run["phase_ms_per_step_rank0"],
        }
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()
    return 0


def self_launch(args):
    """`--gpus N > 1` without torchrun: re-execute this command under torch.distributed.run
    (one process per GPU, rendezvous on 127.0.0.1, a free port), as the driver would launch it."""
    import socket
    with socket.socket() as sk:
        sk.bind(("127.0.0.1", 0))
        port = sk.getsockname()[1]
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", str(args.gpus),
           "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.abspath(__file__)] + sys.argv[1:]
    sys.stdout.flush()
    return subprocess.call(cmd)


def rendezvous_only(args):
    import torch.distributed as dist
    world, rank, _ = dist_env()
    dist.init_process_group("gloo")
    dist.barrier()
    # one write per line: the ranks share the launcher's stdout pipe
    sys.stdout.write(json.dumps({"rendezvous": True, "rank": rank, "world": world}) + "\n")
    sys.stdout.flush()
    dist.destroy_process_group()
    return 0


def main():
    args = parse()
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        return self_launch(args)
    if args.rendezvous_only:
        return rendezvous_only(args)
    if args.impl == "reference":
        return run_reference(args)
    return run_ours(args)


if __name__ == "__main__":
    sys.exit(main())
