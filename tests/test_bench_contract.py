"""bench.py's reference arm (the CPU oracle timed on host cores, BASELINE metric and config):
one JSON line with the contract's keys, runnable without a GPU. The GPU arm's line is checked
on the B200 by the driver (and its keys by tests/test_gpu_fullsize.py's bench usage)."""
import json
import re
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_reference_arm_json_line():
    p = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--workload",
                        "cfg1_er1024", "--steps", "1", "--warmup", "3"], capture_output=True, text=True,
                       timeout=300, cwd=ROOT)
    assert p.returncode == 0, p.stderr[-2000:]
    lines = [l for l in p.stdout.splitlines() if l.strip().startswith("{")]
    assert len(lines) == 1
    d = json.loads(lines[0])
    for k in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better",
              "scaling", "vs_baseline", "dtype", "data", "config", "impl", "cpu_baseline", "e2e"):
        assert k in d, k
    assert d["impl"] == "reference" and d["n_gpus"] == 1 and d["higher_is_better"] is True
    assert d["unit"] == "relax/s" and d["value"] > 0
    assert d["config"]["workload"] == "cfg1_er1024"
    cb = d["cpu_baseline"]
    assert cb["kind"] == "oracle" and cb["cores"] >= 1 and cb["value"] == d["value"] and cb["sample"]
    assert d["e2e"]["value"] == d["value"] and d["e2e"]["h2d_bytes_per_step"] == 0
    with open(os.path.join(ROOT, "BASELINE.json")) as f:
        assert d["metric"] == json.load(f)["metric"]


def test_self_launch_two_ranks_rendezvous():
    """`bench.py --gpus 2` without torchrun re-executes itself under torch.distributed.run (127.0.0.1,
    a free port); both ranks reach the process-group rendezvous (gloo here, NCCL on the GPU box)."""
    env = {k: v for k, v in os.environ.items() if k not in ("WORLD_SIZE", "RANK", "LOCAL_RANK",
                                                             "MASTER_ADDR", "MASTER_PORT")}
    p = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "2", "--rendezvous-only"],
                       capture_output=True, text=True, timeout=300, cwd=ROOT, env=env)
    assert p.returncode == 0, p.stderr[-2000:]
    objs = re.findall(r"\{[^{}]*\}", p.stdout)  # robust to two ranks' lines interleaving
    got = sorted(json.loads(o)["rank"] for o in objs if '"rendezvous"' in o)
    assert got == [0, 1]


def test_default_workload_is_the_metric_config():
    """BASELINE.json quotes the metric 'at 1/2/4/8 B200' on configs[2] (n=65536): every N uses it."""
    sys.path.insert(0, ROOT)
    import bench
    import graphgen as gg
    for n_gpus in (1, 2, 4, 8):
        assert bench.default_workload(n_gpus) == "cfg3_er65536"
    with open(os.path.join(ROOT, "BASELINE.json")) as f:
        assert "n=65536" in json.load(f)["configs"][2]


def test_oracle_steady_rate_counts_full_iterations():
    """The steady-state CPU sample does every relaxation of every outer iteration (no INF skip):
    its rate on a sparse graph is below the whole-run rate of the same oracle, never above it by
    the early-iteration skip (the r1 cpu_baseline bias)."""
    sys.path.insert(0, ROOT)
    import bench
    import graphgen as gg
    g = gg.erdos_renyi(1536, 1536 * 2, seed=11)  # sparse: many rows skipped early in a real run
    seen = []
    for _ in range(3):  # wall-clock rates: a busy host can slow one measurement; one clean pair decides
        whole, _, _ = bench.oracle_whole_run(g, 2)
        steady, cores, sample, rates, _ = bench.oracle_steady_rate(g, warm_s=0.2, step_s=0.3, steps=2)
        assert cores >= 1 and len(rates) == 2 and "steady-state" in sample
        seen.append((steady, whole))
        if steady <= whole * 1.3:
            break
    else:
        raise AssertionError("steady-state rate above the whole-run rate in every attempt: %r" % seen)
