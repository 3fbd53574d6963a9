"""GPU path on the textbook worked examples under tests/golden/ (CLRS 3e Figs. 24.4,
24.6, 25.4): every schedule and arithmetic the C ABI offers reproduces the values
printed in the figures, not only the oracle's. n = 5 pads to one 128-wide tile, so
this is also the ragged single-tile case of phase 1."""
import numpy as np
import pytest

import graphgen as gg
import golden_io

pytestmark = pytest.mark.gpu

FIXTURES = ["clrs_fig25_4.txt", "clrs_fig24_4.txt", "clrs_fig24_6.txt"]
BASE = {"clrs_fig25_4.txt": 1}


def load(name, dtype=np.int32):
    arcs, src, dist = golden_io.load(name, base=BASE.get(name, 0))
    s, d, w = zip(*arcs)
    g = gg.csr_from_arcs(5, np.array(s, np.int64), np.array(d, np.int64), np.array(w, dtype))
    return g, src, dist


def check(got, src, dist):
    got = np.asarray(got)
    if src is None:
        assert got.tolist() == dist
    else:
        assert got[src].tolist() == dist[0]
    assert np.all(np.diag(got) == 0)


@pytest.mark.parametrize("schedule", [0, 1, 2, 3], ids=["auto", "per_phase", "dataflow128", "small64"])
@pytest.mark.parametrize("name", FIXTURES)
def test_golden_fw_i32(lib, name, schedule):
    g, src, dist = load(name)
    c = lib.apsp_config_default(device=0)
    c.schedule = schedule
    check(lib.solve(g, cfg=c).astype(np.int64), src, dist)


@pytest.mark.parametrize("schedule", [0, 2], ids=["auto", "dataflow128"])
@pytest.mark.parametrize("name", FIXTURES)
def test_golden_fw_f32(lib, name, schedule):
    g, src, dist = load(name, np.float32)
    got = lib.solve(g, cfg=lib.apsp_config_default(device=0, schedule=schedule))
    assert got.dtype == np.float32
    check(got.astype(np.int64), src, dist)  # small integers: exact in fp32


@pytest.mark.parametrize("legacy", [0, 1], ids=["dataflow", "per_phase"])
def test_golden_packed16(lib, legacy):
    g, src, dist = load("clrs_fig24_6.txt")  # non-negative weights: int16-eligible
    c = lib.apsp_config_default(device=0, packed16=1)
    c.schedule = legacy
    with lib.apsp_init_from_csr(g.n, g.row_ptr, g.col, g.w, cfg=c) as h:
        assert lib.apsp_get_info(h).packed16_eligible
        lib.apsp_fw_blocked(h)
        check(lib.apsp_get_dist(h).astype(np.int64), src, dist)


@pytest.mark.parametrize("name", FIXTURES)
def test_golden_johnson(lib, name):
    g, src, dist = load(name)
    check(lib.solve_johnson(g, cfg=lib.apsp_config_default(device=0)).astype(np.int64), src, dist)
