"""C-ABI boundary checks that need no GPU: the library loads, exports every symbol
include/apsp.h declares, validates its inputs on the host, and fails loudly
(APSP_ECUDA, no CPU fallback) when no device is visible."""
import os
import re

import numpy as np
import pytest

import graphgen as gg

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def header_functions():
    src = open(os.path.join(ROOT, "include", "apsp.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(apsp_[a-z0-9_]+)\s*\(", src)))


def test_library_exports_every_declared_symbol(lib):
    import ctypes
    names = header_functions()
    assert "apsp_init_from_csr" in names and "apsp_fw_blocked" in names and "apsp_get_dist" in names
    so = ctypes.CDLL(lib.LIB_PATH)
    for name in names:
        assert hasattr(so, name), name
    assert set(names) == set(lib.EXPORTED_SYMBOLS)
    assert "sm_100a" in lib.apsp_version()


def test_config_struct_layout(lib):
    import ctypes
    cfg = lib.apsp_config_default()
    assert cfg.struct_size == ctypes.sizeof(lib.apsp_config)
    assert cfg.device == -1 and cfg.world_size == 1 and cfg.rank == 0


@pytest.mark.parametrize("n,world", [(0, 1), (1, 1), (127, 1), (128, 1), (129, 1), (1000, 2), (65536, 8),
                                     (300, 4), (131072, 8)])
def test_partition(lib, n, world):
    rows = []
    for r in range(world):
        n_pad, rb, rc = lib.apsp_partition(n, world, r)
        assert n_pad % (128 * world) == 0 and n_pad >= max(n, 1) and n_pad - n < 128 * world + (n == 0) * 128
        assert rb == r * n_pad // world
        assert rc == max(0, min(rb + n_pad // world, n) - rb)
        rows += list(range(rb, rb + rc))
    assert rows == list(range(n))


def _bad(lib, n, rp, col, w, status, dtype=None):
    with pytest.raises(lib.ApspError) as e:
        lib.apsp_init_from_csr(n, rp, col, w, dtype=dtype)
    assert e.value.status == status, str(e.value)
    assert lib.apsp_last_error() != ""


def test_input_validation(lib):
    E = lib.APSP_EINVAL
    _bad(lib, 3, [0, 1, 0, 1], [1], [1], E)             # row_ptr not monotone
    _bad(lib, 3, [1, 1, 1, 1], [], [], E)               # row_ptr[0] != 0
    _bad(lib, 3, [0, 1, 1, 1], [3], [1], E)             # col out of range
    _bad(lib, 3, [0, 1, 1, 1], [-1], [1], E)            # negative col
    _bad(lib, 2, [0, 1, 1], [1], [np.nan], E, lib.APSP_F32)
    _bad(lib, 2, [0, 1, 1], [1], [np.inf], E, lib.APSP_F32)


def test_erange(lib):
    # (n-1)*max|w| >= 2^30-1 with non-negative weights
    _bad(lib, 3, [0, 1, 1, 1], [1], [600_000_000], lib.APSP_ERANGE)
    # negative weights tighten the bound to 2^28
    _bad(lib, 3, [0, 2, 2, 2], [1, 2], [-1, 140_000_000], lib.APSP_ERANGE)


def _has_gpu():
    try:
        import torch
        return torch.cuda.is_available()
    except Exception:
        return False


@pytest.mark.skipif(_has_gpu(), reason="checks the no-GPU failure mode")
def test_no_gpu_fails_loudly(lib):
    g = gg.erdos_renyi(50, 200, seed=1)
    with pytest.raises(lib.ApspError) as e:
        lib.apsp_init_from_csr(g.n, g.row_ptr, g.col, g.w)
    assert e.value.status == lib.APSP_ECUDA


def test_binding_constants_match_header(lib):
    """Every `#define APSP_*` integer constant and `apsp_status` / `apsp_dtype` enumerator in
    include/apsp.h has the same value in the Python binding."""
    src = open(os.path.join(ROOT, "include", "apsp.h")).read()
    src_nc = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    consts = {k: int(v, 0) for k, v in re.findall(r"#define\s+(APSP_[A-Z0-9_]+)\s+(0x[0-9A-Fa-f]+|\d+)\b", src_nc)}
    for body in re.findall(r"typedef\s+enum\s*\{(.*?)\}", src_nc, flags=re.S):
        nxt = 0
        for item in body.split(","):
            item = item.strip()
            if not item:
                continue
            if "=" in item:
                name, val = (s.strip() for s in item.split("="))
                nxt = int(val, 0)
            else:
                name = item
            consts[name] = nxt
            nxt += 1
    assert "APSP_MODE_BOUNDARY" in consts and "APSP_ENEGCYCLE" in consts
    for name, val in consts.items():
        if name.startswith("APSP_") and not name.endswith("_H"):
            assert getattr(lib, name) == val, name


@pytest.mark.parametrize("short", ["col", "w"])
def test_binding_refuses_short_csr_arrays(lib, short):
    """The C side reads exactly row_ptr[n] arcs; the binding refuses shorter col_idx / weights
    (APSP_EINVAL) before any pointer crosses the boundary."""
    g = gg.erdos_renyi(50, 200, seed=3)
    col = g.col[:-1] if short == "col" else g.col
    w = g.w[:-1] if short == "w" else g.w
    comp = np.zeros(g.n, np.int32)
    calls = [lambda: lib.apsp_init_from_csr(g.n, g.row_ptr, col, w),
             lambda: lib.apsp_init_johnson(g.n, g.row_ptr, col, w),
             lambda: lib.apsp_init_boundary(g.n, g.row_ptr, col, w, comp, 1),
             lambda: lib.apsp_select(g.n, g.row_ptr, col, w)]
    for call in calls:
        with pytest.raises(lib.ApspError) as e:
            call()
        assert e.value.status == lib.APSP_EINVAL and "row_ptr[n]" in str(e.value)


def test_config_named_fields_and_reserved(lib):
    """The schedule / test switches are named apsp_config fields; reserved[] must stay zero
    (checked before any device work, so APSP_EINVAL even without a GPU)."""
    names = [f[0] for f in lib.apsp_config._fields_]
    for f in ("dist_device", "dist_device_bytes", "schedule", "no_lookahead", "ooc_stream_all", "force_nccl",
              "minplus_variant", "dataflow_delay", "exact_f32", "reserved"):
        assert f in names, f
    hdr = open(os.path.join(ROOT, "include", "apsp.h")).read()
    body = hdr[hdr.index("typedef struct {\n  int32_t struct_size;"):hdr.index("} apsp_config;")]
    body = re.sub(r"/\*.*?\*/", "", body, flags=re.S)
    assert re.findall(r"\b(\w+)(?:\[\d+\])?;", body) == names  # same order as the C struct
    assert (lib.APSP_SCHED_AUTO, lib.APSP_SCHED_PER_PHASE, lib.APSP_SCHED_DATAFLOW) == (0, 1, 2)
    g = gg.erdos_renyi(20, 60, seed=1)
    for field, val in (("reserved", 1), ("schedule", 7), ("minplus_variant", 3), ("dataflow_delay", -1),
                       ("exact_f32", 2)):
        cfg = lib.apsp_config_default()
        if field == "reserved":
            cfg.reserved[2] = val
        else:
            setattr(cfg, field, val)
        with pytest.raises(lib.ApspError) as e:
            lib.apsp_init_from_csr(g.n, g.row_ptr, g.col, g.w, cfg=cfg)
        assert e.value.status == lib.APSP_EINVAL, field


@pytest.mark.parametrize("n,world,virt", [(1, 1, 0), (300, 1, 0), (16384, 1, 0), (1000, 2, 0), (1000, 4, 1),
                                          (65536, 8, 0)])
def test_dist_device_bytes(lib, n, world, virt):
    n_pad, _, _ = lib.apsp_partition(n, world, 0)
    want = (n_pad // world) * n_pad * 4 * (world if virt else 1)
    assert lib.apsp_dist_device_bytes(n, world, virt) == want


def test_dist_device_too_small_or_misaligned_is_refused(lib):
    g = gg.erdos_renyi(300, 900, seed=2)
    need = lib.apsp_dist_device_bytes(g.n)
    for ptr, nbytes in ((1 << 20, need - 4), ((1 << 20) + 64, need)):  # never dereferenced: refused first
        cfg = lib.apsp_config_default(dist_device=ptr, dist_device_bytes=nbytes)
        with pytest.raises(lib.ApspError) as e:
            lib.apsp_init_from_csr(g.n, g.row_ptr, g.col, g.w, cfg=cfg)
        assert e.value.status == lib.APSP_EINVAL
    cfg = lib.apsp_config_default(dist_device=1 << 20, dist_device_bytes=need)
    comp = np.zeros(g.n, np.int32)
    for call in (lambda: lib.apsp_init_johnson(g.n, g.row_ptr, g.col, g.w, cfg=cfg),
                 lambda: lib.apsp_init_boundary(g.n, g.row_ptr, g.col, g.w, comp, 1, cfg=cfg)):
        with pytest.raises(lib.ApspError) as e:
            call()
        assert e.value.status == lib.APSP_EINVAL


def test_kernel_ids_match_header(lib):
    hdr = open(os.path.join(ROOT, "include", "apsp.h")).read()
    ids = {int(v): k for k, v in re.findall(r"#define APSP_KERNEL_([A-Z0-9_]+) (\d+)", hdr)}
    assert sorted(ids) == list(range(1, 8))
    names = {"PER_PHASE": "per_phase", "DATAFLOW": "dataflow", "DATAFLOW_PAIR": "dataflow_pair", "SMALL": "small64",
             "DATAFLOW16": "dataflow16", "SHARDED": "sharded_dataflow", "OUT_OF_CORE": "out_of_core"}
    for v, k in ids.items():
        assert lib.KERNEL_NAMES[v] == names[k]
    assert [f[0] for f in lib.apsp_info._fields_][-2:] == ["kernel", "exact_f32_eligible"]
