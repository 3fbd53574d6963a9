"""Build the sm_100a C-ABI library ``libapsp.so`` in-tree with nvcc.

Used by ``__graft_entry__.build()``. The library links the CUDA runtime
statically and NCCL dynamically from the torch wheel's copy (the one torch
itself loads), with an rpath so it also loads without torch.
"""
from __future__ import annotations

import glob
import os
import subprocess
import sys
import sysconfig

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
BUILD = os.path.join(ROOT, "build", "obj")
LIB = os.path.join(PKG, "libapsp.so")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")


def nccl_dirs():
    purelib = sysconfig.get_paths()["purelib"]
    cands = [os.path.join(purelib, "nvidia", "nccl")]
    try:
        import nvidia.nccl  # noqa: F401
        cands.insert(0, os.path.dirname(nvidia.nccl.__file__) if nvidia.nccl.__file__
                     else list(nvidia.nccl.__path__)[0])
    except Exception:
        pass
    for c in cands:
        if os.path.exists(os.path.join(c, "include", "nccl.h")):
            return os.path.join(c, "include"), os.path.join(c, "lib")
    return "/usr/include", "/usr/lib/x86_64-linux-gnu"


def _run(cmd):
    p = subprocess.run(cmd, stdout=subprocess.PIPE, stderr=subprocess.STDOUT, text=True)
    if p.returncode != 0:
        sys.stderr.write(" ".join(cmd) + "\n" + p.stdout)
        raise RuntimeError("build failed: %s" % cmd[-1])
    return p.stdout


def build_lib(force: bool = False, verbose: bool = False) -> str:
    os.makedirs(BUILD, exist_ok=True)
    inc, libdir = nccl_dirs()
    srcs = sorted(glob.glob(os.path.join(CSRC, "*.cu")))
    headers = glob.glob(os.path.join(CSRC, "*.cuh")) + glob.glob(os.path.join(CSRC, "*.h")) + \
        glob.glob(os.path.join(ROOT, "include", "*.h"))
    newest_hdr = max(os.path.getmtime(h) for h in headers)
    common = [NVCC, "-O3", "-std=c++17", *ARCH, "-lineinfo", "-Xcompiler", "-fPIC,-O2",
              "-I", os.path.join(ROOT, "include"), "-I", inc]
    common += os.environ.get("APSP_NVCC_EXTRA", "").split()  # experiments (pass force=True)
    procs, objs = [], []
    for s in srcs:
        o = os.path.join(BUILD, os.path.basename(s) + ".o")
        objs.append(o)
        if force or not os.path.exists(o) or os.path.getmtime(o) < max(os.path.getmtime(s), newest_hdr):
            cmd = common + (["-Xptxas", "-v"] if verbose else []) + ["-c", s, "-o", o]
            procs.append((cmd, subprocess.Popen(cmd, stdout=subprocess.PIPE, stderr=subprocess.STDOUT, text=True)))
    for cmd, p in procs:
        out = p.communicate()[0]
        if p.returncode != 0:
            sys.stderr.write(" ".join(cmd) + "\n" + out)
            raise RuntimeError("nvcc failed on %s" % cmd[-3])
        if verbose:
            sys.stdout.write(out)
    if force or procs or not os.path.exists(LIB):
        tmp = LIB + ".tmp%d" % os.getpid()
        _run([NVCC, *ARCH, "-shared", "-cudart", "static", "-o", tmp, *objs,
              "-L", libdir, "-l:libnccl.so.2", "-Xlinker", "-rpath=" + libdir])
        os.replace(tmp, LIB)
    return LIB


def build_micro(force: bool = False) -> str:
    out = os.path.join(ROOT, "build", "dpx_peak")
    src = os.path.join(CSRC, "micro", "dpx_peak.cu")
    if force or not os.path.exists(out) or os.path.getmtime(out) < os.path.getmtime(src):
        _run([NVCC, "-O3", *ARCH, "-lineinfo", "-o", out, src])
    return out


if __name__ == "__main__":
    print(build_lib(force="--force" in sys.argv, verbose="-v" in sys.argv))
    print(build_micro())
