#!/usr/bin/env python
"""Build an A/B variant of libapsp.so with extra nvcc flags into build/var_<name>/, next to a copy of
the binding and links to graphgen / oracle / tools, so `cd build/var_<name> && python tools/fw_ab.py ...`
times the variant beside the default build in the same gpurun call.

    python tools/build_variant.py jp -DAPSP_F32_JP_OUTER=1
"""
import importlib.util
import os
import shutil
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def main():
    name, flags = sys.argv[1], sys.argv[2:]
    spec = importlib.util.spec_from_file_location("_apsp_build", os.path.join(ROOT, "paper_conf_ipps_xia0ar22_b200",
                                                                             "_build.py"))
    b = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(b)
    vdir = os.path.join(ROOT, "build", "var_" + name)
    pkg = os.path.join(vdir, "paper_conf_ipps_xia0ar22_b200")
    os.makedirs(pkg, exist_ok=True)
    b.BUILD = os.path.join(vdir, "obj")
    b.LIB = os.path.join(pkg, "libapsp.so")
    os.environ["APSP_NVCC_EXTRA"] = " ".join(flags)
    b.build_lib(force=True)
    shutil.copy(os.path.join(ROOT, "paper_conf_ipps_xia0ar22_b200", "__init__.py"), pkg)
    for d in ("graphgen", "oracle", "tools", "tests", "include"):
        link = os.path.join(vdir, d)
        if not os.path.lexists(link):
            os.symlink(os.path.join("..", "..", d), link)
    print(b.LIB)


if __name__ == "__main__":
    main()
