#!/usr/bin/env python
"""A/B kernel variants: builds libdbg.so with extra -D flags into lib/variants/<name>/ (git-ignored)
for a same-box comparison (`DBG_LIB_PATH=... python bench.py`).

    python tools/build_variants.py base= pred=-DDBG_PROBE_PRED=1 ...
"""
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_icdcs_qiul17_b200 import build as B  # noqa: E402


def build_variant(name: str, defs: list[str]) -> str:
    out = os.path.join(B.LIBDIR, "variants", name)
    os.makedirs(out, exist_ok=True)
    objs = []
    for s in B.SOURCES:
        o = os.path.join(out, s.replace(".cu", ".o"))
        subprocess.check_call([B.NVCC, *B.ARCH, *B.FLAGS, *defs, "-c", os.path.join(B.CSRC, s), "-o", o])
        objs.append(o)
    lib = os.path.join(out, "libdbg.so")
    subprocess.check_call([B.NVCC, *B.ARCH, "-shared", "-o", lib, *objs])
    for o in objs:
        os.remove(o)
    return lib


if __name__ == "__main__":
    for arg in sys.argv[1:]:
        name, _, flags = arg.partition("=")
        print(build_variant(name, [f for f in flags.split(",") if f]))
