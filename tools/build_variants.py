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


def build_variant(name: str, defs: list[str], rev: str | None = None) -> str:
    """rev: build the csrc/ of that git revision (same-box comparison against a previous commit)."""
    out = os.path.join(B.LIBDIR, "variants", name)
    os.makedirs(out, exist_ok=True)
    csrc = B.CSRC
    if rev:
        top = os.path.join("/tmp", f"vsrc_{name}")
        csrc = os.path.join(top, "pkg", "csrc")  # csrc/../../include/dbg.h as in the tree
        os.makedirs(csrc, exist_ok=True)
        os.makedirs(os.path.join(top, "include"), exist_ok=True)
        blob = subprocess.run(["git", "-C", ROOT, "show", f"{rev}:include/dbg.h"], check=True,
                              capture_output=True).stdout
        open(os.path.join(top, "include", "dbg.h"), "wb").write(blob)
        names = subprocess.run(["git", "-C", ROOT, "ls-tree", "--name-only", rev, "paper_conf_icdcs_qiul17_b200/csrc/"],
                               check=True, capture_output=True, text=True).stdout.split()
        for path in names:
            blob = subprocess.run(["git", "-C", ROOT, "show", f"{rev}:{path}"], check=True,
                                  capture_output=True).stdout
            open(os.path.join(csrc, os.path.basename(path)), "wb").write(blob)
    objs = []
    for s in B.SOURCES:
        o = os.path.join(out, s.replace(".cu", ".o"))
        subprocess.check_call([B.NVCC, *B.ARCH, *B.FLAGS, *defs, "-c", os.path.join(csrc, s), "-o", o])
        objs.append(o)
    lib = os.path.join(out, "libdbg.so")
    subprocess.check_call([B.NVCC, *B.ARCH, "-shared", "-o", lib, *objs])
    for o in objs:
        os.remove(o)
    return lib


if __name__ == "__main__":
    for arg in sys.argv[1:]:  # name[@rev]=flag,flag
        name, _, flags = arg.partition("=")
        name, _, rev = name.partition("@")
        print(build_variant(name, [f for f in flags.split(",") if f], rev or None))
