#!/usr/bin/env python3
"""Build an experimental copy of the library with extra compile-time defines
into exp/<name>/ (git-ignored; travels to the GPU box with gpurun), for A/B
timing with SWB_LIB=exp/<name>/libcudalign_b200.so:

    python tools/build_variant.py fmode3 -DSWB_FMODE=3
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

from paper_conf_ipps_sandesm11_b200 import build  # noqa: E402

if __name__ == "__main__":
    name, defs = sys.argv[1], sys.argv[2:]
    print(build.build(defs=defs, out_dir=os.path.join(ROOT, "exp", name)))
