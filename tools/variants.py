#!/usr/bin/env python
"""Build experimental variants of libmdnorm.so into variants/ (git-ignored) for tools/time_kernels.py.

  python tools/variants.py NAME:DEF1=1,DEF2=3 NAME2:...
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_sc_hahnfgmmshvvs24_b200 import build  # noqa: E402

os.makedirs(os.path.join(ROOT, "variants"), exist_ok=True)
from concurrent.futures import ThreadPoolExecutor  # noqa: E402


def one(spec):
    name, _, defs = spec.partition(":")
    out = os.path.join(ROOT, "variants", f"lib_{name}.so")
    build.build(out=out, defines=tuple(d for d in defs.split(",") if d))
    return out


with ThreadPoolExecutor(8) as ex:
    for out in ex.map(one, sys.argv[1:]):
        print(out)
