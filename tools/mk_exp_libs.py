#!/usr/bin/env python
"""Build experiment variants of libagraph.so into exp_libs/ (A/B on the GPU with tools/cmp_libs.sh).

    python tools/mk_exp_libs.py [--keep] NAME=DEF1,DEF2 NAME2= ...   (empty define list = the default build;
                                                                   --keep: do not clear exp_libs/ first)
"""
import os
import sys
from concurrent.futures import ThreadPoolExecutor

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_ipps_lib13_b200 import build as B  # noqa: E402


def one(spec):
    name, _, defs = spec.partition("=")
    out = os.path.join(ROOT, "exp_libs", f"{name}.so")
    B.build(force=True, out=out, defines=[d for d in defs.split(",") if d])
    return out


if __name__ == "__main__":
    os.makedirs(os.path.join(ROOT, "exp_libs"), exist_ok=True)
    specs = [a for a in sys.argv[1:] if a != "--keep"]
    if "--keep" not in sys.argv:
        for f in os.listdir(os.path.join(ROOT, "exp_libs")):
            os.remove(os.path.join(ROOT, "exp_libs", f))
    with ThreadPoolExecutor(len(specs)) as ex:
        for o in ex.map(one, specs):
            print(o)
