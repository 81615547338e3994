#!/usr/bin/env python
"""Per-iteration CTA timing of one query, from a diagnostic build (-DAG_PROF):

    python -m paper_conf_ipps_lib13_b200.build --force -DAG_PROF --out=exp_libs/prof.so
    AGRAPH_LIB=$PWD/exp_libs/prof.so python tools/prof_iters.py --config C2 --alg bfs

For every iteration: |WS|, and in microseconds from the iteration's first CTA start: when the
first / median / last CTA finished its tile loop and its hub drain, and when the next iteration
started (= barrier release).  A large gap between the median and the last CTA is a tail.
"""
import argparse
import ctypes
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import aggen  # noqa: E402
from paper_conf_ipps_lib13_b200 import agraph as A  # noqa: E402

PROF_IT, PROF_CTA = 64, 2048


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C2")
    ap.add_argument("--alg", default="bfs")
    ap.add_argument("--src", type=int, default=0)
    args = ap.parse_args()
    g = aggen.config(args.config)
    G = A.Graph.from_csr(g)
    src = int(aggen.sources(g, 64, seed=3)[args.src])
    fn = G.bfs if args.alg == "bfs" else G.sssp
    for _ in range(2):
        _, _, st = fn(src, stats=True, trace_cap=256)
    buf = np.zeros((PROF_IT, PROF_CTA, 6), dtype=np.uint64)
    L = A.lib()
    L.ag_debug_prof.restype = ctypes.c_int
    L.ag_debug_prof.argtypes = [ctypes.c_void_p, ctypes.c_size_t]
    if L.ag_debug_prof(buf.ctypes.data, buf.nbytes) < 0:
        sys.exit("library built without -DAG_PROF")
    nb = int((buf[0, :, 0] > 0).sum())
    print(f"{args.config} {args.alg} src={src} ms={st.device_ms:.3f} iters={st.iterations} ctas={nb}")
    print(" it      |WS|   start->tiles done (first/med/last)   drains done (first/med/last)   next start"
          "   gated edges: slowest-tile CTA / max / median   hub tasks per CTA: min / med / max (last CTA)"
          "   first task at: min / med / max")
    for it in range(min(st.iterations, PROF_IT)):
        b = buf[it, :nb].astype(np.int64)
        t0 = b[:, 0].min()
        tiles, drain = (b[:, 1] - t0) / 1e3, (b[:, 2] - t0) / 1e3
        nxt = (buf[it + 1, :nb, 0].astype(np.int64).min() - t0) / 1e3 if it + 1 < st.iterations else float("nan")
        ws = int(st.trace_ws[it]) if it < len(st.trace_ws) else -1
        print(f"{it:3d} {ws:9d}   {tiles.min():7.1f} {np.median(tiles):7.1f} {tiles.max():7.1f}        "
              f"{drain.min():7.1f} {np.median(drain):7.1f} {drain.max():7.1f}       {nxt:7.1f}"
              f"   {int(b[np.argmax(tiles), 3]):9d} {int(b[:, 3].max()):9d} {int(np.median(b[:, 3])):9d}"
              f"   {int(b[:, 4].min()):4d} {int(np.median(b[:, 4])):4d} {int(b[:, 4].max()):4d} ({int(b[np.argmax(drain), 4]):4d})"
              + (lambda f: f"   {f.min():7.1f} {np.median(f):7.1f} {f.max():7.1f}" if f.size else "   -")(
                  (b[b[:, 5] > 0, 5] - t0) / 1e3))


if __name__ == "__main__":
    main()
