"""Write the oracle's results for a config's seeded sources to an .npz (test infrastructure).

    python -m tests.oracle_expect --config C2 --sources 2 [--seed 3] -o gpurun_out/expect_C2.npz

tools/sweep.py --expect <file> compares every timed run element by element against these arrays
before it records a time (the static-vs-adaptive table only lists verified runs).  Only this
script touches oracle/; the sweep reads plain arrays.
"""
import argparse
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

import aggen  # noqa: E402
import oracle  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C2")
    ap.add_argument("--sources", type=int, default=2)
    ap.add_argument("--seed", type=int, default=3)
    ap.add_argument("-o", "--out", required=True)
    a = ap.parse_args()
    g = aggen.config(a.config)
    srcs = [int(s) for s in aggen.sources(g, a.sources, seed=a.seed)]
    arrs = {"sources": np.array(srcs, np.uint32)}
    for s in srcs:
        arrs[f"bfs_{s}"] = oracle.bfs(g, s, want_parents=False)[0]
        arrs[f"sssp_{s}"] = oracle.dijkstra(g, s, want_parents=False)[0]
    np.savez(a.out, **arrs)
    print(f"wrote {a.out}: {a.config} sources {srcs}")


if __name__ == "__main__":
    main()
