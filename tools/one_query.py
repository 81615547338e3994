#!/usr/bin/env python
"""Run a few queries of one config (target for ncu captures).

    python tools/one_query.py --config C2 --alg bfs --n 3 [--order 0] [--mapping 0 --workset 0 --kind 1]
"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import aggen  # noqa: E402
from paper_conf_ipps_lib13_b200 import agraph as A  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C2")
    ap.add_argument("--alg", default="bfs")
    ap.add_argument("--n", type=int, default=3)
    ap.add_argument("--order", type=int, default=0)
    ap.add_argument("--mapping", type=int, default=0)
    ap.add_argument("--workset", type=int, default=0)
    ap.add_argument("--kind", type=int, default=1)
    ap.add_argument("--delta", type=int, default=1)
    args = ap.parse_args()
    g = aggen.config(args.config)
    G = A.Graph.from_csr(g)
    p = A.policy_default(0)
    p.order, p.mapping, p.workset, p.kind, p.delta = args.order, args.mapping, args.workset, args.kind, args.delta
    srcs = aggen.sources(g, 64, seed=3)
    for k in range(args.n):
        fn = G.bfs if args.alg == "bfs" else G.sssp
        _, _, st = fn(int(srcs[k % 64]), policy=p, stats=True)
        print(f"{args.alg} src={int(srcs[k % 64])} ms={st.device_ms:.3f} iters={st.iterations} "
              f"Er={st.reached_edges} GTEPS={st.reached_edges / st.device_ms / 1e6:.1f}", flush=True)


if __name__ == "__main__":
    main()
