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
    ap.add_argument("--set", action="append", default=[], help="policy field=value")
    ap.add_argument("--summary", action="store_true", help="print one median line (skips the first query)")
    args = ap.parse_args()
    g = aggen.config(args.config, weighted=args.alg == "sssp")
    G = A.Graph.from_csr(g, weighted=args.alg == "sssp")
    p = A.policy_default(0)
    p.order, p.mapping, p.workset, p.kind, p.delta = args.order, args.mapping, args.workset, args.kind, args.delta
    for kv in args.set:
        k, v = kv.split("=")
        setattr(p, k, int(v))
    srcs = aggen.sources(g, 64, seed=3)
    ms = []
    for k in range(args.n):
        if args.alg == "cc":
            _, _, st = G.cc(policy=p, stats=True)
        else:
            fn = G.bfs if args.alg == "bfs" else G.sssp
            _, _, st = fn(int(srcs[k % 64]), policy=p, stats=True)
        ms.append(st.device_ms)
        if not args.summary:
            print(f"{args.alg} src={int(srcs[k % 64])} ms={st.device_ms:.3f} iters={st.iterations} "
                  f"Er={st.reached_edges} GTEPS={st.reached_edges / st.device_ms / 1e6:.1f}", flush=True)
    if args.summary:
        import statistics
        t = ms[1:] if len(ms) > 1 else ms
        print(f"{args.config} {args.alg} {' '.join(args.set)} n={len(t)} median_ms={statistics.median(t):.3f} "
              f"mean_ms={statistics.mean(t):.3f} max_ms={max(t):.3f}", flush=True)


if __name__ == "__main__":
    main()
