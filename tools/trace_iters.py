#!/usr/bin/env python
"""Per-iteration trace of one query: |WS|, edges inspected, device us, edges/us.

    python tools/trace_iters.py --config C2 --alg sssp [--src-index 1] [--set field=value ...]
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
    ap.add_argument("--src-index", type=int, default=1)
    ap.add_argument("--set", action="append", default=[])
    args = ap.parse_args()
    g = aggen.config(args.config, weighted=args.alg == "sssp")
    G = A.Graph.from_csr(g, weighted=args.alg == "sssp")
    p = A.policy_default(0)
    for kv in args.set:
        k, v = kv.split("=")
        setattr(p, k, int(v))
    s = int(aggen.sources(g, 64, seed=3)[args.src_index])
    for rep in range(2):
        if args.alg == "cc":
            _, _, st = G.cc(policy=p, stats=True, trace_cap=4096)
        else:
            fn = G.bfs if args.alg == "bfs" else G.sssp
            _, _, st = fn(s, policy=p, stats=True, trace_cap=4096)
    print(f"{args.config} {args.alg} src={s} ms={st.device_ms:.3f} iters={st.iterations} "
          f"edges={st.edges_inspected} Er={st.reached_edges}")
    us = getattr(st, "trace_us", None)
    for i in range(len(st.trace_ws)):
        t = us[i] if us is not None else float("nan")
        e = int(st.trace_edges[i])
        print(f"  it {i:4d} ws {int(st.trace_ws[i]):9d} edges {e:10d} us {t:8.1f} "
              f"Medges/ms {e / max(t, 1e-3) / 1e3:8.1f} var {int(st.trace_variant[i])}")


if __name__ == "__main__":
    main()
