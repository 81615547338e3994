#!/usr/bin/env python
"""Static-variant vs adaptive sweep (the paper's Tables 2/3 study, X4/X5, re-run on B200).

    python tools/sweep.py --config C2 [--sources 4] [--alg bfs,sssp] [--trace] [--variants ...]

For each variant (order x mapping x workset, plus the paper and tuned adaptive policies) prints the
median device time over the sources, GTEPS (E_r / t), iterations and optionally the per-iteration
trace (|WS|, edges, variant, microseconds).  Device times come from the library's CUDA events.

--expect FILE (written by `python -m tests.oracle_expect`, the oracle's levels / distances for the
same seeded sources): every run's output is compared element by element before its time is kept;
a mismatch is recorded as {"verified": false, ...} with no time.  Rows carry "verified": true.
"""
import argparse
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import aggen  # noqa: E402
from paper_conf_ipps_lib13_b200 import agraph as A  # noqa: E402


def variants(orders, kinds=(1,)):
    out = []
    for o in orders:
        for k in kinds:
            for m in (1, 2, 3, 4):
                for w in (1, 2):
                    name = f"{'O' if o else 'U'}_{A.MAP_LETTER[m]}_{A.WS_NAME[w]}" + ("" if k == 1 else "_paper")
                    out.append((name, dict(order=o, mapping=m, workset=w, kind=k)))
        out.append((f"{'O' if o else 'U'}_adaptive_paper", dict(order=o, kind=0)))
        out.append((f"{'O' if o else 'U'}_adaptive_tuned", dict(order=o, kind=1)))
        if o:   # NEXT-3: the ordered bucket width adapted per iteration
            out.append(("O_adaptive_tuned_delta0", dict(order=1, kind=1, delta=0)))
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C2")
    ap.add_argument("--sources", type=int, default=4)
    ap.add_argument("--alg", default="bfs,sssp")
    ap.add_argument("--orders", default="0,1")
    ap.add_argument("--kinds", default="1", help="policy kinds of the static variants: 0 paper kernels, 1 tuned")
    ap.add_argument("--trace", action="store_true")
    ap.add_argument("--only", default="")
    ap.add_argument("--reps", type=int, default=2)
    ap.add_argument("--delta", type=int, default=1)
    ap.add_argument("--set", default="", help="extra policy fields k=v,k=v")
    ap.add_argument("--expect", default="", help="oracle results (.npz from tests/oracle_expect.py)")
    args = ap.parse_args()
    expect = np.load(args.expect) if args.expect else None
    g = aggen.config(args.config)
    G = A.Graph.from_csr(g)
    srcs = [int(s) for s in aggen.sources(g, args.sources, seed=3)]
    extra = dict(kv.split("=") for kv in args.set.split(",") if kv)
    print(json.dumps({"config": args.config, "V": g.V, "E": g.E, "max_deg": G.info.max_deg}), flush=True)
    for alg in args.alg.split(","):
        for name, kw in variants([int(x) for x in args.orders.split(",")],
                                 [int(x) for x in args.kinds.split(",")]):
            if args.only and not any(t in name for t in args.only.split(",")):
                continue
            if alg == "bfs" and kw.get("order") == 1 and False:
                continue
            p = A.policy_default(0)
            p.delta = args.delta
            for k, v in kw.items():
                setattr(p, k, v)
            for k, v in extra.items():
                setattr(p, k, int(v))
            times, edges, iters, traces, red = [], [], [], [], []
            bad = None
            try:
                for s in srcs:
                    best = None
                    for _ in range(args.reps):
                        fn = G.bfs if alg == "bfs" else G.sssp
                        out, _, st = fn(s, policy=p, stats=True, trace_cap=1 << 20 if args.trace else 0)
                        if expect is not None and not np.array_equal(out, expect[f"{alg}_{s}"]):
                            bad = (s, int(np.count_nonzero(out != expect[f"{alg}_{s}"])))
                        if best is None or st.device_ms < best.device_ms:
                            best = st
                    times.append(best.device_ms)
                    edges.append(best.reached_edges)
                    iters.append(best.iterations)
                    red.append(best.edges_inspected / max(1, best.reached_edges))
                    if args.trace:
                        traces.append([(int(a), int(b), A.variant_name(int(c)), round(float(d), 1))
                                       for a, b, c, d in zip(best.trace_ws, best.trace_edges, best.trace_variant,
                                                             best.trace_us)][:64])
            except A.AgError as e:
                print(json.dumps({"alg": alg, "variant": name, "error": str(e)}), flush=True)
                continue
            if bad is not None:
                print(json.dumps({"alg": alg, "variant": name, "verified": False, "source": bad[0],
                                  "mismatches": bad[1]}), flush=True)
                continue
            rec = {"alg": alg, "variant": name, "verified": expect is not None, "ms_median": statistics.median(times),
                   "gteps": sum(edges) / (sum(times) * 1e-3) / 1e9, "iters": statistics.median(iters),
                   "redundancy": round(statistics.median(red), 3),
                   "ms_all": [round(t, 3) for t in times]}
            if args.trace:
                rec["trace"] = traces[0]
            print(json.dumps(rec), flush=True)


if __name__ == "__main__":
    main()
