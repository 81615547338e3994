#!/usr/bin/env python
"""The paper's threshold calibration, re-run on B200 (PAPER.md:28.s17-34, §VII.B).

X7 (T2): per-iteration device time of the thread mapping vs the block mapping over the queue
(T_QU vs B_QU) as a function of |WS| — the paper sets T2 where the block mapping stops losing on
small working sets (28.s24-27).  Rows: config, source, iteration, |WS|, m_F, us(T_QU), us(B_QU).

X8 (T3): total time of the paper policy with T3 swept over 1..13% of V on the uniform-degree graph
(C4; the paper's Fig. 13 sweep on Amazon-like graphs, 28.s31-34).

Every run is checked against the oracle results (--expect, from `python -m tests.oracle_expect`)
before its time is kept.

    python tools/calibrate.py --x7 --config C2 --expect gpurun_out/expect_C2.npz
    python tools/calibrate.py --x8 --config C4 --expect gpurun_out/expect_C4.npz
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


def run(G, alg, s, p, expect, trace=False):
    fn = G.bfs if alg == "bfs" else G.sssp
    best = None
    for _ in range(2):
        out, _, st = fn(s, policy=p, stats=True, trace_cap=1 << 16 if trace else 0)
        if expect is not None and not np.array_equal(out, expect[f"{alg}_{s}"]):
            return None
        if best is None or st.device_ms < best.device_ms:
            best = st
    return best


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C2")
    ap.add_argument("--x7", action="store_true")
    ap.add_argument("--x8", action="store_true")
    ap.add_argument("--sources", type=int, default=2)
    ap.add_argument("--expect", default="")
    ap.add_argument("--alg", default="bfs,sssp")
    a = ap.parse_args()
    expect = np.load(a.expect) if a.expect else None
    g = aggen.config(a.config)
    G = A.Graph.from_csr(g)
    srcs = [int(s) for s in aggen.sources(g, a.sources, seed=3)]
    if a.x7:
        for alg in a.alg.split(","):
            for s in srcs:
                res = {}
                for m in (A.MAP_THREAD, A.MAP_CTA):
                    p = A.policy_default(0)
                    p.kind = A.POLICY_PAPER   # both forced variants in the same (general) kernel
                    p.mapping, p.workset = m, A.WS_QUEUE
                    st = run(G, alg, s, p, expect, trace=True)
                    res[m] = st
                if any(v is None for v in res.values()):
                    print(json.dumps({"x": "X7", "config": a.config, "alg": alg, "source": s, "verified": False}), flush=True)
                    continue
                t, b = res[A.MAP_THREAD], res[A.MAP_CTA]
                for i in range(min(len(t.trace_ws), len(b.trace_ws))):
                    if int(t.trace_ws[i]) != int(b.trace_ws[i]):
                        break   # (unordered SSSP traces may diverge)
                    print(json.dumps({"x": "X7", "config": a.config, "alg": alg, "source": s, "it": i,
                                      "ws": int(t.trace_ws[i]), "edges": int(t.trace_edges[i]),
                                      "us_T_QU": round(float(t.trace_us[i]), 2), "us_B_QU": round(float(b.trace_us[i]), 2),
                                      "verified": True}), flush=True)
    if a.x8:
        for alg in a.alg.split(","):
            for ppm in [10000, 20000, 30000, 40000, 50000, 60000, 70000, 80000, 90000, 100000, 110000, 120000, 130000]:
                ms = []
                ok = True
                for s in srcs:
                    p = A.policy_default(0)
                    p.kind = A.POLICY_PAPER
                    p.t3_ppm = ppm
                    st = run(G, alg, s, p, expect)
                    if st is None:
                        ok = False
                        break
                    ms.append(st.device_ms)
                print(json.dumps({"x": "X8", "config": a.config, "alg": alg, "t3_pct": ppm / 1e4,
                                  "ms_median": statistics.median(ms) if ok else None, "ms_all": [round(x, 3) for x in ms],
                                  "verified": ok}), flush=True)


if __name__ == "__main__":
    main()
