#!/usr/bin/env python
"""Per-iteration roofline table of one traversal from the device trace (trace_ns): |WS|, edges inspected,
microseconds, algorithmic bytes of the iteration (edges x 4 B col [+ 4 B weight for SSSP] + |WS| x
(row-offset pair + status word)), achieved GB/s and the fraction of the measured HBM peak.

    python tools/level_roofline.py --config C2 --alg bfs [--src-index 1] [--reps 3]
"""
import argparse
import json
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
    ap.add_argument("--reps", type=int, default=3)
    args = ap.parse_args()
    try:
        peak = float(json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"])
    except Exception:
        peak = 6650.0
    g = aggen.config(args.config, weighted=args.alg == "sssp")
    G = A.Graph.from_csr(g, weighted=args.alg == "sssp")
    s = int(aggen.sources(g, 64, seed=3)[args.src_index])
    fn = G.bfs if args.alg == "bfs" else G.sssp
    best = None
    for _ in range(args.reps):
        _, _, st = fn(s, stats=True, trace_cap=1 << 16)
        if best is None or st.device_ms < best.device_ms:
            best = st
    off = G.info.offset_bytes
    per_edge = 8 if args.alg == "sssp" else 4
    print(f"{args.config} {args.alg} src={s} total {best.device_ms:.3f} ms, {best.iterations} iterations, "
          f"E_r={best.reached_edges}, peak {peak:.0f} GB/s")
    print(f"{'it':>4} {'|WS|':>9} {'edges':>11} {'us':>8} {'alg MB':>8} {'GB/s':>7} {'frac':>6} {'share':>6}")
    tot = sum(best.trace_us)
    for i in range(len(best.trace_ws)):
        ws, e, us = int(best.trace_ws[i]), int(best.trace_edges[i]), float(best.trace_us[i])
        b = e * per_edge + ws * (2 * off + 4)
        gbs = b / (us * 1e-6) / 1e9 if us > 0 else 0.0
        print(f"{i:4d} {ws:9d} {e:11d} {us:8.1f} {b / 1e6:8.1f} {gbs:7.0f} {gbs / peak:6.3f} {us / tot:6.1%}")


if __name__ == "__main__":
    main()
