#!/usr/bin/env python
"""Summarise tools/sweep.py output: per (config, algorithm, order) the best static variant against the
paper's and the tuned adaptive policies (the paper's Tables 2/3 comparison, re-run on B200).

    python tools/sweep_table.py profiles/sweeps/r01_static_C2.jsonl [...]
"""
import json
import sys


def main(paths):
    print("| config | alg | order | best static, paper kernels (ms) | adaptive paper (ms) | best static, tuned kernels (ms)"
          " | adaptive tuned (ms) | tuned adaptive / best static |")
    print("|---|---|---|---|---|---|---|---|")
    for path in paths:
        cfg, rows = None, []
        for line in open(path):
            line = line.strip()
            if not line.startswith("{"):
                continue
            r = json.loads(line)
            if "config" in r:
                cfg = r["config"]
            elif "ms_median" in r:
                rows.append(r)
            elif r.get("verified") is False:
                print(f"<!-- NOT VERIFIED: {path}: {r} -->")
        for alg in ("bfs", "sssp"):
            for order in ("U", "O"):
                sel = [r for r in rows if r["alg"] == alg and r["variant"].startswith(order + "_")]
                static = [r for r in sel if "adaptive" not in r["variant"]]
                if not static:
                    continue
                best = min(static, key=lambda r: r["ms_median"])
                sp = [r for r in static if r["variant"].endswith("_paper")]
                st = [r for r in static if not r["variant"].endswith("_paper")]
                bp = min(sp, key=lambda r: r["ms_median"]) if sp else None
                bt = min(st, key=lambda r: r["ms_median"]) if st else None
                ap = next((r for r in sel if r["variant"].endswith("adaptive_paper")), None)
                at = next((r for r in sel if r["variant"].endswith("adaptive_tuned")), None)
                ad = next((r for r in sel if r["variant"].endswith("adaptive_tuned_delta0")), None)
                if ad and at and ad["ms_median"] < at["ms_median"]:
                    at = dict(ad, ms_median=ad["ms_median"])   # the adaptive-delta tuned run, when better
                f = lambda r: (f"{r['ms_median']:.3f}" + (" (delta adaptive)" if r.get("variant", "").endswith("delta0") else "")) if r else "-"
                g = lambda r: f"{r['variant']} {r['ms_median']:.3f}" if r else "-"
                ratio = f"{at['ms_median'] / best['ms_median']:.2f}" if at else "-"
                print(f"| {cfg} | {alg} | {order} | {g(bp)} | {f(ap)} | {g(bt)} | {f(at)} | {ratio} |")


if __name__ == "__main__":
    main(sys.argv[1:])
