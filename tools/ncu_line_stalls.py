#!/usr/bin/env python
"""Stall-reason breakdown of the hottest CUDA source lines of an ncu report (first kernel).

    python tools/ncu_line_stalls.py report.ncu-rep [N]
"""
import csv
import io
import subprocess
import sys


def main():
    rep = sys.argv[1]
    top = int(sys.argv[2]) if len(sys.argv) > 2 else 15
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source=cuda,sass"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    fname, hdr, seen = None, None, set()
    agg = {}
    for r in rows:
        if not r:
            continue
        if r[0] == "File Path":
            fname = r[1].split("/")[-1]
            continue
        if r[0] == "Function Name":
            seen.add(r[1])
            if len(seen) > 1:
                break
            continue
        if r[0] == "Line No":
            hdr = r
            continue
        if hdr is None or len(r) != len(hdr) or r[2] != "-":
            continue
        col = {k: i for i, k in enumerate(hdr)}
        sc = [k for k in hdr if k.startswith("stall_") and "Not Issued" not in k]
        try:
            s = float(r[col["Warp Stall Sampling (All Samples)"]] or 0)
        except ValueError:
            continue
        a = agg.setdefault((fname, int(r[0])), {"s": 0.0, "src": r[1], "st": {}})
        a["s"] += s
        for k in sc:
            try:
                a["st"][k[6:]] = a["st"].get(k[6:], 0.0) + float(r[col[k]] or 0)
            except ValueError:
                pass
    tot = sum(v["s"] for v in agg.values()) or 1
    for (f, ln), a in sorted(agg.items(), key=lambda x: -x[1]["s"])[:top]:
        br = sorted(((v, k) for k, v in a["st"].items()), reverse=True)[:3]
        bs = ", ".join(f"{k}={v / max(a['s'], 1) * 100:.0f}%" for v, k in br if v > 0)
        print(f"{f}:{ln:<5d} {a['s'] / tot * 100:5.1f}%  [{bs}]  {a['src'].strip()[:80]}")


if __name__ == "__main__":
    main()
