#!/usr/bin/env python
"""Warp-level instructions executed per CUDA source line of an ncu report (first kernel), top N.

    python tools/ncu_line_insts.py report.ncu-rep [N]
"""
import csv
import io
import subprocess
import sys


def main():
    rep = sys.argv[1]
    top = int(sys.argv[2]) if len(sys.argv) > 2 else 30
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source=cuda,sass"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    fname, hdr, seen, agg = None, None, set(), {}
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
        try:
            ex = float(r[col["Instructions Executed"]] or 0)
        except ValueError:
            continue
        a = agg.setdefault((fname, int(r[0])), [0.0, r[1]])
        a[0] += ex
    tot = sum(v[0] for v in agg.values()) or 1
    print(f"total warp instructions {tot:.0f}")
    for (f, ln), (ex, src) in sorted(agg.items(), key=lambda x: -x[1][0])[:top]:
        print(f"{f}:{ln:<5d} {ex / tot * 100:5.1f}%  {ex:12.0f}  {src.strip()[:90]}")


if __name__ == "__main__":
    main()
