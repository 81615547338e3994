#!/usr/bin/env python
"""Per-CUDA-source-line warp-stall attribution from an ncu report (first kernel of the report).

    python tools/ncu_lines.py report.ncu-rep [--top N]
"""
import csv
import io
import subprocess
import sys


def main():
    rep = sys.argv[1]
    top = int(sys.argv[sys.argv.index("--top") + 1]) if "--top" in sys.argv else 40
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source=cuda,sass"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    fname, fn, hdr = None, None, None
    agg = {}
    seen_fn = set()
    for r in rows:
        if not r:
            continue
        if r[0] == "File Path":
            fname = r[1].split("/")[-1]
            continue
        if r[0] == "Function Name":
            fn = r[1]
            seen_fn.add(fn)
            if len(seen_fn) > 1:
                break
            continue
        if r[0] == "Line No":
            hdr = r
            continue
        if hdr is None or len(r) != len(hdr) or r[2] != "-":
            continue
        try:
            s = float(r[4])
            ex = float(r[7])
        except ValueError:
            continue
        k = (fname, int(r[0]))
        a = agg.setdefault(k, [0.0, 0.0, r[1]])
        a[0] += s
        a[1] += ex
    tot = sum(v[0] for v in agg.values()) or 1
    for (f, ln), (s, ex, src) in sorted(agg.items(), key=lambda x: -x[1][0])[:top]:
        print(f"{f}:{ln:<5d} {s / tot * 100:5.1f}%  ex={ex:>12.0f}  {src.strip()[:100]}")


if __name__ == "__main__":
    main()
