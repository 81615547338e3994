#!/usr/bin/env python
"""Per-instruction memory table of an ncu report: every global memory instruction with its executions,
L1 tag requests, L2 theoretical sectors (ideal / excessive) and stall share, sorted by L2 sectors.

    python tools/ncu_mem_insts.py report.ncu-rep [N]
"""
import csv
import io
import subprocess
import sys


def main():
    rep = sys.argv[1]
    n = int(sys.argv[2]) if len(sys.argv) > 2 else 30
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source=sass"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr = rows[1]
    col = {k: hdr.index(k) for k in hdr}

    def f(r, k):
        try:
            return float(r[col[k]].replace(',', '') or 0)
        except (ValueError, IndexError):
            return 0.0
    data = [r for r in rows[2:] if len(r) == len(hdr)]
    tot_st = sum(f(r, "Warp Stall Sampling (All Samples)") for r in data) or 1
    tot_l2 = sum(f(r, "L2 Theoretical Sectors Global") for r in data) or 1
    mem = [r for r in data if f(r, "L1 Tag Requests Global") > 0 or f(r, "L2 Theoretical Sectors Global") > 0]
    mem.sort(key=lambda r: -f(r, "L2 Theoretical Sectors Global"))
    print(f"{'idx':>5} {'exec':>10} {'L1tagreq':>10} {'L2sect':>11} {'%L2':>5} {'sect/req':>8} {'stall%':>6}  sass")
    for r in mem[:n]:
        ex = f(r, "Instructions Executed")
        l1 = f(r, "L1 Tag Requests Global")
        l2 = f(r, "L2 Theoretical Sectors Global")
        st = f(r, "Warp Stall Sampling (All Samples)")
        print(f"{data.index(r):5d} {ex:10.0f} {l1:10.0f} {l2:11.0f} {l2 / tot_l2 * 100:5.1f} {l2 / max(ex, 1):8.1f} "
              f"{st / tot_st * 100:6.1f}  {r[col['Source']][:90]}")
    print(f"total L2 theoretical sectors {tot_l2:.0f}")


if __name__ == "__main__":
    main()
