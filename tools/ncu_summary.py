#!/usr/bin/env python
"""Summarise an ncu report: key metrics + top stall reasons + hottest SASS lines.

    python tools/ncu_summary.py report.ncu-rep [--sass N]
"""
import csv
import io
import subprocess
import sys

KEYS = ['gpu__time_duration.sum', 'dram__bytes_read.sum', 'dram__bytes_write.sum',
        'dram__throughput.avg.pct_of_peak_sustained_elapsed', 'lts__t_sector_hit_rate.pct',
        'l1tex__t_sector_hit_rate.pct', 'sm__warps_active.avg.pct_of_peak_sustained_active',
        'smsp__thread_inst_executed_per_inst_executed.ratio', 'smsp__inst_executed.sum', 'lts__t_sectors.sum',
        'lts__throughput.avg.pct_of_peak_sustained_elapsed', 'l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum',
        'l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum', 'sm__throughput.avg.pct_of_peak_sustained_elapsed',
        'l1tex__throughput.avg.pct_of_peak_sustained_active', 'launch__registers_per_thread', 'launch__grid_size',
        'smsp__inst_executed_op_global_atom.sum', 'smsp__inst_executed_op_global_red.sum',
        'lts__t_sectors_op_atom.sum', 'lts__t_sectors_op_red.sum', 'lts__t_sectors_op_read.sum']


def ncu(args):
    return subprocess.run(["ncu", "-i"] + args, capture_output=True, text=True).stdout


def main():
    rep = sys.argv[1]
    nsass = int(sys.argv[sys.argv.index("--sass") + 1]) if "--sass" in sys.argv else 0
    rows = list(csv.reader(io.StringIO(ncu([rep, "--page", "raw", "--csv"]))))
    hdr, units = rows[0], rows[1]
    for vals in rows[2:]:
        print("--- kernel:", vals[hdr.index("Kernel Name")][:80] if "Kernel Name" in hdr else "?")
        for k in KEYS:
            if k in hdr:
                i = hdr.index(k)
                print(f"  {k:60s} {vals[i]:>16s} {units[i]}")

        def f(x):
            try:
                return float(x.replace(',', ''))
            except ValueError:
                return 0.0
        st = [(hdr[i], f(vals[i])) for i in range(len(hdr))
              if hdr[i].startswith('smsp__pcsamp_warps_issue_stalled') and not hdr[i].endswith('not_issued')]
        tot = sum(v for _, v in st) or 1
        print("  stall samples:", ", ".join(f"{k.replace('smsp__pcsamp_warps_issue_stalled_', '')}={v / tot:.0%}"
                                           for k, v in sorted(st, key=lambda x: -x[1])[:7]))
    if nsass:
        rows = list(csv.reader(io.StringIO(ncu([rep, "--page", "source", "--csv", "--print-source=sass"]))))
        hdr = rows[1]
        data = [r for r in rows[2:] if len(r) == len(hdr) and r[hdr.index("Warp Stall Sampling (All Samples)")].replace('.', '', 1).isdigit()]
        iss = hdr.index("Warp Stall Sampling (All Samples)")
        isrc = hdr.index("Source")
        iex = hdr.index("Instructions Executed")
        tot = sum(float(r[iss] or 0) for r in data) or 1
        top = sorted(range(len(data)), key=lambda i: -float(data[i][iss] or 0))[:nsass]
        for i in sorted(top):
            r = data[i]
            print(f"  {i:5d} {float(r[iss]) / tot * 100:5.1f}%  ex={r[iex]:>10}  {r[isrc][:100]}")


if __name__ == "__main__":
    main()
