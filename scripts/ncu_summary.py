#!/usr/bin/env python
"""Summarise an ncu report (--set full) or a launch-list CSV into markdown for profiles/.

usage: ncu_summary.py full  <report.ncu-rep> [names.txt]  > profiles/<round>_full.md
       ncu_summary.py launches <launches.csv>             > profiles/<round>_launches.md
"""
import csv
import io
import subprocess
import sys

METRICS = [
    ("gpu__time_duration.sum", "time"),
    ("dram__bytes_read.sum", "dram rd"),
    ("dram__bytes_write.sum", "dram wr"),
    ("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "dram %"),
    ("sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active", "tensor %"),
    ("sm__throughput.avg.pct_of_peak_sustained_elapsed", "SM %"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "warps act %"),
    ("launch__registers_per_thread", "regs"),
    ("smsp__inst_executed.sum", "inst"),
    ("launch__grid_size", "grid"),
    ("launch__block_size", "block"),
]


def full(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True,
                         text=True, check=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    tensor_cols = [h for h in hdr if "pipe_tensor" in h and "pct_of_peak_sustained_active" in h]
    cols = [(m, n) for m, n in METRICS if m in hdr]
    if "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active" not in hdr and tensor_cols:
        cols.insert(4, (tensor_cols[0], "tensor %"))
    print(f"ncu --set full report `{rep}`\n")
    print("| # | kernel | " + " | ".join(f"{n} ({units[hdr.index(m)]})" for m, n in cols) + " |")
    print("|" + "---|" * (len(cols) + 2))
    for i, r in enumerate(rows[2:]):
        name = r[hdr.index("Kernel Name")][:40]
        print(f"| {i} | {name} | " + " | ".join(r[hdr.index(m)] for m, _ in cols) + " |")


def launches(path):
    rows = list(csv.reader(open(path)))
    # find header row
    k = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
    hdr = rows[k]
    iname, imet, ival = hdr.index("Kernel Name"), hdr.index("Metric Name"), hdr.index("Metric Value")
    iunit = hdr.index("Metric Unit")
    agg = {}
    order = []
    for r in rows[k + 1:]:
        if len(r) <= ival or r[imet] != "gpu__time_duration.sum":
            continue
        nm = r[iname].split("(")[0]
        v = float(r[ival].replace(",", ""))
        if r[iunit] in ("usecond", "us"):
            v *= 1e3
        elif r[iunit] in ("msecond", "ms"):
            v *= 1e6
        if nm not in agg:
            agg[nm] = [0, 0.0]
            order.append(nm)
        agg[nm][0] += 1
        agg[nm][1] += v
    tot = sum(v for _, v in agg.values())
    print(f"ncu launch list `{path}` (gpu__time_duration.sum, --clock-control none; cold, serialised)\n")
    print("| kernel | launches | total us | share |")
    print("|---|---|---|---|")
    for nm in sorted(order, key=lambda n: -agg[n][1]):
        c, v = agg[nm]
        print(f"| {nm} | {c} | {v / 1e3:.1f} | {100 * v / tot:.1f}% |")


if __name__ == "__main__":
    {"full": full, "launches": launches}[sys.argv[1]](sys.argv[2])
