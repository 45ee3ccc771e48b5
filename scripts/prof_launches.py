"""Summarise an ncu launch list (--metrics gpu__time_duration.sum,dram__bytes_read.sum,
dram__bytes_write.sum, --clock-control none) of one bench step into profiles/: a per-launch
markdown table and the traffic JSON bench.py reads for roofline.traffic.
usage: prof_launches.py launches.csv TAG bits batch"""
import csv
import json
import sys

path, tag, bits, batch = sys.argv[1], sys.argv[2], int(sys.argv[3]), int(sys.argv[4])
rows = list(csv.reader(open(path)))
k = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
hdr = rows[k]
iid, iname, imet, ival, iunit = (hdr.index(c) for c in ("ID", "Kernel Name", "Metric Name", "Metric Value",
                                                          "Metric Unit"))
launch = {}
for r in rows[k + 1:]:
    if len(r) <= ival:
        continue
    d = launch.setdefault(int(r[iid]), {"name": r[iname]})
    v = float(r[ival].replace(",", ""))
    u = r[iunit]
    if r[imet] == "gpu__time_duration.sum":
        v *= {"nsecond": 1e-3, "ns": 1e-3, "usecond": 1.0, "us": 1.0, "msecond": 1e3, "ms": 1e3}.get(u, 1.0)
        d["us"] = v
    else:
        v *= {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "KB": 1e3, "MB": 1e6, "GB": 1e9}.get(u, 1)
        d[r[imet]] = v
ids = sorted(launch)
conv = [launch[i] for i in ids if "qconv" in launch[i]["name"]]
tot_us = sum(d["us"] for d in launch.values())
lines = [f"ncu launch list `{path}` of one bench step (A{bits}W{bits}, batch {batch}; gpu__time_duration.sum, "
         "dram bytes; --clock-control none; cold-cache, serialised: compare SHARES)\n",
         "| # | kernel | us | share | DRAM MB |", "|---|---|---|---|---|"]
for n, i in enumerate(ids):
    d = launch[i]
    mb = (d.get("dram__bytes_read.sum", 0) + d.get("dram__bytes_write.sum", 0)) / 1e6
    lines.append(f"| {n} | {d['name'].split('(')[0][:70]} | {d['us']:.1f} | {100 * d['us'] / tot_us:.1f}% | {mb:.1f} |")
open(f"profiles/{tag}_launches.md", "w").write("\n".join(lines) + "\n")
traffic = sum(d.get("dram__bytes_read.sum", 0) + d.get("dram__bytes_write.sum", 0) for d in conv)
json.dump({"source": f"ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum over one "
                     f"bench step ({path}), A{bits}W{bits} batch {batch}",
           "conv_dram_bytes_per_step": traffic, "conv_launches": len(conv), "bits": bits, "batch": batch,
           "conv_us_serialised": sum(d["us"] for d in conv)},
          open(f"profiles/{tag}_traffic.json", "w"), indent=1)
print(tag, len(launch), "launches", len(conv), "conv", round(traffic / 1e9, 3), "GB conv DRAM", round(tot_us, 1), "us")
