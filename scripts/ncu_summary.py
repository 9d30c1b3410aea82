#!/usr/bin/env python
"""Summarise ncu outputs into profiles/: launch-list shares and key metrics
of full captures.  Usage: ncu_summary.py <gpurun_out/tag> <profiles/tag>"""
import collections
import csv
import json
import os
import subprocess
import sys

src, dst = sys.argv[1], sys.argv[2]
os.makedirs(dst, exist_ok=True)
out = []
lc = os.path.join(src, "launches.csv")
if os.path.exists(lc):
    rows = [r for r in csv.reader(open(lc)) if len(r) > 10]
    h = rows[0]
    ki, vi, ui, gi = h.index("Kernel Name"), h.index("Metric Value"), h.index("Metric Unit"), h.index("Grid Size")
    agg = collections.defaultdict(lambda: [0, 0.0])
    scale = {"ns": 1e-3, "nsecond": 1e-3, "us": 1.0, "usecond": 1.0, "ms": 1e3, "msecond": 1e3}
    for r in rows[1:]:
        name = r[ki].split("(")[0].strip() + f" grid={r[gi]}"
        agg[name][0] += 1
        agg[name][1] += float(r[vi].replace(",", "")) * scale[r[ui]]
    tot = sum(v[1] for v in agg.values())
    out.append("# ncu launch list (gpu__time_duration.sum, --clock-control none; cold-cache, serialised)")
    out.append(f"{'kernel':90s} {'n':>5s} {'total_us':>12s} {'avg_us':>10s} {'share':>7s}")
    for k, v in sorted(agg.items(), key=lambda x: -x[1][1]):
        out.append(f"{k[:90]:90s} {v[0]:5d} {v[1]:12.1f} {v[1] / v[0]:10.2f} {v[1] / tot:7.4f}")
    out.append("")
WANT = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum", "dram__bytes.sum.per_second",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "lts__throughput.avg.pct_of_peak_sustained_elapsed", "l1tex__throughput.avg.pct_of_peak_sustained_active",
        "launch__registers_per_thread", "launch__grid_size", "launch__block_size", "launch__occupancy_limit_registers",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active", "smsp__inst_executed.sum",
        "sm__cycles_elapsed.avg.per_second", "launch__shared_mem_per_block_dynamic"]
traffic = {}
for f in sorted(os.listdir(src)):
    if not f.endswith(".ncu-rep"):
        continue
    raw = subprocess.run(["ncu", "-i", os.path.join(src, f), "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(raw.splitlines()))
    if len(rows) < 3:
        continue
    h, u = rows[0], rows[1]
    for v in rows[2:]:
        kn = v[h.index("Kernel Name")] if "Kernel Name" in h else f
        out.append(f"# {f}: {kn[:120]}")
        for w in WANT:
            if w in h:
                i = h.index(w)
                out.append(f"  {w:65s} {v[i]:>22s} {u[i]}")
        if "dram__bytes_read.sum" in h:
            def tobytes(i):
                x = float(v[i].replace(",", ""))
                return x * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}.get(u[i], 1)
            traffic[f] = tobytes(h.index("dram__bytes_read.sum")) + tobytes(h.index("dram__bytes_write.sum"))
            out.append(f"  dram read+write bytes per launch: {traffic[f]:.6g}")
        out.append("")
open(os.path.join(dst, "ncu_summary.txt"), "w").write("\n".join(out) + "\n")
json.dump(traffic, open(os.path.join(dst, "dram_traffic.json"), "w"), indent=1)
print("\n".join(out))
