"""Summarise an ncu launch list (`--metrics gpu__time_duration.sum --csv`) per kernel.
usage: python scripts/launch_summary.py gpurun_out/<tag>_launches.csv > profiles/<tag>_launches_summary.md"""
import csv
import sys
from collections import defaultdict

rows = [r for r in csv.reader(open(sys.argv[1])) if len(r) > 10]
hdr = rows[0]
ki, mi, vi, ui = hdr.index("Kernel Name"), hdr.index("Metric Name"), hdr.index("Metric Value"), hdr.index("Metric Unit")
agg = defaultdict(lambda: [0, 0.0])
for r in rows[1:]:
    if r[mi] != "gpu__time_duration.sum":
        continue
    scale = {"nsecond": 1e-6, "ns": 1e-6, "usecond": 1e-3, "us": 1e-3, "msecond": 1.0, "ms": 1.0, "second": 1e3, "s": 1e3}[r[ui]]
    name = r[ki].replace("(int)", "").replace("(bool)", "")
    name = name.split("(gsword")[0][:70]
    agg[name][0] += 1
    agg[name][1] += float(r[vi].replace(",", "")) * scale
tot = sum(v[1] for v in agg.values())
print(f"# ncu launch list of `python bench.py --steps 2 --warmup 1 --no-cpu-baseline` (cold-cache, serialised;\n"
      f"# compare shares, not absolute times). Generated from {sys.argv[1].split('/')[-1]}.")
print("kernel | launches | total ms | share | mean us")
for k, (n, t) in sorted(agg.items(), key=lambda kv: -kv[1][1]):
    print(f"{k} | {n} | {t:.3f} | {t / tot:.3f} | {1e3 * t / n:.1f}")
