"""Summarise an ncu launch list (`--metrics gpu__time_duration.sum --csv`) per kernel.
usage: python scripts/launch_summary.py gpurun_out/<tag>_launches.csv > profiles/<tag>_launches_summary.md"""
import csv
import sys
from collections import defaultdict

rows = [r for r in csv.reader(open(sys.argv[1])) if len(r) > 10]
hdr = rows[0]
ki, mi, vi, ui = hdr.index("Kernel Name"), hdr.index("Metric Name"), hdr.index("Metric Value"), hdr.index("Metric Unit")
agg = defaultdict(lambda: [0, 0.0])
durs = defaultdict(list)
for r in rows[1:]:
    if r[mi] != "gpu__time_duration.sum":
        continue
    scale = {"nsecond": 1e-6, "ns": 1e-6, "usecond": 1e-3, "us": 1e-3, "msecond": 1.0, "ms": 1.0, "second": 1e3, "s": 1e3}[r[ui]]
    name = r[ki].replace("(int)", "").replace("(bool)", "")
    name = name.split("(gsword")[0][:70]
    agg[name][0] += 1
    agg[name][1] += float(r[vi].replace(",", "")) * scale
    durs[name].append(float(r[vi].replace(",", "")) * scale)
tot = sum(v[1] for v in agg.values())
print(f"# ncu launch list of `python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-qerror --no-cyclic`\n"
      f"# (cold-cache, serialised;\n"
      f"# compare shares, not absolute times). Generated from {sys.argv[1].split('/')[-1]}.")
print("kernel | launches | total ms | share | mean us")
for k, (n, t) in sorted(agg.items(), key=lambda kv: -kv[1][1]):
    print(f"{k} | {n} | {t:.3f} | {t / tot:.3f} | {1e3 * t / n:.1f}")

# The bench step = per method one estimate-mode sampling kernel at the bench size + the grid
# reduction.  The bench-size launches are the long ones of each estimate instantiation (autotune
# pilots run 1e6 / 8e6 samples): keep launches >= 40 % of that kernel's longest and compare the
# dominant kernel's share of the step with the bench line's kernel_ms / ms_per_step.
def step_ms(prefix):
    best = None
    for k, ds in durs.items():
        if k.startswith(prefix) and (best is None or sum(ds) > sum(durs[best])):
            best = k
    if best is None:
        return 0.0, None
    big = [d for d in durs[best] if d >= 0.4 * max(durs[best])]
    return sorted(big)[len(big) // 2], best

wj, kw = step_ms("void gsword::<unnamed>::sample_kernel<0, 0,")
al, ka = step_ms("void gsword::<unnamed>::sample_kernel<1, 0,")
red = [d for k, ds in durs.items() if "reduce_kernel" in k for d in ds]
rd = sorted(red)[len(red) // 2] if red else 0.0
step = wj + al + 2 * rd
if step > 0:
    print(f"\nstep (median bench-size launches): WanderJoin {wj:.3f} ms ({kw}), Alley {al:.3f} ms ({ka}), "
          f"2 x reduce {2 * rd:.3f} ms; Alley share of the step {al / step:.3f}, WanderJoin {wj / step:.3f}")
