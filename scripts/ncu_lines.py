"""Summarise an ncu report's source page per CUDA line: warp-stall samples,
instructions executed and the average active threads per executed instruction.
usage: python scripts/ncu_lines.py report.ncu-rep [kernel-substring] [top]"""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
want = sys.argv[2] if len(sys.argv) > 2 else ""
top = int(sys.argv[3]) if len(sys.argv) > 3 else 25
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
kernel = None
blocks = {}
hdrs = {}  # the source page's column set can differ per kernel
hdr = None
for row in csv.reader(io.StringIO(out)):
    if not row:
        continue
    if row[0] == "Function Name":
        kernel = row[1]
        blocks.setdefault(kernel, [])
        continue
    if row[0] == "Line No":
        hdr = row
        if kernel is not None:
            hdrs[kernel] = row
        continue
    if hdr and kernel and row[0].isdigit() and len(row) == len(hdr) and row[2] == "-":
        blocks[kernel].append(row)
for k, rows in blocks.items():
    if want not in k:
        continue
    hdr = hdrs[k]
    i_st = hdr.index("Warp Stall Sampling (All Samples)")
    i_ie = hdr.index("Instructions Executed")
    i_te = hdr.index("Thread Instructions Executed")
    names = [h for h in hdr if h.startswith("stall_") and "Not Issued" not in h]
    tot_st = sum(float(r[i_st] or 0) for r in rows) or 1
    tot_ie = sum(float(r[i_ie] or 0) for r in rows) or 1
    print(f"== {k[:110]}\n   stall samples {tot_st:.0f}, warp instructions {tot_ie:.3e}")
    rows.sort(key=lambda r: -float(r[i_st] or 0))
    for r in rows[:top]:
        st, ie, te = float(r[i_st] or 0), float(r[i_ie] or 0), float(r[i_te] or 0)
        reasons = sorted(((float(r[hdr.index(n)] or 0), n[6:]) for n in names), reverse=True)[:2]
        rs = ",".join(f"{n}:{v / max(st, 1):.0%}" for v, n in reasons if v > 0)
        print(f"  L{r[0]:>4} stall {st / tot_st:6.1%} inst {ie / tot_ie:6.1%} thr/inst {te / max(ie, 1):5.1f} "
              f"[{rs}] {r[1].strip()[:70]}")
