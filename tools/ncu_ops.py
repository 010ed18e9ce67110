"""Warp instructions and stall samples per SASS opcode of one kernel (ncu source page):
    python tools/ncu_ops.py report.ncu-rep [top_n]"""
import csv
import io
import subprocess
import sys

raw = subprocess.run(["ncu", "-i", sys.argv[1], "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(raw)))
hdr = next(r for r in rows if r and r[0] == "Address")
data = [r for r in rows[rows.index(hdr) + 1:] if len(r) == len(hdr)]
iS, iI = hdr.index("Warp Stall Sampling (All Samples)"), hdr.index("Instructions Executed")
agg = {}
for r in data:
    op = r[1].strip().split()
    op = (op[1] if op[0].startswith("@") else op[0]).split(".")[0]
    a = agg.setdefault(op, [0.0, 0.0])
    a[0] += float(r[iI] or 0)
    a[1] += float(r[iS] or 0)
T = sum(a[0] for a in agg.values()) or 1
TS = sum(a[1] for a in agg.values()) or 1
print(f"total warp instructions {T:.4g}, stall samples {TS:.4g}")
for k, a in sorted(agg.items(), key=lambda x: -x[1][0])[: int(sys.argv[2]) if len(sys.argv) > 2 else 25]:
    print(f"{k:12s} inst {100 * a[0] / T:5.2f}%  samples {100 * a[1] / TS:5.2f}%")
