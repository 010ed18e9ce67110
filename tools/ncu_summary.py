"""Summarise an ncu report (--set full) or an ncu launch-list CSV into a short text table.

    python tools/ncu_summary.py report.ncu-rep        # per-kernel SOL / DRAM / L2 / occupancy
    python tools/ncu_summary.py launches.csv          # per-kernel launch count, avg time, share
"""
import csv
import io
import subprocess
import sys
from collections import defaultdict

METRICS = [
    ("gpu__time_duration.sum", "time_us", 1.0),
    ("dram__bytes_read.sum", "dram_rd_MB", 1.0),
    ("dram__bytes_write.sum", "dram_wr_MB", 1.0),
    ("gpu__compute_memory_throughput.avg.pct_of_peak_sustained_elapsed", "mem_sol%", 1.0),
    ("sm__throughput.avg.pct_of_peak_sustained_elapsed", "sm_sol%", 1.0),
    ("lts__throughput.avg.pct_of_peak_sustained_elapsed", "l2_sol%", 1.0),
    ("lts__t_sector_hit_rate.pct", "l2_hit%", 1.0),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "occup%", 1.0),
    ("launch__registers_per_thread", "regs", 1.0),
    ("smsp__inst_executed.sum", "warp_inst_M", 1e-6),
]


def report(path):
    raw = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    hdr, units = rows[0], rows[1]
    print("kernel".ljust(34) + "".join(n.rjust(12) for _, n, _ in METRICS))
    for r in rows[2:]:
        name = r[hdr.index("Kernel Name")].split("(")[0][:33]
        vals = []
        for m, _, sc in METRICS:
            if m not in hdr:
                vals.append("-")
                continue
            v = r[hdr.index(m)].replace(",", "")
            u = units[hdr.index(m)]
            try:
                x = float(v)
                if u == "Gbyte":
                    x *= 1e3
                elif u == "Kbyte":
                    x *= 1e-3
                elif u == "byte":
                    x *= 1e-6
                elif u == "msecond":
                    x *= 1e3
                elif u == "nsecond":
                    x *= 1e-3
                vals.append(f"{x * sc:.2f}")
            except ValueError:
                vals.append(v)
        print(name.ljust(34) + "".join(v.rjust(12) for v in vals))


def launches(path):
    rows = list(csv.reader(open(path)))
    hdr = None
    agg = defaultdict(list)
    for r in rows:
        if "Kernel Name" in r:
            hdr = r
            continue
        if hdr and len(r) == len(hdr):
            d = dict(zip(hdr, r))
            agg[d["Kernel Name"].split("(")[0]].append(float(d["Metric Value"].replace(",", "")))
    tot = sum(sum(v) for v in agg.values())
    print("kernel".ljust(34) + "launches".rjust(10) + "avg_us".rjust(12) + "share".rjust(8))
    for k, v in sorted(agg.items(), key=lambda kv: -sum(kv[1])):
        print(k[:33].ljust(34) + str(len(v)).rjust(10) + f"{sum(v) / len(v) / 1e3:12.1f}" + f"{sum(v) / tot:8.3f}")


if __name__ == "__main__":
    p = sys.argv[1]
    (report if p.endswith(".ncu-rep") else launches)(p)
