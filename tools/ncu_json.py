"""Per-kernel JSON summary of an ncu report: DRAM bytes, time, issue/occupancy, top stall reasons."""
import csv
import io
import json
import subprocess
import sys

SCALE = {"Gbyte": 1e9, "Mbyte": 1e6, "Kbyte": 1e3, "byte": 1.0}
TSCALE = {"msecond": 1e3, "usecond": 1.0, "nsecond": 1e-3}


def summarise(path):
    raw = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    hdr, units = rows[0], rows[1]
    out = []
    for r in rows[2:]:
        def g(m, scale=SCALE):
            i = hdr.index(m)
            return float(r[i].replace(",", "")) * scale.get(units[i], 1.0)
        st = [(h, r[i]) for i, h in enumerate(hdr) if "smsp__pcsamp_warps_issue_stalled" in h and not h.endswith("not_issued")]
        vals = sorted(((float(v.replace(",", "") or 0), k.replace("smsp__pcsamp_warps_issue_stalled_", ""))
                       for k, v in st if v not in ("", "n/a")), reverse=True)
        tot = sum(v for v, _ in vals) or 1.0
        out.append(dict(kernel=r[hdr.index("Kernel Name")].split("(")[0],
                        time_us=g("gpu__time_duration.sum", TSCALE),
                        dram_read=g("dram__bytes_read.sum"), dram_write=g("dram__bytes_write.sum"),
                        issue_active_pct=g("smsp__issue_active.avg.pct_of_peak_sustained_active"),
                        warps_active_pct=g("sm__warps_active.avg.pct_of_peak_sustained_active"),
                        warp_inst=g("smsp__inst_executed.sum"),
                        stalls={k: round(v / tot, 3) for v, k in vals[:8]}))
    return out


if __name__ == "__main__":
    print(json.dumps(summarise(sys.argv[1]), indent=1))
