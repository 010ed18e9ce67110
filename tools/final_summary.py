"""Assemble the round's ncu evidence from one tools/gpu_measure.sh output directory into the text summary
committed under profiles/:  python tools/final_summary.py gpurun_out/TAG "header line" > profiles/..._ncu_summary.txt
(per-kernel table, KBF limiter metrics, instructions / stalls by source region, stall reasons by region,
shared-memory wavefronts by source line, per-tile phase clocks, the launch list)."""
import contextlib
import csv
import io
import os
import re
import subprocess
import sys

sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
import ncu_phases  # noqa: E402
import ncu_stalls  # noqa: E402

LIMITERS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum", "smsp__inst_executed.sum",
            "smsp__issue_active.avg.pct_of_peak_sustained_active",
            "l1tex__data_pipe_lsu_wavefronts.avg.pct_of_peak_sustained_elapsed",
            "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum", "l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum",
            "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum",
            "l1tex__data_pipe_lsu_wavefronts_mem_shared_op_atom.sum",
            "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_atom.sum",
            "l1tex__data_pipe_lsu_wavefronts_mem_shared_op_st.sum",
            "sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active",
            "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread",
            "launch__shared_mem_per_block_dynamic", "launch__occupancy_limit_shared_mem",
            "launch__occupancy_limit_registers", "launch__grid_size"]


def raw_metrics(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units, vals = rows[0], rows[1], rows[2]
    return {h: (v, u) for h, u, v in zip(hdr, units, vals)}


def wavefronts_by_line(rep, top=22):
    raw = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    hdr = next(r for r in rows if r and r[0] == "Line No")
    iw, ii = hdr.index("L1 Wavefronts Shared"), hdr.index("L1 Wavefronts Shared Ideal")
    agg, fname, tot = {}, None, [0.0, 0.0]

    def f(x):
        try:
            return float(x.replace(",", ""))
        except ValueError:
            return 0.0
    for r in rows:
        if r and r[0] == "File Path":
            fname = r[1].split("/")[-1]
        elif r and re.match(r"^\d+$", r[0] or ""):
            a = agg.setdefault((fname, int(r[0])), [0.0, 0.0, r[1].strip()[:100]])
            a[0] += f(r[iw])
            a[1] += f(r[ii])
            tot[0] += f(r[iw])
            tot[1] += f(r[ii])
    print(f"total {tot[0]:.4g}, ideal {tot[1]:.4g}")
    for (fn, ln), a in sorted(agg.items(), key=lambda kv: -kv[1][0])[:top]:
        print(f"{fn}:{ln:<6d} {a[0] / 1e6:6.2f}M ({100 * a[0] / tot[0]:4.1f}%) ideal {a[1] / 1e6:5.2f}M  {a[2]}")


def main(d, header):
    print(header)
    print()
    print("## per-kernel summary")
    for rep in ("kbf.ncu-rep", "kg.ncu-rep"):
        p = os.path.join(d, rep)
        if os.path.exists(p):
            print(subprocess.run([sys.executable, os.path.join(os.path.dirname(__file__), "ncu_summary.py"), p],
                                 capture_output=True, text=True).stdout.rstrip())
    kbf = os.path.join(d, "kbf.ncu-rep")
    print()
    print("## KBF (tile_bulk<1,1>) limiters")
    m = raw_metrics(kbf)
    for k in LIMITERS:
        if k in m:
            print(f"{k:70s} {m[k][0]:>16s} {m[k][1]}")
    print()
    print("## KBF warp instructions / stall samples by source region (tools/ncu_phases.py)")
    with contextlib.redirect_stdout(io.StringIO()) as buf:
        ncu_phases.main(kbf)
    print(buf.getvalue().rstrip())
    print()
    print("## KBF stall samples by region and reason (tools/ncu_stalls.py)")
    with contextlib.redirect_stdout(io.StringIO()) as buf:
        ncu_stalls.main(kbf)
    print(buf.getvalue().rstrip())
    print()
    print("## shared-memory wavefronts by source line (L1 Wavefronts Shared; ideal = without bank conflicts)")
    wavefronts_by_line(kbf)
    tp = os.path.join(d, "tile_phases.txt")
    if os.path.exists(tp):
        print()
        print("## per-tile phase clocks (tools/tprof.py, -DDGR_DIAG=1 build)")
        print(open(tp).read().rstrip())
    lc = os.path.join(d, "launches.csv")
    if os.path.exists(lc):
        print()
        print("## launch list (ncu --metrics gpu__time_duration.sum --clock-control none)")
        print(subprocess.run([sys.executable, os.path.join(os.path.dirname(__file__), "ncu_summary.py"), lc],
                             capture_output=True, text=True).stdout.rstrip())


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2] if len(sys.argv) > 2 else "# ncu evidence")
