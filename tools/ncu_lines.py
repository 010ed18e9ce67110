"""Per-source-line instruction counts and stall samples of one kernel in an ncu report.

    python tools/ncu_lines.py report.ncu-rep [top_n]
Prints the top lines by warp instructions executed, then totals per line range of the source file
(function regions) so the cost of each phase can be read off.
"""
import csv
import io
import re
import subprocess
import sys


def lines(path):
    raw = subprocess.run(["ncu", "-i", path, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    hdr = next(r for r in rows if r and r[0] == "Line No")
    i_inst = hdr.index("Instructions Executed")
    i_samp = hdr.index("Warp Stall Sampling (All Samples)")
    out, fname = [], None
    for r in rows:
        if r and r[0] == "File Path":
            fname = r[1].split("/")[-1]
        elif r and r[0] not in ("", "Line No", "Function Name", "File Path") and re.match(r"^\d+$", r[0]):
            def num(v):
                try:
                    return float(v.replace(",", ""))
                except ValueError:
                    return 0.0
            out.append((fname, int(r[0]), num(r[i_inst]), num(r[i_samp]), r[1].strip()))
    return out


if __name__ == "__main__":
    L = lines(sys.argv[1])
    top = int(sys.argv[2]) if len(sys.argv) > 2 else 40
    tot_i = sum(x[2] for x in L) or 1
    tot_s = sum(x[3] for x in L) or 1
    print(f"total warp instructions {tot_i:.4g}, stall samples {tot_s:.4g}")
    print(f"{'file:line':28s} {'inst%':>6s} {'samp%':>6s}  source")
    for f, ln, i, s, src in sorted(L, key=lambda x: -x[2])[:top]:
        print(f"{f + ':' + str(ln):28s} {100 * i / tot_i:6.2f} {100 * s / tot_s:6.2f}  {src[:90]}")
    print("\n# by stall samples")
    for f, ln, i, s, src in sorted(L, key=lambda x: -x[3])[:top]:
        print(f"{f + ':' + str(ln):28s} {100 * i / tot_i:6.2f} {100 * s / tot_s:6.2f}  {src[:90]}")


def stall_lines(path, reason, top=15):
    """Source lines with the most samples of one stall reason (e.g. 'stall_long_sb')."""
    raw = subprocess.run(["ncu", "-i", path, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    hdr = next(r for r in rows if r and r[0] == "Line No")
    col = hdr.index(reason)
    out, fname = [], None
    for r in rows:
        if r and r[0] == "File Path":
            fname = r[1].split("/")[-1]
        elif r and re.match(r"^\d+$", r[0] or ""):
            try:
                v = float(r[col].replace(",", ""))
            except ValueError:
                v = 0.0
            out.append((v, f"{fname}:{r[0]}", r[1].strip()[:90]))
    tot = sum(v for v, _, _ in out) or 1
    for v, loc, src in sorted(out, reverse=True)[:top]:
        print(f"{loc:28s} {100 * v / tot:6.2f}  {src}")
