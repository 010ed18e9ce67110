"""Warp-stall samples of the tile kernel by source region AND stall reason, from an ncu report captured
with --import-source on:  python tools/ncu_stalls.py kbf.ncu-rep
(regions as in ncu_phases.py).  Shows what each phase waits on: long_sb (global memory), short_sb /
mio_throttle / lg_throttle (shared memory and the LSU queue), barrier, selected (issuing), ..."""
import csv
import io
import re
import subprocess
import sys
from collections import defaultdict

sys.path.insert(0, __import__("os").path.dirname(__file__))
from ncu_phases import MARKERS, full_source  # noqa: E402


def main(path):
    src = full_source(path)
    region_of, region = {}, "other"
    for ln in sorted(src):
        for pat, name in MARKERS:
            if re.search(pat, src[ln]):
                region = name
                break
        region_of[ln] = region
    raw = subprocess.run(["ncu", "-i", path, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    hdr = next(r for r in rows if r and r[0] == "Line No")
    cols = [i for i, h in enumerate(hdr) if h.startswith("stall_") and "Not Issued" not in h]
    agg = defaultdict(lambda: defaultdict(float))
    fname = None
    for r in rows:
        if r and r[0] == "File Path":
            fname = r[1].split("/")[-1]
        elif r and re.match(r"^\d+$", r[0] or "") and fname == "dgr_kernels.cu":
            reg = region_of.get(int(r[0]), "other")
            for i in cols:
                try:
                    agg[reg][hdr[i]] += float(r[i].replace(",", ""))
                except (ValueError, IndexError):
                    pass
    tot = sum(sum(d.values()) for d in agg.values()) or 1
    reasons = defaultdict(float)
    for d in agg.values():
        for k, v in d.items():
            reasons[k] += v
    top = [k for k, _ in sorted(reasons.items(), key=lambda kv: -kv[1])[:9]]
    short = [k.replace("stall_", "")[:11] for k in top]
    print(f"stall samples by region (% of all) and reason; columns: top reasons overall")
    print(f"{'region':32s} {'all':>6s} " + " ".join(f"{s:>11s}" for s in short))
    print(f"{'(all regions)':32s} {100.0:6.1f} " + " ".join(f"{100 * reasons[k] / tot:11.1f}" for k in top))
    for reg, d in sorted(agg.items(), key=lambda kv: -sum(kv[1].values())):
        s = sum(d.values())
        if s / tot < 0.005:
            continue
        print(f"{reg:32s} {100 * s / tot:6.1f} " + " ".join(f"{100 * d[k] / tot:11.1f}" for k in top))


if __name__ == "__main__":
    main(sys.argv[1])
