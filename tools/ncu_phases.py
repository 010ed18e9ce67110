"""Warp instructions and stall samples of the tile kernel by source region (function / phase),
from an ncu report captured with --import-source on:  python tools/ncu_phases.py kbf.ncu-rep
Regions are delimited by the function definitions and phase comments of dgr_kernels.cu as embedded
in the report, so the split follows the source version that was profiled.  Inlined helpers are
counted in their own region (path_cost, softmax, seg_reduce, ...), not at their call sites."""
import re
import sys
from collections import defaultdict

sys.path.insert(0, __import__("os").path.dirname(__file__))
from ncu_lines import lines  # noqa: E402

MARKERS = [   # (regex on the source line, region name); a region runs until the next marker
    (r"uint4 philox4x32_10|uint4 philox_rk", "philox"),
    (r"float gumbel_word", "gumbel_word"),
    (r"float gumbel\(", "gumbel"),
    (r"struct Lane \{|void lane_setup|void lane_from", "lane decode"),
    (r"T seg_reduce", "seg_reduce"),
    (r"void dq_add|double dq_get", "dq limbs"),
    (r"void red64", "red64"),
    (r"long long beta_fold|void tp_fold_global", "tp fold (global)"),
    (r"void flush_window", "flush"),
    (r"long long warp_sum_ll", "warp_sum"),
    (r"void adam_update", "adam"),
    (r"struct Win \{", "win"),
    (r"double path_cost", "path_cost"),
    (r"int lane_wl|void red_shared_add", "red_shared"),
    (r"void c_events", "c_events"),
    (r"float softmax_from_noise", "softmax"),
    (r"void reverse_warp", "slow reverse"),
    (r"void forward_warp", "slow forward"),
    (r"void slow_tile", "slow tile"),
    (r"struct StageLayout|void mbar_|void bulk_|void issue_tile_loads|void cp16|void lsu_tile_loads|void prefetch_tile|void tma_2d", "stage"),
    (r"void process_tile", "process_tile: setup"),
    (r"-- reverse of iteration k --", "process_tile: reverse"),
    (r"-- net level", "process_tile: net level + noise"),
    (r"-- forward of iteration k_next --", "process_tile: forward"),
    (r"write back the tile's group slot state", "process_tile: write-back + flush"),
    (r"void __launch_bounds__\(kBThreads, kBPerSM\) tile_bulk", "tile_bulk entry"),
    (r"^// KG", "KG"),
]


def full_source(path, fname="dgr_kernels.cu"):
    """line number -> text of every line of the profiled source file embedded in the report"""
    import csv
    import io
    import subprocess
    raw = subprocess.run(["ncu", "-i", path, "--page", "source", "--print-source", "cuda", "--csv"],
                         capture_output=True, text=True).stdout
    out, cur = {}, None
    for r in csv.reader(io.StringIO(raw)):
        if len(r) >= 2 and r[0] == "File Name":
            cur = r[1].split("/")[-1]
        elif cur == fname and len(r) >= 2 and r[0].isdigit():
            out[int(r[0])] = r[1]
    return out


def main(path):
    src = full_source(path)
    region_of, region = {}, "other"
    for ln in sorted(src):
        for pat, name in MARKERS:
            if re.search(pat, src[ln]):
                region = name
                break
        region_of[ln] = region
    agg = defaultdict(lambda: [0.0, 0.0])
    for f, ln, inst, samp, _ in lines(path):
        if f != "dgr_kernels.cu":
            continue
        r = region_of.get(ln, "other")
        agg[r][0] += inst
        agg[r][1] += samp
    ti = sum(v[0] for v in agg.values()) or 1
    ts = sum(v[1] for v in agg.values()) or 1
    print(f"total warp instructions {ti:.4g} (dgr_kernels.cu lines), stall samples {ts:.4g}")
    print(f"{'region':34s} {'inst%':>7s} {'Minst':>8s} {'samp%':>7s}")
    for k, (i, s) in sorted(agg.items(), key=lambda kv: -kv[1][0]):
        print(f"{k:34s} {100 * i / ti:7.2f} {i / 1e6:8.2f} {100 * s / ts:7.2f}")


if __name__ == "__main__":
    main(sys.argv[1])
