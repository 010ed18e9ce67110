"""BASELINE.json configs[4]: the scaling sweep 10^4 .. 4x10^6 nets at fixed pin density on one B200.

    python tools/sweep.py [--steps 100] [--warmup 10] [--configs sweep1e4,sweep1e5,sweep1e6,sweep4e6]

One JSON line per config: solver iterations/s (CUDA events around one dgr_step(K) after W warm-up
iterations, the forest resident in HBM), path-candidate updates/s, the whole iteration's algorithmic
bytes against MEASURED_PEAKS.json hbm_gbs (bench.py's accounting) and the HBM
footprint of the solver's workspace.  Synthetic inputs from forestgen (DESIGN.md §3 recipe).
"""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import bench  # noqa: E402
import forestgen  # noqa: E402
import paper_conf_dac_0159layhrr24_b200 as dgr  # noqa: E402


def one(name: str, steps: int, warmup: int, peak: float) -> dict:
    t0 = time.time()
    f = forestgen.generate(name)
    gen_s = time.time() - t0
    W = dgr.Weights()
    s = dgr.Solver(f)
    s.step(warmup, 1.0, 0.3, W, want_loss=False)
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    s.step(steps, 1.0, 0.3, W, want_loss=False)
    b.record()
    b.synchronize()
    ms = a.elapsed_time(b)
    info = s.info()
    st = dict(paths=f.n_paths, single_paths=bench.single_paths(f), subnets=f.n_subnets, trees=f.n_trees,
              nets=f.n_nets,
              bundles=info["n_bundles"], cells=f.X * f.Y)
    sv = bench.survey_bytes(st, f.X, f.Y)   # SURVEY.md 8(d) per-unit figures
    sb = bench.stage_bytes(st)               # this design's stricter minimum
    alg = sv["KG"] + sv["KBF"]
    alg_strict = sb["KG"] + sb["KBF"]
    ips = steps / (ms / 1e3)
    s.close()
    return {"config": name, "grid": f"{f.X}x{f.Y}", "nets": int(f.n_nets), "paths": int(f.n_paths),
            "iters_per_s": ips, "path_cand_per_s": ips * f.n_paths, "ms_per_iter": ms / steps,
            "alg_bytes_per_iter": int(alg), "achieved_gbs": alg * ips / 1e9, "peak_gbs": peak,
            "roofline_frac": alg * ips / 1e9 / peak,
            "roofline_frac_strict": alg_strict * ips / 1e9 / peak, "hbm_footprint_bytes": int(info["workspace_bytes"]),
            "tiles": info["n_tiles"], "steps": steps, "warmup": warmup, "gen_s": round(gen_s, 1)}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--steps", type=int, default=100)
    ap.add_argument("--warmup", type=int, default=10)
    ap.add_argument("--configs", default="sweep1e4,sweep1e5,sweep1e6,sweep4e6")
    args = ap.parse_args()
    peak, _ = bench.measured_peak()
    for name in args.configs.split(","):
        print(json.dumps(one(name, args.steps, args.warmup, peak)), flush=True)


if __name__ == "__main__":
    main()
