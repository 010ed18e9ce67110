"""Per-rank compute of the sharded iteration, measured on one B200 (DESIGN.md §7's time model):
    python tools/rank_model.py [CONFIG] [R ...]
Rank r of R runs alone with a no-op exchange callback (timing only: its demand lacks the other
ranks' events), so its KBF covers exactly its shard's tiles and its KG exactly its bands — what
each of R GPUs computes per iteration.  One JSON line per (R, r): per-kernel milliseconds per launch
(CUDA events on the launching stream, dgr_profile), the shard's tiles and candidates."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import forestgen  # noqa: E402
import paper_conf_dac_0159layhrr24_b200 as dgr  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "ispd19"
Rs = [int(x) for x in sys.argv[2:]] or [1, 2, 4, 8]
f = forestgen.generate(cfg)


def noop(buf, n, dtype, stream):
    return 0


for R in Rs:
    for r in sorted({0, R // 2, R - 1}):
        s = dgr.Solver(f, rank=r, world=R, allreduce=noop if R > 1 else None)
        s.step(10, 1.0, 0.3, want_loss=False)
        torch.cuda.synchronize()
        s.profile(True)
        s.step(50, 1.0, 0.3, want_loss=False)
        ms, n = s.profile_read()
        s.profile(False)
        info = s.info()
        print(json.dumps({"config": cfg, "R": R, "rank": r, "tiles": info["n_tiles"], "bundles": info["n_bundles"],
                          "stage_ms": {k: ms[k] / n[k] for k in ms if n[k]}}), flush=True)
        s.close()
