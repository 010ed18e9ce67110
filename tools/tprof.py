"""Per-tile phase clocks of one KBF launch (DGR_DEBUG_SKIP=256): where a tile's lifetime goes."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ["DGR_DEBUG_SKIP"] = str(256 | int(os.environ.get("EXTRA_SKIP", "0")))
out = os.environ.setdefault("DGR_PROF_OUT", "/tmp/tprof.bin")
import numpy as np, torch, forestgen
import paper_conf_dac_0159layhrr24_b200 as dgr
f = forestgen.generate("ispd19")
s = dgr.Solver(f)
s.step(3, 1.0, 0.3, want_loss=False); torch.cuda.synchronize()
s.step(1, 1.0, 0.3, want_loss=False); torch.cuda.synchronize()
a = np.fromfile(out, dtype=np.int64).reshape(-1, 8)
a = a[a[:, 0] > 0]
d = np.diff(a[:, :6], axis=1).astype(np.float64)
names = ["wait stage", "reverse", "net level+noise+clear", "forward", "flush"]
tot = d.sum(1)
print(f"tiles {len(a)}  mean lifetime {tot.mean():.0f} cycles  (sum over tiles {tot.sum()/1.965e3/148:.1f} us per SM at 1965 MHz)")
for i, n in enumerate(names):
    print(f"  {n:24s} mean {d[:, i].mean():8.0f}  share {100*d[:, i].sum()/tot.sum():5.1f}%  p90 {np.percentile(d[:, i], 90):8.0f}")
gt = a[:, 7]; sm = a[:, 6]
print("kernel span (globaltimer of first/last tile start) us:", (gt.max() - gt.min()) / 1e3)
# concurrency: average CTAs per SM over time = sum lifetimes / (148 * span)
span_cyc = (gt.max() - gt.min()) / 1e3 * 1965
print("avg resident tiles per SM (lifetime-weighted):", tot.sum() / (148 * span_cyc))
