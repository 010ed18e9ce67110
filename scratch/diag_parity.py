"""Diagnostic: GPU-vs-oracle logit/demand error distributions and oracle self-sensitivity."""
import sys, time, copy
import numpy as np
sys.path.insert(0, '.')
import forestgen, oracle
import paper_conf_dac_0159layhrr24_b200 as dgr

def err(a, b):
    return np.abs(np.asarray(a, np.float64) - b) / np.maximum(np.abs(b), 1.0)

for name, iters in [("c1e4", 1), ("ispd18", 1), ("c1e4", 100), ("tiny", 200)]:
    f = forestgen.generate(name)
    s = dgr.Solver(f); o = oracle.Oracle(f)
    fp = copy.deepcopy(f)
    rng = np.random.default_rng(1)
    fp.w_path0 = (f.w_path0.astype(np.float64) * (1 + 1e-6 * rng.choice([-1, 1], f.n_paths))).astype(np.float32)
    fp.w_tree0 = (f.w_tree0.astype(np.float64) * (1 + 1e-6 * rng.choice([-1, 1], f.n_trees))).astype(np.float32)
    o2 = oracle.Oracle(fp)
    W = oracle.weights()
    t0 = time.time()
    done = 0
    while done < iters:
        n = min(100, iters - done)
        t = 0.9 ** (done // 100)
        gl = s.step(n, t, 0.3); ol = o.step(n, t, 0.3, W); o2.step(n, t, 0.3, W)
        done += n
    ew = err(s.logits()[1], o.logits()[1]); es = err(o2.logits()[1], o.logits()[1])
    ed = np.concatenate([err(a, b).ravel() for a, b in zip(s.demand(), o.demand())])
    esd = np.concatenate([err(a, b).ravel() for a, b in zip(o2.demand(), o.demand())])
    print(f"{name} iters={iters} ({time.time()-t0:.1f}s) loss gpu {gl[0]:.6f} or {ol[0]:.6f} rel {abs(gl[0]-ol[0])/abs(ol[0]):.2e}")
    print(f"  w_path gpu-err q[.5,.99,.999,max] {np.quantile(ew,[.5,.99,.999]).round(9)} {ew.max():.3e} n>1e-4: {(ew>1e-4).sum()} of {len(ew)}")
    print(f"  w_path oracle self-sens max {es.max():.3e} n>1e-5: {(es>1e-5).sum()}; gpu n>1e-4 where sens<=1e-5: {((ew>1e-4)&(es<=1e-5)).sum()}")
    print(f"  demand gpu-err max {ed.max():.3e} n>1e-4 {(ed>1e-4).sum()}; self-sens max {esd.max():.3e}")
