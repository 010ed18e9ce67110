"""Oracle fp64 gradients at iteration 0 of the elements that differ after one iteration."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, forestgen, oracle
import paper_conf_dac_0159layhrr24_b200 as dgr
f = forestgen.generate(sys.argv[1])
W = dgr.Weights(); ow = oracle.weights()
s = dgr.Solver(f); o = oracle.Oracle(f)
s.step(0, 1.0, 0.3); o.step(0, 1.0, 0.3, ow); s.step(1, 1.0, 0.3); o.step(1, 1.0, 0.3, ow)
gwt, gwp = s.logits(); owt, owp = o.logits()
o0 = oracle.Oracle(f); o0.forward(1.0, ow); dw0, du0 = o0.backward(1.0, ow)
bad = np.nonzero(np.abs(gwp - owp) > 1e-2)[0]
print("bad", bad.tolist())
print("their |dw0|", np.abs(dw0[bad]).tolist())
a = np.abs(dw0[dw0 != 0])
print("|dw0| quantiles (nonzero)", np.quantile(a, [1e-6, 1e-5, 1e-4, 1e-3, 0.5]).tolist(), "exact zeros", int((dw0 == 0).sum()))
print("count |dw0| < 1e-5:", int((np.abs(dw0) < 1e-5).sum()), "< 1e-6:", int((np.abs(dw0) < 1e-6).sum()), "of", dw0.size)
