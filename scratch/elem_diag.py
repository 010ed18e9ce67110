"""Inspect one logit that differs from the oracle after one iteration (sweep4e6)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, forestgen, oracle
import paper_conf_dac_0159layhrr24_b200 as dgr
name = sys.argv[1]; idx = int(sys.argv[2])
f = forestgen.generate(name)
s = dgr.Solver(f); o = oracle.Oracle(f); W = dgr.Weights(); ow = oracle.weights()
s.step(0, 1.0, 0.3); o.step(0, 1.0, 0.3, ow)
s.step(1, 1.0, 0.3); o.step(1, 1.0, 0.3, ow)
gwt, gwp = s.logits(); owt, owp = o.logits()
spo = np.asarray(f.sub_path_off); tso = np.asarray(f.tree_sub_off); nto = np.asarray(f.net_tree_off)
sub = int(np.searchsorted(spo, idx, side="right") - 1); tree = int(np.searchsorted(tso, sub, side="right") - 1)
net = int(np.searchsorted(nto, tree, side="right") - 1)
print("path", idx, "sub", sub, "tree", tree, "net", net, "net trees", nto[net + 1] - nto[net], "subs of tree", tso[tree + 1] - tso[tree])
print("sub_xy", np.asarray(f.sub_xy)[sub])
w0 = np.asarray(f.w_path0)
for i in range(spo[sub], spo[sub + 1]):
    g0, g1 = np.asarray(f.path_seg_off)[i], np.asarray(f.path_seg_off)[i + 1]
    print(i, "w0 %.6f gpu %.6f orc %.6f" % (w0[i], gwp[i], owp[i]), "segs", np.asarray(f.seg)[g0:g1].tolist())
for j in range(nto[net], nto[net + 1]):
    print("tree", j, "w0 %.6f gpu %.6f orc %.6f" % (np.asarray(f.w_tree0)[j], gwt[j], owt[j]))
bad = np.nonzero(np.abs(gwp - owp) > 1e-2)[0]
print("elements off by > 1e-2:", len(bad), bad[:10])
