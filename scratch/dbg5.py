import numpy as np, sys, os
sys.path.insert(0, '.')
from oracle import core as oracle
from paper_conf_ipps_wangxc17_b200 import phmm, synth
h = phmm.PairHMM(precision="fp32")
b = synth.random_pairs_batch(4, 400, m_range=(1, 60), n_range=(1, 60))
n = b.hap_lengths()[b.pairs[:,1]]
p = int(np.nonzero((n >= 43) & (n <= 46))[0][0])
ref = oracle.batch_log10(b.subset([p]))[0]
for cnt in [1, 2, 5, 10, 20, 21, 22, 40, 100, 170, 171, 200]:
    o = h.compute_batch(b.subset([p] * cnt))[0]
    u = np.unique(o)
    bad = np.nonzero(np.abs(o - ref) > 1e-6)[0]
    print(cnt, "distinct", len(u), "bad idx", bad[:20], "maxerr %.2e" % np.max(np.abs(o - ref)))
