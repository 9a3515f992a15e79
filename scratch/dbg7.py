import numpy as np, sys, os
sys.path.insert(0, '.')
from oracle import core as oracle
from paper_conf_ipps_wangxc17_b200 import phmm, synth
h = phmm.PairHMM(precision="fp32")
b = synth.random_pairs_batch(4, 400, m_range=(1, 60), n_range=(1, 60))
n = b.hap_lengths()[b.pairs[:,1]]
p = int(np.nonzero((n >= 43) & (n <= 46))[0][0])
ref = oracle.batch_log10(b.subset([p]))[0]
o = h.compute_batch(b.subset([p] * 40))[0]
print("nbad", int(np.sum(np.abs(o - ref) > 1e-6)))
