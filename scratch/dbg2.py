import numpy as np, sys
sys.path.insert(0, '.')
from oracle import core as oracle
from paper_conf_ipps_wangxc17_b200 import phmm, synth
h = phmm.PairHMM(precision="fp32")
for seed in [4,5,6]:
    b = synth.random_pairs_batch(seed, 400, m_range=(1, 60), n_range=(1, 60))
    got, st = h.compute_batch(b)
    ref = oracle.batch_log10(b)
    with np.errstate(invalid='ignore'):
        d = np.abs(got - ref)
    d[np.isneginf(got) & np.isneginf(ref)] = 0
    bad = np.nonzero(~(d < 1e-3))[0]
    m = b.read_lengths()[b.pairs[:,0]]; n = b.hap_lengths()[b.pairs[:,1]]
    print(seed, "bad", len(bad), [(int(p), int(m[p]), int(n[p]), int(st[p]), round(float(got[p]),3), round(float(ref[p]),3)) for p in bad[:12]])
