import numpy as np, sys
sys.path.insert(0, '.')
from oracle import core as oracle
from paper_conf_ipps_wangxc17_b200 import phmm, synth
for prec in ["fp64", "fp32"]:
    h = phmm.PairHMM(precision=prec)
    for seed in [1,2,3]:
        b = synth.random_pairs_batch(seed, 400, m_range=(1, 60), n_range=(1, 60))
        got, st = h.compute_batch(b)
        ref = oracle.batch_log10(b)
        d = np.abs(got - ref); d[np.isneginf(got) & np.isneginf(ref)] = 0
        bad = np.nonzero(~(d < 1e-3))[0]
        m = b.read_lengths()[b.pairs[:,0]]; n = b.hap_lengths()[b.pairs[:,1]]
        print(prec, seed, "bad", len(bad), [(int(p), int(m[p]), int(n[p]), float(got[p]), float(ref[p])) for p in bad[:10]])
    print(h.stats())
