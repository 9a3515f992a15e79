import numpy as np, sys
sys.path.insert(0, '.')
from oracle import core as oracle
from paper_conf_ipps_wangxc17_b200 import phmm, synth
h = phmm.PairHMM(precision="fp32")
b = synth.random_pairs_batch(4, 400, m_range=(1, 60), n_range=(1, 60))
ref = oracle.batch_log10(b)
n = b.hap_lengths()[b.pairs[:,1]]; m = b.read_lengths()[b.pairs[:,0]]
# restrict to one bin: ncols 44..48 -> N 42..46
for lo_, hi_ in [(38, 38), (39, 42), (43, 46), (47, 50), (51,54), (55,58)]:
    sel = np.nonzero((n >= lo_) & (n <= hi_))[0]
    sb = b.subset(sel)
    outs = [h.compute_batch(sb)[0] for _ in range(4)]
    nd = [int(np.sum(o != outs[0])) for o in outs[1:]]
    err = np.abs(outs[0] - ref[sel]); err[np.isneginf(ref[sel])] = 0
    print(f"N {lo_}-{hi_}: pairs {len(sel)} blocks~{int(np.sum((m[sel]+3+3)//4))} nondet {nd} maxerr {err.max():.2e}")
# identical pairs
p = int(np.nonzero((n >= 43) & (n <= 46))[0][0])
sb = b.subset([p] * 200)
o = h.compute_batch(sb)[0]
print("identical x200: distinct values", len(np.unique(o)), "ref", ref[p], "vals", np.unique(o)[:5])
