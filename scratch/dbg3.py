import numpy as np, sys
sys.path.insert(0, '.')
from oracle import core as oracle
from paper_conf_ipps_wangxc17_b200 import phmm, synth
h = phmm.PairHMM(precision="fp32")
b = synth.random_pairs_batch(4, 400, m_range=(1, 60), n_range=(1, 60))
ref = oracle.batch_log10(b)
outs = [h.compute_batch(b)[0] for _ in range(6)]
for o in outs[1:]:
    diff = np.nonzero(~((o == outs[0]) | (np.isneginf(o) & np.isneginf(outs[0]))))[0]
    print("run-to-run differing pairs:", len(diff), diff[:10])
m = b.read_lengths()[b.pairs[:,0]]; n = b.hap_lengths()[b.pairs[:,1]]
for o in outs[:3]:
    with np.errstate(invalid='ignore'):
        d = np.abs(o - ref)
    d[np.isneginf(o) & np.isneginf(ref)] = 0
    bad = np.nonzero(~(d < 1e-3))[0]
    print("bad", len(bad), [(int(p), int(m[p]), int(n[p])) for p in bad[:10]])
# single-pair batches for the bad ones
bad = np.nonzero(~(np.abs(outs[0]-ref) < 1e-3))[0]
for p in bad[:5]:
    sb = b.subset([p])
    o = h.compute_batch(sb)[0][0]
    print("alone", p, o, ref[p])
# bucket 1
h1 = phmm.PairHMM(precision="fp32", col_bucket=1)
o = h1.compute_batch(b)[0]
with np.errstate(invalid='ignore'):
    d = np.abs(o - ref)
d[np.isneginf(o) & np.isneginf(ref)] = 0
print("bucket1 bad", int(np.sum(~(d < 1e-3))))
