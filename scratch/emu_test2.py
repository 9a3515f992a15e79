import sys, numpy as np
sys.path.insert(0, '.'); sys.path.insert(0, 'scratch')
import emu
from oracle import core as oracle
from paper_conf_ipps_wangxc17_b200 import synth
b = synth.random_pairs_batch(4, 400, m_range=(1, 60), n_range=(1, 60))
n = b.hap_lengths()[b.pairs[:,1]]; m = b.read_lengths()[b.pairs[:,0]]
p = int(np.nonzero((n >= 43) & (n <= 46))[0][0])
print("m", m[p], "n", n[p], "nb", (m[p]+3+3)//4)
sb = b.subset([p] * 200)
ref = oracle.batch_log10(sb)
got = emu.run_batch(sb)
print("ref", ref[0], "emu distinct", np.unique(got)[:6], "maxerr", np.max(np.abs(got - ref)))
