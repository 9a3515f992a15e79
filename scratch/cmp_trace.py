import sys, numpy as np
sys.path.insert(0, '.'); sys.path.insert(0, 'scratch')
import emu
from paper_conf_ipps_wangxc17_b200 import synth
b = synth.random_pairs_batch(4, 400, m_range=(1, 60), n_range=(1, 60))
n = b.hap_lengths()[b.pairs[:,1]]
p = int(np.nonzero((n >= 43) & (n <= 46))[0][0])
sb = b.subset([p] * 40)
emu.TRACE.clear()
got = emu.run_batch(sb)
et = np.array(emu.TRACE)
gt = np.load("gpurun_out/trace.npy")
print("emu steps", et.shape, "gpu steps", gt.shape)
S = min(len(et), len(gt))
for s in range(S):
    a, g = et[s], gt[s]
    bad = ~np.isclose(a, g, rtol=1e-5, atol=1e-30)
    if bad.any():
        li, ci = np.nonzero(bad)
        print("first diff at step", s, "lanes", sorted(set(li.tolist()))[:10], "cols", sorted(set(ci.tolist())))
        for l in sorted(set(li.tolist()))[:4]:
            print("  lane", l, "emu", a[l], "\n         gpu", g[l])
        break
