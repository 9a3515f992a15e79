import numpy as np, sys, os, ctypes
sys.path.insert(0, '.')
from paper_conf_ipps_wangxc17_b200 import phmm, synth
h = phmm.PairHMM(precision="fp32")
L = phmm.load_library()
b = synth.random_pairs_batch(4, 400, m_range=(1, 60), n_range=(1, 60))
n = b.hap_lengths()[b.pairs[:,1]]
p = int(np.nonzero((n >= 43) & (n <= 46))[0][0])
o = h.compute_batch(b.subset([p] * 40))[0]
buf = np.zeros(4096 * 32 * 6, np.float32)
L.phmm_debug_trace.argtypes = [ctypes.c_void_p, ctypes.c_int]
steps = L.phmm_debug_trace(buf.ctypes.data, 4096)
os.makedirs("gpurun_out", exist_ok=True)
np.save("gpurun_out/trace.npy", buf[:steps * 32 * 6].reshape(steps, 32, 6))
np.save("gpurun_out/trace_out.npy", o)
print("steps", steps)
