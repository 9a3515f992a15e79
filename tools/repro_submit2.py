import sys, os, time
sys.path.insert(0, os.environ.get("GRAFT_REPO_ROOT", "/root/repo"))
import numpy as np
from paper_conf_ipps_wangxc17_b200 import phmm, synth
regions = [synth.config_batch("C3", n_regions=1, region_start=r) for r in range(256)]
ctx = phmm.PairHMM(precision="fp32")
ctx.compute_batch(regions[0])
for t in [ctx.submit(b) for b in regions]: t.wait()   # warm the queue's buffers
t0 = time.perf_counter()
ts = []
for b in regions:
    ts.append(ctx.submit(b))
t1 = time.perf_counter()
st0 = ctx.stats()
for t in ts: t.wait()
t2 = time.perf_counter()
print("submit loop %.1f ms, wait %.1f ms, stats at end of loop n_pairs %d, last run n_pairs %d" % (1e3*(t1-t0), 1e3*(t2-t1), st0["n_pairs"], ctx.stats()["n_pairs"]), flush=True)
ctx.close()
