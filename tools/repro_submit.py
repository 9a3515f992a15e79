import sys, os, faulthandler
faulthandler.enable()
sys.path.insert(0, os.environ.get("GRAFT_REPO_ROOT", "/root/repo"))
import numpy as np
from paper_conf_ipps_wangxc17_b200 import phmm, synth
mode = sys.argv[1]
regions = [synth.config_batch("C3", n_regions=1, region_start=r) for r in range(int(sys.argv[2]) if len(sys.argv) > 2 else 64)]
ctx = phmm.PairHMM(precision="fp32")
print("created", flush=True)
if mode in ("submit", "all"):
    ts = [ctx.submit(b) for b in regions]
    for t in ts: t.wait()
    print("submitted", flush=True)
if mode in ("host", "all"):
    for b in regions: ctx.compute_batch(b)
    print("host done", flush=True)
ctx.close()
print("closed", flush=True)
