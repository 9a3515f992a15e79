import sys, os, faulthandler
faulthandler.enable()
sys.path.insert(0, os.environ.get("GRAFT_REPO_ROOT", "/root/repo"))
import numpy as np
import torch
from paper_conf_ipps_wangxc17_b200 import phmm, synth
n = int(sys.argv[1]); timing = sys.argv[2] == "1"; mode = sys.argv[3]
regions = [synth.config_batch("C3", n_regions=1, region_start=r) for r in range(n)]
ctx = phmm.PairHMM(precision="fp32", timing=timing)
if mode == "dev":
    dbs = [phmm.DeviceBatch.from_host(b, device="cuda:0") for b in regions]
    for db in dbs: ctx.compute_batch_dev(db)
    torch.cuda.synchronize()
elif mode == "host":
    for b in regions: ctx.compute_batch(b)
elif mode == "whole":
    w = synth.config_batch("C3", n_regions=n)
    db = phmm.DeviceBatch.from_host(w, device="cuda:0")
    ctx.compute_batch_dev(db)
    ctx.compute_batch(w)
ctx.close()
print("closed", flush=True)
