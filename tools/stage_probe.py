"""Pageable vs page-locked host buffers through phmm_compute_batch on C2 (e2e per call),
for several staging thread counts (PHMM_STAGE_THREADS)."""
import json, os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
from paper_conf_ipps_wangxc17_b200 import phmm, synth

b = synth.config_batch("C2")
keys = ("read_bases", "base_quals", "ins_quals", "del_quals", "gcp_quals", "read_offsets", "hap_bases", "hap_offsets", "pairs")
pin = synth.Batch(**{k: torch.from_numpy(np.ascontiguousarray(getattr(b, k))).pin_memory().numpy() for k in keys})
n = b.n_pairs
pout = torch.empty(n, dtype=torch.float64).pin_memory().numpy()
pst = torch.empty(n, dtype=torch.uint8).pin_memory().numpy()
res = {}
for th in [int(x) for x in sys.argv[1:]] or [8]:
    os.environ["PHMM_STAGE_THREADS"] = str(th)
    ctx = phmm.PairHMM(precision="fp32")
    for _ in range(2):
        ctx.compute_batch(b); ctx.compute_batch(pin, out=pout, status=pst)
    t = {"pageable": [], "pinned": []}
    for _ in range(5):
        for kind, bb, o, s in (("pageable", b, None, None), ("pinned", pin, pout, pst)):
            t0 = time.perf_counter(); ctx.compute_batch(bb, out=o, status=s); t[kind].append(time.perf_counter() - t0)
    res[th] = {k: 1e3 * float(np.median(v)) for k, v in t.items()}
    res[th]["ratio"] = res[th]["pinned"] / res[th]["pageable"]
    ctx.close()
print(json.dumps({"workload": "C2 (2^20 pairs)", "ms_per_call_median_of_5": res, "cores": os.cpu_count()}))
