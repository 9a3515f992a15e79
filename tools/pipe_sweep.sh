#!/bin/bash
# C2 host-buffer call, page-locked and pageable inputs, 3 repetitions: PIPE_ON=1 (default,
# pipelined) or 0 (one pass); PHMM_PIPE_FIRST / PHMM_PIPE_MAXCH override the chunk plan
for rep in 1 2 3; do
  PHMM_PIPE=${PIPE_ON:-1} python - <<'PY'
import os, sys, time, json, numpy as np, torch
sys.path.insert(0, os.getcwd())
from paper_conf_ipps_wangxc17_b200 import phmm, synth
KEYS = ("read_bases", "base_quals", "ins_quals", "del_quals", "gcp_quals", "read_offsets", "hap_bases", "hap_offsets", "pairs")
b = synth.config_batch("C2")
pin = synth.Batch(**{k: torch.from_numpy(np.ascontiguousarray(getattr(b, k))).pin_memory().numpy() for k in KEYS})
out = torch.empty(b.n_pairs, dtype=torch.float64).pin_memory().numpy(); st = torch.empty(b.n_pairs, dtype=torch.uint8).pin_memory().numpy()
ctx = phmm.PairHMM(precision="fp32")
def t(bb, o, s_):
    ctx.compute_batch(bb, out=o, status=s_); r = []
    for _ in range(7):
        t0 = time.perf_counter(); ctx.compute_batch(bb, out=o, status=s_); r.append((time.perf_counter() - t0) * 1e3)
    return round(float(np.median(r)), 3)
o2 = np.empty(b.n_pairs); s2 = np.empty(b.n_pairs, dtype=np.uint8)
print(json.dumps({"pipe": os.environ["PHMM_PIPE"], "pinned_ms": t(pin, out, st), "n_chunks": ctx.stats()["n_chunks"], "pageable_ms": t(b, o2, s2)}), flush=True)
PY
done
