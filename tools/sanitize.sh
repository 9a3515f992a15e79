#!/bin/bash
# compute-sanitizer passes on small inputs (each bounded by timeout)
cat > /tmp/san_case.py <<'PY'
import sys; sys.path.insert(0, '.')
import numpy as np
from paper_conf_ipps_wangxc17_b200 import phmm, synth
b = synth.concat_batches([synth.config_batch("C2", n_regions=4), synth.random_pairs_batch(3, 100, m_range=(1, 60), n_range=(1, 80)),
                          synth.config_batch("C3", n_regions=1), synth.config_batch("C4", n_regions=1).subset(range(6))])
import os, torch
pin = synth.Batch(**{k: torch.from_numpy(np.ascontiguousarray(getattr(b, k))).pin_memory().numpy()
                     for k in ("read_bases", "base_quals", "ins_quals", "del_quals", "gcp_quals", "read_offsets",
                               "hap_bases", "hap_offsets", "pairs")})
for prec in ("fp32", "fp64"):
    with phmm.PairHMM(precision=prec) as h:
        out, st = h.compute_batch(b)
        print(prec, "ok", np.isfinite(out).sum(), "rescued", int((st == 1).sum()))
    # the pipelined host call (two streams, copy thread), pageable and page-locked inputs
    os.environ["PHMM_PIPE_MIN"] = "64"
    with phmm.PairHMM(precision=prec) as h:
        o2, s2 = h.compute_batch(b)
        n2 = h.stats()["n_chunks"]
        o3, s3 = h.compute_batch(pin)
        n3 = h.stats()["n_chunks"]
    del os.environ["PHMM_PIPE_MIN"]
    print(prec, "pipelined ok" if np.array_equal(o2, out) and np.array_equal(o3, out) else "pipelined MISMATCH",
          "chunks", n2, n3)
PY
for tool in memcheck racecheck synccheck; do
  echo "== $tool"
  timeout 600 compute-sanitizer --tool $tool --print-limit 5 python /tmp/san_case.py 2>&1 | grep -E "ERROR SUMMARY|hazard|ok|Invalid|RACECHECK" | head -8
done
