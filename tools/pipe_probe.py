"""Probe of the pipelined host-buffer call (compute_host_pipe): wall time of phmm_compute_batch
on C2 from page-locked and pageable buffers, unpipelined (PHMM_PIPE=0 context) vs pipelined with
first-chunk divisors F, plus one PHMM_PIPE_TRACE timeline. Prints one JSON line per setting."""
import json
import os
import sys
import time

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_wangxc17_b200 import phmm, synth  # noqa: E402

KEYS = ("read_bases", "base_quals", "ins_quals", "del_quals", "gcp_quals", "read_offsets", "hap_bases",
        "hap_offsets", "pairs")


def timeit(ctx, b, out, st, reps=5):
    ctx.compute_batch(b, out=out, status=st)
    ts = []
    for _ in range(reps):
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        ctx.compute_batch(b, out=out, status=st)
        ts.append((time.perf_counter() - t0) * 1e3)
    return min(ts), float(np.median(ts))


def main():
    wl = sys.argv[1] if len(sys.argv) > 1 else "C2"
    b = synth.config_batch(wl)
    n = b.n_pairs
    pin = synth.Batch(**{k: torch.from_numpy(np.ascontiguousarray(getattr(b, k))).pin_memory().numpy() for k in KEYS})
    out_p = torch.empty(n, dtype=torch.float64).pin_memory().numpy()
    st_p = torch.empty(n, dtype=torch.uint8).pin_memory().numpy()
    out = np.empty(n)
    st = np.empty(n, dtype=np.uint8)
    os.environ["PHMM_PIPE"] = "0"
    flat = phmm.PairHMM(precision="fp32", timing=True)
    del os.environ["PHMM_PIPE"]
    ctx = phmm.PairHMM(precision="fp32", timing=True)
    db = phmm.DeviceBatch.from_host(b, device="cuda:0")
    ctx.compute_batch_dev(db)
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for _ in range(5):
        ctx.compute_batch_dev(db)
    torch.cuda.synchronize()
    print(json.dumps({"workload": wl, "mode": "device call", "ms": (time.perf_counter() - t0) * 200}))
    for name, c, env in [("flat", flat, None)] + [(f"pipe F={f}", ctx, str(f)) for f in (2, 4, 8, 16)]:
        if env:
            os.environ["PHMM_PIPE_FIRST"] = env
        r = {"workload": wl, "mode": name}
        r["pinned_ms_min_med"] = timeit(c, pin, out_p, st_p)
        r["pageable_ms_min_med"] = timeit(c, b, out, st)
        r["n_chunks"] = c.stats()["n_chunks"]
        print(json.dumps(r), flush=True)
    os.environ["PHMM_PIPE_FIRST"] = "8"
    os.environ["PHMM_PIPE_TRACE"] = "1"
    tr = phmm.PairHMM(precision="fp32", timing=True)
    tr.compute_batch(pin, out=out_p, status=st_p)
    tr.compute_batch(pin, out=out_p, status=st_p)
    tr.compute_batch(b, out=out, status=st)


if __name__ == "__main__":
    main()
