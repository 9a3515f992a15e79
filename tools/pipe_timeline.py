"""Device timeline (CUPTI through torch.profiler) of one pipelined host-buffer call
(phmm_compute_batch from page-locked buffers, compute_host_pipe): every kernel / copy with its
start and duration, so the per-chunk overheads (prep, sync gaps, wavefront tails) can be read.
Usage: python tools/pipe_timeline.py [C2] [first-chunk divisor]"""
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

KEYS = ("read_bases", "base_quals", "ins_quals", "del_quals", "gcp_quals", "read_offsets", "hap_bases",
        "hap_offsets", "pairs")


def main():
    import torch
    from torch.profiler import ProfilerActivity, profile

    from paper_conf_ipps_wangxc17_b200 import phmm, synth

    work = sys.argv[1] if len(sys.argv) > 1 else "C2"
    if len(sys.argv) > 2:
        os.environ["PHMM_PIPE_FIRST"] = sys.argv[2]
    b = synth.config_batch(work)
    n = b.n_pairs
    pin = synth.Batch(**{k: torch.from_numpy(np.ascontiguousarray(getattr(b, k))).pin_memory().numpy() for k in KEYS})
    out = torch.empty(n, dtype=torch.float64).pin_memory().numpy()
    st = torch.empty(n, dtype=torch.uint8).pin_memory().numpy()
    ctx = phmm.PairHMM(precision="fp32")
    for _ in range(3):
        ctx.compute_batch(pin, out=out, status=st)
    torch.cuda.synchronize()
    with profile(activities=[ProfilerActivity.CUDA, ProfilerActivity.CPU]) as prof:
        ctx.compute_batch(pin, out=out, status=st)
        torch.cuda.synchronize()
    evs = sorted((e.time_range.start, e.time_range.end, e.name) for e in prof.events() if e.device_type.name == "CUDA")
    t00 = evs[0][0]
    for t0, t1, name in evs:
        print(json.dumps({"t_us": round(t0 - t00, 1), "dur_us": round(t1 - t0, 1), "name": name[:70]}))


if __name__ == "__main__":
    main()
