"""Device timeline (CUPTI via torch.profiler) of C2 batches streamed through
phmm_compute_batch_async with two in flight (page-locked buffers): when each batch's prefetch
copies and kernels run."""
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
KEYS = ("read_bases", "base_quals", "ins_quals", "del_quals", "gcp_quals", "read_offsets", "hap_bases",
        "hap_offsets", "pairs")


def main():
    import torch
    from torch.profiler import ProfilerActivity, profile

    from paper_conf_ipps_wangxc17_b200 import phmm, synth
    b = synth.config_batch("C2")
    pin = synth.Batch(**{k: torch.from_numpy(np.ascontiguousarray(getattr(b, k))).pin_memory().numpy() for k in KEYS})
    outs = [torch.empty(b.n_pairs, dtype=torch.float64).pin_memory().numpy() for _ in range(2)]
    ctx = phmm.PairHMM(precision="fp32")

    def stream(k):
        q = []
        t0 = time.perf_counter()
        for i in range(k):
            q.append(ctx.compute_batch_async(pin, out=outs[i % 2]))
            if len(q) >= 2:
                q.pop(0).wait()
        while q:
            q.pop(0).wait()
        return (time.perf_counter() - t0) * 1e3 / k

    print(json.dumps({"warm_ms_per_step": stream(6)}))
    with profile(activities=[ProfilerActivity.CUDA]) as prof:
        ms = stream(4)
    print(json.dumps({"profiled_ms_per_step": ms}))
    evs = sorted((e.time_range.start, e.time_range.end, e.name) for e in prof.events() if e.device_type.name == "CUDA")
    t00 = evs[0][0]
    for t0, t1, name in evs:
        if t1 - t0 > 30 or "wavefront" in name:
            print(json.dumps({"t_us": round(t0 - t00, 1), "dur_us": round(t1 - t0, 1), "name": name[:60]}))


if __name__ == "__main__":
    main()
