"""Device timeline of one compute_batch_dev call (CUPTI through torch.profiler): every kernel
and memcpy/memset of the call with its start/end, the GPU-idle gaps between them, and the
busy time per kernel name. Prints one JSON object (profiles/r02_timeline_<workload>.json).
Usage: python tools/timeline.py [C2|C3|...] [n_regions]"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import torch
    from torch.profiler import ProfilerActivity, profile

    from paper_conf_ipps_wangxc17_b200 import phmm, synth

    work = sys.argv[1] if len(sys.argv) > 1 else "C2"
    nreg = int(sys.argv[2]) if len(sys.argv) > 2 else None
    b = synth.config_batch(work, n_regions=nreg) if nreg else synth.config_batch(work)
    db = phmm.DeviceBatch.from_host(b, device="cuda:0")
    ctx = phmm.PairHMM(precision=synth.CONFIGS[work]["precision"])
    for _ in range(3):
        ctx.compute_batch_dev(db)
    torch.cuda.synchronize()
    with profile(activities=[ProfilerActivity.CUDA, ProfilerActivity.CPU]) as prof:
        ctx.compute_batch_dev(db)
        torch.cuda.synchronize()
    evs = []
    for e in prof.events():
        if e.device_type.name != "CUDA":
            continue
        t0 = e.time_range.start
        t1 = e.time_range.end
        evs.append((t0, t1, e.name))
    evs.sort()
    if not evs:
        print(json.dumps({"error": "no CUDA events"}))
        return
    span = evs[-1][1] - evs[0][0]
    gaps = []
    busy = 0.0
    cur_end = evs[0][0]
    prev = None
    for t0, t1, name in evs:
        if t0 > cur_end:
            gaps.append((t0 - cur_end, prev, name))
        busy += max(0.0, t1 - max(t0, cur_end)) if t1 > cur_end else 0.0
        if t1 > cur_end:
            cur_end = t1
        prev = name
    per = {}
    for t0, t1, name in evs:
        per[name] = per.get(name, 0.0) + (t1 - t0)
    gaps.sort(reverse=True)
    out = {
        "workload": work, "pairs": b.n_pairs, "span_us": span, "busy_us": busy, "idle_us": span - busy,
        "n_device_ops": len(evs),
        "top_gaps_us": [{"us": g, "after": (a or "")[:70], "before": (n or "")[:70]} for g, a, n in gaps[:12]],
        "busy_by_name_us": {k[:80]: v for k, v in sorted(per.items(), key=lambda kv: -kv[1])[:25]},
        "timeline": [{"t_us": round(t0 - evs[0][0], 1), "dur_us": round(t1 - t0, 1), "name": n[:60]} for t0, t1, n in evs],
    }
    print(json.dumps(out))


if __name__ == "__main__":
    main()
