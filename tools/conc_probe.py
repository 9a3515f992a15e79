"""Co-residency probe: can the FP64 rescue run beside the FP32 wavefront on the same SMs?

Times, on one workload (C3 by default): the FP32 call alone, the FP64 call over the pairs the
FP32 call rescued (default launch shape, and with PHMM_F64_CONC one-warp CTAs per SM), and the
two calls running at the same time on two streams from two host threads. Prints JSON lines.
"""
import json
import os
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import torch

    from paper_conf_ipps_wangxc17_b200 import phmm, synth

    work = sys.argv[1] if len(sys.argv) > 1 else "C3"
    nreg = int(sys.argv[2]) if len(sys.argv) > 2 else 4096
    b = synth.config_batch(work, n_regions=nreg)
    dev = "cuda:0"
    db = phmm.DeviceBatch.from_host(b, device=dev)
    s32, s64 = torch.cuda.Stream(), torch.cuda.Stream()
    c32 = phmm.PairHMM(precision="fp32", stream=s32.cuda_stream)
    o, st = c32.compute_batch_dev(db)
    torch.cuda.synchronize()
    st = st.cpu().numpy()
    resc = np.nonzero(st == 1)[0]
    sub = b.subset(resc)
    dsub = phmm.DeviceBatch.from_host(sub, device=dev)
    # the FP32 side runs the pairs it keeps (no rescue inside the timed FP32 call)
    keep = b.subset(np.nonzero(st == 0)[0])
    db = phmm.DeviceBatch.from_host(keep, device=dev)
    conc = os.environ.get("PHMM_F64_CONC", "0")

    def timed(fn, reps=3):
        fn()
        torch.cuda.synchronize()
        ts = []
        for _ in range(reps):
            t0 = time.perf_counter()
            fn()
            torch.cuda.synchronize()
            ts.append(time.perf_counter() - t0)
        return 1e3 * min(ts)

    os.environ.pop("PHMM_F64_CONC", None)
    c64d = phmm.PairHMM(precision="fp64", stream=s64.cuda_stream)
    os.environ["PHMM_F64_CONC"] = conc
    c64c = phmm.PairHMM(precision="fp64", stream=s64.cuda_stream)
    ref64, _ = c64d.compute_batch_dev(dsub)
    t32 = timed(lambda: c32.compute_batch_dev(db))
    t64d = timed(lambda: c64d.compute_batch_dev(dsub))
    t64c = timed(lambda: c64c.compute_batch_dev(dsub))
    o64c, _ = c64c.compute_batch_dev(dsub)
    torch.cuda.synchronize()
    same = bool(torch.equal(o64c, ref64))

    def both(c64):
        def run():
            th = threading.Thread(target=lambda: c64.compute_batch_dev(dsub))
            th.start()
            c32.compute_batch_dev(db)
            th.join()
        return run

    tbd = timed(both(c64d))
    tbc = timed(both(c64c))
    print(json.dumps({"workload": work, "regions": nreg, "pairs": b.n_pairs, "fp32_pairs": keep.n_pairs, "rescued": int(resc.size),
                      "f64_conc_ctas_per_sm": int(conc), "fp32_call_ms": t32, "fp64_default_ms": t64d,
                      "fp64_conc_ms": t64c, "both_default_ms": tbd, "both_conc_ms": tbc,
                      "sequential_ms": t32 + t64d, "conc_bitwise_equal": same}), flush=True)


if __name__ == "__main__":
    main()
