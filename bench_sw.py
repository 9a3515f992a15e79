#!/usr/bin/env python3
"""Smith-Waterman benchmark (the paper's SW1/SW2 workload, PAPER.md
§V-B, Fig. 10: re-batched haplotype-vs-reference tasks).

    python bench_sw.py [--workload SW2] [--steps K] [--warmup W] [--no-cpu-baseline]

Prints one JSON line: GCUPS of phmm_sw_align_batch_dev on device-resident inputs (fill
+ traceback + the per-call prep; CUDA events), the fill kernel alone (`roofline`,
integer-ALU bound), the host-buffer call (`e2e`), and the CPU oracle on a bounded sample
(`cpu_baseline`). The oracle is imported only for that leg.
"""
from __future__ import annotations

import argparse
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

# ALU-pipe roofline of the fill kernel: integer ops per cell of the running-max recurrence
# (DESIGN.md §12): 2 adds + compare + 2 selects (vertical), the same (horizontal), match
# select + add (diagonal), 3 compares + 3 selects (choose), 1 compare + 2 selects (0 term)
# = 20 ALU-pipe ops; 64 ALU lanes per SM per clock (profiles/r01_microbench_issue_rates.jsonl).
SW_ALU_OPS_PER_CELL = 20
ALU_LANES_PER_SM = 64


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="SW2", choices=["SW1", "SW2"])
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-seconds", type=float, default=10.0)
    args = ap.parse_args()

    import torch

    from paper_conf_ipps_wangxc17_b200 import phmm, synth

    b = synth.sw_config_batch(args.workload)
    cells = b.cells()
    dev = "cuda:0"
    T = {"ref_bases": torch.from_numpy(b.ref_bases).to(dev), "ref_offsets": torch.from_numpy(b.ref_offsets).to(dev),
         "alt_bases": torch.from_numpy(b.alt_bases).to(dev), "alt_offsets": torch.from_numpy(b.alt_offsets).to(dev),
         "tasks": torch.from_numpy(b.tasks).to(dev), "total_ref_bases": int(b.ref_offsets[-1]),
         "total_alt_bases": int(b.alt_offsets[-1])}
    off = b.ops_capacity()
    ops = torch.zeros(int(off[-1]), dtype=torch.int32, device=dev)
    res = torch.zeros((b.n_tasks, 6), dtype=torch.int32, device=dev)
    ctx = phmm.PairHMM(device=0, timing=True)
    for _ in range(args.warmup):
        ctx.sw_align_batch_dev(T, res=res, ops=ops)
    torch.cuda.synchronize()
    ms, fill = [], []
    for _ in range(args.steps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        e0.record()
        ctx.sw_align_batch_dev(T, res=res, ops=ops)  # synchronous: returns when results are final
        e1.record()
        torch.cuda.synchronize()
        ms.append(e0.elapsed_time(e1))
        fill.append(ctx.stats()["ms_wavefront"])
    t = float(np.mean(ms))
    tf = float(np.mean(fill))
    nsm = torch.cuda.get_device_properties(0).multi_processor_count
    try:
        sm_max = float(json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json"))).get("sm_max_mhz", 1965))
    except (OSError, ValueError):
        sm_max = 1965.0
    peak = nsm * ALU_LANES_PER_SM * sm_max * 1e6 / SW_ALU_OPS_PER_CELL / 1e9
    # end to end through the host-buffer call
    t0 = time.perf_counter()
    for _ in range(args.steps):
        ctx.sw_align_batch(b)
    te = (time.perf_counter() - t0) / args.steps
    out = {"metric": "Smith-Waterman GCUPS (fill + traceback)", "value": cells / (t / 1e3) / 1e9, "unit": "GCUPS",
           "n_gpus": 1, "steps": args.steps, "warmup": args.warmup, "ms_per_step": t, "higher_is_better": True,
           "dtype": "int32", "data": "synthetic",
           "config": {"workload": args.workload, "desc": synth.SW_CONFIGS[args.workload]["desc"],
                      "tasks": b.n_tasks, "cells": cells, "params": list(phmm.SW_GATK_HC)},
           "roofline": {"bound": "alu", "kernel": "k_sw_fill", "achieved": cells / (tf / 1e3) / 1e9, "peak": peak,
                        "unit": "GCUPS", "frac": cells / (tf / 1e3) / 1e9 / peak, "fill_ms": tf,
                        "peak_basis": f"{nsm} SM x {ALU_LANES_PER_SM} ALU lanes x {sm_max:.0f} MHz / "
                                      f"{SW_ALU_OPS_PER_CELL} int ops per cell"},
           "e2e": {"value": cells / te / 1e9, "unit": "GCUPS", "ms_per_step": te * 1e3,
                   "h2d_bytes_per_step": int(b.ref_bases.nbytes + b.alt_bases.nbytes + b.ref_offsets.nbytes
                                             + b.alt_offsets.nbytes + b.tasks.nbytes),
                   "d2h_bytes_per_step": int(b.n_tasks * 24 + 4 * int(res[:, 5].sum().item()))},
           "paper": "SW2 on Titan X: 19.6 GCUPS peak, 18.5 average with 3,200 re-batched tasks (L24@1700)"}
    if not args.no_cpu_baseline:
        from oracle import sw as oracle_sw

        rng = np.random.default_rng(0)
        per = max(1, cells // b.n_tasks)
        k = int(min(b.n_tasks, max(16, args.cpu_seconds * 2e8 / per)))
        idx = np.sort(rng.choice(b.n_tasks, size=k, replace=False))
        sub = synth.SwBatch(b.ref_bases, b.ref_offsets, b.alt_bases, b.alt_offsets, b.tasks[idx])
        nt = os.cpu_count() or 1
        t0 = time.perf_counter()
        ref, _, _ = oracle_sw.batch(sub.ref_bases, sub.ref_offsets, sub.alt_bases, sub.alt_offsets, sub.tasks,
                                    nthreads=nt)
        tc = time.perf_counter() - t0
        got = res.cpu().numpy()[idx]
        out["cpu_baseline"] = {"value": sub.cells() / tc / 1e9, "unit": "GCUPS", "cores": nt, "kind": "oracle",
                               "sample": f"{k} seeded-random tasks ({sub.cells()} cells, {tc:.1f} s)",
                               "parity_exact": bool(np.array_equal(got, ref))}
    print(json.dumps(out))


if __name__ == "__main__":
    main()
