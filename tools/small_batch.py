"""Per-call cost at the paper's batch size: one HaplotypeCaller region per call (C3 regions,
~240 pairs; the paper's PairHMM batches average 189 pairs, PAPER.md L24@575), against the
same regions in one call. Prints one JSON line (profiles/r02_small_batch.json)."""
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import torch

    from paper_conf_ipps_wangxc17_b200 import phmm, synth

    n_regions = int(sys.argv[1]) if len(sys.argv) > 1 else 256
    regions = [synth.config_batch("C3", n_regions=1, region_start=r) for r in range(n_regions)]
    whole = synth.config_batch("C3", n_regions=n_regions)
    cells = whole.cells()
    res = {"workload": "C3 regions (HaplotypeCaller-shaped, 250 bp reads x 4-8 haplotypes of 250-500 bp)",
           "regions": n_regions, "pairs": whole.n_pairs, "mean_pairs_per_region": whole.n_pairs / n_regions,
           "cells": cells}
    ctx = phmm.PairHMM(precision="fp32", timing=True)
    dbs = [phmm.DeviceBatch.from_host(b, device="cuda:0") for b in regions]
    dwhole = phmm.DeviceBatch.from_host(whole, device="cuda:0")
    for db in dbs[:8]:
        ctx.compute_batch_dev(db)
    ctx.compute_batch_dev(dwhole)
    torch.cuda.synchronize()
    # one call per region, device buffers
    launches, syncs = [], []
    t0 = time.perf_counter()
    outs = []
    for db in dbs:
        o, _ = ctx.compute_batch_dev(db)
        outs.append(o)
        launches.append(ctx.stats()["kernel_launches"])
    torch.cuda.synchronize()
    t_dev = time.perf_counter() - t0
    # one call per region, host buffers
    t0 = time.perf_counter()
    for b in regions:
        ctx.compute_batch(b)
    t_host = time.perf_counter() - t0
    # one submission per region (phmm_submit), then wait for all (after one untimed round
    # that sizes the queue's host buffers)
    for t in [ctx.submit(b) for b in regions]:
        t.wait()
    t0 = time.perf_counter()
    tickets = [ctx.submit(b) for b in regions] if not os.environ.get("NO_SUBMIT") else []
    for t in tickets:
        t.wait()
    t_sub = max(time.perf_counter() - t0, 1e-9)
    same_sub = all(np.array_equal(t.out, o.cpu().numpy()) for t, o in zip(tickets, outs))
    # all regions in one call
    reps = 5
    t0 = time.perf_counter()
    for _ in range(reps):
        o_all, _ = ctx.compute_batch_dev(dwhole)
    torch.cuda.synchronize()
    t_one = (time.perf_counter() - t0) / reps
    same = bool(np.array_equal(torch.cat(outs).cpu().numpy(), o_all.cpu().numpy()))
    res.update({
        "per_region_dev": {"ms_per_call": 1e3 * t_dev / n_regions, "gcups": cells / t_dev / 1e9,
                           "kernel_launches_per_call": float(np.mean(launches))},
        "per_region_host": {"ms_per_call": 1e3 * t_host / n_regions, "gcups": cells / t_host / 1e9},
        "one_call": {"ms": 1e3 * t_one, "gcups": cells / t_one / 1e9},
        "per_region_submit": {"ms_per_region": 1e3 * t_sub / n_regions, "gcups": cells / t_sub / 1e9,
                              "bitwise_equal_to_per_region_calls": bool(same_sub),
                              "how": "phmm_submit of each region (host buffers), then phmm_wait on every ticket"},
        "bitwise_equal_to_one_call": same,
        "timing": "host wall clock (time.perf_counter) around the synchronous C-ABI calls",
        "paper_context": "PH2 average 6.0 GCUPS on GTX Titan X incl. transfers (PAPER.md L24@2258)",
    })
    print(json.dumps(res), flush=True)
    ctx.close()
    print("closed", file=sys.stderr, flush=True)


if __name__ == "__main__":
    main()
