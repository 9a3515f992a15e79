#!/usr/bin/env python3
"""bench.py -- batched GATK PairHMM forward on B200: GCUPS per GPU and whole job.

Contract (see the task statement / DESIGN.md §7):
  python bench.py [--gpus N] [--steps K] [--warmup W] [--workload C2] [--impl reference]
  N > 1: launched by torch.distributed.run, one rank per GPU (NCCL).

A "step" is one pass of the whole hot path (validate, per-read tables,
length binning, FP32 wavefront, finalize, FP64 rescue) over one batch of
synthetic input: ``phmm_compute_batch_dev`` on
device-resident inputs for ``value``; ``phmm_compute_batch`` from pinned and
from pageable host buffers (H2D + compute + D2H of every result) for ``e2e``.
Each rank generates its own regions from (seed, region id) -- no input moves --
and for N > 1 the step ends with one NCCL all-gather of the results plus their
global pair ids (the path's one exchange step; parallel.py):
  * C5 (default --scaling strong): the fixed 2^26-pair job is split into
    whole-region ranges balanced by cells; ``result_sha256`` (the job's results
    in global pair order) is the same for every GPU count;
  * C2..C4 (default --scaling weak): every rank runs the config's region count.

metric = GCUPS = sum over pairs of m*N / seconds / 1e9 (PAPER.md L22@1416:
the three M/I/D updates of one cell count as one cell update).
"""
from __future__ import annotations

import argparse
import glob
import hashlib
import json
import os
import statistics
import subprocess
import sys
import tempfile
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

# FP32 pipe roofline: 8 FP32-pipe ops per cell (3 FFMA + 4 FMUL + 1 FADD),
# 128 FP32 lanes per SM per clock.
FP32_OPS_PER_CELL = 8
FP32_LANES_PER_SM = 128
FP64_LANES_PER_SM = 64
DFMA_MEASURED_PER_SM = 57.13  # microbench/issue_rates.cu "dfma" (profiles/r01_microbench_issue_rates.jsonl)
SM_MAX_MHZ_FALLBACK = 1965.0

WORKLOADS = {
    "C2": "C2: 1M pairs (8192 regions x 16 reads x 8 haplotypes), 101 bp reads x 300 bp haplotypes, "
          "2% decoy reads, FP32 + FP64 underflow rescue",
    "C3": "C3: HaplotypeCaller-shaped regions, 250 bp reads x 4-8 haplotypes of 250-500 bp",
    "C4": "C4: long-read stress, 1000 bp reads x 1500 bp haplotypes",
    "C5": "C5: 64M pairs (262144 regions x 32 reads x 8 haplotypes), mixed 100-250 bp reads, N ~ U{m..2m}",
}
# regions per rank (weak split) or of the whole job (strong split: C5, the full 2^26 pairs)
DEFAULT_REGIONS = {"C2": 8192, "C3": 4096, "C4": 256, "C5": 262144}
# The paper's PairHMM numbers: other hardware and its HCC1954 dataset,
# context only (vs_baseline stays null).
PAPER_CONTEXT = {
    "PH2_peak_gcups": 34.8, "PH2_avg_gcups": 6.0,
    "hardware": "NVIDIA GTX Titan X (Maxwell), 6,611 GFLOP/s FP32",
    "workload": "HCC1954 PairHMM batches of GATK 3.6 HaplotypeCaller (avg 189 pairs), incl. host<->device transfer",
    "PH2_over_PH1": "2.1x on Quadro K1200 (kernel time)",
    "source": "PAPER.md L24@2217, L24@2258, L26@1631",
}


def _ncu_traffic(workload):
    """dram__bytes_read.sum + dram__bytes_write.sum of one k_wavefront<float> launch from the
    latest committed ncu --set full capture (profiles/r*_wavefront_traffic.json), for the
    workload that capture was taken on (C2); None otherwise."""
    if workload != "C2":
        return None, None
    files = sorted(glob.glob(os.path.join(ROOT, "profiles", "r*_wavefront_traffic.json")))
    for fn in reversed(files):
        try:
            d = json.load(open(fn))
        except (OSError, ValueError):
            continue
        if d.get("kernel") == "k_wavefront<float>":
            return float(d["dram_bytes_read_plus_write"]), os.path.relpath(fn, ROOT)
    return None, None


def _algorithmic_bytes(b):
    """Bytes the FP32 pass must move at least once: read bases + 4 quality
    arrays, haplotype bases, pair indices, one float result per pair."""
    return int(5 * b.read_bases.size + b.hap_bases.size + 8 * b.n_pairs + 4 * b.n_pairs)


def _measured_peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            return json.load(f)
    except Exception:  # noqa: BLE001
        return {}


class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled every 200 ms during the timed region."""

    FIELDS = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu_index: int):
        self.gpu = gpu_index
        self.proc = None
        self.path = None

    def start(self):
        fd, self.path = tempfile.mkstemp(prefix="clk_", suffix=".csv")
        os.close(fd)
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.gpu), f"--query-gpu={self.FIELDS}",
                                          "--format=csv,noheader,nounits", "-lms", "200"],
                                         stdout=open(self.path, "w"), stderr=subprocess.DEVNULL)
        except Exception:  # noqa: BLE001
            self.proc = None

    def stop(self) -> dict:
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        time.sleep(0.25)
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:  # noqa: BLE001
            self.proc.kill()
        sm, smax, power, reasons = [], [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        with open(self.path) as f:
            for line in f:
                parts = [p.strip() for p in line.split(",")]
                if len(parts) < 9:
                    continue
                try:
                    sm.append(float(parts[1]))
                    smax.append(float(parts[2]))
                    power.append(float(parts[3]))
                except ValueError:
                    continue
                for nm, v in zip(names, parts[5:9]):
                    if v.lower().startswith("active"):
                        reasons.add(nm)
        os.unlink(self.path)
        if not sm:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["no samples"]}
        return {"sm_mhz": statistics.median(sm), "sm_max_mhz": max(smax), "power_w_max": max(power),
                "samples": len(sm), "reasons": sorted(reasons)}


def _dist():
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return ws, rank, local


def run_reference(args, ws, rank):
    """--impl reference: the oracle (plain C, fp64, OpenMP) as it stands on the
    host cores, on a bounded sample of the same workload each step."""
    if rank != 0:
        return 0
    from oracle import core as oracle
    from paper_conf_ipps_wangxc17_b200 import synth

    n_regions = max(1, int(args.ref_regions))
    cores = oracle.max_threads()
    batches = [synth.config_batch(args.workload, n_regions=n_regions, region_start=i * n_regions)
               for i in range(args.warmup + args.steps)]
    for b in batches[:args.warmup]:
        oracle.batch_log10(b)
    t_total, cells = 0.0, 0
    for b in batches[args.warmup:]:
        t0 = time.perf_counter()
        oracle.batch_log10(b)
        t_total += time.perf_counter() - t0
        cells += b.cells()
    gcups = cells / t_total / 1e9
    sample = f"{n_regions} regions ({batches[-1].n_pairs} pairs, {batches[-1].cells()} cells) of {args.workload} per step"
    line = {"metric": "PairHMM GCUPS", "value": gcups, "unit": "GCUPS", "n_gpus": ws, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": 1e3 * t_total / max(1, args.steps), "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "impl": "reference",
            "config": {"workload": WORKLOADS[args.workload], "sample": sample},
            "cpu_baseline": {"value": gcups, "unit": "GCUPS", "cores": cores, "kind": "oracle", "sample": sample},
            "e2e": {"value": gcups, "unit": "GCUPS", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


def cpu_baseline(args, batch):
    """The oracle timed on this box's host cores on a bounded sample (~10-30 s)."""
    from oracle import core as oracle

    cores = oracle.max_threads()
    rng = np.random.default_rng(7)
    cells_per_pair = batch.pair_cells()
    # size the sample: probe, then aim for ~args.cpu_seconds
    probe = rng.choice(batch.n_pairs, size=min(batch.n_pairs, 64 * cores), replace=False)
    t0 = time.perf_counter()
    oracle.batch_log10(batch, pair_idx=probe)
    dt = time.perf_counter() - t0
    rate = cells_per_pair[probe].sum() / max(dt, 1e-6)
    n_target = int(min(batch.n_pairs, max(len(probe), args.cpu_seconds * rate / cells_per_pair.mean())))
    sample = np.sort(rng.choice(batch.n_pairs, size=n_target, replace=False))
    t0 = time.perf_counter()
    ref = oracle.batch_log10(batch, pair_idx=sample)
    dt = time.perf_counter() - t0
    cells = int(cells_per_pair[sample].sum())
    # the same oracle on one core (SURVEY §8d asks for both), ~3 s of work
    rate1 = cells / dt / max(1, cores)
    n1 = int(min(len(sample), max(16, 3.0 * rate1 / cells_per_pair.mean())))
    s1 = sample[:n1]
    t0 = time.perf_counter()
    oracle.batch_log10(batch, pair_idx=s1, nthreads=1)
    dt1 = time.perf_counter() - t0
    oracle.batch_log10(batch, pair_idx=s1[:1], nthreads=cores)  # restore the OpenMP thread count
    c1 = int(cells_per_pair[s1].sum())
    return {"value": cells / dt / 1e9, "unit": "GCUPS", "cores": cores, "kind": "oracle",
            "sample": f"{n_target} seeded-random pairs of the timed batch ({cells} cells, {dt:.1f} s)",
            "value_1core": c1 / dt1 / 1e9,
            "sample_1core": f"first {n1} pairs of that sample ({c1} cells, {dt1:.1f} s, 1 thread)"}, sample, ref


def _e2e_leg(args, ctx, batch, ws, flush, stream, gloo, n_slot, pair_start, pinned: bool, inflight: int = 1):
    """Same metric through the host-buffer C-ABI call: H2D of the step's inputs, the whole
    path, D2H of the results, every step (wall clock around the synchronous call, max over
    ranks). pinned: inputs and outputs in page-locked host memory; otherwise plain numpy
    (pageable) arrays, which the library stages through its own pinned buffers. N > 1: every
    rank's results land in its own host memory -- a distributed caller consumes its shard
    where it computed it; the cross-rank gather of the results is the device step's (NCCL)."""
    import torch
    import torch.distributed as dist

    from paper_conf_ipps_wangxc17_b200 import phmm

    keys = ("read_bases", "base_quals", "ins_quals", "del_quals", "gcp_quals", "read_offsets", "hap_bases",
            "hap_offsets", "pairs")
    host = {}
    for k in keys:
        a = np.ascontiguousarray(getattr(batch, k))
        host[k] = torch.from_numpy(a).pin_memory() if pinned else torch.from_numpy(a.copy())
    s = phmm._Batch()
    for k, t in host.items():
        setattr(s, k, t.data_ptr())
    s.n_reads, s.n_haps, s.n_pairs = batch.n_reads, batch.n_haps, batch.n_pairs
    s.total_read_bases = int(batch.read_offsets[-1])
    s.total_hap_bases = int(batch.hap_offsets[-1])
    n = batch.n_pairs
    hslot = torch.full((n_slot + 2,), float("nan"), dtype=torch.float64)
    if pinned:
        hslot = hslot.pin_memory()
    hslot[0], hslot[1] = float(pair_start), float(n)
    hout = hslot[2:2 + n]
    hst = torch.empty(n, dtype=torch.uint8)
    if pinned:
        hst = hst.pin_memory()
    h2d = int(sum(t.numel() * t.element_size() for t in host.values()))
    d2h = n * (8 + 1)

    def one():
        rc = ctx.compute_batch_raw(s, hout.data_ptr(), hst.data_ptr())
        assert rc == 0, rc

    for _ in range(max(1, args.warmup)):
        one()
    if ws > 1:
        dist.barrier()
    torch.cuda.synchronize()
    if inflight > 1:
        # phmm_compute_batch_async with `inflight` batches in flight: step k's inputs are copied
        # to the device while step k-1 computes; every step still copies its inputs and reads
        # its results back (alternating result buffers); timed from the first submission to the
        # last result
        outs = [(hout, hst)] + [(torch.empty(n, dtype=torch.float64).pin_memory(),
                                 torch.empty(n, dtype=torch.uint8).pin_memory()) for _ in range(inflight - 1)]
        # warm-up of the async path itself (its device input regions are allocated on first use)
        wq = [ctx.compute_batch_async_raw(s, o.data_ptr(), st_.data_ptr()) for o, st_ in outs]
        for t in wq:
            assert ctx.wait_raw(t) == 0
        if ws > 1:
            dist.barrier()
        t0 = time.perf_counter()
        q = []
        for i in range(args.steps):
            o, st_ = outs[i % inflight]
            q.append(ctx.compute_batch_async_raw(s, o.data_ptr(), st_.data_ptr()))
            if len(q) >= inflight:
                assert ctx.wait_raw(q.pop(0)) == 0
        while q:
            assert ctx.wait_raw(q.pop(0)) == 0
        t_e = time.perf_counter() - t0
        if ws > 1:
            tt = torch.tensor([t_e], dtype=torch.float64)
            dist.all_reduce(tt, op=dist.ReduceOp.MAX, group=gloo)
            t_e = float(tt.item())
        return {"unit": "GCUPS", "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h,
                "ms_per_step": 1e3 * t_e / args.steps, "seconds": t_e, "batches_in_flight": inflight,
                "host_buffers": "pinned (page-locked)",
                "api": "phmm_compute_batch_async + phmm_wait (no input copy; the next batch's H2D overlaps "
                       "this batch's compute)"}
    e_ms = []
    for i in range(args.steps):
        with torch.cuda.stream(stream):
            flush.fill_(i & 0xff)
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        one()
        e_ms.append((time.perf_counter() - t0) * 1e3)
    t_e = sum(e_ms) / 1e3
    if ws > 1:
        tt = torch.tensor([t_e], dtype=torch.float64)
        dist.all_reduce(tt, op=dist.ReduceOp.MAX, group=gloo)
        t_e = float(tt.item())
    return {"unit": "GCUPS", "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h,
            "ms_per_step": 1e3 * t_e / args.steps, "seconds": t_e,
            "host_buffers": "pinned (page-locked)" if pinned else "pageable numpy (library-staged)"}


def run_extra(ctx, workload, n_regions, args, stream, flush):
    """A secondary workload on the same context (the HaplotypeCaller-shaped C3 beside C2):
    device-resident GCUPS, wavefront and rescue time."""
    import torch

    from paper_conf_ipps_wangxc17_b200 import phmm, synth

    b = synth.config_batch(workload, n_regions=n_regions)
    with torch.cuda.stream(stream):
        db = phmm.DeviceBatch.from_host(b, device=torch.cuda.current_device())
        out = torch.empty(b.n_pairs, dtype=torch.float64, device=db.pairs.device)
        st = torch.empty(b.n_pairs, dtype=torch.uint8, device=db.pairs.device)
    for _ in range(2):
        ctx.compute_batch_dev(db, out=out, status=st)
    torch.cuda.synchronize()
    ms, wf, rs = [], [], []
    for i in range(max(3, args.steps // 2)):
        with torch.cuda.stream(stream):
            flush.fill_(i & 0xff)
        a, z = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(stream)
        ctx.compute_batch_dev(db, out=out, status=st)
        z.record(stream)
        z.synchronize()
        ms.append(a.elapsed_time(z))
        x = ctx.stats()
        wf.append(x["ms_wavefront"])
        rs.append(x["ms_rescue"])
    cells = b.cells()
    st_h = st.cpu().numpy()
    return {"workload": WORKLOADS[workload], "regions": n_regions, "pairs": b.n_pairs, "cells": cells,
            "value": cells / (np.mean(ms) / 1e3) / 1e9, "unit": "GCUPS", "ms_per_step": float(np.mean(ms)),
            "wavefront_ms": float(np.mean(wf)), "kernel_gcups": cells / (np.mean(wf) / 1e3) / 1e9,
            "rescue_ms": float(np.mean(rs)), "rescued_pairs": int(np.sum(st_h >= 1))}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--workload", default="C2", choices=sorted(WORKLOADS))
    ap.add_argument("--regions", type=int, default=None,
                    help="strong: the job's regions; weak: regions per rank (default: the config's)")
    ap.add_argument("--scaling", default=None, choices=["weak", "strong"],
                    help="N > 1 split (default: strong for C5 -- the fixed 2^26-pair job split by cells "
                         "(SURVEY §8e) -- weak, a fixed shard per rank, otherwise)")
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--ref-regions", type=int, default=16, help="regions per step for --impl reference")
    ap.add_argument("--cpu-seconds", type=float, default=12.0)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-extra", action="store_true", help="skip the secondary C3 object")
    ap.add_argument("--profile-steps", action="store_true", help="short run for ncu (no clocks/cpu)")
    args = ap.parse_args()

    ws, rank, local = _dist()
    if args.impl == "reference":
        return run_reference(args, ws, rank)

    import torch
    import torch.distributed as dist

    from paper_conf_ipps_wangxc17_b200 import parallel, phmm, synth

    # PHMM_BENCH_BACKEND=gloo (tests only): ranks may share a GPU and the result gather goes
    # through host memory -- exercises the N > 1 path on a one-GPU box; NCCL is the product path
    backend = os.environ.get("PHMM_BENCH_BACKEND", "nccl")
    if backend not in ("nccl", "gloo"):
        raise SystemExit(f"PHMM_BENCH_BACKEND must be nccl or gloo, not {backend!r}")
    local = local % max(1, torch.cuda.device_count()) if backend == "gloo" else local
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    gloo = None
    if ws > 1:
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=dev)
            gloo = dist.new_group(backend="gloo")  # host-side reductions / the e2e legs' host gather
        else:
            dist.init_process_group("gloo")
            gloo = dist.group.WORLD

    scaling = args.scaling or ("strong" if args.workload == "C5" else "weak")
    n_regions = args.regions or DEFAULT_REGIONS[args.workload]
    r0, r1, pair_start, total_pairs, total_cells, cells = parallel.shard(args.workload, rank, ws, scaling,
                                                                         n_regions)
    batch = synth.config_batch(args.workload, n_regions=r1 - r0, region_start=r0)
    assert batch.cells() == cells
    n_pairs = batch.n_pairs

    stream = torch.cuda.Stream(device=dev)
    ctx = phmm.PairHMM(device=local, precision="fp32", stream=stream.cuda_stream, timing=True)
    # the result gather (parallel.py): every rank's slot = [pair_start, count, results, pad]
    n_slot = n_pairs
    if ws > 1:
        nn = torch.tensor([n_pairs], dtype=torch.int64)
        dist.all_reduce(nn, op=dist.ReduceOp.MAX, group=gloo)
        n_slot = int(nn.item())
    with torch.cuda.stream(stream):
        db = phmm.DeviceBatch.from_host(batch, device=dev)
        slot = parallel.pack_slot(torch.empty(0, dtype=torch.float64, device=dev), pair_start, n_slot)
        slot[1] = float(n_pairs)
        out = slot[2:2 + n_pairs]  # the library writes its results straight into the slot
        status = torch.empty(n_pairs, dtype=torch.uint8, device=dev)
        flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)  # > 126 MB L2
    torch.cuda.synchronize()
    gathered = [None]

    def step():
        ctx.compute_batch_dev(db, out=out, status=status)
        if ws > 1:
            with torch.cuda.stream(stream):
                gathered[0] = parallel.gather_slots(slot if backend == "nccl" else slot.cpu(), ws)

    for _ in range(max(args.warmup, 0)):
        step()
    torch.cuda.synchronize()

    clk = ClockSampler(local)
    if not args.profile_steps:
        clk.start()
        time.sleep(0.3)
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    wf_ms, resc_ms, launches, rescued = [], [], 0, 0
    if ws > 1:
        dist.barrier()
    torch.cuda.synchronize()
    for i in range(args.steps):
        with torch.cuda.stream(stream):
            flush.fill_(i & 0xff)  # L2 flush between timed steps (not timed)
            ev[i][0].record(stream)
        step()
        ev[i][1].record(stream)
        st = ctx.stats()
        wf_ms.append(st["ms_wavefront"])
        resc_ms.append(st["ms_rescue"])
        launches += st["kernel_launches"]
        rescued = st["n_rescued"]
    torch.cuda.synchronize()
    if ws > 1:
        dist.barrier()
    step_ms = [a.elapsed_time(b) for a, b in ev]
    clocks = clk.stop() if not args.profile_steps else {}
    t_rank = sum(step_ms) / 1e3
    if ws > 1:
        tt = torch.tensor([t_rank], dtype=torch.float64)
        dist.all_reduce(tt, op=dist.ReduceOp.MAX, group=gloo)
        t_max = float(tt.item())
    else:
        t_max = t_rank
    # the whole job's cells (strong: the fixed region set; weak: every rank's shard)
    job_cells = total_cells
    value = job_cells * args.steps / t_max / 1e9

    # the job's results in global pair order (rank 0), and their hash: identical for every GPU
    # count under the strong split (every pair's arithmetic is independent of its shard)
    result_hash = None
    if rank == 0:
        g = gathered[0].cpu().numpy() if ws > 1 else slot.view(1, -1).cpu().numpy()
        glob = parallel.unpack_global(g, total_pairs)
        result_hash = hashlib.sha256(glob.tobytes()).hexdigest()

    # ---- e2e: host API (H2D + compute + D2H each step), pinned and pageable host buffers
    e2e = None
    if not args.no_e2e and not args.profile_steps:
        e_pin = _e2e_leg(args, ctx, batch, ws, flush, stream, gloo, n_slot, pair_start, pinned=True)
        e_pag = _e2e_leg(args, ctx, batch, ws, flush, stream, gloo, n_slot, pair_start, pinned=False)
        e2e = {"value": job_cells * args.steps / e_pin["seconds"] / 1e9, "unit": "GCUPS",
               "h2d_bytes_per_step": e_pin["h2d_bytes_per_step"], "d2h_bytes_per_step": e_pin["d2h_bytes_per_step"],
               "ms_per_step": e_pin["ms_per_step"], "host_buffers": e_pin["host_buffers"],
               "timing": "host wall clock around phmm_compute_batch (synchronous C-ABI call), max over ranks",
               "pageable": {"value": job_cells * args.steps / e_pag["seconds"] / 1e9, "unit": "GCUPS",
                            "ms_per_step": e_pag["ms_per_step"], "host_buffers": e_pag["host_buffers"]}}
        e2e["pageable_over_pinned"] = e2e["pageable"]["value"] / e2e["value"]
        e_asy = _e2e_leg(args, ctx, batch, ws, flush, stream, gloo, n_slot, pair_start, pinned=True, inflight=2)
        e2e["streamed"] = {"value": job_cells * args.steps / e_asy["seconds"] / 1e9, "unit": "GCUPS",
                           "ms_per_step": e_asy["ms_per_step"], "batches_in_flight": e_asy["batches_in_flight"],
                           "host_buffers": e_asy["host_buffers"], "api": e_asy["api"],
                           "timing": "host wall clock from the first submission to the last result, max over ranks"}

    # ---- roofline of the dominant kernel (the FP32 wavefront), live CUDA events
    nsm = torch.cuda.get_device_properties(dev).multi_processor_count
    peaks = _measured_peaks()
    sm_max = float(peaks.get("sm_max_mhz", SM_MAX_MHZ_FALLBACK))
    peak_gcups = nsm * FP32_LANES_PER_SM * sm_max * 1e6 / FP32_OPS_PER_CELL / 1e9
    wf = float(np.mean(wf_ms)) if wf_ms else float("nan")
    achieved = cells / (wf / 1e3) / 1e9 if wf > 0 else None
    sm_run = clocks.get("sm_mhz") if clocks else None
    traffic, traffic_src = _ncu_traffic(args.workload if args.regions is None else None)
    roofline = {"bound": "alu", "achieved": achieved, "peak": peak_gcups, "unit": "GCUPS",
                "frac": (achieved / peak_gcups) if achieved else None, "traffic": traffic,
                "traffic_unit": "bytes per launch (dram read + write)", "traffic_source": traffic_src,
                "algorithmic_bytes_per_launch": _algorithmic_bytes(batch),
                "kernel": "k_wavefront<float>",
                "peak_basis": f"{nsm} SM x {FP32_LANES_PER_SM} FP32 lanes x {sm_max:.0f} MHz (MEASURED_PEAKS sm_max_mhz)"
                              f" / {FP32_OPS_PER_CELL} FP32-pipe ops per cell (3 FFMA + 4 FMUL + 1 FADD)",
                "frac_at_run_clock": (achieved / (peak_gcups * sm_run / sm_max)) if (achieved and sm_run) else None,
                "wavefront_ms": wf, "wavefront_share_of_step": wf / (sum(step_ms) / len(step_ms))}

    # ---- the FP64 rescue pass (table build + k_wavefront<double> on the compacted list) against
    # the FP64 pipe roofline: 64 FP64 lanes per SM, same 8 ops per cell
    st_host = status.cpu().numpy()
    resc_cells = int(batch.pair_cells()[st_host >= 1].sum())
    peak64 = nsm * FP64_LANES_PER_SM * sm_max * 1e6 / FP32_OPS_PER_CELL / 1e9
    rms = float(np.mean(resc_ms)) if resc_ms else 0.0
    r_gcups = resc_cells / (rms / 1e3) / 1e9 if rms > 0 else None
    rescue = {"pairs": int(np.sum(st_host >= 1)), "cells": resc_cells, "ms": rms, "achieved": r_gcups,
              "peak": peak64, "unit": "GCUPS", "frac": (r_gcups / peak64) if r_gcups else None,
              "kernel": "k_wavefront<double> (+ its per-read table build)",
              "peak_basis": f"{nsm} SM x {FP64_LANES_PER_SM} FP64 lanes x {sm_max:.0f} MHz / {FP32_OPS_PER_CELL} ops per cell",
              # the DFMA rate the microbenchmark measured on this pool's B200 (57.1 lane-ops/clk/SM,
              # profiles/r01_microbench_issue_rates.jsonl) instead of the nominal 64
              "peak_measured_dfma": nsm * DFMA_MEASURED_PER_SM * sm_max * 1e6 / FP32_OPS_PER_CELL / 1e9,
              "frac_measured_dfma": (r_gcups / (nsm * DFMA_MEASURED_PER_SM * sm_max * 1e6 / FP32_OPS_PER_CELL / 1e9))
              if r_gcups else None}

    cpu = None
    if rank == 0 and ws == 1 and not args.no_cpu_baseline and not args.profile_steps:
        cpu, sample_idx, ref = cpu_baseline(args, batch)
        got = out.cpu().numpy()[sample_idx]
        fin = np.isfinite(ref)
        cpu["parity_max_abs_log10"] = float(np.max(np.abs(got[fin] - ref[fin]))) if fin.any() else 0.0

    extra = None
    if ws == 1 and not args.no_extra and not args.profile_steps and args.workload == "C2" and args.regions is None:
        extra = {"C3": run_extra(ctx, "C3", DEFAULT_REGIONS["C3"], args, stream, flush)}
        # the FP64 path (PHMM_PREC_FP64, BASELINE configs[0]'s precision) on the whole of C2,
        # against the FP64 pipe roofline (64 FP64 lanes per SM, 8 ops per cell)
        ctx64 = phmm.PairHMM(device=local, precision="fp64", stream=stream.cuda_stream, timing=True)
        x = run_extra(ctx64, "C2", DEFAULT_REGIONS["C2"], args, stream, flush)
        ctx64.close()
        peak64 = nsm * FP64_LANES_PER_SM * sm_max * 1e6 / FP32_OPS_PER_CELL / 1e9
        x.update({"precision": "fp64 (every pair)", "kernel": "k_wavefront<double>",
                  "kernel_frac_fp64_roofline": x["kernel_gcups"] / peak64, "fp64_roofline_gcups": peak64})
        extra["C2_fp64"] = x

    if rank == 0:
        split = (f"strong: the fixed {n_regions}-region job split over {ws} rank(s) by cells (whole regions)"
                 if scaling == "strong" else f"weak: {n_regions} regions per rank")
        line = {"metric": "PairHMM GCUPS", "value": value, "unit": "GCUPS", "n_gpus": ws, "steps": args.steps,
                "warmup": args.warmup, "ms_per_step": 1e3 * t_max / args.steps,
                "ms_per_step_median": float(np.median(step_ms)), "higher_is_better": True,
                "scaling": scaling, "vs_baseline": None, "dtype": "f32", "data": "synthetic",
                "config": {"workload": WORKLOADS[args.workload], "split": split,
                           "regions_rank0": r1 - r0, "pairs_rank0": n_pairs, "cells_rank0": cells,
                           "job_pairs": total_pairs, "job_cells": total_cells,
                           "padded_cells_rank0": ctx.stats()["padded_cells"],
                           "rescued_pairs_rank0": rescued, "chunks_rank0": ctx.stats()["n_chunks"],
                           "l2": "flushed between timed steps (256 MiB write, untimed)",
                           "parallelism": f"dp{ws} (independent region shards, one NCCL all-gather of results)"},
                "result_sha256": result_hash,
                "gpu_launches": launches,
                "roofline": roofline, "rescue": rescue, "cpu_baseline": cpu, "e2e": e2e, "clocks": clocks,
                "extra": extra, "paper_context": PAPER_CONTEXT}
        print(json.dumps(line), flush=True)
    ctx.close()
    if ws > 1:
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
