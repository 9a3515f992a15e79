"""The host-buffer call's copies and the device call's chunking.

* phmm_compute_batch stages pageable host buffers through the context's pinned ring
  (host_stage.h) and copies page-locked ones directly: results bitwise equal to the device
  call for either kind of buffer, staged_bytes counting the staged input + output bytes.
* phmm_compute_batch_dev runs batches of more than kDevChunkPairs pairs as consecutive
  chunks (the full 2^26-pair C5 on one GPU): bitwise equal to the one-pass call.
"""
import os

import numpy as np
import pytest

from oracle import core as oracle
from paper_conf_ipps_wangxc17_b200 import phmm, synth

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def batch():
    b = synth.config_batch("C2", n_regions=2048)  # 2^18 pairs, 26 MB per read array: several 8 MiB pieces
    assert b.n_pairs == 1 << 18
    return b


@pytest.fixture(scope="module")
def ctx():
    h = phmm.PairHMM(precision="fp32")
    yield h
    h.close()


def test_pageable_and_pinned_host_buffers_are_bitwise_the_device_call(ctx, batch):
    import torch

    db = phmm.DeviceBatch.from_host(batch, device="cuda:0")
    dev, dst = ctx.compute_batch_dev(db)
    torch.cuda.synchronize()
    dev, dst = dev.cpu().numpy(), dst.cpu().numpy()
    # pageable numpy arrays, pageable outputs
    got, st = ctx.compute_batch(batch)
    assert np.array_equal(got, dev) and np.array_equal(st, dst)
    n = batch.n_pairs
    staged = ctx.stats()["staged_bytes"]
    assert staged == batch.nbytes_inputs() + 9 * n, (staged, batch.nbytes_inputs() + 9 * n)
    # page-locked inputs and outputs: no staging
    pin = {k: torch.from_numpy(np.ascontiguousarray(getattr(batch, k))).pin_memory().numpy()
           for k in ("read_bases", "base_quals", "ins_quals", "del_quals", "gcp_quals", "read_offsets",
                     "hap_bases", "hap_offsets", "pairs")}
    pb = synth.Batch(**pin)
    out = torch.empty(n, dtype=torch.float64).pin_memory().numpy()
    sto = torch.empty(n, dtype=torch.uint8).pin_memory().numpy()
    got2, st2 = ctx.compute_batch(pb, out=out, status=sto)
    assert np.array_equal(got2, dev) and np.array_equal(st2, dst)
    assert ctx.stats()["staged_bytes"] == 0
    # a small batch (below one piece) and an odd-sized one agree with the oracle
    small = synth.random_pairs_batch(3, 77)
    g3, _ = ctx.compute_batch(small)
    ref = oracle.batch_log10(small)
    fin = np.isfinite(ref)
    assert np.max(np.abs(g3[fin] - ref[fin])) <= 1e-3


@pytest.mark.parametrize("prec", ["fp32", "fp64"])
def test_device_call_chunking_is_bitwise(prec):
    """compute_dev runs batches of more than kDevChunkPairs pairs (2^23; PHMM_CHUNK_PAIRS
    lowers it here) as consecutive chunks of pairs over the reads / haplotypes each chunk uses
    (so the full 2^26-pair C5 fits one GPU): results, statuses and the statistics' cell count
    must equal the one-pass call bit for bit, also when a chunk's pairs use reads scattered
    over the whole batch (shuffled pair order) and for a ragged last chunk."""
    import torch

    b = synth.concat_batches([synth.config_batch("C3", n_regions=4), synth.random_pairs_batch(8, 300)])
    b = b.subset(np.random.default_rng(1).permutation(b.n_pairs))
    whole = phmm.PairHMM(precision=prec)
    os.environ["PHMM_CHUNK_PAIRS"] = "1000"
    try:
        chunked = phmm.PairHMM(precision=prec, timing=True)
    finally:
        del os.environ["PHMM_CHUNK_PAIRS"]
    try:
        db = phmm.DeviceBatch.from_host(b, device="cuda:0")
        o1, s1 = whole.compute_batch_dev(db)
        o2, s2 = chunked.compute_batch_dev(db)
        torch.cuda.synchronize()
        assert np.array_equal(o1.cpu().numpy(), o2.cpu().numpy())
        assert np.array_equal(s1.cpu().numpy(), s2.cpu().numpy())
        st = chunked.stats()
        assert st["n_chunks"] == (b.n_pairs + 999) // 1000 and st["cells"] == b.cells()
        assert st["ms_wavefront"] > 0
        h, _ = chunked.compute_batch(b)  # the host variant chunks the same way
        assert np.array_equal(h, o1.cpu().numpy())
        # an index error in the last chunk: no output written
        bad = b.subset(np.arange(b.n_pairs))
        bad.pairs[-1, 0] = b.n_reads
        out = np.full(b.n_pairs, 5.0)
        with pytest.raises(phmm.PhmmError) as ei:
            chunked.compute_batch(bad, out=out)
        assert ei.value.code == -5 and np.all(out == 5.0)
    finally:
        whole.close()
        chunked.close()


def test_submit_queue_coalesces_regions_bitwise():
    """phmm_submit / phmm_wait: 300 region-sized batches (C3 regions, ~240 pairs each)
    submitted one by one are coalesced into few runs; every batch's results equal its own
    synchronous call bit for bit. A batch with an invalid base fails alone (-2, outputs
    untouched) while the batches coalesced with it succeed."""
    ctx = phmm.PairHMM(precision="fp32")
    try:
        regions = [synth.config_batch("C3", n_regions=1, region_start=r) for r in range(300)]
        bad_k = 137
        bad = regions[bad_k].subset(np.arange(regions[bad_k].n_pairs))
        bad.read_bases = bad.read_bases.copy()
        bad.read_bases[5] = ord("Z")
        tickets = []
        for k, b in enumerate(regions):
            src = bad if k == bad_k else b
            out = np.full(src.n_pairs, 7.0)
            tickets.append(ctx.submit(src, out=out))
        for k, t in enumerate(tickets):
            if k == bad_k:
                with pytest.raises(phmm.PhmmError) as ei:
                    t.wait()
                assert ei.value.code == -2 and np.all(t.out == 7.0)
            else:
                got, st = t.wait()
                ref, rst = ctx.compute_batch(regions[k])
                assert np.array_equal(got, ref) and np.array_equal(st, rst), k
        # a ticket can be waited for once
        with pytest.raises(phmm.PhmmError):
            tickets[0].wait()
    finally:
        ctx.close()


@pytest.mark.parametrize("prec", ["fp32", "fp64"])
def test_pipelined_host_call_is_bitwise_the_one_pass_call(prec):
    """A host batch of 2^17 .. 2^23 pairs in region order runs pipelined (compute_host_pipe):
    chunks of n/8 + 7n/8 pairs, alternating between two streams and two buffer sets, whose input bytes reach the
    device on a copy stream while the previous chunk computes; one FP64 rescue over the whole
    batch at the end. Results and statuses must equal the device call and the unpipelined host
    call (PHMM_PIPE=0) bit for bit, pageable and page-locked; staged_bytes counts every input
    byte once; an invalid base or an out-of-range pair index in the LAST chunk fails the call
    with the outputs untouched; a batch whose first chunk uses the last read is not pipelined."""
    import torch

    b = synth.concat_batches([synth.config_batch("C2", n_regions=1536), synth.config_batch("C3", n_regions=128)])
    n = b.n_pairs
    assert n >= 1 << 17
    ctx = phmm.PairHMM(precision=prec)
    os.environ["PHMM_PIPE"] = "0"
    try:
        flat = phmm.PairHMM(precision=prec)
    finally:
        del os.environ["PHMM_PIPE"]
    try:
        db = phmm.DeviceBatch.from_host(b, device="cuda:0")
        dev, dst = ctx.compute_batch_dev(db)
        torch.cuda.synchronize()
        dev, dst = dev.cpu().numpy(), dst.cpu().numpy()
        got, st = ctx.compute_batch(b)
        stats = ctx.stats()
        assert stats["n_chunks"] == 2, stats
        assert stats["staged_bytes"] == b.nbytes_inputs() + 9 * n
        assert stats["cells"] == b.cells()
        assert np.array_equal(got, dev) and np.array_equal(st, dst)
        got0, st0 = flat.compute_batch(b)
        assert flat.stats()["n_chunks"] == 1
        assert np.array_equal(got0, dev) and np.array_equal(st0, dst)
        if prec == "fp32":
            assert stats["n_rescued"] == flat.stats()["n_rescued"] > 0
        pin = {k: torch.from_numpy(np.ascontiguousarray(getattr(b, k))).pin_memory().numpy()
               for k in ("read_bases", "base_quals", "ins_quals", "del_quals", "gcp_quals", "read_offsets",
                         "hap_bases", "hap_offsets", "pairs")}
        out = torch.empty(n, dtype=torch.float64).pin_memory().numpy()
        sto = torch.empty(n, dtype=torch.uint8).pin_memory().numpy()
        got2, st2 = ctx.compute_batch(synth.Batch(**pin), out=out, status=sto)
        assert np.array_equal(got2, dev) and np.array_equal(st2, dst)
        assert ctx.stats()["staged_bytes"] == 0 and ctx.stats()["n_chunks"] == 2
        # errors in the last chunk's bytes / pairs: outputs untouched
        bad = b.subset(np.arange(n))
        bad.read_bases = bad.read_bases.copy()
        bad.read_bases[-3] = ord("x")
        o = np.full(n, 3.0)
        with pytest.raises(phmm.PhmmError) as ei:
            ctx.compute_batch(bad, out=o)
        assert ei.value.code == -2 and np.all(o == 3.0)
        bad = b.subset(np.arange(n))
        bad.pairs[-1, 1] = b.n_haps
        with pytest.raises(phmm.PhmmError) as ei:
            ctx.compute_batch(bad, out=o)
        assert ei.value.code == -5 and np.all(o == 3.0)
        # the context is still usable after the errors
        got3, _ = ctx.compute_batch(b)
        assert np.array_equal(got3, dev)
        # first chunk touching the last read: one pass
        perm = np.arange(n)
        last = int(np.nonzero(b.pairs[:, 0] == b.n_reads - 1)[0][0])
        perm[[0, last]] = perm[[last, 0]]
        sw = b.subset(perm)
        got4, _ = ctx.compute_batch(sw)
        assert ctx.stats()["n_chunks"] == 1
        assert np.array_equal(got4, dev[perm])
    finally:
        ctx.close()
        flat.close()


@pytest.mark.parametrize("prec", ["fp32", "fp64"])
def test_pipelined_small_ragged_batches_are_bitwise(prec):
    """The pipelined host call on small, ragged batches (PHMM_PIPE_MIN lowers its threshold):
    multi-bin C3 regions, long C4 rows, random pairs of 1..60 x 1..80 bases (some below the
    40-column minimum) and decoys, with chunks of a few pairs each; pageable and page-locked
    inputs give the one-pass results bit for bit, statuses included (the C4 pairs too: their ring
    rescale happens at the same rows in any batch, R14); also for 16..100 pairs, where a chunk
    may hold a single pair."""
    import torch

    big = synth.concat_batches([synth.config_batch("C2", n_regions=4),
                                synth.random_pairs_batch(3, 100, m_range=(1, 60), n_range=(1, 80)),
                                synth.config_batch("C3", n_regions=2), synth.config_batch("C4", n_regions=1).subset(range(6))])
    flat_env = {"PHMM_PIPE": "0"}
    os.environ.update(flat_env)
    try:
        flat = phmm.PairHMM(precision=prec)
    finally:
        del os.environ["PHMM_PIPE"]
    os.environ["PHMM_PIPE_MIN"] = "16"
    try:
        pipe = phmm.PairHMM(precision=prec)
    finally:
        del os.environ["PHMM_PIPE_MIN"]
    try:
        for n in (16, 17, 31, 100, big.n_pairs):
            b = big.subset(np.arange(n)) if n < big.n_pairs else big
            ref, rst = flat.compute_batch(b)
            got, gst = pipe.compute_batch(b)
            assert np.array_equal(got, ref) and np.array_equal(gst, rst), n
            assert pipe.stats()["n_chunks"] >= 2, (n, pipe.stats()["n_chunks"])
            pin = synth.Batch(**{k: torch.from_numpy(np.ascontiguousarray(getattr(b, k))).pin_memory().numpy()
                                 for k in ("read_bases", "base_quals", "ins_quals", "del_quals", "gcp_quals",
                                           "read_offsets", "hap_bases", "hap_offsets", "pairs")})
            got2, gst2 = pipe.compute_batch(pin)
            assert np.array_equal(got2, ref) and np.array_equal(gst2, rst), n
    finally:
        flat.close()
        pipe.close()


def test_async_no_copy_batches_are_bitwise_and_prefetched():
    """phmm_compute_batch_async: batches streamed with two in flight (page-locked: the next
    batch's inputs are prefetched into the other device input region while one computes;
    pageable: each runs as phmm_compute_batch) give phmm_compute_batch's results bit for bit,
    in any mix with synchronous calls; a batch with an invalid base fails alone (outputs
    untouched) and the following ones still succeed."""
    import torch

    ctx = phmm.PairHMM(precision="fp32")
    try:
        batches = [synth.config_batch("C2", n_regions=256, region_start=256 * k) for k in range(3)]
        batches.append(synth.config_batch("C3", n_regions=16))
        batches.append(synth.random_pairs_batch(5, 500))
        keys = ("read_bases", "base_quals", "ins_quals", "del_quals", "gcp_quals", "read_offsets", "hap_bases",
                "hap_offsets", "pairs")
        pinned = [synth.Batch(**{k: torch.from_numpy(np.ascontiguousarray(getattr(b, k))).pin_memory().numpy()
                                 for k in keys}) for b in batches]
        refs = [ctx.compute_batch(b) for b in batches]
        bad = batches[1].subset(np.arange(batches[1].n_pairs))
        bad.read_bases = bad.read_bases.copy()
        bad.read_bases[7] = ord("Q")
        badp = synth.Batch(**{k: torch.from_numpy(np.ascontiguousarray(getattr(bad, k))).pin_memory().numpy()
                              for k in keys})
        for rnd in range(2):
            srcs = pinned if rnd == 0 else batches  # page-locked (prefetched), then pageable
            ts = []
            for k, b in enumerate(srcs):
                if k == 2:
                    o = torch.empty(bad.n_pairs, dtype=torch.float64).pin_memory().numpy()
                    o[:] = 9.0
                    ts.append(("bad", ctx.compute_batch_async(badp if rnd == 0 else bad, out=o)))
                ts.append((k, ctx.compute_batch_async(b)))
                if len(ts) >= 3:  # keep two or three in flight
                    k0, t0 = ts.pop(0)
                    _check(k0, t0, refs)
            # a synchronous call in between must not disturb the queued batches
            mid, _ = ctx.compute_batch(batches[0])
            assert np.array_equal(mid, refs[0][0])
            for k0, t0 in ts:
                _check(k0, t0, refs)
    finally:
        ctx.close()


def _check(k, t, refs):
    if k == "bad":
        with pytest.raises(phmm.PhmmError) as ei:
            t.wait()
        assert ei.value.code == -2 and np.all(t.out == 9.0)
        return
    got, st = t.wait()
    assert np.array_equal(got, refs[k][0]) and np.array_equal(st, refs[k][1]), k


def test_pipelined_call_above_the_device_chunk_is_bitwise():
    """A host batch larger than one device chunk (PHMM_CHUNK_PAIRS lowers it to 5,000 pairs
    here) runs pipelined in chunks of at most that many pairs, each with its own FP64 rescue
    (as the chunked device call): bitwise the one-pass call, pageable and page-locked."""
    import torch

    b = synth.concat_batches([synth.config_batch("C2", n_regions=160), synth.config_batch("C3", n_regions=24)])
    os.environ["PHMM_PIPE"] = "0"
    try:
        flat = phmm.PairHMM(precision="fp32")
    finally:
        del os.environ["PHMM_PIPE"]
    os.environ["PHMM_CHUNK_PAIRS"] = "5000"
    os.environ["PHMM_PIPE_MIN"] = "64"
    try:
        pipe = phmm.PairHMM(precision="fp32")
    finally:
        del os.environ["PHMM_CHUNK_PAIRS"]
        del os.environ["PHMM_PIPE_MIN"]
    try:
        ref, rst = flat.compute_batch(b)
        got, gst = pipe.compute_batch(b)
        st = pipe.stats()
        assert st["n_chunks"] >= (b.n_pairs + 4999) // 5000 and st["n_rescued"] == flat.stats()["n_rescued"]
        assert np.array_equal(got, ref) and np.array_equal(gst, rst)
        pin = synth.Batch(**{k: torch.from_numpy(np.ascontiguousarray(getattr(b, k))).pin_memory().numpy()
                             for k in ("read_bases", "base_quals", "ins_quals", "del_quals", "gcp_quals",
                                       "read_offsets", "hap_bases", "hap_offsets", "pairs")})
        got2, gst2 = pipe.compute_batch(pin)
        assert np.array_equal(got2, ref) and np.array_equal(gst2, rst)
    finally:
        flat.close()
        pipe.close()


@pytest.mark.parametrize("window", [1000, 30000, 0])
def test_pipelined_call_with_overlapping_chunk_ranges(window):
    """Pairs shuffled inside windows of `window` pairs (0: the whole batch) so that consecutive
    chunks use overlapping read / haplotype index ranges (a chunk's reads partly brought by the
    previous chunk's bytes; with a full shuffle the first chunk needs everything and the call runs
    as one chunk): bitwise the one-pass call, page-locked and pageable."""
    import torch

    b = synth.concat_batches([synth.config_batch("C2", n_regions=1200), synth.config_batch("C3", n_regions=40)])
    n = b.n_pairs
    rng = np.random.default_rng(window + 5)
    if window:
        perm = np.concatenate([s + rng.permutation(min(window, n - s)) for s in range(0, n, window)])
    else:
        perm = rng.permutation(n)
    bs = b.subset(perm)
    os.environ["PHMM_PIPE"] = "0"
    try:
        flat = phmm.PairHMM(precision="fp32")
    finally:
        del os.environ["PHMM_PIPE"]
    pipe = phmm.PairHMM(precision="fp32")
    try:
        ref, rst = flat.compute_batch(bs)
        got, gst = pipe.compute_batch(bs)
        assert np.array_equal(got, ref) and np.array_equal(gst, rst)
        assert pipe.stats()["n_chunks"] == (1 if window == 0 else 2), pipe.stats()["n_chunks"]
        pin = synth.Batch(**{k: torch.from_numpy(np.ascontiguousarray(getattr(bs, k))).pin_memory().numpy()
                             for k in ("read_bases", "base_quals", "ins_quals", "del_quals", "gcp_quals",
                                       "read_offsets", "hap_bases", "hap_offsets", "pairs")})
        got2, gst2 = pipe.compute_batch(pin)
        assert np.array_equal(got2, ref) and np.array_equal(gst2, rst)
    finally:
        flat.close()
        pipe.close()


def test_random_shapes_stress_bitwise():
    """tools/pipe_stress.py for 15 rounds: random batch shapes (C2/C3/C4 region mixes incl. long
    reads against long haplotypes, local pair shuffles, page-locked or pageable, FP32 or FP64)
    through the pipelined host call, the streamed async call, the device call in 3,000-pair
    chunks and the submission queue (three slices coalesced by the worker), each bit for bit the
    one-pass call (R14)."""
    import subprocess
    import sys

    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    r = subprocess.run([sys.executable, os.path.join(root, "tools", "pipe_stress.py"), "15"], capture_output=True,
                       text=True, timeout=900, cwd=root)
    assert r.returncode == 0 and "all 15 rounds bitwise equal" in r.stdout, r.stdout[-3000:] + r.stderr[-2000:]
