"""GPU parity: libphmm (through the C ABI) against the CPU oracle, element by
element on the same seeded inputs (BASELINE.json north_star tolerances):
  * FP64 path: |d log10| <= 1e-9 * max(|ref|, 1e-3)   (relative, R15)
  * FP32 + rescue path: |d log10| <= 1e-3 absolute
Every pair the oracle computes is compared; -inf must match -inf.
"""
import dataclasses
import math

import numpy as np
import pytest

from oracle import core as oracle
from paper_conf_ipps_wangxc17_b200 import phmm, synth

pytestmark = pytest.mark.gpu

TOL_FP64_REL = 1e-9
TOL_FP32_ABS = 1e-3


@pytest.fixture(scope="module")
def ctx32():
    h = phmm.PairHMM(precision="fp32")
    yield h
    h.close()


@pytest.fixture(scope="module")
def ctx64():
    h = phmm.PairHMM(precision="fp64")
    yield h
    h.close()


def _check(got, ref, mode):
    got = np.asarray(got, dtype=np.float64)
    ref = np.asarray(ref, dtype=np.float64)
    assert got.shape == ref.shape
    ninf_ref = np.isneginf(ref)
    assert np.array_equal(np.isneginf(got), ninf_ref), "−inf mismatch"
    ok = ~ninf_ref
    assert np.all(np.isfinite(got[ok]))
    d = np.abs(got[ok] - ref[ok])
    if mode == "fp64":
        bound = TOL_FP64_REL * np.maximum(np.abs(ref[ok]), 1e-3)
    else:
        bound = np.full_like(d, TOL_FP32_ABS)
    bad = np.nonzero(d > bound)[0]
    assert bad.size == 0, f"{bad.size} pairs out of tolerance; worst {d.max():.3e} at ref {ref[ok][np.argmax(d)]}"
    return float(d.max()) if d.size else 0.0


def test_c1_fp64(ctx64):
    b = synth.config_batch("C1")
    got, st = ctx64.compute_batch(b)
    _check(got, oracle.batch_log10(b), "fp64")
    assert np.all(st == 0)


def test_c1_fp32(ctx32):
    b = synth.config_batch("C1")
    got, st = ctx32.compute_batch(b)
    _check(got, oracle.batch_log10(b), "fp32")


@pytest.mark.parametrize("seed", [1, 2, 3])
def test_random_edge_pairs_fp64(ctx64, seed):
    """Ragged tiny pairs: m, N in 1..60, Q0..60, 'N' bases, m > N."""
    b = synth.random_pairs_batch(seed, 400, m_range=(1, 60), n_range=(1, 60))
    got, _ = ctx64.compute_batch(b)
    _check(got, oracle.batch_log10(b), "fp64")


@pytest.mark.parametrize("seed", [4, 5, 6])
def test_random_edge_pairs_fp32(ctx32, seed):
    b = synth.random_pairs_batch(seed, 400, m_range=(1, 60), n_range=(1, 60))
    got, st = ctx32.compute_batch(b)
    _check(got, oracle.batch_log10(b), "fp32")
    assert set(np.unique(st)) <= {0, 1, 2}


def test_single_cell_pairs(ctx32, ctx64):
    b = synth.random_pairs_batch(9, 64, m_range=(1, 1), n_range=(1, 1))
    ref = oracle.batch_log10(b)
    _check(ctx64.compute_batch(b)[0], ref, "fp64")
    _check(ctx32.compute_batch(b)[0], ref, "fp32")


def test_c2_reduced_all_pairs(ctx32):
    """C2 shape (101 x 300, 16 reads x 8 haplotypes per region, 2 % decoys)."""
    b = synth.config_batch("C2", n_regions=48)
    got, st = ctx32.compute_batch(b)
    _check(got, oracle.batch_log10(b), "fp32")
    stats = ctx32.stats()
    assert stats["n_rescued"] == int(np.sum(st == 1) + np.sum(st == 2))
    assert stats["cells"] == b.cells()


def test_c3_reduced_mixed_lengths(ctx32):
    b = synth.config_batch("C3", n_regions=6)
    got, _ = ctx32.compute_batch(b)
    _check(got, oracle.batch_log10(b), "fp32")


def test_c4_reduced_long_reads(ctx32):
    """1000 x 1500: 8 passes of 128 rows per lane stream, ring carry of 1502 columns."""
    b = synth.config_batch("C4", n_regions=1)
    got, st = ctx32.compute_batch(b)
    ref = oracle.batch_log10(b)
    _check(got, ref, "fp32")
    # the ring rescale keeps long pairs inside the FP32 range: most of the
    # pairs below the 1e-28 scaled threshold (log10 P < -64) come back from the FP32 pass
    n_low = int(np.sum(ref < -64.2))
    assert n_low > 10
    assert int(np.sum(st == 1)) < n_low // 2, (int(np.sum(st == 1)), n_low)


def test_forced_rescue_is_fp64_exact(ctx32):
    """Random reads against random haplotypes: log10 P ~ -150, every pair
    underflows FP32 and must come back through the FP64 rescue at FP64
    accuracy."""
    rng = np.random.default_rng(3)
    b = synth.random_pairs_batch(21, 60, m_range=(150, 200), n_range=(200, 260), qual_range=(30, 40),
                                 indel_qual_range=(40, 45), gcp_range=(10, 10), n_frac=0.0)
    got, st = ctx32.compute_batch(b)
    ref = oracle.batch_log10(b)
    assert np.all(ref < -64.2)
    assert np.all(st == 1)
    _check(got, ref, "fp64")


def test_fp64_underflow_gives_minus_inf(ctx32):
    """Q60 mismatches everywhere: P < 1e-700, below even the FP64 scale."""
    m = 400
    b = synth.Batch(read_bases=np.frombuffer(b"A" * m, np.uint8).copy(),
                    base_quals=np.full(m, 60, np.uint8), ins_quals=np.full(m, 60, np.uint8),
                    del_quals=np.full(m, 60, np.uint8), gcp_quals=np.full(m, 60, np.uint8),
                    read_offsets=np.array([0, m], np.int64),
                    hap_bases=np.frombuffer(b"C" * 500, np.uint8).copy(), hap_offsets=np.array([0, 500], np.int64),
                    pairs=np.array([[0, 0]], np.int32))
    got, st = ctx32.compute_batch(b)
    assert oracle.batch_log10(b)[0] < -2000
    assert np.isneginf(got[0]) and st[0] == 2
    assert ctx32.stats()["n_fp64_underflow"] == 1 and ctx32.stats()["n_rescued"] == 1


def test_order_and_batch_invariance_bitwise(ctx32):
    """Each pair's result is bitwise identical whatever the batch order or
    composition (a pair's rows never mix with its neighbours': Z/R pad rows)."""
    b = synth.config_batch("C3", n_regions=3)
    base, _ = ctx32.compute_batch(b)
    perm = np.random.default_rng(0).permutation(b.n_pairs)
    got, _ = ctx32.compute_batch(b.subset(perm))
    assert np.array_equal(got, base[perm])
    half = perm[: b.n_pairs // 2]
    got2, _ = ctx32.compute_batch(b.subset(half))
    assert np.array_equal(got2, base[half])
    mixed = synth.concat_batches([synth.random_pairs_batch(77, 50), b])
    got3, _ = ctx32.compute_batch(mixed)
    assert np.array_equal(got3[50:], base)


def test_host_and_device_variants_agree(ctx32):
    import torch

    b = synth.config_batch("C2", n_regions=6)
    host, hst = ctx32.compute_batch(b)
    db = phmm.DeviceBatch.from_host(b, device="cuda:0")
    dev, dst = ctx32.compute_batch_dev(db)
    torch.cuda.synchronize()
    assert np.array_equal(dev.cpu().numpy(), host)
    assert np.array_equal(dst.cpu().numpy(), hst)


def _sentinel(n):
    return np.full(n, 12345.0), np.full(n, 77, np.uint8)


@pytest.mark.parametrize("kind,code", [("base", -2), ("qual", -3), ("empty", -4), ("index", -5)])
def test_input_errors_leave_outputs_untouched(ctx32, kind, code):
    b = synth.random_pairs_batch(2, 20)
    if kind == "base":
        b.read_bases[3] = ord("x")
    elif kind == "qual":
        b.ins_quals[5] = 200
    elif kind == "empty":
        ro = b.read_offsets.copy()
        ro[4] = ro[3]  # read 3 becomes empty; read 4 absorbs its bases
        b.read_offsets = ro
    elif kind == "index":
        b.pairs = b.pairs.copy()
        b.pairs[7, 1] = 20
    out, st = _sentinel(b.n_pairs)
    with pytest.raises(phmm.PhmmError) as ei:
        ctx32.compute_batch(b, out=out, status=st)
    assert ei.value.code == code
    assert np.all(out == 12345.0) and np.all(st == 77)
    # the context stays usable
    good = synth.random_pairs_batch(2, 5)
    got, _ = ctx32.compute_batch(good)
    _check(got, oracle.batch_log10(good), "fp32")


def test_empty_batch(ctx32):
    b = synth.random_pairs_batch(2, 3)
    b.pairs = np.zeros((0, 2), np.int32)
    got, st = ctx32.compute_batch(b)
    assert got.size == 0


def test_full_c2_sampled(ctx32):
    """BASELINE configs[1] at full size (2^20 pairs), the launch bench.py times:
    a seeded sample of pairs plus every rescued pair against the oracle."""
    import torch

    b = synth.config_batch("C2")
    assert b.n_pairs == 1 << 20
    db = phmm.DeviceBatch.from_host(b, device="cuda:0")
    out, st = ctx32.compute_batch_dev(db)
    torch.cuda.synchronize()
    out = out.cpu().numpy()
    st = st.cpu().numpy()
    rng = np.random.default_rng(123)
    sample = np.unique(np.concatenate([rng.choice(b.n_pairs, 3000, replace=False), np.nonzero(st != 0)[0][:3000]]))
    ref = oracle.batch_log10(b, pair_idx=sample)
    _check(out[sample], ref, "fp32")
    # decoy reads (2 %) make some pairs need the rescue
    assert 0 < np.sum(st == 1) < b.n_pairs // 10


@pytest.mark.parametrize("cfg,regions", [("C4", 256), ("C5", 8192), ("C3", 4096)])
def test_bench_configs_sampled(ctx32, cfg, regions):
    """The other bench workloads at the size bench.py times them (C4: 16,384 pairs of
    1,000 x 1,500 with the ring rescale; C5-shaped shard: 2^21 mixed pairs; C3: ~1e6 mixed
    pairs): a seeded sample of pairs plus rescued and ring-rescaled pairs against the oracle."""
    import torch

    b = synth.config_batch(cfg, n_regions=regions)
    db = phmm.DeviceBatch.from_host(b, device="cuda:0")
    out, st = ctx32.compute_batch_dev(db)
    torch.cuda.synchronize()
    out = out.cpu().numpy()
    st = st.cpu().numpy()
    rng = np.random.default_rng(7)
    cells = b.pair_cells()
    k = max(40, int(2e9 / cells.mean()) // 10)  # ~2e8 oracle cells
    sample = np.unique(np.concatenate([rng.choice(b.n_pairs, min(k, b.n_pairs), replace=False),
                                       rng.permutation(np.nonzero(st != 0)[0])[:k // 4]]))
    ref = oracle.batch_log10(b, pair_idx=sample)
    _check(out[sample], ref, "fp32")
    if cfg == "C4":
        # pairs far below the FP32 range come back from the FP32 pass (ring rescale)
        fp32_low = (st[sample] == 0) & (ref < -70)
        assert fp32_low.sum() > 0


def _long_short_mix(seed, n_long, n_short, long_range=(4000, 4094)):
    """Haplotypes up to the maximum length (4094) mixed with short ones: the long
    bins run in the second, reduced-occupancy wavefront launch."""
    long_ = synth.random_pairs_batch(seed, n_long, m_range=(1, 150), n_range=long_range, qual_range=(20, 40))
    short = synth.random_pairs_batch(seed + 1, n_short, m_range=(1, 120), n_range=(1, 300))
    b = synth.concat_batches([short, long_])
    return b


def test_max_hap_length_fp32(ctx32):
    b = _long_short_mix(31, 12, 300)
    assert int(b.hap_lengths().max()) <= 4094
    got, _ = ctx32.compute_batch(b)
    _check(got, oracle.batch_log10(b), "fp32")


def test_max_hap_length_fp64(ctx64):
    b = _long_short_mix(33, 8, 200)
    got, _ = ctx64.compute_batch(b)
    _check(got, oracle.batch_log10(b), "fp64")


def test_exact_max_hap_length(ctx32, ctx64):
    b = synth.random_pairs_batch(35, 6, m_range=(1, 80), n_range=(4094, 4094))
    ref = oracle.batch_log10(b)
    _check(ctx32.compute_batch(b)[0], ref, "fp32")
    _check(ctx64.compute_batch(b)[0], ref, "fp64")


def test_hap_too_long_is_invalid_arg(ctx32):
    b = synth.random_pairs_batch(36, 2, m_range=(5, 10), n_range=(4095, 4095))
    with pytest.raises(phmm.PhmmError) as ei:
        ctx32.compute_batch(b)
    assert ei.value.code == -1


def test_c4_reduced_fp64(ctx64):
    """FP64 mode with 1500-column haplotypes (32-byte ring slots: the second launch class)."""
    b = synth.config_batch("C4", n_regions=1)
    got, _ = ctx64.compute_batch(b)
    _check(got, oracle.batch_log10(b), "fp64")


def test_long_rows_flat_gap_chains_no_overflow(ctx32):
    """The ring rescale's overflow bound (every cell after a rescale to 2^112
    is <= 2 * ncols * the ring row's max) near its worst: gap continuation Q1 (mu = epsilon =
    0.79: D chains that barely decay along a row; Q0 would make beta = 0 and P = 0) and the
    largest gap-open probabilities R16 allows (Q4), on long reads of the C4 shape. Every pair
    must come out finite and within the FP32 tolerance, whether the FP32 pass keeps it or the
    FP64 rescue takes it."""
    b = synth.config_batch("C4", n_regions=1).subset(range(24))
    b.gcp_quals = np.ones_like(b.gcp_quals)
    b.ins_quals = np.full_like(b.ins_quals, 4)
    b.del_quals = np.full_like(b.del_quals, 4)
    got, st = ctx32.compute_batch(b)
    ref = oracle.batch_log10(b)
    assert np.all(np.isfinite(got))
    _check(got, ref, "fp32")
    assert np.sum(st == 0) > 0  # some pairs stay in the FP32 pass (through the rescale)


def test_rescue_tables_shared_by_read(ctx32):
    """The FP64 rescue builds one table per distinct read of the rescued pairs (DESIGN.md
    §4.6): 6 random reads against 10 random haplotypes each (every pair far below the FP32
    range), the pairs shuffled so that a read's pairs are scattered through the rescue list,
    plus a few in-range pairs in between. Rescued pairs must match the oracle at FP64
    accuracy; the result must not depend on the pair order."""
    b = synth.random_pairs_batch(31, 60, m_range=(120, 160), n_range=(180, 240), qual_range=(30, 40),
                                 indel_qual_range=(40, 45), gcp_range=(10, 10), n_frac=0.0)
    pairs = np.stack([np.repeat(np.arange(6), 10), np.arange(60)], axis=1).astype(np.int32)
    good = np.stack([np.arange(6, 12), np.arange(6, 12)], axis=1).astype(np.int32)  # read i vs its own hap i
    perm = np.random.default_rng(4).permutation(66)
    b.pairs = np.ascontiguousarray(np.concatenate([pairs, good])[perm])
    b.hap_offsets = b.hap_offsets.copy()
    # haplotypes 6..11 become copies of reads 6..11 (in-range pairs)
    reads = [b.read_bases[b.read_offsets[i]:b.read_offsets[i + 1]] for i in range(b.n_reads)]
    haps = [b.hap_bases[b.hap_offsets[i]:b.hap_offsets[i + 1]] for i in range(b.n_haps)]
    for i in range(6, 12):
        haps[i] = reads[i].copy()
    b.hap_bases = np.ascontiguousarray(np.concatenate(haps))
    b.hap_offsets = np.concatenate([[0], np.cumsum([h.size for h in haps])]).astype(np.int64)
    got, st = ctx32.compute_batch(b)
    ref = oracle.batch_log10(b)
    resc = st == 1
    assert resc.sum() == 60 and np.all(st[~resc] == 0)
    _check(got[resc], ref[resc], "fp64")
    _check(got[~resc], ref[~resc], "fp32")
    inv = np.argsort(perm)
    got2, _ = ctx32.compute_batch(b.subset(inv))
    assert np.array_equal(got2, got[inv])


def test_full_c2_fp64_mode_sampled(ctx64):
    """The FP64 path (PHMM_PREC_FP64) on the whole of BASELINE configs[1] (2^20 pairs):
    a seeded sample against the oracle at the north star's 1e-9 relative tolerance."""
    import torch

    b = synth.config_batch("C2")
    db = phmm.DeviceBatch.from_host(b, device="cuda:0")
    out, st = ctx64.compute_batch_dev(db)
    torch.cuda.synchronize()
    out = out.cpu().numpy()
    sample = np.random.default_rng(321).choice(b.n_pairs, 2000, replace=False)
    _check(out[sample], oracle.batch_log10(b, pair_idx=sample), "fp64")


@pytest.mark.parametrize("seed", [41, 42])
def test_fully_ragged_one_batch(ctx32, ctx64, seed):
    """One batch that spans every launch kind at once: random m in 1..400 and N in 1..2000
    (many length bins, multi-block reads, long-row launches with ring carry) with random
    Q0..60 base qualities (part of the pairs fall below the FP32 range and are rescued)."""
    b = synth.random_pairs_batch(seed, 160, m_range=(1, 400), n_range=(1, 2000))
    ref = oracle.batch_log10(b)
    got32, st = ctx32.compute_batch(b)
    _check(got32, ref, "fp32")
    assert set(np.unique(st)) <= {0, 1, 2}
    _check(ctx64.compute_batch(b)[0], ref, "fp64")


@pytest.mark.parametrize("seed,iq", [(51, (60, 127)), (52, (60, 127)), (53, (4, 127))])
def test_high_indel_and_gcp_qualities_near_rescue_threshold(ctx32, ctx64, seed, iq):
    """Indel and gap-continuation qualities drawn per base from Q60-127 (or Q4-127): the
    rescaled 5-op form stores M^ = a_i M with a_i = k_i zeta_i down to 10^-12.7, so these
    push the FP32 pass's values toward the subnormal range. Reads with 8-22 substitutions
    against their own haplotype put log10 P on both sides of the rescue threshold (-64.1);
    the pairs the FP32 pass keeps must be within 1e-3 like every other pair, and the FP64
    mode within 1e-9 relative."""
    b = synth.near_threshold_batch(seed, 400, indel_qual_range=iq, gcp_range=iq)
    ref = oracle.batch_log10(b)
    near = (ref > -64.1236) & (ref < -58.0)
    assert near.sum() >= 20 and (ref < -64.2).sum() >= 50
    got, st = ctx32.compute_batch(b)
    _check(got, ref, "fp32")
    # the near-threshold pairs are the FP32 pass's own results (scaled sum >= 1e-28)
    assert np.all(st[near & (ref > -63.5)] == 0)
    _check(ctx64.compute_batch(b)[0], ref, "fp64")


@pytest.mark.parametrize("qi,qd", [(3, 3), (0, 10), (2, 3), (10, 0)])
def test_r16_non_distribution_transitions_rejected(ctx32, ctx64, qi, qd):
    """DESIGN.md reading R16: e(qi) + e(qd) > 1 (only possible with qi or qd <= 3) makes the
    transitions out of M exceed 1; the call returns PHMM_E_INVALID_QUAL and leaves the
    outputs untouched, in both precisions."""
    b = synth.random_pairs_batch(3, 10, indel_qual_range=(20, 40))
    b.ins_quals = b.ins_quals.copy()
    b.del_quals = b.del_quals.copy()
    k = int(b.read_offsets[4]) + 1 if b.read_offsets[5] - b.read_offsets[4] > 1 else int(b.read_offsets[4])
    b.ins_quals[k] = qi
    b.del_quals[k] = qd
    for ctx in (ctx32, ctx64):
        out, st = _sentinel(b.n_pairs)
        with pytest.raises(phmm.PhmmError) as ei:
            ctx.compute_batch(b, out=out, status=st)
        assert ei.value.code == -3
        assert np.all(out == 12345.0) and np.all(st == 77)
    # qi = qd = 4: e(4) + e(4) = 0.796 <= 1 is accepted
    b.ins_quals[k] = 4
    b.del_quals[k] = 4
    _check(ctx32.compute_batch(b)[0], oracle.batch_log10(b), "fp32")


def test_unused_read_longer_than_cap_is_harmless(ctx32, ctx64):
    """A read of 2^20 + 1 bases that no pair uses (reads longer than 2^20 are only an error
    when a pair uses them, include/phmm.h): the per-read table pass must not write past its
    1-block reservation into other reads' tables. Every other pair must match
    the oracle; a pair that does use the long read returns PHMM_E_INVALID_ARG."""
    small = synth.random_pairs_batch(61, 40, m_range=(1, 120), n_range=(1, 200))
    L = (1 << 20) + 1
    rng = np.random.default_rng(5)
    longb = synth.Batch(read_bases=np.frombuffer(b"ACGT", np.uint8)[rng.integers(0, 4, L)].copy(),
                        base_quals=np.full(L, 30, np.uint8), ins_quals=np.full(L, 45, np.uint8),
                        del_quals=np.full(L, 45, np.uint8), gcp_quals=np.full(L, 10, np.uint8),
                        read_offsets=np.array([0, L], np.int64),
                        hap_bases=np.frombuffer(b"ACGT" * 10, np.uint8).copy(),
                        hap_offsets=np.array([0, 40], np.int64), pairs=np.array([[0, 0]], np.int32))
    # the long read sits in the middle of the read array: its table slot precedes others
    b = synth.concat_batches([synth.random_pairs_batch(62, 20, m_range=(1, 120)), longb, small])
    used = np.ones(b.n_pairs, bool)
    used[20] = False  # the long read's own pair
    ok = b.subset(np.nonzero(used)[0])
    ref = oracle.batch_log10(ok)
    _check(ctx32.compute_batch(ok)[0], ref, "fp32")
    _check(ctx64.compute_batch(ok)[0], ref, "fp64")
    out, st = _sentinel(b.n_pairs)
    with pytest.raises(phmm.PhmmError) as ei:
        ctx32.compute_batch(b, out=out, status=st)
    assert ei.value.code == -1
    assert np.all(out == 12345.0)


def test_dev_variant_follows_torch_stream_and_leaves_outputs_on_error(ctx32):
    """compute_batch_dev on a context without an explicit stream runs on torch's current
    stream (phmm_set_stream): inputs produced by a still-running op on that stream are seen
    complete. On an input error the device outputs keep their contents (results reach them
    only after the whole path succeeded)."""
    import torch

    b = synth.config_batch("C2", n_regions=4)
    ref, _ = ctx32.compute_batch(b)
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        db = phmm.DeviceBatch.from_host(b, device="cuda:0")
        # delay the stream, then overwrite the pairs with the real ones: a library call that
        # did not wait for this stream would read the zeros
        real = db.pairs.clone()
        db.pairs.zero_()
        torch.cuda._sleep(200_000_000)
        db.pairs.copy_(real)
        out, st = ctx32.compute_batch_dev(db)
        got = out.cpu().numpy()
    assert np.array_equal(got, ref)
    with torch.cuda.stream(s):
        bad = phmm.DeviceBatch.from_host(b, device="cuda:0")
        bad.read_bases[7] = ord("x")
        o = torch.full((b.n_pairs,), 12345.0, dtype=torch.float64, device="cuda:0")
        t = torch.full((b.n_pairs,), 77, dtype=torch.uint8, device="cuda:0")
        with pytest.raises(phmm.PhmmError) as ei:
            ctx32.compute_batch_dev(bad, out=o, status=t)
        assert ei.value.code == -2
        assert bool(torch.all(o == 12345.0)) and bool(torch.all(t == 77))
        with pytest.raises(ValueError):
            ctx32.compute_batch_dev(db, out=torch.empty(b.n_pairs, dtype=torch.float32, device="cuda:0"))
        with pytest.raises(ValueError):
            ctx32.compute_batch_dev(db, out=torch.empty(b.n_pairs - 1, dtype=torch.float64, device="cuda:0"))


def test_full_c5_one_gpu_sampled(ctx32):
    """BASELINE configs[4] at its stated size on one B200: 2^26 pairs (262,144 regions, 3.28e12
    cells) in one device call, which runs as 8 chunks of 2^23 pairs. A seeded sample of pairs
    plus rescued pairs against the oracle (1e-3), every result finite or -inf with a status,
    and the chunked call's cell count equal to the job's."""
    import torch

    b = synth.config_batch("C5")
    assert b.n_pairs == 1 << 26
    db = phmm.DeviceBatch.from_host(b, device="cuda:0")
    out, st = ctx32.compute_batch_dev(db)
    torch.cuda.synchronize()
    stats = ctx32.stats()
    assert stats["n_chunks"] == 8 and stats["cells"] == b.cells()
    out = out.cpu().numpy()
    st = st.cpu().numpy()
    del db
    torch.cuda.empty_cache()
    assert np.all(np.isfinite(out) | np.isneginf(out)) and set(np.unique(st)) <= {0, 1, 2}
    assert stats["n_rescued"] == int(np.sum(st >= 1))
    rng = np.random.default_rng(55)
    sample = np.unique(np.concatenate([rng.choice(b.n_pairs, 4000, replace=False),
                                       rng.permutation(np.nonzero(st != 0)[0])[:1000]]))
    _check(out[sample], oracle.batch_log10(b, pair_idx=sample), "fp32")
    # the host-buffer call on the same job (pipelined: 2^23-pair chunks whose inputs a copy thread
    # moves while the previous chunk computes, a rescue per chunk): bitwise the device call
    hout, hst = ctx32.compute_batch(b)
    assert ctx32.stats()["n_chunks"] >= 8
    assert np.array_equal(hout, out) and np.array_equal(hst, st)


@pytest.mark.parametrize("seed", [71, 72, 73, 74])
def test_full_quality_ranges(ctx32, ctx64, seed):
    """Base qualities over the whole accepted range Q0-127, indel qualities Q4-127 (R16 keeps
    e(qi) + e(qd) <= 1), gap continuation Q1-127, 10 % 'N' bases, ragged lengths incl. m > N:
    FP32 + rescue within 1e-3, FP64 within 1e-9 relative, -inf exactly where the oracle's is."""
    b = synth.random_pairs_batch(seed, 300, m_range=(1, 150), n_range=(1, 220), qual_range=(0, 127),
                                 indel_qual_range=(4, 127), gcp_range=(1, 127), n_frac=0.1)
    ref = oracle.batch_log10(b)
    # Q127 mismatches take P below the FP64 pass's range (scale 2^1020, R7): the scaled
    # FP64 sum is subnormal below log10 P = -614.7 (status 2, imprecise by design, not compared)
    # and 0 below ~ -630 (-inf, status 2)
    cmp = ref > -614
    low = ref < -640
    for ctx, mode in ((ctx32, "fp32"), (ctx64, "fp64")):
        got, st = ctx.compute_batch(b)
        _check(got[cmp], ref[cmp], mode)
        assert np.all(np.isneginf(got[low])) and np.all(st[low] == 2)
        assert np.all(st[~cmp] == 2)


def test_device_call_argument_errors(ctx32):
    """The device-buffer call rejects inconsistent sizes and offsets with PHMM_E_INVALID_ARG
    (offsets not starting at 0, decreasing, or not ending at the total) and out-of-range pair
    indices with PHMM_E_INDEX, leaving the outputs untouched."""
    import torch

    b = synth.random_pairs_batch(5, 30)
    cases = []
    ro = b.read_offsets.copy(); ro[3], ro[4] = ro[4], ro[3]       # decreasing
    cases.append(("read_offsets", ro, -1))
    ho = b.hap_offsets.copy(); ho[0] = 1                          # does not start at 0
    cases.append(("hap_offsets", ho, -1))
    pr = b.pairs.copy(); pr[4, 1] = -1                            # negative haplotype index
    cases.append(("pairs", pr, -5))
    for field, arr, code in cases:
        bb = synth.Batch(**{**{k: getattr(b, k) for k in ("read_bases", "base_quals", "ins_quals", "del_quals",
                                                         "gcp_quals", "read_offsets", "hap_bases",
                                                         "hap_offsets", "pairs")}, field: arr})
        db = phmm.DeviceBatch.from_host(bb, device="cuda:0")
        o = torch.full((b.n_pairs,), 3.0, dtype=torch.float64, device="cuda:0")
        with pytest.raises(phmm.PhmmError) as ei:
            ctx32.compute_batch_dev(db, out=o)
        assert ei.value.code == code, (field, ei.value.code)
        assert bool(torch.all(o == 3.0))
    # a total that disagrees with the offsets (the host variant checks it on the host)
    import ctypes

    st, keep = phmm._host_struct(b)
    st.total_read_bases -= 1
    out = np.full(b.n_pairs, 3.0)
    rc = ctx32._L.phmm_compute_batch(ctx32._h, ctypes.byref(st), out.ctypes.data_as(phmm._f64p), None)
    assert rc == -1 and np.all(out == 3.0)
    del keep


def _shifted(t, k):
    """The same bytes at an address k bytes past a 256-byte-aligned allocation."""
    import torch

    buf = torch.empty(t.numel() + 64, dtype=t.dtype, device=t.device)
    v = buf[k:k + t.numel()]
    v.copy_(t)
    return v


@pytest.mark.parametrize("shift", [(0, 0), (3, 3), (1, 5), (4, 4)])
def test_validation_every_alignment_and_position(ctx32, shift):
    """k_validate reads the five read arrays as 16-byte vectors when they share their
    alignment mod 16, as 4-byte words when they share it mod 4, else bytes, and the
    haplotype bases as 16-byte vectors after a scalar head: a bad byte in the head, inside a
    vector or in the tail, at every alignment class, is reported (PHMM_E_INVALID_BASE /
    PHMM_E_INVALID_QUAL) and the outputs stay untouched; the clean batch gives the oracle."""
    import torch

    base = synth.random_pairs_batch(11, 40)
    nrb, nhb = int(base.read_offsets[-1]), int(base.hap_offsets[-1])
    ref = oracle.batch_log10(base)
    rs, qs = shift  # shift of read_bases and of the four quality arrays

    def dev_batch(b):
        db = phmm.DeviceBatch.from_host(b, device="cuda:0")
        db.read_bases = _shifted(db.read_bases, rs)
        for k in ("base_quals", "ins_quals", "del_quals", "gcp_quals"):
            setattr(db, k, _shifted(getattr(db, k), qs))
        db.hap_bases = _shifted(db.hap_bases, rs + 1)
        return db

    got, _ = ctx32.compute_batch_dev(dev_batch(base))
    _check(got.cpu().numpy(), ref, "fp32")
    for pos in sorted({0, 1, 5, 15, 16, 17, 31, nrb // 2, nrb - 2, nrb - 1}):
        for arr, bad, code in (("read_bases", ord("x"), -2), ("del_quals", 200, -3), ("ins_quals", 2, -3)):
            b = dataclasses.replace(base, **{arr: getattr(base, arr).copy()})
            getattr(b, arr)[pos] = bad
            if arr == "ins_quals":  # Q2 insertion with a Q2 deletion: R16 (e(qi) + e(qd) > 1)
                b.del_quals = b.del_quals.copy()
                b.del_quals[pos] = 2
            out = torch.full((b.n_pairs,), 12345.0, dtype=torch.float64, device="cuda:0")
            st = torch.full((b.n_pairs,), 77, dtype=torch.uint8, device="cuda:0")
            with pytest.raises(phmm.PhmmError) as ei:
                ctx32.compute_batch_dev(dev_batch(b), out=out, status=st)
            assert ei.value.code == code, (arr, pos)
            assert bool(torch.all(out == 12345.0)) and bool(torch.all(st == 77))
    for pos in sorted({0, 1, 15, 16, nhb // 2, nhb - 1}):
        b = dataclasses.replace(base, hap_bases=base.hap_bases.copy())
        b.hap_bases[pos] = ord("u")
        with pytest.raises(phmm.PhmmError) as ei:
            ctx32.compute_batch_dev(dev_batch(b))
        assert ei.value.code == -2, pos
