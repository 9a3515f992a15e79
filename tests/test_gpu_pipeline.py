"""The host-buffer call's optional copy/compute pipeline (phmm_compute_batch with
PHMM_CHUNKS=n; off by default, measured slower): large batches are cut into chunks whose H2D overlaps the previous chunk's FP32 pass, with one
FP64 rescue over the whole batch at the end. Results must be bitwise those of the
device-buffer call (one pass over the whole batch) and of the unchunked host call, for any
pair order, and an input error in a late chunk must still leave the outputs untouched."""
import os

import numpy as np
import pytest

from oracle import core as oracle
from paper_conf_ipps_wangxc17_b200 import phmm, synth

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def batch():
    b = synth.config_batch("C2", n_regions=2048)  # 2^18 pairs: 4 chunks
    assert b.n_pairs == 1 << 18
    return b


@pytest.fixture(scope="module")
def ctx():
    os.environ["PHMM_CHUNKS"] = "4"
    try:
        h = phmm.PairHMM(precision="fp32")
    finally:
        del os.environ["PHMM_CHUNKS"]
    yield h
    h.close()


@pytest.fixture(scope="module")
def ctx_one_shot():
    os.environ["PHMM_CHUNKS"] = "1"
    try:
        h = phmm.PairHMM(precision="fp32")
    finally:
        del os.environ["PHMM_CHUNKS"]
    yield h
    h.close()


@pytest.fixture(scope="module")
def reference(batch, ctx):
    import torch

    db = phmm.DeviceBatch.from_host(batch, device="cuda:0")
    out, st = ctx.compute_batch_dev(db)
    torch.cuda.synchronize()
    return out.cpu().numpy(), st.cpu().numpy(), ctx.stats()["n_rescued"]


def test_chunked_host_call_is_bitwise_the_device_call(batch, ctx, ctx_one_shot, reference):
    ref, ref_st, n_resc = reference
    got, st = ctx.compute_batch(batch)
    assert ctx.stats()["n_rescued"] == n_resc > 0
    assert np.array_equal(got, ref) and np.array_equal(st, ref_st)
    one, st1 = ctx_one_shot.compute_batch(batch)
    assert np.array_equal(one, ref) and np.array_equal(st1, ref_st)
    # and against the oracle on a sample (plus rescued pairs)
    rng = np.random.default_rng(5)
    sample = np.unique(np.concatenate([rng.choice(batch.n_pairs, 500, replace=False), np.nonzero(st)[0][:500]]))
    d = np.abs(got[sample] - oracle.batch_log10(batch, pair_idx=sample))
    assert d.max() <= 1e-3


def test_chunked_any_pair_order(batch, ctx, reference):
    """Shuffled pairs: every chunk references reads all over the batch (wide chunk ranges)."""
    ref, ref_st, _ = reference
    perm = np.random.default_rng(9).permutation(batch.n_pairs)
    got, st = ctx.compute_batch(batch.subset(perm))
    assert np.array_equal(got, ref[perm]) and np.array_equal(st, ref_st[perm])
    # reversed order: the reads of the first chunk are the last ones copied
    rev = np.arange(batch.n_pairs)[::-1].copy()
    got, _ = ctx.compute_batch(batch.subset(rev))
    assert np.array_equal(got, ref[rev])


@pytest.mark.parametrize("kind,code", [("base", -2), ("qual", -3), ("index", -5)])
def test_error_in_last_chunk_leaves_outputs_untouched(batch, ctx, kind, code):
    b = batch.subset(np.arange(batch.n_pairs))
    b.read_bases = b.read_bases.copy()
    b.ins_quals = b.ins_quals.copy()
    b.pairs = b.pairs.copy()
    last_read = int(b.pairs[-1, 0])
    x = int(b.read_offsets[last_read]) + 1
    if kind == "base":
        b.read_bases[x] = ord("x")
    elif kind == "qual":
        b.ins_quals[x] = 200
    else:
        b.pairs[-1, 1] = b.n_haps
    out = np.full(b.n_pairs, 12345.0)
    st = np.full(b.n_pairs, 77, np.uint8)
    with pytest.raises(phmm.PhmmError) as ei:
        ctx.compute_batch(b, out=out, status=st)
    assert ei.value.code == code
    assert np.all(out == 12345.0) and np.all(st == 77)
    small = synth.random_pairs_batch(3, 8)
    got, _ = ctx.compute_batch(small)
    assert np.max(np.abs(got - oracle.batch_log10(small))) <= 1e-3
