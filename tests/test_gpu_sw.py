"""GPU parity of the Smith-Waterman path (phmm_sw_align_batch, csrc/sw.cuh) against the
CPU oracle (oracle/sw_oracle.c): integer DP, so every output is compared exactly --
score, end cell, start cell, CIGAR runs (readings R20-R25)."""
import numpy as np
import pytest

from oracle import sw as oracle_sw
from paper_conf_ipps_wangxc17_b200 import phmm, synth

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def ctx():
    h = phmm.PairHMM(precision="fp32")
    yield h
    h.close()


def _check(ctx, b, params=phmm.SW_GATK_HC):
    res, ops, off = ctx.sw_align_batch(b, params)
    ref, rops, roff = oracle_sw.batch(b.ref_bases, b.ref_offsets, b.alt_bases, b.alt_offsets, b.tasks, params)
    assert off[-1] == ops.size  # packed: the runs of all tasks back to back
    bad = np.nonzero((res != ref).any(axis=1))[0]
    assert bad.size == 0, f"{bad.size} tasks differ, first {bad[0]}: gpu {res[bad[0]]} oracle {ref[bad[0]]}"
    for t in range(b.n_tasks):
        n = ref[t, 5]
        assert np.array_equal(ops[off[t]:off[t] + n], rops[roff[t]:roff[t] + n]), t
    return res


@pytest.mark.parametrize("params", [phmm.SW_GATK_HC, (1, -1, -1, -1), (2, -1, -2, -1), (5, -4, -10, -1)])
def test_random_ragged_tasks(ctx, params):
    b = synth.sw_random_batch(5, 400, m_range=(1, 70), n_range=(1, 70))
    _check(ctx, b, params)


def test_single_cell_and_tiny(ctx):
    b = synth.sw_random_batch(6, 200, m_range=(1, 3), n_range=(1, 3))
    _check(ctx, b)
    _check(ctx, b, (1, -1, -1, -1))


def test_multi_stripe_rows(ctx):
    """M up to 1,100 rows: up to 5 stripes of 256 rows, the ring carry between them."""
    b = synth.sw_random_batch(7, 24, m_range=(200, 1100), n_range=(50, 700), related=0.8)
    _check(ctx, b)
    _check(ctx, b, (1, -1, -1, -1))


def test_sw1_config_all_tasks(ctx):
    """The paper's re-batched size: 3,200 haplotype-vs-reference tasks (SW1)."""
    b = synth.sw_config_batch("SW1")
    res = _check(ctx, b)
    assert (res[:, 0] > 0).all()
    assert ctx.stats()["cells"] == b.cells()


def test_maximum_columns(ctx):
    b = synth.sw_random_batch(8, 3, m_range=(300, 600), n_range=(4096, 4096), related=1.0)
    _check(ctx, b)


def test_device_variant_equals_host(ctx):
    import torch

    b = synth.sw_config_batch("SW1", n_regions=40)
    res, ops, off = ctx.sw_align_batch(b)
    dev = "cuda:0"
    T = {"ref_bases": torch.from_numpy(b.ref_bases).to(dev), "ref_offsets": torch.from_numpy(b.ref_offsets).to(dev),
         "alt_bases": torch.from_numpy(b.alt_bases).to(dev), "alt_offsets": torch.from_numpy(b.alt_offsets).to(dev),
         "tasks": torch.from_numpy(b.tasks).to(dev), "total_ref_bases": int(b.ref_offsets[-1]),
         "total_alt_bases": int(b.alt_offsets[-1])}
    dops = torch.zeros(int(b.ops_capacity()[-1]), dtype=torch.int32, device=dev)
    dres, _ = ctx.sw_align_batch_dev(T, ops=dops)
    torch.cuda.synchronize()
    assert np.array_equal(dres.cpu().numpy(), res)
    got = dops.cpu().numpy().view(np.uint32)
    for t in range(b.n_tasks):
        assert np.array_equal(got[off[t]:off[t] + res[t, 5]], ops[off[t]:off[t] + res[t, 5]])


@pytest.mark.parametrize("kind,code", [("base", -2), ("index", -5), ("empty", -4), ("too_long", -1),
                                       ("params", -1)])
def test_input_errors(ctx, kind, code):
    b = synth.sw_random_batch(9, 10)
    params = phmm.SW_GATK_HC
    if kind == "base":
        b.alt_bases = b.alt_bases.copy()
        b.alt_bases[2] = ord("x")
    elif kind == "index":
        b.tasks = b.tasks.copy()
        b.tasks[3, 0] = 99
    elif kind == "empty":
        ro = b.ref_offsets.copy()
        ro[2] = ro[1]
        b.ref_offsets = ro
    elif kind == "too_long":
        b = synth.sw_random_batch(9, 2, m_range=(5, 10), n_range=(4097, 4097))
    elif kind == "params":
        params = (200, -150, -5, -11)  # gap_open > gap_extend
    with pytest.raises(phmm.PhmmError) as ei:
        ctx.sw_align_batch(b, params)
    assert ei.value.code == code
    # the context stays usable
    _check(ctx, synth.sw_random_batch(10, 20))
