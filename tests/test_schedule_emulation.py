"""The FP32 kernel's schedule, modelled on the CPU (tests/support/emu_wavefront.py):
64 virtual lanes, group switch events, PAD-code idle columns, the ring and the
Z/R/S pad rows. The model must reproduce the oracle within the FP32 tolerance for
both row counts the kernel can be built with, and be independent of pair order."""
import os
import sys

import numpy as np
import pytest

from oracle import core as oracle
from paper_conf_ipps_wangxc17_b200 import synth

sys.path.insert(0, os.path.join(os.path.dirname(__file__), "support"))
import emu_wavefront as emu  # noqa: E402


@pytest.mark.parametrize("K", [4, 8])
def test_emulated_schedule_matches_oracle_multi_pass(K):
    b = synth.random_pairs_batch(12, 40, m_range=(1, 40), n_range=(30, 48))
    ref = oracle.batch_log10(b)
    got = emu.run_batch(b, K=K)
    fin = np.isfinite(ref)
    assert np.array_equal(np.isneginf(got), np.isneginf(ref))
    assert np.max(np.abs(got[fin] - ref[fin])) < 1e-3


def test_emulated_schedule_is_order_independent():
    b = synth.random_pairs_batch(13, 30, m_range=(1, 30), n_range=(38, 44))
    a = emu.run_batch(b)
    perm = list(np.random.default_rng(1).permutation(b.n_pairs))
    c = emu.run_batch(b, order=perm)
    assert np.array_equal(a, c)


def test_emulated_ring_rescale_long_rows():
    """Long rows (ncols >= 768): the ring rescale carries pairs far below
    the FP32 range (log10 P down to about -100) through the FP32 schedule."""
    b = synth.config_batch("C4", n_regions=1).subset(range(10))
    ref = oracle.batch_log10(b)
    got = emu.run_batch(b)
    assert np.min(ref) < -70
    ok = np.isfinite(got)
    assert ok.sum() >= 8
    assert np.max(np.abs(got[ok] - ref[ok])) < 1e-3
