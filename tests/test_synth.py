"""The seeded generator: determinism, addressability per region, shapes of
the BASELINE.json configs."""
import numpy as np

from paper_conf_ipps_wangxc17_b200 import synth


def test_region_addressable_and_deterministic():
    a = synth.config_batch("C2", n_regions=4, region_start=10)
    b = synth.config_batch("C2", n_regions=4, region_start=10)
    for k in ("read_bases", "base_quals", "hap_bases", "pairs", "read_offsets"):
        assert np.array_equal(getattr(a, k), getattr(b, k))
    whole = synth.config_batch("C2", n_regions=14)
    r10 = synth.config_batch("C2", n_regions=1, region_start=10)
    # region 10 of the whole batch is byte-identical to region 10 generated alone
    ro = whole.read_offsets
    assert whole.read(10 * 16) == r10.read(0)


def test_c1_shape():
    b = synth.config_batch("C1")
    assert b.n_pairs == 64
    assert set(b.read_lengths()) == {100} and set(b.hap_lengths()) == {120}
    assert b.cells() == 64 * 100 * 120


def test_c2_shape_small():
    b = synth.config_batch("C2", n_regions=8)
    assert b.n_pairs == 8 * 16 * 8
    assert set(b.read_lengths()) == {101} and set(b.hap_lengths()) == {300}
    assert set(np.unique(b.ins_quals)) == {45} and set(np.unique(b.gcp_quals)) == {10}
    assert set(np.unique(b.base_quals)) <= {6, 12, 23, 37}


def test_c3_c5_mixed_lengths():
    b3 = synth.config_batch("C3", n_regions=6)
    assert b3.read_lengths().min() >= 150 and b3.read_lengths().max() == 250
    assert 250 <= b3.hap_lengths().min() and b3.hap_lengths().max() <= 500
    b5 = synth.config_batch("C5", n_regions=6)
    m = b5.read_lengths()[b5.pairs[:, 0]]
    n = b5.hap_lengths()[b5.pairs[:, 1]]
    assert np.all(n >= m) and np.all(n <= 2 * m)


def test_alphabet_and_quality_range():
    b = synth.random_pairs_batch(5, 50)
    assert set(np.unique(b.read_bases)) <= set(b"ACGTN")
    assert set(np.unique(b.hap_bases)) <= set(b"ACGTN")
    assert b.base_quals.max() <= 127


def test_generator_heap_is_intact_after_many_regions():
    """Regression: an insertion that filled a haplotype to its target length was followed by
    one more write (one byte past the end); glibc caught the corrupted heap only at exit.
    Generate 2,048 regions of every config in a fresh process and require a clean exit."""
    import subprocess
    import sys

    code = ("import sys; sys.path.insert(0, %r)\n"
            "from paper_conf_ipps_wangxc17_b200 import synth\n"
            "for c in ('C2', 'C3', 'C4', 'C5'):\n"
            "    bs = [synth.config_batch(c, n_regions=1, region_start=r) for r in range(512)]\n"
            "    w = synth.config_batch(c, n_regions=2048)\n"
            "print('ok')\n") % __import__("os").path.dirname(__import__("os").path.dirname(__file__))
    r = subprocess.run([sys.executable, "-c", code], capture_output=True, text=True, timeout=600,
                       env=dict(__import__("os").environ, MALLOC_CHECK_="3"))
    assert r.returncode == 0 and r.stdout.strip() == "ok", r.stderr[-2000:]
