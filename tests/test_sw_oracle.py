"""Pins of the Smith-Waterman oracle (oracle/sw_oracle.c) against things other than
itself (Eq. 5, L16@3413; readings R20-R25 in DESIGN.md §12):

* S1 brute force: H from an explicit enumeration of every move path (oracle/sw_brute.py);
* S2 the literal Eq. 5 (max over k, l by loops) == the running-max form, H and btrack;
* S3 closed forms: identical sequences, one mismatch, one insertion, one deletion;
* S4 transpose symmetry of the best score over the last row and column;
* S5 every traceback rescored from the sequences equals the reported score and ends at
  the end cell; the end cell holds the maximum of row M and column N;
* S6 hand values (tests/golden/sw_hand_values.tsv).
"""
import os

import numpy as np
import pytest

from oracle import sw, sw_brute

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "sw_hand_values.tsv")
PARAMS = [sw.GATK_HC, (1, -1, -1, -1), (2, -1, -2, -1), (5, -4, -10, -1)]


def _rand_seq(rng, n, alphabet=b"ACGTN"):
    return rng.choice(np.frombuffer(alphabet, dtype=np.uint8), size=n).tobytes()


@pytest.mark.parametrize("params", PARAMS)
def test_s1_brute_force_tiny(params):
    rng = np.random.default_rng(hash(params) & 0xFFFF)
    for _ in range(30):
        a = _rand_seq(rng, int(rng.integers(1, 5)), b"ACGN")
        b = _rand_seq(rng, int(rng.integers(1, 5)), b"ACGN")
        ref = sw_brute.sw_brute_H(a, b, params)
        for literal in (True, False):
            got = sw.align(a, b, params, literal=literal)["H"]
            assert np.array_equal(got, ref), (a, b, params, literal)


@pytest.mark.parametrize("params", PARAMS)
def test_s2_literal_equals_running(params):
    rng = np.random.default_rng(7 + (hash(params) & 0xFF))
    for _ in range(60):
        a = _rand_seq(rng, int(rng.integers(1, 26)), b"ACGT")
        b = _rand_seq(rng, int(rng.integers(1, 26)), b"ACGT")
        x = sw.align(a, b, params, literal=True)
        y = sw.align(a, b, params, literal=False)
        assert np.array_equal(x["H"], y["H"]) and np.array_equal(x["bt"], y["bt"])
        assert (x["score"], x["end"], x["start"], x["cigar"]) == (y["score"], y["end"], y["start"], y["cigar"])


def test_s3_identical_sequences():
    for n in (1, 2, 7, 40, 300):
        s = _rand_seq(np.random.default_rng(n), n, b"ACGT")
        r = sw.align(s, s)
        assert r["score"] == 200 * n and r["end"] == (n, n) and r["start"] == (1, 1) and r["cigar"] == f"{n}M"


def test_s3_one_mismatch():
    a = b"ACGTACGTACGTACGTACGT"
    b = a[:9] + (b"A" if a[9:10] != b"A" else b"C") + a[10:]
    r = sw.align(a, b)
    assert r["score"] == 19 * 200 - 150 and r["cigar"] == "20M" and r["start"] == (1, 1)


def test_s3_one_insertion_and_deletion():
    a = b"ACGTTGCAACGGTACCATGA"  # 20 bases
    b = a[:10] + b"T" + a[10:]   # one extra column base: 'I' (horizontal gap of length 1)
    r = sw.align(a, b)
    assert r["score"] == 20 * 200 - 260
    assert r["cigar"] == "10M1I10M" and r["start"] == (1, 1) and r["end"] == (20, 21)
    r2 = sw.align(b, a)  # transposed: a vertical gap, 'D'
    assert r2["score"] == r["score"] and r2["cigar"] == "10M1D10M"
    b3 = a[:8] + b"GGG" + a[8:]  # gap of length 3: open + 2 extends
    assert sw.align(a, b3)["score"] == 20 * 200 - 260 - 2 * 11


@pytest.mark.parametrize("params", PARAMS)
def test_s4_transpose_symmetry(params):
    rng = np.random.default_rng(11)
    for _ in range(50):
        a = _rand_seq(rng, int(rng.integers(1, 40)))
        b = _rand_seq(rng, int(rng.integers(1, 40)))
        assert sw.align(a, b, params)["score"] == sw.align(b, a, params)["score"]


@pytest.mark.parametrize("params", PARAMS)
def test_s5_traceback_rescores_and_end_is_max(params):
    rng = np.random.default_rng(13)
    for _ in range(80):
        m, n = int(rng.integers(1, 60)), int(rng.integers(1, 60))
        a = _rand_seq(rng, m)
        b = bytearray(a[: min(m, n)]) + bytearray(_rand_seq(rng, max(0, n - m)))
        for k in range(len(b)):  # mutate: similar sequences give long alignments
            if rng.random() < 0.15:
                b[k] = int(rng.choice(list(b"ACGT")))
        b = bytes(b[:n]) if len(b) >= n else bytes(b) + _rand_seq(rng, n - len(b))
        r = sw.align(a, b, params)
        H = r["H"]
        cand = np.concatenate([H[1:, n], H[m, 1:]])
        assert r["score"] == cand.max()
        assert H[r["end"]] == r["score"]
        assert (H >= 0).all()
        s, (ie, je) = sw.rescore(a, b, r["start"], r["ops"], params)
        assert s == r["score"] and (ie, je) == r["end"]
        # the path starts on the boundary or at a cell whose H came from the 0 term
        si, sj = r["start"]
        assert si == 1 or sj == 1 or r["bt"][si - 1, sj - 1] == sw.BT_STOP or r["ops"].size == 0


def test_s5_batch_equals_single():
    rng = np.random.default_rng(17)
    refs = [_rand_seq(rng, int(rng.integers(1, 50))) for _ in range(6)]
    alts = [_rand_seq(rng, int(rng.integers(1, 50))) for _ in range(5)]
    ro = np.concatenate([[0], np.cumsum([len(x) for x in refs])])
    ao = np.concatenate([[0], np.cumsum([len(x) for x in alts])])
    tasks = np.array([(i, j) for i in range(6) for j in range(5)], dtype=np.int32)
    res, ops, off = sw.batch(b"".join(refs), ro, b"".join(alts), ao, tasks, nthreads=4)
    for t, (i, j) in enumerate(tasks):
        r = sw.align(refs[i], alts[j])
        assert tuple(res[t, :5]) == (r["score"], *r["end"], *r["start"])
        assert np.array_equal(ops[off[t]: off[t] + res[t, 5]], r["ops"])


def test_s6_hand_values():
    rows = [l.rstrip("\n").split("\t") for l in open(GOLDEN) if l.strip() and not l.startswith("#")]
    assert len(rows) >= 6
    for a, b, params, score, end, start, cigar, _why in rows:
        p = tuple(int(x) for x in params.split(","))
        r = sw.align(a.encode(), b.encode(), p)
        assert r["score"] == int(score), (a, b)
        assert r["end"] == tuple(int(x) for x in end.split(",")), (a, b)
        assert r["start"] == tuple(int(x) for x in start.split(",")), (a, b)
        assert r["cigar"] == cigar, (a, b, r["cigar"])
