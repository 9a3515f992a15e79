"""Pins for the PairHMM oracle (oracle/phmm_oracle.c) against things other
than itself: exact path enumeration, closed forms, hand-derived values,
invariants. CPU only (-m "not gpu").

PAPER.md prints no PairHMM value, so the pins are:
  P1 brute-force path enumeration (oracle/brute.py), exact in Fractions;
  P2 the m = 1 closed form; P3 the ungapped (delta = zeta = 0) closed form on
  long inputs, evaluated in mpmath -- this also pins the row renormalisation
  far below the double range; P4 hand values (tests/golden/hand_values.tsv);
  P5 reversal symmetry of the M-terminated part; P6 dominance; P7 bounds;
  P8 power-of-two / constant prior scaling.
"""
import math
import os
import random
from fractions import Fraction

import mpmath
import numpy as np
import pytest

from oracle import brute, core
from paper_conf_ipps_wangxc17_b200 import synth

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "hand_values.tsv")


def _rel(a, b):
    return abs(a - b) / max(abs(b), 1e-300)


def _rand_prob(rng, allow_zero=True):
    den = rng.randint(1, 50)
    num = rng.randint(0 if allow_zero else 1, den)
    return Fraction(num, den)


# ---------------------------------------------------------------- P1 brute force
@pytest.mark.parametrize("seed", range(60))
def test_p1_bruteforce_exact_fractions(seed):
    """Probability-domain DP vs exact path enumeration, general (non-GATK)
    alpha..mu so that swapped coefficients or indices are caught."""
    rng = random.Random(1000 + seed)
    m, n = rng.randint(1, 4), rng.randint(1, 4)
    tr = [[_rand_prob(rng) for _ in range(m)] for _ in range(7)]
    prior = [[_rand_prob(rng, allow_zero=False) for _ in range(n)] for _ in range(m)]
    bm, bi = brute.brute_parts(*tr, prior)
    lm, li, lp = core.prob_parts(*[[float(x) for x in t] for t in tr], [[float(x) for x in r] for r in prior])
    for got, exact in ((lm, bm), (li, bi), (lp, bm + bi)):
        if exact == 0:
            assert got == -math.inf
        else:
            assert _rel(10.0 ** got, float(exact)) < 1e-12, (got, exact)


@pytest.mark.parametrize("seed", range(40))
def test_p1_bruteforce_phred(seed):
    """Phred wrapper vs path enumeration (mpmath, 40 digits) with N bases,
    Q0..60, random indel/gcp qualities, m > N allowed."""
    rng = random.Random(seed)
    m, n = rng.randint(1, 5), rng.randint(1, 5)
    alpha = "ACGTN"
    read = "".join(rng.choice(alpha) for _ in range(m))
    hap = "".join(rng.choice(alpha) for _ in range(n))
    q = [rng.randint(0, 60) for _ in range(m)]
    qi = [rng.randint(5, 60) for _ in range(m)]
    qd = [rng.randint(5, 60) for _ in range(m)]
    qg = [rng.randint(3, 40) for _ in range(m)]
    bm, bi = brute.brute_phred(read, q, qi, qd, qg, hap)
    lm, li, lp = core.phred_parts(read, q, qi, qd, qg, hap)
    for got, exact in ((lm, bm), (li, bi), (lp, bm + bi)):
        if exact == 0:
            assert got == -math.inf
        else:
            assert abs(got - float(mpmath.log10(exact))) < 1e-12 * max(1.0, abs(got)), (got, exact)


def test_p1_bruteforce_5x5_float():
    """A few 5x5 cases in Fractions (the largest size the enumerator does quickly)."""
    rng = random.Random(7)
    for _ in range(3):
        m = n = 5
        tr = [[_rand_prob(rng) for _ in range(m)] for _ in range(7)]
        prior = [[_rand_prob(rng, allow_zero=False) for _ in range(n)] for _ in range(m)]
        bm, bi = brute.brute_parts(*tr, prior)
        _, _, lp = core.prob_parts(*[[float(x) for x in t] for t in tr], [[float(x) for x in r] for r in prior])
        assert _rel(10.0 ** lp, float(bm + bi)) < 1e-12


# ---------------------------------------------------------------- P2 m = 1
@pytest.mark.parametrize("seed", range(10))
def test_p2_single_base_read_closed_form(seed):
    """m = 1: I(1,.) = 0, so P = (gamma_1/N) * sum_j P(1,j)."""
    rng = random.Random(seed)
    n = rng.randint(1, 300)
    hap = "".join(rng.choice("ACGTN") for _ in range(n))
    rb = rng.choice("ACGTN")
    q, qg = rng.randint(0, 60), rng.randint(1, 40)
    eb = mpmath.mpf(10) ** (-mpmath.mpf(q) / 10)
    eg = mpmath.mpf(10) ** (-mpmath.mpf(qg) / 10)
    s = sum((1 - eb) if (rb == h or rb == "N" or h == "N") else eb / 3 for h in hap)
    exact = (1 - eg) / n * s
    lp = core.phred_log10(rb, [q], [45], [45], [qg], hap)
    if exact == 0:
        assert lp == -math.inf
    else:
        assert abs(lp - float(mpmath.log10(exact))) < 1e-12 * max(1, abs(lp))


# ---------------------------------------------------------------- P3 ungapped
@pytest.mark.parametrize("m,n,seed", [(1, 7, 0), (30, 30, 1), (150, 400, 2), (400, 420, 3), (700, 1500, 4)])
def test_p3_ungapped_closed_form_long(m, n, seed):
    """delta = zeta = 0 removes every gap: P = (gamma_1/N) * sum_{c=0}^{N-m}
    prod_i P(i, c+i) * prod_{i>=2} alpha_i. With mismatch priors ~1e-4 the
    terms reach 1e-2000 and beyond, far under the double range, so this also
    pins the power-of-two row renormalisation."""
    rng = np.random.default_rng(seed)
    prior = np.where(rng.random((m, n)) < 0.7, rng.uniform(0.5, 1.0, (m, n)), rng.uniform(1e-5, 1e-3, (m, n)))
    alpha = rng.uniform(0.5, 1.0, m)
    beta = rng.uniform(0.1, 1.0, m)
    gamma = rng.uniform(0.1, 1.0, m)
    eps = rng.uniform(0.0, 0.5, m)
    mu = rng.uniform(0.0, 0.5, m)
    zeros = np.zeros(m)
    _, li, lp = core.prob_parts(alpha, beta, gamma, zeros, eps, zeros, mu, prior)
    with mpmath.workdps(30):
        la = sum(mpmath.log(mpmath.mpf(float(a))) for a in alpha[1:])
        terms = []
        for c in range(0, n - m + 1):
            terms.append(sum(mpmath.log(mpmath.mpf(float(prior[i, c + i]))) for i in range(m)))
        mx = max(terms)
        lse = mx + mpmath.log(sum(mpmath.exp(t - mx) for t in terms))
        exact = mpmath.log(mpmath.mpf(float(gamma[0])) / n) + la + lse
        exact10 = float(exact / mpmath.log(10))
    assert li == -math.inf
    assert abs(lp - exact10) < 1e-12 * max(1.0, abs(exact10)), (lp, exact10)


# ---------------------------------------------------------------- P4 hand values
def _golden():
    rows = []
    with open(GOLDEN) as f:
        for line in f:
            if line.startswith("#") or line.startswith("read\t") or not line.strip():
                continue
            read, hap, val, _ = line.rstrip("\n").split("\t")
            rows.append((read, hap, float(val)))
    return rows


@pytest.mark.parametrize("read,hap,expected", _golden())
def test_p4_hand_values(read, hap, expected):
    m = len(read)
    lp = core.phred_log10(read, [30] * m, [45] * m, [45] * m, [10] * m, hap)
    assert abs(lp - expected) < 1e-13 * max(1.0, abs(expected))


GOLDEN_ROWS = os.path.join(os.path.dirname(__file__), "golden", "hand_values_rows.tsv")


def _golden_rows():
    rows = []
    with open(GOLDEN_ROWS) as f:
        for line in f:
            if line.startswith("#") or line.startswith("read\t") or not line.strip():
                continue
            read, hap, q, qi, qd, qg, val, _ = line.rstrip("\n").split("\t")
            ints = lambda s: [int(x) for x in s.split(",")]
            rows.append((read, hap, ints(q), ints(qi), ints(qd), ints(qg), float(val)))
    return rows


@pytest.mark.parametrize("read,hap,q,qi,qd,qg,expected", _golden_rows())
def test_p4_hand_values_per_row_qualities(read, hap, q, qi, qd, qg, expected):
    """qi != qd and per-row qualities: pins which quality feeds M->I and M->D (R2) and
    that a transition uses its destination row's qualities (R3)."""
    lp = core.phred_log10(read, q, qi, qd, qg, hap)
    assert abs(lp - expected) < 1e-13 * max(1.0, abs(expected)), (lp, expected)
    # the same inputs with qi and qd swapped must NOT give the hand value (the pin is not
    # symmetric in the two gap-open qualities)
    swapped = core.phred_log10(read, q, qd, qi, qg, hap)
    assert abs(swapped - expected) > 0.1, (swapped, expected)


@pytest.mark.parametrize("seed", range(20))
def test_insertion_quality_governs_extra_read_base(seed):
    """A 2-base read against a 1-base haplotype can only be explained by an insertion
    after the first base (column 0 of row 2 is 0): P = e(qi_2) * (1 - e(qg_1)) * pm_1,
    exactly, for ANY deletion qualities (R2: delta = e(qi) is the M->I transition, R3:
    the destination row's qi)."""
    rng = random.Random(seed)
    q = [rng.randint(6, 60) for _ in range(2)]
    qi = [rng.randint(4, 60) for _ in range(2)]
    qg = [rng.randint(4, 60) for _ in range(2)]
    e = lambda x: 10.0 ** (-x / 10.0)
    want = math.log10(e(qi[1]) * (1.0 - e(qg[0])) * (1.0 - e(q[0])))
    vals = set()
    for _ in range(4):
        qd = [rng.randint(4, 127) for _ in range(2)]
        lp = core.phred_log10("AA", q, qi, qd, qg, "A")
        assert abs(lp - want) < 1e-13 * abs(want), (lp, want)
        vals.add(lp)
    assert len(vals) == 1  # bitwise independent of qd


@pytest.mark.parametrize("qd1", [15, 20, 25, 30])
def test_deletion_quality_governs_missing_hap_base(qd1):
    """Read "AC" against haplotype "AGC" at Q80 base qualities and a tiny insertion rate:
    every path but the deletion of the haplotype's G (M(1,1) -> D(1,2) -> M(2,3)) carries a
    mismatch (px = 3.3e-9) or an insertion (1e-9), so P is proportional to zeta_1 = e(qd_1),
    the deletion quality of the row the deletion happens in (R2, R3): P(qd1) / P(qd1 + 10)
    = 10 to 1e-3."""
    q, qi, qg = [80, 80], [90, 90], [10, 10]
    a = core.phred_log10("AC", q, qi, [qd1, 40], qg, "AGC")
    b = core.phred_log10("AC", q, qi, [qd1 + 10, 40], qg, "AGC")
    assert abs((a - b) - 1.0) < 1e-3, a - b
    # the row-2 deletion quality barely matters (a D move in row 2 ends in D, not counted)
    c = core.phred_log10("AC", q, qi, [qd1, 10], qg, "AGC")
    assert abs(c - a) < 1e-4


def test_p4_q0_zero_probability():
    """Q0 base quality gives pm = 1 - 10^0 = 0: a 1-base read that matches a
    1-base haplotype has P = 0 exactly (log10 = -inf), SURVEY §8c P7."""
    assert core.phred_log10("A", [0], [45], [45], [10], "A") == -math.inf
    assert core.phred_log10("A", [0], [45], [45], [10], "C") > -1.0  # px = 1/3


# ---------------------------------------------------------------- P5 symmetry
@pytest.mark.parametrize("seed", range(30))
def test_p5_reversal_symmetry_of_m_part(seed):
    """With qi, qd, qg constant along the read, reversing (read, base quals,
    haplotype) maps every path ending in M onto one starting in M and back,
    so sum_j M(m,j) is invariant (the full M+I is NOT: a read cannot start in
    I; reading R8 restates the north-star invariant this way)."""
    rng = random.Random(seed)
    m, n = rng.randint(1, 60), rng.randint(1, 80)
    read = "".join(rng.choice("ACGTN") for _ in range(m))
    hap = "".join(rng.choice("ACGTN") for _ in range(n))
    q = [rng.randint(0, 50) for _ in range(m)]
    ci, cd, cg = rng.randint(10, 50), rng.randint(10, 50), rng.randint(3, 30)
    a = core.phred_parts(read, q, [ci] * m, [cd] * m, [cg] * m, hap)[0]
    b = core.phred_parts(read[::-1], q[::-1], [ci] * m, [cd] * m, [cg] * m, hap[::-1])[0]
    if a == -math.inf:
        assert b == -math.inf
    else:
        assert abs(a - b) < 1e-11 * max(1.0, abs(a))


# ---------------------------------------------------------------- P6 dominance
@pytest.mark.parametrize("seed", range(20))
def test_p6_identical_dominates_single_mismatch(seed):
    rng = random.Random(seed)
    m = rng.randint(2, 120)
    read = "".join(rng.choice("ACGT") for _ in range(m))
    q = [rng.randint(20, 45) for _ in range(m)]
    ones = lambda v: [v] * m
    ident = core.phred_log10(read, q, ones(45), ones(45), ones(10), read)
    for _ in range(5):
        pos = rng.randrange(m)
        alt = "ACGT".replace(read[pos], "")
        hap = read[:pos] + rng.choice(alt) + read[pos + 1:]
        assert ident > core.phred_log10(read, q, ones(45), ones(45), ones(10), hap)


# ---------------------------------------------------------------- P7 bounds
def test_p7_probability_bounds():
    rng = random.Random(5)
    for _ in range(400):
        m, n = rng.randint(1, 12), rng.randint(1, 12)
        read = "".join(rng.choice("ACGTN") for _ in range(m))
        hap = "".join(rng.choice("ACGTN") for _ in range(n))
        lp = core.phred_log10(read, [rng.randint(6, 60) for _ in range(m)],
                              [rng.randint(6, 60) for _ in range(m)], [rng.randint(6, 60) for _ in range(m)],
                              [rng.randint(6, 40) for _ in range(m)], hap)
        assert -math.inf < lp <= 0.0


# ---------------------------------------------------------------- P8 scaling
@pytest.mark.parametrize("c", [2.0 ** -40, 1e-7, 3.0])
def test_p8_constant_prior_scaling(c):
    """Every path visits exactly one M or I state per row (D moves stay in the
    row). An M visit carries P(i,j); an I visit carries delta_i or eps_i. So
    multiplying every P(i,j), delta_i and eps_i by c multiplies P by c^m:
    log10 P shifts by m*log10(c). With c = 1e-7 and m = 300 the unscaled value
    is ~1e-2100 (renormalisation pinned again)."""
    rng = np.random.default_rng(11)
    m, n = 300, 350
    prior = rng.uniform(1e-3, 1.0, (m, n))
    tr = [rng.uniform(0.01, 1.0, m) for _ in range(7)]
    _, _, a = core.prob_parts(*tr, prior)
    a_, b_, g_, d_, e_, z_, u_ = tr
    _, _, b = core.prob_parts(a_, b_, g_, d_ * c, e_ * c, z_, u_, prior * c)
    assert abs((b - a) - m * math.log10(c)) < 1e-11 * max(1.0, abs(b))


# ---------------------------------------------------------------- batch entry point
def test_batch_matches_single_calls_and_checks_indices():
    b = synth.random_pairs_batch(3, 25)
    out = core.batch_log10(b)
    for p in range(b.n_pairs):
        r, h = b.pairs[p]
        s, e = b.read_offsets[r], b.read_offsets[r + 1]
        exp = core.phred_log10(b.read_bases[s:e], b.base_quals[s:e], b.ins_quals[s:e], b.del_quals[s:e],
                               b.gcp_quals[s:e], b.hap(h))
        assert out[p] == exp or (math.isinf(out[p]) and math.isinf(exp))
    bad = synth.random_pairs_batch(3, 2)
    bad.pairs = np.array([[0, 5]], dtype=np.int32)
    with pytest.raises(IndexError):
        core.batch_log10(bad)
