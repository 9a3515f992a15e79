"""Brute-force PairHMM: explicit enumeration of every HMM path.

TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

This is the independent pin for the DP oracle on tiny inputs (m, N <= 5). It
never evaluates the recurrence of Eq. 6 (PAPER.md L18@541); it walks the
state graph of the PairHMM model (Fig. 5, L16@2878) one path at a time and
sums the product of the edge weights along each path, so a dropped term, a
wrong index or a transposed operand in the DP shows up as a mismatch.

Path semantics (reading R6, GATK initial row):
  * a path starts in D(0, c) for c = 0..N-1 with weight 1/N (the initial row
    D(0, .) = 1/N; D(0, N) has no successor);
  * moves, weights indexed by the DESTINATION row (reading R3):
      X(i-1, j-1) -> M(i, j)   alpha_i (X=M) | beta_i (X=I) | gamma_i (X=D), times P(i, j)
      M(i-1, j)   -> I(i, j)   delta_i          I(i-1, j) -> I(i, j)   eps_i
      M(i, j-1)   -> D(i, j)   zeta_i           D(i, j-1) -> D(i, j)   mu_i    (rows i >= 1)
    where a start state D(0, c) only has the move to M(1, c+1) (there is no
    M(0, .) or I(0, .) mass, and no D -> D move inside row 0: every D(0, c) is
    its own start);
  * a path ends in M(m, j) or I(m, j), j = 1..N (termination reading R1, the
    "match and insertion" last-row sum of L20@2262).
P is the sum of the weights of all such paths.

Arithmetic is whatever the inputs are: Fractions give the exact rational
answer; mpmath mpf gives a high-precision one for irrational (Phred) inputs.
"""
from __future__ import annotations

from fractions import Fraction
from typing import Sequence


def enumerate_paths(m: int, n: int, alpha, beta, gamma, delta, eps, zeta, mu, prior,
                    one=Fraction(1)):
    """Return (sum over paths ending in M(m,.), sum over paths ending in I(m,.)).

    Transition sequences are indexed by row i = 1..m at position i-1; prior is
    an m x n nested sequence, prior[i-1][j-1] = P(i, j). ``one`` sets the
    number type (Fraction(1) or mpmath.mpf(1)).
    """
    zero = one * 0
    tot_m = [zero]
    tot_i = [zero]

    def visit(state: str, i: int, j: int, w):
        # record termination
        if i == m:
            if state == "M":
                tot_m[0] += w
            elif state == "I":
                tot_i[0] += w
            # from row m only D(m, .) states are reachable, never M/I again
            if state == "D" or state == "M":
                pass
            return
        # moves to the next row
        if j + 1 <= n:  # diagonal -> M(i+1, j+1)
            t = {"M": alpha, "I": beta, "D": gamma}[state][i]  # destination row i+1 -> index i
            visit("M", i + 1, j + 1, w * t * prior[i][j])
        if state in ("M", "I") and j >= 1:  # vertical -> I(i+1, j)
            t = delta[i] if state == "M" else eps[i]
            visit("I", i + 1, j, w * t)
        # horizontal -> D(i, j+1): only inside rows >= 1
        if i >= 1 and state in ("M", "D") and j + 1 <= n:
            t = zeta[i - 1] if state == "M" else mu[i - 1]
            visit("D", i, j + 1, w * t)

    for c in range(0, n):
        visit("D", 0, c, one / n)
    return tot_m[0], tot_i[0]


def brute_parts(alpha, beta, gamma, delta, eps, zeta, mu, prior, one=Fraction(1)):
    m = len(prior)
    n = len(prior[0])
    return enumerate_paths(m, n, alpha, beta, gamma, delta, eps, zeta, mu, prior, one)


def phred_inputs(read: str, q: Sequence[int], qi: Sequence[int], qd: Sequence[int],
                 qg: Sequence[int], hap: str, one):
    """GATK Phred mapping (readings R2, R4, R5), written out again in
    the number type of ``one`` for the brute force."""
    ten = one * 10

    def err(Q):
        return ten ** (-(one * Q) / 10)

    m = len(read)
    alpha, beta, gamma, delta, eps, zeta, mu, prior = [], [], [], [], [], [], [], []
    for i in range(m):
        ei, ed, eg, eb = err(qi[i]), err(qd[i]), err(qg[i]), err(q[i])
        s = ei + ed
        alpha.append(one - (s if s < one else one))
        beta.append(one - eg)
        gamma.append(one - eg)
        delta.append(ei)
        eps.append(eg)
        zeta.append(ed)
        mu.append(eg)
        row = []
        for hj in hap:
            match = read[i] == hj or read[i] == "N" or hj == "N"
            row.append(one - eb if match else eb / 3)
        prior.append(row)
    return alpha, beta, gamma, delta, eps, zeta, mu, prior


def brute_phred(read, q, qi, qd, qg, hap, dps: int = 40):
    """(M-part, I-part) of P(read | hap) by path enumeration in mpmath."""
    import mpmath

    with mpmath.workdps(dps):
        one = mpmath.mpf(1)
        args = phred_inputs(read, q, qi, qd, qg, hap, one)
        sm, si = brute_parts(*args, one=one)
        return sm, si
