"""CPU model of the schedule of k_wavefront_f32 (float32 numpy, vectorised over the 64
virtual lanes of a warp). It models what the kernel computes, independent of how the
virtual lanes are packed into physical lanes / register halves:

* a warp streams through the blocks of one length bin; pass q gives block 64q+v to
  virtual lane v (K rows each, the Z/R/read/S pad-row layout of DESIGN.md §4.2);
* virtual lane v computes column x of its block at step T_q + 1 + SH + v + x; a pass is
  P = max(ncols + G + SH, 72) steps; virtual lanes switch blocks in groups of G = 8 at the
  events T_q + 8e (e = 0..7), taking column -1 - (v mod 8) - SH next (SH = 4 PAD columns,
  the staged switch of DESIGN.md §4.4): the switch writes the finished pair's result and
  points the lane at its new block's codes and priors, and 4 steps later the group COMMITS
  the new block's coefficients and initial state (M = I = 0, D = the virtual row 0 on the
  R row) -- until then the lane computes PAD columns with its old coefficients and state;
* columns outside a block read the PAD code (prior 0) -- no per-lane branch;
* virtual lane v takes the row above from v-1's last row one step later; v = 0 from
  a ring indexed by column + 1 (slot 0 = boundary column) written by v = 63 of the
  previous pass;
* the result of a pair is D of its S row, read at the next switch event.

The GPU kernel's per-step state was compared against this model with a trace build
(DESIGN.md §4.4); tests/test_schedule_emulation.py checks the model against the oracle.
"""
import numpy as np

G, PADC, MINP = 8, 5, 72
RESCALE_COLS = 768  # long rows: passes 64 steps longer, ring rescale on
RS_TARGET, RS_TRIG, RS_CAP = 112, 104, 126  # ring rescale: below 2^RS_TRIG -> ~2^RS_TARGET, saturating at 2^RS_CAP


SH = 4  # PAD columns a lane runs before its block (staged switch)


def pass_len(ncols):
    if ncols >= RESCALE_COLS:
        return ncols + G + 64 + SH
    return max(ncols + G + SH, MINP)
E = np.float32


def ncols_of(n, bucket=4):
    c = ((n + 2 + bucket - 1) // bucket) * bucket
    lo = ((40 + bucket - 1) // bucket) * bucket
    return max(c, lo)


def qerr(q):
    return E(10.0 ** (-float(q) / 10.0))


def read_rows(rb, q, qi, qd, qg, K):
    """(nb*K rows of (u, w, ep', mu, prior[5])), nb, f = number of Z rows (>= 1).

    The kernel's 5-op form of Eq. 6: per row i the stored values are
    M^ = a_i M, I^ = b_i I, D^ = d_i D with a_i = k_i zeta_i, d_i = k_i, b_i = a_{i-1}/delta_i,
    k_i = min(1, delta_{i+1}/zeta_i) (k_m = 1), a_R = delta_1, b_R = d_R = 1, so that
      D^ = M^(left) + mu D^(left)
      I^ = M^(up) + ep' I^(up)                  ep' = eps_i b_i / b_{i-1}
      M^ = T[code] (M^(diag) + u I^(diag) + w D^(diag))
           T = a_i alpha_i P / a_{i-1},  u = beta_i a_{i-1} / (alpha_i b_{i-1}),
           w = beta_i a_{i-1} / (alpha_i d_{i-1})
    and the S row: T = 1/a_m, u = a_m/b_m, w = 0, ep' = 0, mu = 1 -> M^_S(j) = (M+I)(m,j-1),
    D^_S = running sum."""
    m = len(rb)
    nb = (m + 3 + K - 1) // K
    f = nb * K - (m + 2)
    e = lambda qq: 10.0 ** (-float(qq) / 10.0)
    de = [None] + [e(qi[x]) for x in range(m)]
    ze = [None] + [e(qd[x]) for x in range(m)]
    kk = [1.0] + [min(1.0, de[i + 1] / ze[i]) if i < m else 1.0 for i in range(1, m + 1)]
    a = [de[1]] + [kk[i] * ze[i] for i in range(1, m + 1)]
    b = [1.0, 1.0] + [a[i - 1] / de[i] for i in range(2, m + 1)]
    d = [1.0] + [kk[i] for i in range(1, m + 1)]
    rows = []
    for row in range(nb * K):
        uu = ww = ep = mu = 0.0
        pr = [0.0] * 5
        if row < f:
            pass  # Z
        elif row == f:
            mu = 1.0  # R
        elif row <= f + m:
            i = row - f
            x = i - 1
            ei, ed, eg, eb = de[i], ze[i], e(qg[x]), e(q[x])
            al = 1.0 - min(ei + ed, 1.0)
            be = 1.0 - eg
            uu = be * a[i - 1] / (al * b[i - 1])
            ww = be * a[i - 1] / (al * d[i - 1])
            ep = eg * b[i] / b[i - 1]
            mu = eg
            pm, px = 1.0 - eb, eb / 3.0
            base = chr(rb[x])
            t = a[i] * al / a[i - 1]
            pr = [t * (pm if (base == c or base == 'N') else px) for c in "ACGT"] + [t * pm]
        else:  # S
            uu = a[m] / b[m]
            mu = 1.0
            pr = [1.0 / a[m]] * 5
        rows.append((E(uu), E(ww), E(ep), E(mu), [E(v) for v in pr]))
    return rows, nb, f


def hap_code_row(hap, ncols, P):
    """codes[c] for c in [-P, P+8): 0..4 inside, 'N' (4) at column N, PAD elsewhere."""
    n = len(hap)
    codes = np.full(3 * P + 64, PADC, dtype=np.int64)
    off = P
    for c in range(n):
        codes[off + c] = "ACGTN".index(chr(hap[c]))
    codes[off + n] = 4
    return codes, off


TRACE = []


def run_stream(blocks, ncols, K, rescale=True):
    P = pass_len(ncols)
    nblk = len(blocks)
    npass = (nblk + 63) // 64
    d0 = E(2.0 ** 120) / E(ncols)
    V = 64
    co = np.zeros((4, V, K), E)
    pri = np.zeros((V, 6, K), E)
    M = np.zeros((V, K), E); I = np.zeros_like(M); D = np.zeros_like(M)
    up = np.zeros((V, 3), E); dg = np.zeros((V, 3), E)
    col = np.full(V, -(1 << 20), np.int64)  # column computed next step
    codes = [None] * V
    offs = np.zeros(V, np.int64)
    pad = np.full(10 * P, PADC, np.int64)
    for v in range(V):
        codes[v] = pad
    out = [-1] * V
    ring = np.zeros((P + 8, 3), E)
    res = {}
    exps = {}

    def code_of(v):
        c = col[v]
        if c < -P or c >= P + 8 or codes[v] is pad:
            return PADC
        return int(codes[v][offs[v] + c])

    def step():
        pr = np.stack([pri[v, code_of(v)] for v in range(V)])
        uu, ww, ep, mu = co
        for u in range(K - 1, -1, -1):
            md = dg[:, 0] if u == 0 else M[:, u - 1]
            id_ = dg[:, 1] if u == 0 else I[:, u - 1]
            dd = dg[:, 2] if u == 0 else D[:, u - 1]
            nD = (mu[:, u] * D[:, u] + M[:, u]).astype(E)
            y = (uu[:, u] * id_ + md).astype(E)
            x = (ww[:, u] * dd + y).astype(E)
            M[:, u] = (pr[:, u] * x).astype(E)
            D[:, u] = nD
        m_up, i_up = up[:, 0].copy(), up[:, 1].copy()
        for u in range(K):
            ni = (ep[:, u] * i_up + m_up).astype(E)
            m_up = M[:, u].copy(); i_up = ni; I[:, u] = ni
        # exchange: v <- v-1 (this step's last row); v = 0 <- ring slot of its next column
        c63 = col[63]
        if -1 <= c63 < ncols:
            ring[c63 + 1] = [M[63, K - 1], I[63, K - 1], D[63, K - 1]]
        dg[:] = up
        new_up = np.zeros_like(up)
        new_up[1:, 0] = M[:-1, K - 1]; new_up[1:, 1] = I[:-1, K - 1]; new_up[1:, 2] = D[:-1, K - 1]
        nc0 = col[0] + 1
        new_up[0] = ring[min(max(nc0 + 1, 0), len(ring) - 1)] if nc0 >= -1 else 0
        up[:] = new_up
        TRACE.append(np.stack([M[:, K - 1], I[:, K - 1], D[:, K - 1]], 1).copy())
        col[:] += 1

    rescale = ncols >= RESCALE_COLS

    def ring_scale(sh):
        # saturating at 2^RS_CAP (a saturated pair goes to the FP64 rescue)
        x = ring[0:ncols + 1].astype(np.float64) * 2.0 ** sh
        ring[0:ncols + 1] = np.minimum(x, 2.0 ** RS_CAP).astype(E)
        return bool(np.any(x > 2.0 ** RS_CAP))

    for q in range(npass + 1):
        for e in range(8):
            if rescale and e == 0:
                # ring rescale: lane 0's block continues the pair of lane 63's
                b = q * 64
                cont = q < npass and b < nblk and not blocks[b]["first"]
                sh = 0
                rm = float(np.max(ring[0:ncols + 1])) if cont else 0.0  # the whole ring row
                if cont and 0 < rm <= 3.0e38:
                    Ex = int(np.floor(np.log2(rm)))
                    if -90 <= Ex < RS_TRIG:
                        sh = min(RS_TARGET - Ex, 126)
                if sh:
                    pr_ = blocks[b]["pair"]
                    sat = ring_scale(sh)
                    exps[pr_] = exps.get(pr_, 0) + (-(1 << 24) if sat else sh)
            staged = {}
            for v in range(8 * e, 8 * e + 8):  # switch
                gi = v % G
                b = q * 64 + v
                if out[v] >= 0:
                    res[out[v]] = float(D[v, K - 1])
                out[v] = -1
                if q < npass and b < nblk:
                    blk = blocks[b]
                    for u in range(K):
                        for cc in range(5):
                            pri[v, cc, u] = blk["rows"][u][4][cc]
                    codes[v], offs[v] = blk["codes"]
                    if blk["last"]:
                        out[v] = blk["pair"]
                    staged[v] = blk
                else:
                    codes[v] = pad; offs[v] = 0
                    staged[v] = None
                col[v] = -1 - gi - SH
            for k in range(4):
                step()
            for v, blk in staged.items():  # commit, 4 steps after the switch
                if blk is None:
                    co[:, v, :] = 0; M[v] = 0; I[v] = 0; D[v] = 0
                    continue
                for u in range(K):
                    for fi in range(4):
                        co[fi, v, u] = blk["rows"][u][fi]
                    M[v, u] = 0; I[v, u] = 0
                    D[v, u] = d0 if blk["rrow"] == u else E(0)
            nsteps = 4 if e < 7 else (P - 7 * G - 4 if q < npass else 0)
            for k in range(nsteps):
                step()
    return res, exps


def run_batch(batch, order=None, bucket=4, K=8):
    """All pairs of a batch through the schedule, one stream per ncols bin."""
    pairs = batch.pairs
    order = list(range(len(pairs))) if order is None else order
    bins = {}
    for p in order:
        r, h = pairs[p]
        n = int(batch.hap_offsets[h + 1] - batch.hap_offsets[h])
        bins.setdefault(ncols_of(n, bucket), []).append(p)
    out, exps = {}, {}
    for nc, plist in bins.items():
        P = pass_len(nc)
        blocks = []
        for p in plist:
            r, h = pairs[p]
            s, e = batch.read_offsets[r], batch.read_offsets[r + 1]
            rows, nb, f = read_rows(batch.read_bases[s:e], batch.base_quals[s:e], batch.ins_quals[s:e],
                                    batch.del_quals[s:e], batch.gcp_quals[s:e], K)
            codes = hap_code_row(batch.hap(h), nc, P)
            for j in range(nb):
                blocks.append(dict(rows=rows[K * j:K * j + K], codes=codes, pair=p, last=(j == nb - 1), first=(j == 0),
                                   rrow=(f % K) if f // K == j else 15))
        r_, x_ = run_stream(blocks, nc, K)
        out.update(r_)
        exps.update(x_)
    res = np.zeros(len(pairs))
    for p in range(len(pairs)):
        r, h = pairs[p]
        n = int(batch.hap_offsets[h + 1] - batch.hap_offsets[h])
        s = out[p]
        x = exps.get(p, 0)
        if x < -(1 << 23):  # saturated by the ring rescale: the FP64 rescue's job
            res[p] = np.nan
            continue
        res[p] = (np.log10(s) if s > 0 else -np.inf) - (120 + x) * np.log10(2) + \
            np.log10(ncols_of(n, bucket) / n)
    return res
