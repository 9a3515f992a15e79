"""CPU model of the schedule of k_wavefront_f32 (float32 numpy, vectorised over the 64
virtual lanes of a warp). It models what the kernel computes, independent of how the
virtual lanes are packed into physical lanes / register halves:

* a warp streams through the blocks of one length bin; pass q gives block 64q+v to
  virtual lane v (K rows each, the Z/R/read/S1/S2 pad-row layout of DESIGN.md §4.2);
* virtual lane v computes column x of its block at step T_q + 1 + v + x; a pass is
  P = max(ncols + G, 72) steps; virtual lanes switch blocks in groups of G = 8 at the
  events T_q + 8e (e = 0..7), taking column -1 - (v mod 8) next;
* columns outside a block read the PAD code (prior 0) -- no per-lane branch;
* virtual lane v takes the row above from v-1's last row one step later; v = 0 from
  a ring indexed by column + 1 (slot 0 = boundary column) written by v = 63 of the
  previous pass;
* the result of a pair is D of its S2 row, read at the next switch event.

The GPU kernel's per-step state was compared against this model with a trace build
(DESIGN.md §4.4); tests/test_schedule_emulation.py checks the model against the oracle.
"""
import numpy as np

G, PADC, MINP = 8, 5, 72
E = np.float32


def ncols_of(n, bucket=4):
    c = ((n + 2 + bucket - 1) // bucket) * bucket
    lo = ((40 + bucket - 1) // bucket) * bucket
    return max(c, lo)


def qerr(q):
    return E(10.0 ** (-float(q) / 10.0))


def read_rows(rb, q, qi, qd, qg, K):
    """(nb*K rows of (al, be, de, ep, ze, mu, prior[5])), nb, f = number of Z rows."""
    m = len(rb)
    nb = (m + 3 + K - 1) // K
    f = nb * K - (m + 3)
    rows = []
    for row in range(nb * K):
        al = be = de = ep = ze = mu = E(0)
        pr = [E(0)] * 5
        if row < f:
            pass  # Z
        elif row == f:
            mu = E(1)  # R
        elif row <= f + m:
            x = row - f - 1
            ei, ed, eg, eb = qerr(qi[x]), qerr(qd[x]), qerr(qg[x]), qerr(q[x])
            s = E(ei + ed)
            al = E(E(1) - min(s, E(1)))
            be = E(E(1) - eg); de = ei; ep = eg; ze = ed; mu = eg
            pm, px = E(E(1) - eb), E(eb / E(3))
            base = chr(rb[x])
            pr = [pm if (base == c or base == 'N') else px for c in "ACGT"] + [pm]
        elif row == f + m + 1:
            de = ep = mu = E(1)  # S1
        else:
            be = ze = mu = E(1)  # S2
            pr = [E(1)] * 5
        rows.append((al, be, de, ep, ze, mu, pr))
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


def run_stream(blocks, ncols, K):
    P = max(ncols + G, MINP)
    nblk = len(blocks)
    npass = (nblk + 63) // 64
    d0 = E(2.0 ** 120) / E(ncols)
    V = 64
    co = np.zeros((6, V, K), E)
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

    def code_of(v):
        c = col[v]
        if c < -P or c >= P + 8 or codes[v] is pad:
            return PADC
        return int(codes[v][offs[v] + c])

    def step():
        pr = np.stack([pri[v, code_of(v)] for v in range(V)])
        al, be, de, ep, ze, mu = co
        lastM, lastI, lastD = M[:, K - 1].copy(), I[:, K - 1].copy(), D[:, K - 1].copy()
        for u in range(K - 1, -1, -1):
            md = dg[:, 0] if u == 0 else M[:, u - 1]
            id_ = dg[:, 1] if u == 0 else I[:, u - 1]
            dd = dg[:, 2] if u == 0 else D[:, u - 1]
            nD = (ze[:, u] * M[:, u] + mu[:, u] * D[:, u]).astype(E)
            x = (al[:, u] * md + be[:, u] * (id_ + dd).astype(E)).astype(E)
            M[:, u] = (pr[:, u] * x).astype(E)
            D[:, u] = nD
        m_up, i_up = up[:, 0].copy(), up[:, 1].copy()
        for u in range(K):
            ni = (ep[:, u] * i_up + de[:, u] * m_up).astype(E)
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

    for q in range(npass + 1):
        for e in range(8):
            for v in range(8 * e, 8 * e + 8):
                gi = v % G
                b = q * 64 + v
                if out[v] >= 0:
                    res[out[v]] = float(D[v, K - 1])
                out[v] = -1
                if q < npass and b < nblk:
                    blk = blocks[b]
                    for u in range(K):
                        r = blk["rows"][u]
                        for fi in range(6):
                            co[fi, v, u] = r[fi]
                        for cc in range(5):
                            pri[v, cc, u] = r[6][cc]
                        M[v, u] = 0; I[v, u] = 0
                        D[v, u] = d0 if blk["rrow"] == u else E(0)
                    codes[v], offs[v] = blk["codes"]
                    if blk["last"]:
                        out[v] = blk["pair"]
                else:
                    co[:, v, :] = 0; pri[v] = 0; M[v] = 0; I[v] = 0; D[v] = 0
                    codes[v] = pad; offs[v] = 0
                col[v] = -1 - gi
                if v == 0:
                    up[0] = ring[0]
            nsteps = G if e < 7 else (P - 7 * G if q < npass else 0)
            for _ in range(nsteps):
                step()
    return res


def run_batch(batch, order=None, bucket=4, K=8):
    """All pairs of a batch through the schedule, one stream per ncols bin."""
    pairs = batch.pairs
    order = list(range(len(pairs))) if order is None else order
    bins = {}
    for p in order:
        r, h = pairs[p]
        n = int(batch.hap_offsets[h + 1] - batch.hap_offsets[h])
        bins.setdefault(ncols_of(n, bucket), []).append(p)
    out = {}
    for nc, plist in bins.items():
        P = max(nc + G, MINP)
        blocks = []
        for p in plist:
            r, h = pairs[p]
            s, e = batch.read_offsets[r], batch.read_offsets[r + 1]
            rows, nb, f = read_rows(batch.read_bases[s:e], batch.base_quals[s:e], batch.ins_quals[s:e],
                                    batch.del_quals[s:e], batch.gcp_quals[s:e], K)
            codes = hap_code_row(batch.hap(h), nc, P)
            for j in range(nb):
                blocks.append(dict(rows=rows[K * j:K * j + K], codes=codes, pair=p, last=(j == nb - 1),
                                   rrow=(f % K) if f // K == j else 15))
        out.update(run_stream(blocks, nc, K))
    res = np.zeros(len(pairs))
    for p in range(len(pairs)):
        r, h = pairs[p]
        n = int(batch.hap_offsets[h + 1] - batch.hap_offsets[h])
        s = out[p]
        res[p] = (np.log10(s) if s > 0 else -np.inf) - 120 * np.log10(2) + np.log10(ncols_of(n, bucket) / n)
    return res
