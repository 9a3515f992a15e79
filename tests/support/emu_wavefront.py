"""CPU emulator of k_wavefront_f32's schedule (float32, numpy over 32 lanes x 2 halves)."""
import numpy as np

K, G, PADC, MINP, FRONT = 4, 8, 5, 72, 16
E = np.float32


def ncols_of(n, bucket=4):
    c = ((n + 2 + bucket - 1) // bucket) * bucket
    lo = ((40 + bucket - 1) // bucket) * bucket
    return max(c, lo)


def qerr(q):
    return E(10.0 ** (-float(q) / 10.0))


def read_table(rb, q, qi, qd, qg):
    m = len(rb)
    nb = (m + 3 + K - 1) // K
    f = nb * K - (m + 3)
    rows = []
    for row in range(nb * K):
        al = be = de = ep = ze = mu = E(0)
        pr = [E(0)] * 5
        if row < f:
            pass
        elif row == f:
            mu = E(1)
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
            de = ep = mu = E(1)
        else:
            be = ze = mu = E(1)
            pr = [E(1)] * 5
        rows.append((al, be, de, ep, ze, mu, pr))
    return rows, nb, f


def hap_codes(hap, bucket=4):
    n = len(hap)
    nc = ncols_of(n, bucket)
    p = max(nc + G, MINP)
    slot = FRONT + p + 8
    codes = np.full(slot, PADC, dtype=np.int64)
    for c in range(n):
        codes[FRONT + c] = "ACGTN".index(chr(hap[c]))
    codes[FRONT + n] = 4
    return codes


TRACE = []


def run_stream(blocks, ncols):
    """blocks: list of dicts with rows (4 rows), codes (array, col 0 at FRONT), rrow, last, pair.
    Returns {pair: scaled sum}."""
    P = max(ncols + G, MINP)
    nblk = len(blocks)
    npass = (nblk + 63) // 64
    d0 = E(2.0 ** 120) / E(ncols)
    # state [lane, half, row]
    co = np.zeros((6, 32, 2, 4), E)  # al be de ep ze mu
    pri = np.zeros((32, 2, 6, 4), E)  # prior table per lane/half/code
    M = np.zeros((32, 2, 4), E); I = np.zeros_like(M); D = np.zeros_like(M)
    upM = np.zeros((32, 2), E); upI = np.zeros_like(upM); upD = np.zeros_like(upM)
    dgM = np.zeros_like(upM); dgI = np.zeros_like(upM); dgD = np.zeros_like(upM)
    codes = [[None, None] for _ in range(32)]  # code arrays
    idx = np.zeros((32, 2), np.int64)
    code_nx = np.full((32, 2), PADC, np.int64)
    out = [[-1, -1] for _ in range(32)]
    ring = np.zeros((P + 8, 3), E)
    res = {}
    c0 = -(1 << 20); c31B = -(1 << 20)
    padcodes = np.full(100000, PADC, np.int64)
    for l in range(32):
        for h in range(2):
            codes[l][h] = padcodes; idx[l, h] = 0

    def step():
        nonlocal c0, c31B
        rv = ring[min(c0 + 2, len(ring) - 1)].copy() if True else None
        code = code_nx.copy()
        for l in range(32):
            for h in range(2):
                code_nx[l, h] = codes[l][h][idx[l, h]]
                idx[l, h] += 1
        pr = np.zeros((32, 2, 4), E)
        for l in range(32):
            for h in range(2):
                pr[l, h] = pri[l, h, code[l, h]]
        al, be, de, ep, ze, mu = co
        for u in (3, 2, 1, 0):
            md = dgM if u == 0 else M[:, :, u - 1]
            id_ = dgI if u == 0 else I[:, :, u - 1]
            dd = dgD if u == 0 else D[:, :, u - 1]
            nD = (ze[:, :, u] * M[:, :, u] + mu[:, :, u] * D[:, :, u]).astype(E)
            x = (al[:, :, u] * md + be[:, :, u] * (id_ + dd).astype(E)).astype(E)
            M[:, :, u] = (pr[:, :, u] * x).astype(E)
            D[:, :, u] = nD
        m_up, i_up = upM.copy(), upI.copy()
        for u in range(4):
            ni = (ep[:, :, u] * i_up + de[:, :, u] * m_up).astype(E)
            m_up = M[:, :, u].copy(); i_up = ni; I[:, :, u] = ni
        sA = np.stack([M[:, 0, 3], I[:, 0, 3], D[:, 0, 3]], 1).copy()
        sB = np.stack([M[:, 1, 3], I[:, 1, 3], D[:, 1, 3]], 1).copy()
        sA[31] = rv
        sB[31] = np.array([M[31, 0, 3], I[31, 0, 3], D[31, 0, 3]])
        if -1 <= c31B < ncols:
            ring[c31B + 1] = [M[31, 1, 3], I[31, 1, 3], D[31, 1, 3]]
        dgM[:] = upM; dgI[:] = upI; dgD[:] = upD
        src = (np.arange(32) + 31) % 32
        upM[:, 0] = sA[src, 0]; upI[:, 0] = sA[src, 1]; upD[:, 0] = sA[src, 2]
        upM[:, 1] = sB[src, 0]; upI[:, 1] = sB[src, 1]; upD[:, 1] = sB[src, 2]
        TRACE.append(np.stack([M[:, 0, 3], I[:, 0, 3], D[:, 0, 3], M[:, 1, 3], I[:, 1, 3], D[:, 1, 3]], 1).copy())
        c0 += 1; c31B += 1

    for q in range(npass + 1):
        for e in range(8):
            h, g = e // 4, e % 4
            if e == 0:
                c0 = -1
            if e == 7:
                c31B = -1 - (G - 1)
            for l in range(8 * g, 8 * g + 8):
                gi = l % G
                b = q * 64 + h * 32 + l
                if out[l][h] >= 0:
                    res[out[l][h]] = float(D[l, h, 3])
                out[l][h] = -1
                if q < npass and b < nblk:
                    blk = blocks[b]
                    for u in range(4):
                        r = blk["rows"][u]
                        for fi in range(6):
                            co[fi, l, h, u] = r[fi]
                        for cc in range(5):
                            pri[l, h, cc, u] = r[6][cc]
                        M[l, h, u] = 0; I[l, h, u] = 0
                        D[l, h, u] = d0 if blk["rrow"] == u else E(0)
                    codes[l][h] = blk["codes"]; idx[l, h] = FRONT - gi
                    if blk["last"]:
                        out[l][h] = blk["pair"]
                else:
                    co[:, l, h, :] = 0; M[l, h] = 0; I[l, h] = 0; D[l, h] = 0
                    codes[l][h] = padcodes; idx[l, h] = 0
                code_nx[l, h] = PADC
                if h == 0 and l == 0:
                    upM[0, 0], upI[0, 0], upD[0, 0] = ring[0]
            nsteps = G if e < 7 else (P - 7 * G if q < npass else 0)
            for _ in range(nsteps):
                step()
    return res


def run_batch(batch, order=None, bucket=4):
    """All pairs in one stream per ncols bin (in the given order)."""
    pairs = batch.pairs
    order = list(range(len(pairs))) if order is None else order
    bins = {}
    for p in order:
        r, h = pairs[p]
        n = int(batch.hap_offsets[h + 1] - batch.hap_offsets[h])
        bins.setdefault(ncols_of(n, bucket), []).append(p)
    out = {}
    for nc, plist in bins.items():
        blocks = []
        for p in plist:
            r, h = pairs[p]
            s, e = batch.read_offsets[r], batch.read_offsets[r + 1]
            rows, nb, f = read_table(batch.read_bases[s:e], batch.base_quals[s:e], batch.ins_quals[s:e],
                                     batch.del_quals[s:e], batch.gcp_quals[s:e])
            codes = hap_codes(batch.hap(h), bucket)
            for j in range(nb):
                blocks.append(dict(rows=rows[4 * j:4 * j + 4], codes=codes, pair=p, last=(j == nb - 1),
                                   rrow=(f % 4) if f // 4 == j else 15))
        out.update(run_stream(blocks, nc))
    res = np.zeros(len(pairs))
    for p in range(len(pairs)):
        r, h = pairs[p]
        n = int(batch.hap_offsets[h + 1] - batch.hap_offsets[h])
        s = out[p]
        res[p] = (np.log10(s) if s > 0 else -np.inf) - 120 * np.log10(2) + np.log10(ncols_of(n, bucket) / n)
    return res
