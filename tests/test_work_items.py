"""Work items of the wavefront launches (the length-binned scheduler):
a line-by-line Python model of ``k_scan_bins`` (phmm_device.cuh) and of the item -> (bin,
first block, end block) mapping in ``k_wavefront`` (wavefront.cuh). The items of a
launch must tile every bin's blocks exactly once, the short (guided) items must be the
last ones a launch hands out, and with ``lpt`` the bins must come longest-row first."""
import numpy as np
import pytest


def scan_bins(bin_blocks, cut, chunk, chunk_s, tail_div, lpt):
    nb = len(bin_blocks)
    bin_start = np.zeros(nb + 1, dtype=np.int64)
    bin_start[1:] = np.cumsum(bin_blocks)
    c = min(max(cut, 0), nb)
    B0, Ball = int(bin_start[c]), int(bin_start[nb])
    L0, L1 = B0, Ball - B0
    thr0 = L0 - L0 // tail_div if tail_div > 0 else L0
    thr1 = L1 - L1 // tail_div if tail_div > 0 else L1
    vi = np.zeros(nb, dtype=np.int64)
    nbig = np.zeros(nb, dtype=np.int64)
    for i in range(nb):
        vb = int(bin_blocks[i])
        l0 = i < c
        pos = ((B0 if l0 else Ball) - int(bin_start[i + 1])) if lpt else (int(bin_start[i]) - (0 if l0 else B0))
        thr = thr0 if l0 else thr1
        big = 0 if thr <= pos else min(thr - pos, vb)
        nbg = -(-vb // chunk) if big == vb else big // chunk
        used = min(nbg * chunk, vb)
        vi[i] = nbg + -(-(vb - used) // chunk_s)
        nbig[i] = nbg
    item_start = np.zeros(nb + 1, dtype=np.int64)
    item_start[1:] = np.cumsum(vi)
    I0, Iall = int(item_start[c]), int(item_start[nb])
    launch_items = [0, I0, I0, Iall]
    if lpt:
        new = item_start.copy()
        for i in range(nb):
            nxt = int(item_start[i + 1])
            new[i] = I0 - nxt if i < c else I0 + (Iall - nxt)
        item_start = new
    return bin_start, item_start, nbig, launch_items


def item_range(it, bin_lo, bin_hi, bin_start, item_start, nbig, chunk, chunk_s, lpt):
    lo, hi = bin_lo, bin_hi - 1
    if lpt:
        while lo < hi:
            mid = (lo + hi) >> 1
            if item_start[mid] <= it:
                hi = mid
            else:
                lo = mid + 1
    else:
        while lo < hi:
            mid = (lo + hi + 1) >> 1
            if item_start[mid] <= it:
                lo = mid
            else:
                hi = mid - 1
    b = lo
    b0, b1 = int(bin_start[b]), int(bin_start[b + 1])
    k = it - int(item_start[b])
    if k < nbig[b]:
        s = b0 + k * chunk
        e = s + chunk
    else:
        s = b0 + int(nbig[b]) * chunk + (k - int(nbig[b])) * chunk_s
        e = s + chunk_s
    return b, s, min(e, b1), bool(k >= nbig[b])


@pytest.mark.parametrize("lpt", [0, 1])
@pytest.mark.parametrize("seed", range(6))
def test_items_tile_every_bin_once(lpt, seed):
    rng = np.random.default_rng(seed)
    nb = int(rng.integers(1, 60))
    blocks = rng.integers(0, 5000, size=nb) * (rng.random(nb) < 0.7)
    cut = int(rng.integers(0, nb + 1))
    chunk = int(rng.integers(64, 2000))
    chunk_s = max(64, chunk // 8)
    tail_div = int(rng.choice([0, 4, 8]))
    bin_start, item_start, nbig, li = scan_bins(blocks, cut, chunk, chunk_s, tail_div, lpt)
    for launch, (blo, bhi) in enumerate([(0, cut), (cut, nb)]):
        it0, it1 = li[2 * launch], li[2 * launch + 1]
        if bhi <= blo:
            assert it0 == it1
            continue
        seen = np.zeros(int(bin_start[bhi]), dtype=np.int32)
        order, sizes, short = [], [], []
        for it in range(it0, it1):
            b, s, e, sh = item_range(it, blo, bhi, bin_start, item_start, nbig, chunk, chunk_s, lpt)
            assert blo <= b < bhi and bin_start[b] <= s < e <= bin_start[b + 1]
            assert e - s <= (chunk_s if sh else chunk)
            seen[s:e] += 1
            order.append(b)
            sizes.append(e - s)
            short.append(sh)
        assert np.all(seen[int(bin_start[blo]):int(bin_start[bhi])] == 1)
        # bins in launch order: ascending, or descending with lpt
        assert order == sorted(order, reverse=bool(lpt))
        # guided: the short items are the last ones handed out and hold the launch's tail
        L = int(bin_start[bhi]) - int(bin_start[blo])
        if tail_div == 0:
            assert not any(short)
        elif any(short):
            j = short.index(True)
            assert all(short[j:])
            n_short_blocks = sum(sizes[j:])
            assert L // tail_div <= n_short_blocks <= L // tail_div + chunk


def test_no_short_items_without_tail():
    blocks = np.array([1000, 0, 300, 4096])
    bin_start, item_start, nbig, li = scan_bins(blocks, 4, 512, 64, 0, 0)
    assert list(nbig) == [2, 0, 1, 8]
    assert li[1] == 11
