// phmm_device.cuh -- validation, binning, finalize and rescue-list kernels of libphmm.
// Included only by phmm_lib.cu. See phmm_common.cuh for what is computed.
#pragma once
#include "phmm_common.cuh"

namespace phmm {

// ============================================================ prep kernels

// Haplotype bases: validation only (the code regions are written by k_hap_codes_wf).
// (Also used on the Smith-Waterman sequences.)
__global__ void k_validate_haps(const uint8_t* __restrict__ hap, int64_t n, uint32_t* err) {
  uint32_t e = 0;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    if (base_code(hap[i]) == 0xffu) e |= ERR_BASE;
  if (e) atomicOr(err, e);
}

// One read base: alphabet, qualities <= 127, and the transitions out of M a distribution,
// e(qi) + e(qd) <= 1 (reading R16; only qualities <= 3 can violate it).
__device__ __forceinline__ uint32_t read_base_err(uint8_t b, uint8_t q, uint8_t qi, uint8_t qd, uint8_t qg) {
  uint32_t e = 0;
  if (base_code(b) == 0xffu) e |= ERR_BASE;
  if ((q | qi | qd | qg) & 0x80u) e |= ERR_QUAL;
  else if ((qi <= 3 || qd <= 3) && exp10(-(double)qi / 10.0) + exp10(-(double)qd / 10.0) > 1.0) e |= ERR_QUAL;
  return e;
}

// Offsets: start at 0, non-decreasing, end at total.
__device__ __forceinline__ bool offset_bad(const int64_t* __restrict__ off, int64_t i, int64_t n, int64_t total) {
  bool bad = (i == 0) ? off[0] != 0 : off[i] < off[i - 1];
  if (i == n) bad |= off[n] != total;
  return bad;
}

// The whole batch in one launch: every haplotype base, every read base with its four
// qualities (4 bases per thread-step through 32-bit words where the five arrays share their
// alignment), and both offset arrays. Errors are OR-ed into *err (one atomic per warp).
__global__ void k_validate(const uint8_t* __restrict__ hap, int64_t n_hb, const uint8_t* __restrict__ rb,
                           const uint8_t* __restrict__ q, const uint8_t* __restrict__ qi,
                           const uint8_t* __restrict__ qd, const uint8_t* __restrict__ qg, int64_t n_rb,
                           const int64_t* __restrict__ roff, int64_t n_reads, const int64_t* __restrict__ hoff,
                           int64_t n_haps, uint32_t* err) {
  uint32_t e = 0;
  const int64_t tid = blockIdx.x * (int64_t)blockDim.x + threadIdx.x, nthr = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i = tid; i < n_hb; i += nthr)
    if (base_code(hap[i]) == 0xffu) e |= ERR_BASE;
  // reads: a scalar head up to the first 4-aligned read byte, then words (when all five
  // arrays are equally aligned), then a scalar tail
  const uintptr_t mis = (uintptr_t)rb & 3;
  const bool same = (((uintptr_t)q & 3) == mis) && (((uintptr_t)qi & 3) == mis) && (((uintptr_t)qd & 3) == mis) &&
                    (((uintptr_t)qg & 3) == mis);
  const int64_t head = same ? min(n_rb, (int64_t)((4 - mis) & 3)) : n_rb;
  for (int64_t i = tid; i < head; i += nthr) e |= read_base_err(rb[i], q[i], qi[i], qd[i], qg[i]);
  const int64_t nw = (n_rb - head) >> 2;
  const uint32_t *rb4 = reinterpret_cast<const uint32_t*>(rb + head), *q4 = reinterpret_cast<const uint32_t*>(q + head),
                 *i4 = reinterpret_cast<const uint32_t*>(qi + head), *d4 = reinterpret_cast<const uint32_t*>(qd + head),
                 *g4 = reinterpret_cast<const uint32_t*>(qg + head);
  for (int64_t w = tid; w < nw; w += nthr) {
    const uint32_t b = rb4[w], a = q4[w], x = i4[w], y = d4[w], z = g4[w];
    // fast path: every byte an uppercase base letter candidate and no quality byte >= 128 or <= 3
    if (((a | x | y | z) & 0x80808080u) || __vcmpleu4(x, 0x03030303u) || __vcmpleu4(y, 0x03030303u)) {
      for (int k = 0; k < 4; ++k)
        e |= read_base_err((uint8_t)(b >> 8 * k), (uint8_t)(a >> 8 * k), (uint8_t)(x >> 8 * k),
                           (uint8_t)(y >> 8 * k), (uint8_t)(z >> 8 * k));
    } else {
      for (int k = 0; k < 4; ++k)
        if (base_code((uint8_t)(b >> 8 * k)) == 0xffu) e |= ERR_BASE;
    }
  }
  for (int64_t i = head + 4 * nw + tid; i < n_rb; i += nthr) e |= read_base_err(rb[i], q[i], qi[i], qd[i], qg[i]);
  for (int64_t i = tid; i <= n_reads; i += nthr)
    if (offset_bad(roff, i, n_reads, n_rb)) e |= ERR_ARG;
  for (int64_t i = tid; i <= n_haps; i += nthr)
    if (offset_bad(hoff, i, n_haps, n_hb)) e |= ERR_ARG;
  e = __reduce_or_sync(0xffffffffu, e);
  if (e && (threadIdx.x & 31) == 0) atomicOr(err, e);
}

// Offsets (the Smith-Waterman batch): start at 0, non-decreasing, end at total.
__global__ void k_validate_offsets(const int64_t* __restrict__ off, int64_t n, int64_t total, uint32_t* err) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i <= n; i += (int64_t)gridDim.x * blockDim.x)
    if (offset_bad(off, i, n, total)) atomicOr(err, ERR_ARG);
}

// Per pair: validate indices/lengths, bin by column count, count blocks per bin.
// pair_list == nullptr -> pairs 0..n-1, else the listed pair ids (rescue pass).
// Counters are aggregated per warp (match_any + reduce) before one atomic per
// distinct bin and per warp: with one length bin every pair would otherwise hit
// the same address.
template <int K>
__global__ void k_pair_bins(const int32_t* __restrict__ pairs, const int32_t* __restrict__ pair_list,
                            const int64_t* __restrict__ n_list_dev, int64_t n_pairs,
                            const int64_t* __restrict__ roff, int64_t n_reads,
                            const int64_t* __restrict__ hoff, int64_t n_haps, int bucket,
                            int32_t* __restrict__ pair_bin, int32_t* __restrict__ pair_nb,
                            unsigned long long* __restrict__ bin_blocks, unsigned long long* __restrict__ bin_pairs,
                            int* __restrict__ max_ncols, int* __restrict__ min_ncols_c,
                            unsigned long long* __restrict__ cells,
                            unsigned long long* __restrict__ padded_cells, unsigned long long* __restrict__ total_blocks,
                            uint32_t* err) {
  const int64_t n = n_list_dev ? *n_list_dev : n_pairs;
  const int lane = threadIdx.x & 31;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  uint32_t e = 0;
  unsigned long long my_cells = 0, my_padded = 0, my_blocks = 0;
  int my_max = 0, my_minc = 0;  // my_minc = kNcolsComplement - smallest column count
  for (int64_t base = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) & ~31ll; base < n; base += stride) {
    const int64_t k = base + lane;
    int bin = -1, nb = 0;
    if (k < n) {
      const int64_t p = pair_list ? pair_list[k] : k;
      const int32_t r = pairs[2 * p], h = pairs[2 * p + 1];
      if (r < 0 || r >= n_reads || h < 0 || h >= n_haps) {
        e |= ERR_INDEX;
      } else {
        const int64_t m = roff[r + 1] - roff[r], nh = hoff[h + 1] - hoff[h];
        if (m < 1 || nh < 1) {
          e |= ERR_EMPTY;
        } else if (nh > kMaxHapLen || m > kMaxReadLen) {
          e |= ERR_ARG;
        } else {
          const int nc = ncols_of((int)nh, bucket);
          bin = bin_of_ncols(nc, bucket);
          nb = nblocks_of<K>((int)m);
          my_max = max(my_max, nc);
          my_minc = max(my_minc, kNcolsComplement - nc);
          my_cells += (unsigned long long)(m * nh);
          my_padded += (unsigned long long)nb * K * nc;
          my_blocks += (unsigned long long)nb;
        }
      }
      pair_bin[k] = bin;
      pair_nb[k] = nb;
    }
    const unsigned act = __ballot_sync(0xffffffffu, bin >= 0);
    if (bin >= 0) {
      const unsigned peers = __match_any_sync(act, bin);
      const unsigned sum_nb = __reduce_add_sync(peers, (unsigned)nb);
      if (lane == __ffs(peers) - 1) {
        atomicAdd(&bin_blocks[bin], (unsigned long long)sum_nb);
        atomicAdd(&bin_pairs[bin], (unsigned long long)__popc(peers));
      }
    }
  }
  // one atomic per warp for the scalars
  for (int o = 16; o > 0; o >>= 1) {
    my_cells += __shfl_xor_sync(0xffffffffu, my_cells, o);
    my_padded += __shfl_xor_sync(0xffffffffu, my_padded, o);
    my_blocks += __shfl_xor_sync(0xffffffffu, my_blocks, o);
    my_max = max(my_max, __shfl_xor_sync(0xffffffffu, my_max, o));
    my_minc = max(my_minc, __shfl_xor_sync(0xffffffffu, my_minc, o));
    e |= __shfl_xor_sync(0xffffffffu, e, o);
  }
  if (lane == 0) {
    if (my_cells) atomicAdd(cells, my_cells);
    if (my_padded) atomicAdd(padded_cells, my_padded);
    if (my_blocks) atomicAdd(total_blocks, my_blocks);
    if (my_max) atomicMax(max_ncols, my_max);
    if (my_minc) atomicMax(min_ncols_c, my_minc);
    if (e) atomicOr(err, e);
  }
}

// Number of table blocks of each table item (an item is a read, or a rescued pair's read).
template <int K>
__global__ void k_item_nblocks(const int32_t* __restrict__ item_read, int64_t n_items,
                               const int64_t* __restrict__ n_items_dev, const int64_t* __restrict__ roff,
                               int64_t* __restrict__ item_nb) {
  const int64_t n = n_items_dev ? *n_items_dev : n_items;
  for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < n; k += (int64_t)gridDim.x * blockDim.x) {
    const int64_t r = item_read ? item_read[k] : k;
    const int64_t m = r >= 0 ? roff[r + 1] - roff[r] : 0;  // r < 0: unused item
    item_nb[k] = m >= 1 ? nblocks_of<K>((int)(m > kMaxReadLen ? 1 : m)) : 0;
  }
  if (blockIdx.x == 0 && threadIdx.x == 0) item_nb[n] = 0;
}

// ============================================================ finalize

// FP32 pass: log10 of the scaled sum, or queue the pair for the FP64 rescue.
__device__ __forceinline__ double start_mass_correction(const int32_t* __restrict__ pairs,
                                                        const int64_t* __restrict__ hoff, int64_t p, int bucket) {
  const int32_t h = pairs[2 * p + 1];
  const int n = (int)(hoff[h + 1] - hoff[h]);
  return log10((double)ncols_of(n, bucket) / (double)n);
}

// rescue_list gets p + rbase (a chunk of a larger batch lists its pairs by their batch index).
__global__ void k_finalize_fp32(const float* __restrict__ s32, const int32_t* __restrict__ exp32, int64_t n_pairs,
                                const int32_t* __restrict__ pairs,
                                const int64_t* __restrict__ hoff, int bucket, double* __restrict__ out,
                                uint8_t* __restrict__ status, int32_t* __restrict__ rescue_list,
                                int64_t* __restrict__ n_rescue, int write_status, int64_t rbase) {
  const double off = 120.0 * 0.30102999566398119521;
  for (int64_t p = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; p < n_pairs; p += (int64_t)gridDim.x * blockDim.x) {
    const float s = s32[p];
    // NaN-safe: also catches s < 1e-28; exp32 < 0 by 2^23: the ring rescale saturated
    if (!(s >= 1e-28f) || !isfinite(s) || exp32[p] < -(1 << 23)) {
      const unsigned long long k = atomicAdd(reinterpret_cast<unsigned long long*>(n_rescue), 1ull);
      rescue_list[k] = (int32_t)(p + rbase);
    } else {
      // the ring rescale multiplied the pair's later rows by 2^exp32[p]
      out[p] = log10((double)s) - (off + (double)exp32[p] * 0.30102999566398119521) +
               start_mass_correction(pairs, hoff, p, bucket);
      if (write_status) status[p] = 0;
    }
  }
}

// FP64 results (rescue list or all pairs): log10 - 1020 log10 2, status.
__global__ void k_finalize_fp64(const double* __restrict__ s64, const int32_t* __restrict__ list,
                                const int64_t* __restrict__ n_list_dev, int64_t n, const int32_t* __restrict__ pairs,
                                const int64_t* __restrict__ hoff, int bucket, double* __restrict__ out,
                                uint8_t* __restrict__ status, int write_status, uint8_t ok_status,
                                unsigned long long* __restrict__ n_underflow) {
  const double off = 1020.0 * 0.30102999566398119521;
  const int64_t cnt = n_list_dev ? *n_list_dev : n;
  for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < cnt; k += (int64_t)gridDim.x * blockDim.x) {
    const int64_t p = list ? list[k] : k;
    const double s = s64[k];
    uint8_t st = ok_status;
    double v;
    if (!(s > 0.0)) { v = -INFINITY; st = 2; }
    else {
      v = log10(s) - off + start_mass_correction(pairs, hoff, p, bucket);
      if (s < 2.2250738585072014e-308) st = 2;
    }
    if (st == 2) atomicAdd(n_underflow, 1ull);
    out[p] = v;
    if (write_status) status[p] = st;
  }
}

// One chunk of a batch: its pairs relative to its first read / haplotype (rlo, hlo), and the
// offsets of its reads [rlo, rlo + nr) / haplotypes [hlo, hlo + nh). relative = 1 (the host
// variant's copy/compute pipeline, whose chunk arrays start at the chunk's first byte): the
// offsets relative to that byte; relative = 0 (a chunked device call, which addresses the
// batch's base arrays): the offsets keep their values.
__global__ void k_rebase_chunk(const int64_t* __restrict__ roff, int64_t rlo, int64_t nr, int64_t* __restrict__ roff_c,
                               const int64_t* __restrict__ hoff, int64_t hlo, int64_t nh, int64_t* __restrict__ hoff_c,
                               const int32_t* __restrict__ pairs, int64_t p0, int64_t np, int32_t* __restrict__ pairs_c,
                               int relative) {
  const int64_t n = (nr + 1 > nh + 1 ? nr + 1 : nh + 1) > np ? (nr + 1 > nh + 1 ? nr + 1 : nh + 1) : np;
  const int64_t r0 = relative ? roff[rlo] : 0, h0 = relative ? hoff[hlo] : 0;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    if (i <= nr) roff_c[i] = roff[rlo + i] - r0;
    if (i <= nh) hoff_c[i] = hoff[hlo + i] - h0;
    if (i < np) {
      pairs_c[2 * i] = pairs[2 * (p0 + i)] - (int32_t)rlo;
      pairs_c[2 * i + 1] = pairs[2 * (p0 + i) + 1] - (int32_t)hlo;
    }
  }
}

// Index ranges of the chunks of a chunked device call: chunk blockIdx.y = pairs
// [y * chunk_pairs, ...); rng[4y .. 4y+3] = min / max read index, min / max haplotype index
// (minima preset to UINT_MAX, maxima to 0). Out-of-range indices raise ERR_INDEX.
__global__ void k_chunk_ranges(const int32_t* __restrict__ pairs, int64_t n_pairs, int64_t chunk_pairs,
                               int64_t n_reads, int64_t n_haps, uint32_t* __restrict__ rng, uint32_t* err) {
  const int64_t p0 = (int64_t)blockIdx.y * chunk_pairs;
  const int64_t p1 = min(n_pairs, p0 + chunk_pairs);
  uint32_t rmin = 0xffffffffu, rmax = 0, hmin = 0xffffffffu, hmax = 0, e = 0;
  for (int64_t p = p0 + blockIdx.x * (int64_t)blockDim.x + threadIdx.x; p < p1; p += (int64_t)gridDim.x * blockDim.x) {
    const int32_t r = pairs[2 * p], h = pairs[2 * p + 1];
    if (r < 0 || r >= n_reads || h < 0 || h >= n_haps) {
      e |= ERR_INDEX;
      continue;
    }
    rmin = min(rmin, (uint32_t)r); rmax = max(rmax, (uint32_t)r);
    hmin = min(hmin, (uint32_t)h); hmax = max(hmax, (uint32_t)h);
  }
  rmin = __reduce_min_sync(0xffffffffu, rmin); rmax = __reduce_max_sync(0xffffffffu, rmax);
  hmin = __reduce_min_sync(0xffffffffu, hmin); hmax = __reduce_max_sync(0xffffffffu, hmax);
  e = __reduce_or_sync(0xffffffffu, e);
  if ((threadIdx.x & 31) == 0) {
    uint32_t* g = rng + 4 * blockIdx.y;
    if (rmin != 0xffffffffu) {
      atomicMin(g, rmin); atomicMax(g + 1, rmax);
      atomicMin(g + 2, hmin); atomicMax(g + 3, hmax);
    }
    if (e) atomicOr(err, e);
  }
}

// item list of the rescue pass, one table item per distinct read: the rescued pairs' read ids
// were sorted (sorted_read, with their list positions sorted_pos); item j = the j-th distinct
// read, items past the last distinct read are unused (item_read = -1, no blocks)
__global__ void k_rescue_read_keys(const int32_t* __restrict__ pairs, const int32_t* __restrict__ list, int64_t n,
                                   uint32_t* __restrict__ keys, int32_t* __restrict__ vals) {
  for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < n; k += (int64_t)gridDim.x * blockDim.x) {
    keys[k] = (uint32_t)pairs[2 * (int64_t)list[k]];
    vals[k] = (int32_t)k;
  }
}
__global__ void k_rescue_head_flags(const uint32_t* __restrict__ sorted_read, int64_t n, int32_t* __restrict__ head) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    head[i] = (i == 0 || sorted_read[i] != sorted_read[i - 1]) ? 1 : 0;
}
// incl = inclusive scan of the head flags: sorted entry i belongs to item incl[i] - 1
__global__ void k_rescue_items_dedup(const uint32_t* __restrict__ sorted_read, const int32_t* __restrict__ sorted_pos,
                                     const int32_t* __restrict__ head, const int32_t* __restrict__ incl, int64_t n,
                                     int32_t* __restrict__ item_read, int32_t* __restrict__ pair_item) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    const int32_t item = incl[i] - 1;
    pair_item[sorted_pos[i]] = item;
    if (head[i]) item_read[item] = (int32_t)sorted_read[i];
    if (i >= incl[n - 1]) item_read[i] = -1;  // unused items (past the distinct reads)
  }
}


// exclusive scan of bins + work items (single block; nbins <= kMaxBins)
// Work items of each bin (the length-binned scheduler). A launch runs the
// bins [0, cut) or [cut, nbins); in launch order, its blocks before the last 1/tail_div of
// the launch's blocks are cut into items of `chunk` blocks, the rest into items of `chunk_s`
// blocks, so the last items of a launch are short and its warps finish together (guided
// self-scheduling). tail_div = 0: all items full-size. bin_nbig[b] = full-size items of bin b.
__device__ __forceinline__ unsigned long long block_scan_1024(unsigned long long v, unsigned long long* sh,
                                                              unsigned long long* total) {
  // warp inclusive scans by shuffle, then a scan of the 32 warp totals by warp 0
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  unsigned long long x = v;
#pragma unroll
  for (int off = 1; off < 32; off <<= 1) {
    const unsigned long long y = __shfl_up_sync(0xffffffffu, x, off);
    if (lane >= off) x += y;
  }
  if (lane == 31) sh[w] = x;
  __syncthreads();
  if (w == 0) {
    unsigned long long t = sh[lane];
#pragma unroll
    for (int off = 1; off < 32; off <<= 1) {
      const unsigned long long y = __shfl_up_sync(0xffffffffu, t, off);
      if (lane >= off) t += y;
    }
    sh[32 + lane] = t;  // inclusive prefix of the warp totals
  }
  __syncthreads();
  const unsigned long long incl = x + (w > 0 ? sh[32 + w - 1] : 0ull);
  *total = sh[63];
  __syncthreads();
  return incl - v;  // exclusive
}

__global__ void __launch_bounds__(1024) k_scan_bins(const unsigned long long* __restrict__ bin_blocks, int nbins,
                                                    int cut, int64_t chunk, int64_t chunk_s, int tail_div, int lpt,
                                                    unsigned long long* __restrict__ bin_start,
                                                    unsigned long long* __restrict__ item_start,
                                                    unsigned long long* __restrict__ bin_nbig,
                                                    unsigned long long* __restrict__ launch_items) {
  __shared__ unsigned long long sh[1024];
  // pass 1: first block of every bin (serial-by-tile scan: nbins is a few thousand at most)
  unsigned long long carry = 0, tot;
  for (int base = 0; base < nbins; base += 1024) {
    const int i = base + threadIdx.x;
    const unsigned long long vb = (i < nbins) ? bin_blocks[i] : 0ull;
    const unsigned long long ex = block_scan_1024(vb, sh, &tot);
    if (i < nbins) bin_start[i] = carry + ex;
    carry += tot;
  }
  if (threadIdx.x == 0) bin_start[nbins] = carry;
  __syncthreads();
  const int c = cut < 0 ? 0 : (cut > nbins ? nbins : cut);
  const unsigned long long B0 = bin_start[c], Ball = carry;
  const unsigned long long L0 = B0, L1 = Ball - B0;  // blocks of the two launches
  const unsigned long long thr0 = tail_div > 0 ? L0 - L0 / tail_div : L0;
  const unsigned long long thr1 = tail_div > 0 ? L1 - L1 / tail_div : L1;
  // pass 2: items per bin (item_start: exclusive prefix in bin order for now)
  carry = 0;
  for (int base = 0; base < nbins; base += 1024) {
    const int i = base + threadIdx.x;
    unsigned long long vi = 0;
    if (i < nbins) {
      const unsigned long long vb = bin_blocks[i];
      const bool l0 = i < c;
      // position of the bin's first block in its launch's order (ascending or, lpt, descending bins)
      const unsigned long long pos = lpt ? (l0 ? B0 : Ball) - bin_start[i + 1] : bin_start[i] - (l0 ? 0ull : B0);
      const unsigned long long thr = l0 ? thr0 : thr1;
      const unsigned long long big = thr <= pos ? 0ull : (thr - pos < vb ? thr - pos : vb);
      const unsigned long long nbig = (big == vb) ? (vb + chunk - 1) / chunk : big / chunk;
      const unsigned long long used = nbig * chunk < vb ? nbig * chunk : vb;
      vi = nbig + (vb - used + chunk_s - 1) / chunk_s;
      bin_nbig[i] = nbig;
    }
    const unsigned long long ex = block_scan_1024(vi, sh, &tot);
    if (i < nbins) item_start[i] = carry + ex;
    carry += tot;
  }
  if (threadIdx.x == 0) item_start[nbins] = carry;
  __syncthreads();
  const unsigned long long I0 = item_start[c], Iall = carry;
  if (threadIdx.x == 0) {
    launch_items[0] = 0; launch_items[1] = I0; launch_items[2] = I0; launch_items[3] = Iall;
  }
  if (lpt) {  // descending bins inside each launch: item_start[i] = launch base + items of the bins above i
    constexpr int kPer = (kMaxBins + 1 + 1023) / 1024;
    unsigned long long v[kPer];
#pragma unroll
    for (int r = 0; r < kPer; ++r) {  // read every old value before any is overwritten
      const int i = threadIdx.x + 1024 * r;
      const unsigned long long nxt = (i + 1 < nbins) ? item_start[i + 1] : Iall;
      v[r] = (i < c) ? I0 - nxt : I0 + (Iall - nxt);
    }
    __syncthreads();
#pragma unroll
    for (int r = 0; r < kPer; ++r) {
      const int i = threadIdx.x + 1024 * r;
      if (i < nbins) item_start[i] = v[r];
    }
  }
}

}  // namespace phmm
