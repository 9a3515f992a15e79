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

// Four base letters in a 32-bit word, each one of A C G T N (SIMD byte compares).
__device__ __forceinline__ bool bases_ok4(uint32_t w) {
  const uint32_t m = __vcmpeq4(w, 0x41414141u) | __vcmpeq4(w, 0x43434343u) | __vcmpeq4(w, 0x47474747u) |
                     __vcmpeq4(w, 0x54545454u) | __vcmpeq4(w, 0x4e4e4e4eu);
  return m == 0xffffffffu;
}

// 4 read bases with their four qualities (one 32-bit word of each array).
__device__ __forceinline__ uint32_t read_word_err(uint32_t b, uint32_t a, uint32_t x, uint32_t y, uint32_t z) {
  // fast path: every byte a base letter, no quality byte >= 128, no indel quality <= 3
  if (!((a | x | y | z) & 0x80808080u) && !__vcmpleu4(x, 0x03030303u) && !__vcmpleu4(y, 0x03030303u))
    return bases_ok4(b) ? 0u : ERR_BASE;
  uint32_t e = 0;
  for (int k = 0; k < 4; ++k)
    e |= read_base_err((uint8_t)(b >> 8 * k), (uint8_t)(a >> 8 * k), (uint8_t)(x >> 8 * k), (uint8_t)(y >> 8 * k),
                       (uint8_t)(z >> 8 * k));
  return e;
}

// The whole batch in one launch: every haplotype base, every read base with its four
// qualities (16 bases per thread-step through 16-byte vectors where the five arrays share
// their alignment), and both offset arrays. Errors are OR-ed into *err (one atomic per warp).
__global__ void k_validate(const uint8_t* __restrict__ hap, int64_t n_hb, const uint8_t* __restrict__ rb,
                           const uint8_t* __restrict__ q, const uint8_t* __restrict__ qi,
                           const uint8_t* __restrict__ qd, const uint8_t* __restrict__ qg, int64_t n_rb,
                           const int64_t* __restrict__ roff, int64_t n_reads, const int64_t* __restrict__ hoff,
                           int64_t n_haps, uint32_t* err) {
  uint32_t e = 0;
  const int64_t tid = blockIdx.x * (int64_t)blockDim.x + threadIdx.x, nthr = (int64_t)gridDim.x * blockDim.x;
  // haplotypes: a scalar head up to 16-byte alignment, 16-byte vectors, a scalar tail
  {
    const int64_t head = min(n_hb, (int64_t)((16 - ((uintptr_t)hap & 15)) & 15));
    for (int64_t i = tid; i < head; i += nthr)
      if (base_code(hap[i]) == 0xffu) e |= ERR_BASE;
    const int64_t nv = (n_hb - head) >> 4;
    const uint4* h16 = reinterpret_cast<const uint4*>(hap + head);
    for (int64_t v = tid; v < nv; v += nthr) {
      const uint4 w = h16[v];
      if (!(bases_ok4(w.x) && bases_ok4(w.y) && bases_ok4(w.z) && bases_ok4(w.w))) e |= ERR_BASE;
    }
    for (int64_t i = head + 16 * nv + tid; i < n_hb; i += nthr)
      if (base_code(hap[i]) == 0xffu) e |= ERR_BASE;
  }
  // reads: the same, as 16-byte vectors of all five arrays when they share their alignment
  // (else 4-byte words when they share it mod 4, else bytes)
  auto same_mod = [&](uintptr_t m) {
    const uintptr_t r = (uintptr_t)rb & m;
    return (((uintptr_t)q & m) == r) && (((uintptr_t)qi & m) == r) && (((uintptr_t)qd & m) == r) &&
           (((uintptr_t)qg & m) == r);
  };
  const int vec = same_mod(15) ? 16 : (same_mod(3) ? 4 : 1);
  const int64_t head = vec == 1 ? n_rb : min(n_rb, (int64_t)((vec - ((uintptr_t)rb & (vec - 1))) & (vec - 1)));
  for (int64_t i = tid; i < head; i += nthr) e |= read_base_err(rb[i], q[i], qi[i], qd[i], qg[i]);
  int64_t done = head;
  if (vec == 16) {
    const int64_t nv = (n_rb - head) >> 4;
    const uint4 *b16 = reinterpret_cast<const uint4*>(rb + head), *q16 = reinterpret_cast<const uint4*>(q + head),
                *i16 = reinterpret_cast<const uint4*>(qi + head), *d16 = reinterpret_cast<const uint4*>(qd + head),
                *g16 = reinterpret_cast<const uint4*>(qg + head);
    for (int64_t v = tid; v < nv; v += nthr) {
      const uint4 b = b16[v], a = q16[v], x = i16[v], y = d16[v], z = g16[v];
      e |= read_word_err(b.x, a.x, x.x, y.x, z.x) | read_word_err(b.y, a.y, x.y, y.y, z.y) |
           read_word_err(b.z, a.z, x.z, y.z, z.z) | read_word_err(b.w, a.w, x.w, y.w, z.w);
    }
    done = head + 16 * nv;
  } else if (vec == 4) {
    const int64_t nw = (n_rb - head) >> 2;
    const uint32_t *b4 = reinterpret_cast<const uint32_t*>(rb + head), *q4 = reinterpret_cast<const uint32_t*>(q + head),
                   *i4 = reinterpret_cast<const uint32_t*>(qi + head), *d4 = reinterpret_cast<const uint32_t*>(qd + head),
                   *g4 = reinterpret_cast<const uint32_t*>(qg + head);
    for (int64_t w = tid; w < nw; w += nthr) e |= read_word_err(b4[w], q4[w], i4[w], d4[w], g4[w]);
    done = head + 4 * nw;
  }
  for (int64_t i = done + tid; i < n_rb; i += nthr) e |= read_base_err(rb[i], q[i], qi[i], qd[i], qg[i]);
  for (int64_t i = tid; i <= n_reads; i += nthr)
    if (offset_bad(roff, i, n_reads, n_rb)) e |= ERR_ARG;
  for (int64_t i = tid; i <= n_haps; i += nthr)
    if (offset_bad(hoff, i, n_haps, n_hb)) e |= ERR_ARG;
  e = __reduce_or_sync(0xffffffffu, e);
  if (e && (threadIdx.x & 31) == 0) atomicOr(err, e);
}

// Byte fill of device scratch as a kernel: a cudaMemsetAsync is queued behind the host->device
// copies of the pipelined host call (measured: a 0.5 MB memset waited 150 us on another
// stream's copy), a kernel is not. 16-byte stores from the first 16-byte boundary on.
__global__ void k_fill_bytes(uint8_t* __restrict__ p, uint32_t v4, int64_t n) {
  const int64_t tid = blockIdx.x * (int64_t)blockDim.x + threadIdx.x, nthr = (int64_t)gridDim.x * blockDim.x;
  const int64_t head = min(n, (int64_t)((16 - ((uintptr_t)p & 15)) & 15));
  for (int64_t i = tid; i < head; i += nthr) p[i] = (uint8_t)v4;
  const int64_t nv = (n - head) >> 4;
  uint4* q = reinterpret_cast<uint4*>(p + head);
  for (int64_t i = tid; i < nv; i += nthr) q[i] = make_uint4(v4, v4, v4, v4);
  for (int64_t i = head + 16 * nv + tid; i < n; i += nthr) p[i] = (uint8_t)v4;
}

// Offsets (the Smith-Waterman batch): start at 0, non-decreasing, end at total.
__global__ void k_validate_offsets(const int64_t* __restrict__ off, int64_t n, int64_t total, uint32_t* err) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i <= n; i += (int64_t)gridDim.x * blockDim.x)
    if (offset_bad(off, i, n, total)) atomicOr(err, ERR_ARG);
}

// Per pair: validate indices/lengths, bin by column count, count blocks per bin.
// pair_list == nullptr -> pairs 0..n-1, else the listed pair ids (rescue pass).
// Counters are aggregated per warp (match_any + reduce), then per CTA in a shared-memory
// histogram, which is flushed with one global atomic per non-empty bin and CTA: with one
// length bin (C2) every warp would otherwise hit the same global address (32 K same-address
// atomics per 2^20 pairs, 63 us; profiles/r02_timeline_C2.json). 32-bit shared counters:
// the launch gives every CTA at most kPairBinsPerCta pairs of at most 2^18 blocks each
// (nblocks_of<4>(kMaxReadLen)), so a CTA's count stays below 2^30.
constexpr int64_t kPairBinsPerCta = 4096;
constexpr int kPairBinsU = 4;  // pairs per lane per trip
template <int K>
__global__ void k_pair_bins(const int32_t* __restrict__ pairs, const int32_t* __restrict__ pair_list,
                            const int64_t* __restrict__ n_list_dev, int64_t n_pairs,
                            const int64_t* __restrict__ roff, int64_t n_reads,
                            const int64_t* __restrict__ hoff, int64_t n_haps, int bucket, int align,
                            int32_t* __restrict__ pair_bin, int32_t* __restrict__ pair_nb,
                            unsigned long long* __restrict__ bin_blocks, unsigned long long* __restrict__ bin_pairs,
                            int* __restrict__ max_ncols, int* __restrict__ min_ncols_c,
                            unsigned long long* __restrict__ cells,
                            unsigned long long* __restrict__ padded_cells, unsigned long long* __restrict__ total_blocks,
                            uint32_t* err) {
  __shared__ uint32_t s_blk[kMaxBins + 1], s_cnt[kMaxBins + 1];
  for (int i = threadIdx.x; i <= kMaxBins; i += blockDim.x) s_blk[i] = s_cnt[i] = 0u;
  __syncthreads();
  const int64_t n = n_list_dev ? *n_list_dev : n_pairs;
  const int lane = threadIdx.x & 31;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  uint32_t e = 0;
  unsigned long long my_cells = 0, my_padded = 0, my_blocks = 0;
  int my_max = 0, my_minc = 0;  // my_minc = kNcolsComplement - smallest column count
  // kPairBinsU pairs per lane per trip, their loads issued together (the kernel is bound by
  // the latency of the pairs -> offsets gather chain, not by bandwidth)
  constexpr int U = kPairBinsU;
  for (int64_t base = ((blockIdx.x * (int64_t)blockDim.x + threadIdx.x) & ~31ll) * U; base < n; base += stride * U) {
    int32_t r[U], h[U];
    int64_t r0[U], r1[U], h0[U], h1[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const int64_t k = base + 32 * u + lane;
      r[u] = h[u] = -1;
      if (k < n) {
        const int64_t p = pair_list ? pair_list[k] : k;
        r[u] = pairs[2 * p];
        h[u] = pairs[2 * p + 1];
      }
    }
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const bool ok = r[u] >= 0 && r[u] < n_reads && h[u] >= 0 && h[u] < n_haps;
      r0[u] = ok ? roff[r[u]] : 0;
      r1[u] = ok ? roff[r[u] + 1] : 0;
      h0[u] = ok ? hoff[h[u]] : 0;
      h1[u] = ok ? hoff[h[u] + 1] : 0;
    }
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const int64_t k = base + 32 * u + lane;
      int bin = -1, nb = 0;
      if (k < n) {
        if (r[u] < 0 || r[u] >= n_reads || h[u] < 0 || h[u] >= n_haps) {
          e |= ERR_INDEX;
        } else {
          const int64_t m = r1[u] - r0[u], nh = h1[u] - h0[u];
          if (m < 1 || nh < 1) {
            e |= ERR_EMPTY;
          } else if (nh > kMaxHapLen || m > kMaxReadLen) {
            e |= ERR_ARG;
          } else {
            const int nc = ncols_of((int)nh, bucket);
            bin = bin_of_ncols(nc, bucket);
            nb = padded_nb(nblocks_of<K>((int)m), nc, align);
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
          atomicAdd(&s_blk[bin], sum_nb);
          atomicAdd(&s_cnt[bin], (uint32_t)__popc(peers));
        }
      }
    }
  }
  __syncthreads();
  for (int i = threadIdx.x; i <= kMaxBins; i += blockDim.x)
    if (s_cnt[i]) {
      atomicAdd(&bin_blocks[i], (unsigned long long)s_blk[i]);
      atomicAdd(&bin_pairs[i], (unsigned long long)s_cnt[i]);
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

// rng[4k .. 4k+3] = (UINT_MAX, 0, UINT_MAX, 0) for k < n: the identities of k_chunk_ranges
__global__ void k_ranges_init(uint32_t* __restrict__ rng, int64_t n) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < 4 * n; i += (int64_t)gridDim.x * blockDim.x)
    rng[i] = (i & 1) ? 0u : 0xffffffffu;
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
  // every thread owns kPer consecutive bins (serial within the thread, one block scan over
  // the 1024 thread sums per pass); the prefixes are kept in shared memory for the lookups
  // of a neighbouring bin
  constexpr int kPer = (kMaxBins + 1 + 1023) / 1024;
  __shared__ unsigned long long sh[64];
  __shared__ unsigned long long spre[kPer * 1024 + 1];
  const int i0 = threadIdx.x * kPer;
  unsigned long long vb[kPer], loc = 0, tot;
#pragma unroll
  for (int r = 0; r < kPer; ++r) {
    vb[r] = (i0 + r < nbins) ? bin_blocks[i0 + r] : 0ull;
    loc += vb[r];
  }
  // pass 1: first block of every bin
  unsigned long long acc = block_scan_1024(loc, sh, &tot);
  unsigned long long bs[kPer];
#pragma unroll
  for (int r = 0; r < kPer; ++r) {
    bs[r] = acc;
    acc += vb[r];
    if (i0 + r < nbins) {
      bin_start[i0 + r] = bs[r];
      spre[i0 + r] = bs[r];
    }
  }
  const unsigned long long Ball = tot;
  if (threadIdx.x == 0) {
    bin_start[nbins] = Ball;
    spre[nbins] = Ball;
  }
  __syncthreads();
  const int c = cut < 0 ? 0 : (cut > nbins ? nbins : cut);
  const unsigned long long B0 = spre[c];
  const unsigned long long L0 = B0, L1 = Ball - B0;  // blocks of the two launches
  const unsigned long long thr0 = tail_div > 0 ? L0 - L0 / tail_div : L0;
  const unsigned long long thr1 = tail_div > 0 ? L1 - L1 / tail_div : L1;
  // pass 2: items per bin (exclusive prefix in ascending bin order)
  unsigned long long vi[kPer];
  loc = 0;
#pragma unroll
  for (int r = 0; r < kPer; ++r) {
    const int i = i0 + r;
    vi[r] = 0;
    if (i < nbins) {
      const bool l0 = i < c;
      // position of the bin's first block in its launch's order (ascending or, lpt, descending bins)
      const unsigned long long pos = lpt ? (l0 ? B0 : Ball) - spre[i + 1] : bs[r] - (l0 ? 0ull : B0);
      const unsigned long long thr = l0 ? thr0 : thr1;
      const unsigned long long big = thr <= pos ? 0ull : (thr - pos < vb[r] ? thr - pos : vb[r]);
      const unsigned long long nbig = (big == vb[r]) ? (vb[r] + chunk - 1) / chunk : big / chunk;
      const unsigned long long used = nbig * chunk < vb[r] ? nbig * chunk : vb[r];
      vi[r] = nbig + (vb[r] - used + chunk_s - 1) / chunk_s;
      bin_nbig[i] = nbig;
    }
    loc += vi[r];
  }
  unsigned long long Iall;
  acc = block_scan_1024(loc, sh, &Iall);  // (ends with a barrier: spre is free again)
  unsigned long long is[kPer];
#pragma unroll
  for (int r = 0; r < kPer; ++r) {
    is[r] = acc;
    acc += vi[r];
    if (i0 + r < nbins) spre[i0 + r] = is[r];
  }
  if (threadIdx.x == 0) {
    spre[nbins] = Iall;
    item_start[nbins] = Iall;
  }
  __syncthreads();
  const unsigned long long I0 = spre[c];
  if (threadIdx.x == 0) {
    launch_items[0] = 0; launch_items[1] = I0; launch_items[2] = I0; launch_items[3] = Iall;
  }
#pragma unroll
  for (int r = 0; r < kPer; ++r) {
    const int i = i0 + r;
    if (i >= nbins) break;
    // lpt: descending bins inside each launch, item_start[i] = launch base + items of the bins above i
    const unsigned long long nxt = spre[i + 1];
    item_start[i] = !lpt ? is[r] : (i < c) ? I0 - nxt : I0 + (Iall - nxt);
  }
}

}  // namespace phmm
