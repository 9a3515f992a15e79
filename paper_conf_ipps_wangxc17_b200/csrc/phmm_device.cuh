// phmm_device.cuh -- prep, generic (FP64) wavefront and finalize kernels of libphmm.
// Included only by phmm_lib.cu. See phmm_common.cuh for what is computed.
#pragma once
#include "phmm_common.cuh"

namespace phmm {

// ============================================================ prep kernels

// Haplotype bases -> one-hot codes (validation in the same pass).
__global__ void k_hap_codes(const uint8_t* __restrict__ hap, int64_t n, uint8_t* __restrict__ codes,
                            uint32_t* err) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    uint32_t c = base_code(hap[i]);
    if (c == 0xffu) { atomicOr(err, ERR_BASE); c = 0; }
    codes[i] = (uint8_t)c;
  }
}

// Read bases and qualities: validation only (the tables re-read them).
__global__ void k_validate_reads(const uint8_t* __restrict__ rb, const uint8_t* __restrict__ q,
                                 const uint8_t* __restrict__ qi, const uint8_t* __restrict__ qd,
                                 const uint8_t* __restrict__ qg, int64_t n, uint32_t* err) {
  uint32_t e = 0;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    if (base_code(rb[i]) == 0xffu) e |= ERR_BASE;
    if ((q[i] | qi[i] | qd[i] | qg[i]) & 0x80u) e |= ERR_QUAL;
    // the transitions out of M must be a distribution: e(qi) + e(qd) <= 1
    // (reading R16); only qualities <= 3 can violate it
    else if ((qi[i] <= 3 || qd[i] <= 3) && exp10(-(double)qi[i] / 10.0) + exp10(-(double)qd[i] / 10.0) > 1.0)
      e |= ERR_QUAL;
  }
  if (e) atomicOr(err, e);
}

// Offsets: start at 0, non-decreasing, end at total.
__global__ void k_validate_offsets(const int64_t* __restrict__ off, int64_t n, int64_t total, uint32_t* err) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i <= n; i += (int64_t)gridDim.x * blockDim.x) {
    bool bad = false;
    if (i == 0) bad = off[0] != 0;
    else bad = off[i] < off[i - 1];
    if (i == n) bad |= off[n] != total;
    if (bad) atomicOr(err, ERR_ARG);
  }
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
                            int* __restrict__ max_ncols, unsigned long long* __restrict__ cells,
                            unsigned long long* __restrict__ padded_cells, unsigned long long* __restrict__ total_blocks,
                            uint32_t* err) {
  const int64_t n = n_list_dev ? *n_list_dev : n_pairs;
  const int lane = threadIdx.x & 31;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  uint32_t e = 0;
  unsigned long long my_cells = 0, my_padded = 0, my_blocks = 0;
  int my_max = 0;
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
        } else if (nh > kMaxHapLen || m > (1 << 20)) {
          e |= ERR_ARG;
        } else {
          const int nc = ncols_of((int)nh, bucket);
          bin = bin_of_ncols(nc, bucket);
          nb = nblocks_of<K>((int)m);
          my_max = max(my_max, nc);
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
    e |= __shfl_xor_sync(0xffffffffu, e, o);
  }
  if (lane == 0) {
    if (my_cells) atomicAdd(cells, my_cells);
    if (my_padded) atomicAdd(padded_cells, my_padded);
    if (my_blocks) atomicAdd(total_blocks, my_blocks);
    if (my_max) atomicMax(max_ncols, my_max);
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
    const int64_t m = roff[r + 1] - roff[r];
    item_nb[k] = m >= 1 ? nblocks_of<K>((int)(m > (1 << 20) ? 1 : m)) : 0;
  }
  if (blockIdx.x == 0 && threadIdx.x == 0) item_nb[n] = 0;
}

// Build the per-item coefficient table: one thread per padded row.
// Row layout of an item with m read bases, nb = ceil((m+3)/K) blocks:
//   f = nb*K - (m+3) Z rows, R, rows 1..m, S1, S2
template <typename T, int K>
__global__ void k_build_table(const int32_t* __restrict__ item_read, const int64_t* __restrict__ n_items_dev,
                              int64_t n_items, const int64_t* __restrict__ item_tab_off,
                              const int64_t* __restrict__ total_tab_blocks_dev, const int64_t* __restrict__ roff,
                              const uint8_t* __restrict__ rb, const uint8_t* __restrict__ q,
                              const uint8_t* __restrict__ qi, const uint8_t* __restrict__ qd,
                              const uint8_t* __restrict__ qg, TabBlock<T, K>* __restrict__ tab) {
  const int64_t nit = n_items_dev ? *n_items_dev : n_items;
  const int64_t total_rows = (*total_tab_blocks_dev) * K;
  for (int64_t g = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; g < total_rows; g += (int64_t)gridDim.x * blockDim.x) {
    const int64_t b = g / K;
    const int t = (int)(g % K);
    // item owning table block b: last item with item_tab_off[item] <= b
    int64_t lo = 0, hi = nit - 1;
    while (lo < hi) {
      const int64_t mid = (lo + hi + 1) >> 1;
      if (item_tab_off[mid] <= b) lo = mid; else hi = mid - 1;
    }
    const int64_t it = lo;
    const int64_t r = item_read ? item_read[it] : it;
    const int64_t r0 = roff[r];
    const int m = (int)(roff[r + 1] - r0);
    const int nb = nblocks_of<K>(m);
    const int f = nb * K - (m + 3);
    const int row = (int)(b - item_tab_off[it]) * K + t;  // row within the item
    T al = 0, be = 0, de = 0, ep = 0, ze = 0, mu = 0, pm = 0, px = 0;
    uint32_t mk = MASK_BASE;
    if (row < f) {
      // Z row: everything 0
    } else if (row == f) {  // R row
      mu = 1;
      mk |= MASK_D0;
    } else if (row <= f + m) {  // read row i = row - f (1-based)
      const int64_t x = r0 + (row - f - 1);
      const T ei = qual_err<T>(qi[x]), ed = qual_err<T>(qd[x]), eg = qual_err<T>(qg[x]), eb = qual_err<T>(q[x]);
      const T s = ei + ed;
      al = (T)1 - (s < (T)1 ? s : (T)1);
      be = (T)1 - eg;
      de = ei;
      ep = eg;
      ze = ed;
      mu = eg;
      pm = (T)1 - eb;
      px = eb / (T)3;
      uint32_t c = base_code(rb[x]);
      mk = (c == 0xffu) ? 0u : c;
      if (row == f + 1 && t == 0) mk |= MASK_ABOVE_IS_R;
    } else if (row == f + m + 1) {  // S1
      de = 1; ep = 1; mu = 1;
    } else {  // S2
      be = 1; ze = 1; mu = 1; pm = 1; px = 1;
    }
    TabBlock<T, K>& B = tab[b];
    B.coef[0][t] = al; B.coef[1][t] = be; B.coef[2][t] = de; B.coef[3][t] = ep;
    B.coef[4][t] = ze; B.coef[5][t] = mu; B.coef[6][t] = pm; B.coef[7][t] = px;
    B.mask[t] = mk;
  }
}

// Allocate each pair's block range inside its bin and write the descriptors.
template <int K>
__global__ void k_alloc_blocks(const int32_t* __restrict__ pairs, const int32_t* __restrict__ pair_list,
                               const int64_t* __restrict__ n_list_dev, int64_t n_pairs,
                               const int32_t* __restrict__ pair_bin, const int32_t* __restrict__ pair_nb,
                               const unsigned long long* __restrict__ bin_start,
                               unsigned long long* __restrict__ bin_cursor,
                               const int64_t* __restrict__ hoff, const int64_t* __restrict__ item_tab_off,
                               const int32_t* __restrict__ pair_item, int out_by_list,
                               BlkDesc* __restrict__ blk) {
  const int64_t n = n_list_dev ? *n_list_dev : n_pairs;
  for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < n; k += (int64_t)gridDim.x * blockDim.x) {
    const int bin = pair_bin[k];
    if (bin < 0) continue;
    const int nb = pair_nb[k];
    const int64_t p = pair_list ? pair_list[k] : k;
    const int32_t r = pairs[2 * p], h = pairs[2 * p + 1];
    const int64_t item = pair_item ? pair_item[k] : r;
    const unsigned long long g0 = bin_start[bin] + atomicAdd(&bin_cursor[bin], (unsigned long long)nb);
    const uint32_t tab0 = (uint32_t)item_tab_off[item];
    const int nh = (int)(hoff[h + 1] - hoff[h]);
    for (int j = 0; j < nb; ++j) {
      BlkDesc d;
      d.tab_blk = tab0 + j;
      d.hap_off = (uint32_t)hoff[h];
      d.out_idx = (int32_t)(out_by_list ? k : p);
      d.n = (uint16_t)nh;
      d.flags = (uint16_t)((j == nb - 1 ? BLK_LAST : 0) | (j == 0 ? BLK_FIRST : 0));
      blk[g0 + j] = d;
    }
  }
}

// ============================================================ wavefront

template <typename T>
struct WfArgs {
  const BlkDesc* blk;
  const void* tab;               // TabBlock<T,K>[]
  const uint8_t* hcodes;         // haplotype one-hot codes (+ padding)
  const unsigned long long* bin_start;   // [nbins+1] block start of each bin
  const unsigned long long* item_start;  // [nbins+1] first work item of each bin
  int nbins;
  int bucket;
  int64_t chunk_blocks;          // nominal blocks per work item
  unsigned int* item_counter;    // dynamic work queue
  T* out;                        // scaled last-row sum per output slot
  int ring_len;                  // ring entries per warp (>= max ncols)
};

template <typename T>
__device__ __forceinline__ T shfl_up1(T v, int src) {
  return __shfl_sync(0xffffffffu, v, src);
}

template <typename T, int K>
__device__ __forceinline__ void load_block(const TabBlock<T, K>* __restrict__ tab, uint32_t b, T (&c)[8][K],
                                           uint32_t (&mk)[K]) {
  constexpr int NW = (int)(sizeof(TabBlock<T, K>) / 16);
  const uint4* __restrict__ src = reinterpret_cast<const uint4*>(tab + b);
  union U { uint4 w[NW]; TabBlock<T, K> tb; } u;
#pragma unroll
  for (int i = 0; i < NW; ++i) u.w[i] = __ldg(src + i);
#pragma unroll
  for (int f = 0; f < 8; ++f)
#pragma unroll
    for (int t = 0; t < K; ++t) c[f][t] = u.tb.coef[f][t];
#pragma unroll
  for (int t = 0; t < K; ++t) mk[t] = u.tb.mask[t];
}

// One warp streams through blocks [s, s+nblk) of one bin (all with ncols columns).
template <typename T, int K>
__device__ __forceinline__ void run_stream(const WfArgs<T>& A, RingEnt<T>* __restrict__ ring, int lane,
                                           int64_t s, int nblk, int ncols) {
  const TabBlock<T, K>* __restrict__ tab = reinterpret_cast<const TabBlock<T, K>*>(A.tab);
  const T scale = (T)ldexp(1.0, Prec<T>::kScaleExp);
  T cf[8][K];
  uint32_t mk[K];
  T M[K], I[K], D[K];
#pragma unroll
  for (int t = 0; t < K; ++t) {
#pragma unroll
    for (int f = 0; f < 8; ++f) cf[f][t] = 0;
    mk[t] = 0;
    M[t] = 0; I[t] = 0; D[t] = 0;
  }
  T upM = 0, upI = 0, upD = 0, dgM = 0, dgI = 0, dgD = 0;
  const uint8_t* __restrict__ hp = A.hcodes;
  constexpr int kNoCol = -(1 << 30);  // never equal to a lane-local column (c >= -32)
  int ecol = kNoCol, out_idx = 0;
  int c = -lane - 1;  // lane-local column; becomes 0 at step t == lane
  int q = -1;         // lane-local pass
  const int steps = ((nblk - 1) >> 5) * ncols + ((nblk - 1) & 31) + ncols;
  const int src = (lane + 31) & 31;

  for (int step = 0; step < steps; ++step) {
    ++c;
    if (c == ncols) c = 0;
    if (c == 0) {  // switch to the next block of this lane
      ++q;
      const int b = q * 32 + lane;
      if (b < nblk) {
        const BlkDesc d = A.blk[s + b];
        load_block<T, K>(tab, d.tab_blk, cf, mk);
        hp = A.hcodes + d.hap_off;
        // virtual row 0 (the R row): D = s/ncols on every column, so the total
        // start mass over all ncols columns (real + padding) is exactly s and
        // no cell can exceed s; finalize adds log10(ncols/N).
        const T d0 = scale / (T)ncols;
        ecol = (d.flags & BLK_LAST) ? (int)d.n + 1 : kNoCol;
        out_idx = d.out_idx;
#pragma unroll
        for (int t = 0; t < K; ++t) { M[t] = 0; I[t] = 0; D[t] = (mk[t] & MASK_D0) ? d0 : (T)0; }
        dgM = 0; dgI = 0; dgD = (mk[0] & MASK_ABOVE_IS_R) ? d0 : (T)0;
      } else {
#pragma unroll
        for (int t = 0; t < K; ++t) {
#pragma unroll
          for (int f = 0; f < 8; ++f) cf[f][t] = 0;
          mk[t] = 0;
          M[t] = 0; I[t] = 0; D[t] = 0;
        }
        ecol = kNoCol;
        hp = A.hcodes;
      }
    }
    const uint32_t hc = (c >= 0) ? (uint32_t)hp[c] : 0u;

    // ---- one column of K rows (Eq. 6), rows top to bottom
    T nM[K], nI[K], nD[K];
#pragma unroll
    for (int t = 0; t < K; ++t) {
      const T mD = (t == 0) ? dgM : M[t - 1];
      const T iD = (t == 0) ? dgI : I[t - 1];
      const T dD = (t == 0) ? dgD : D[t - 1];
      const T pr = (mk[t] & hc) ? cf[6][t] : cf[7][t];
      nM[t] = pr * fma(cf[0][t], mD, cf[1][t] * (iD + dD));
      nD[t] = fma(cf[4][t], M[t], cf[5][t] * D[t]);
      const T mU = (t == 0) ? upM : nM[t - 1];
      const T iU = (t == 0) ? upI : nI[t - 1];
      nI[t] = fma(cf[2][t], mU, cf[3][t] * iU);
    }
#pragma unroll
    for (int t = 0; t < K; ++t) { M[t] = nM[t]; I[t] = nI[t]; D[t] = nD[t]; }

    if (c == ecol) A.out[out_idx] = nD[K - 1];  // S2 row: the last-row M+I sum (L20@2262)

    // ---- exchange: row K-1 goes down one lane; lane 31 -> ring -> lane 0
    const T sM = nM[K - 1], sI = nI[K - 1], sD = nD[K - 1];
    if (lane == 31 && c >= 0) {
      RingEnt<T> e; e.m = sM; e.i = sI; e.d = sD; e.pad = 0;
      ring[c] = e;
    }
    __syncwarp();
    T rM = shfl_up1(sM, src), rI = shfl_up1(sI, src), rD = shfl_up1(sD, src);
    if (lane == 0) {
      const int cn = (c + 1 == ncols) ? 0 : c + 1;
      const RingEnt<T> e = ring[cn];
      rM = e.m; rI = e.i; rD = e.d;
    }
    dgM = upM; dgI = upI; dgD = upD;
    upM = rM; upI = rI; upD = rD;
  }
}

template <typename T, int K>
__global__ void __launch_bounds__(128) k_wavefront(WfArgs<T> A) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  const int lane = threadIdx.x & 31;
  const int wib = threadIdx.x >> 5;
  RingEnt<T>* ring = reinterpret_cast<RingEnt<T>*>(smem_raw) + (size_t)wib * A.ring_len;
  for (int i = lane; i < A.ring_len; i += 32) {
    RingEnt<T> z; z.m = 0; z.i = 0; z.d = 0; z.pad = 0;
    ring[i] = z;
  }
  __syncwarp();
  const unsigned long long n_items = A.item_start[A.nbins];
  while (true) {
    unsigned int it = 0;
    if (lane == 0) it = atomicAdd(A.item_counter, 1u);
    it = __shfl_sync(0xffffffffu, it, 0);
    if (it >= n_items) break;
    // bin of this item: last bin with item_start[bin] <= it
    int lo = 0, hi = A.nbins - 1;
    while (lo < hi) {
      const int mid = (lo + hi + 1) >> 1;
      if (A.item_start[mid] <= it) lo = mid; else hi = mid - 1;
    }
    const int bin = lo;
    const int64_t b0 = (int64_t)A.bin_start[bin], b1 = (int64_t)A.bin_start[bin + 1];
    const int64_t k = (int64_t)(it - A.item_start[bin]);
    int64_t s = b0 + k * A.chunk_blocks;
    int64_t e = s + A.chunk_blocks;
    if (e > b1) e = b1;
    // move both ends forward to the first block of a pair
    auto advance = [&](int64_t x) -> int64_t {
      while (x < b1) {
        const int64_t y = x + lane;
        const bool first = (y < b1) ? ((A.blk[y].flags & BLK_FIRST) != 0) : true;
        const unsigned bal = __ballot_sync(0xffffffffu, first);
        if (bal) return x + __ffs(bal) - 1;
        x += 32;
      }
      return b1;
    };
    s = advance(s);
    e = (e >= b1) ? b1 : advance(e);
    if (e <= s) continue;
    const int ncols = bin * A.bucket;
    run_stream<T, K>(A, ring, lane, s, (int)(e - s), ncols);
  }
}

// ============================================================ finalize

// FP32 pass: log10 of the scaled sum, or queue the pair for the FP64 rescue.
__device__ __forceinline__ double start_mass_correction(const int32_t* __restrict__ pairs,
                                                        const int64_t* __restrict__ hoff, int64_t p, int bucket) {
  const int32_t h = pairs[2 * p + 1];
  const int n = (int)(hoff[h + 1] - hoff[h]);
  return log10((double)ncols_of(n, bucket) / (double)n);
}

__global__ void k_finalize_fp32(const float* __restrict__ s32, int64_t n_pairs, const int32_t* __restrict__ pairs,
                                const int64_t* __restrict__ hoff, int bucket, double* __restrict__ out,
                                uint8_t* __restrict__ status, int32_t* __restrict__ rescue_list,
                                int64_t* __restrict__ n_rescue, int write_status) {
  const double off = 120.0 * 0.30102999566398119521;
  for (int64_t p = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; p < n_pairs; p += (int64_t)gridDim.x * blockDim.x) {
    const float s = s32[p];
    if (!(s >= 1e-28f) || !isfinite(s)) {  // NaN-safe: also catches s < 1e-28
      const unsigned long long k = atomicAdd(reinterpret_cast<unsigned long long*>(n_rescue), 1ull);
      rescue_list[k] = (int32_t)p;
    } else {
      out[p] = log10((double)s) - off + start_mass_correction(pairs, hoff, p, bucket);
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

// item list of the rescue pass: one table item per rescued pair (its read)
__global__ void k_rescue_items(const int32_t* __restrict__ pairs, const int32_t* __restrict__ list,
                               int64_t n, int32_t* __restrict__ item_read,
                               int32_t* __restrict__ pair_item) {
  for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < n; k += (int64_t)gridDim.x * blockDim.x) {
    item_read[k] = pairs[2 * (int64_t)list[k]];
    pair_item[k] = (int32_t)k;
  }
}

// exclusive scan of bins + work items (single block; nbins <= kMaxBins)
__global__ void k_scan_bins(const unsigned long long* __restrict__ bin_blocks, int nbins, int64_t chunk,
                            unsigned long long* __restrict__ bin_start, unsigned long long* __restrict__ item_start) {
  __shared__ unsigned long long sb[1024], si[1024];
  // serial-by-tile scan: nbins is a few thousand at most
  unsigned long long carry_b = 0, carry_i = 0;
  for (int base = 0; base < nbins; base += 1024) {
    const int i = base + threadIdx.x;
    const unsigned long long vb = (i < nbins) ? bin_blocks[i] : 0ull;
    const unsigned long long vi = (i < nbins) ? (vb + chunk - 1) / chunk : 0ull;
    sb[threadIdx.x] = vb; si[threadIdx.x] = vi;
    __syncthreads();
    for (int off = 1; off < 1024; off <<= 1) {
      unsigned long long ab = 0, ai = 0;
      if (threadIdx.x >= off) { ab = sb[threadIdx.x - off]; ai = si[threadIdx.x - off]; }
      __syncthreads();
      sb[threadIdx.x] += ab; si[threadIdx.x] += ai;
      __syncthreads();
    }
    if (i < nbins) { bin_start[i] = carry_b + sb[threadIdx.x] - vb; item_start[i] = carry_i + si[threadIdx.x] - vi; }
    const unsigned long long tb = sb[1023], ti = si[1023];
    __syncthreads();
    carry_b += tb; carry_i += ti;
  }
  if (threadIdx.x == 0) { bin_start[nbins] = carry_b; item_start[nbins] = carry_i; }
}

}  // namespace phmm
