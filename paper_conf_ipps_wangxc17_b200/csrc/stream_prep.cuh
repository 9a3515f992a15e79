// stream_prep.cuh -- prep kernels of a wavefront pass (FP32 main pass or FP64 pass):
// haplotype code regions, per-read coefficient tables, stable length
// binning and block descriptors (§8a-3). Included only by phmm_lib.cu.
#pragma once
#include "wavefront.cuh"

namespace phmm {

// ---------------------------------------------------------------- haplotype codes
// Code region of one haplotype: 4 copies of wf_hc_copy_len(ncols) bytes; in copy k
// column c sits at byte WF_HC_FRONT + k + c (so a lane picks the copy that makes its
// code words 4-aligned). Byte = code * WF_CB with code A=0 C=1 G=2 T=3 N=4 PAD=5:
// columns c < N carry the haplotype, c == N carries 'N' (matches every row), every
// other byte is PAD (prior 0). BlkDesc.hap_off = region start + WF_HC_FRONT.
// (Moved into bits 8..15 by the kernel, the byte becomes the offset of the code's rows
// in a lane's shared-memory prior table.)
__host__ __device__ inline int64_t wf_hc_region(int n, int bucket) {
  return 4 * (int64_t)wf_hc_copy_len(ncols_of(n, bucket));
}

// One warp per haplotype: its code bytes (copy 0, PAD front and tail) are built once in
// shared memory, then the 4 shifted copies are written as coalesced 32-bit words
// (funnel shifts of two aligned words).
constexpr int kHcThreads = 256;
constexpr int kHcBuf = 4352;  // >= wf_hc_copy_len(ncols_of(kMaxHapLen, 64)) + 4
__global__ void __launch_bounds__(kHcThreads) k_hap_codes_wf(const uint8_t* __restrict__ hap,
                                                             const int64_t* __restrict__ hoff, int64_t n_haps,
                                                             const int64_t* __restrict__ hc_off, int bucket,
                                                             uint8_t* __restrict__ codes) {
  __shared__ __align__(16) uint8_t sbuf[kHcThreads / 32][kHcBuf];
  const int lane = threadIdx.x & 31;
  uint8_t* buf = sbuf[threadIdx.x >> 5];
  const uint32_t* buf32 = reinterpret_cast<const uint32_t*>(buf);
  const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  constexpr uint32_t kPadW = (uint32_t)(WF_PAD * WF_CB) * 0x01010101u;
  for (int64_t h = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5; h < n_haps; h += nwarps) {
    const int64_t h0 = hoff[h];
    const int n = (int)(hoff[h + 1] - h0);
    if (n < 1 || n > kMaxHapLen) continue;
    const int len = wf_hc_copy_len(ncols_of(n, bucket));  // multiple of 4, region start 4-aligned
    __syncwarp();
    // byte b of copy 0 = column b - WF_HC_FRONT; 4 bytes per lane per trip, their loads
    // issued before any is used (the loop is bound by load latency, one haplotype per warp)
    for (int b0 = 0; b0 < len + 4; b0 += 128) {
      uint8_t x[4];
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        const int c = b0 + 32 * j + lane - (int)WF_HC_FRONT;
        x[j] = (c >= 0 && c < n) ? hap[h0 + c] : (uint8_t)0;
      }
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        const int b = b0 + 32 * j + lane;
        const int c = b - (int)WF_HC_FRONT;
        if (b >= len + 4) break;
        uint32_t v = WF_PAD;
        if (c >= 0 && c < n) {
          switch (x[j]) {
            case 'A': v = 0; break;
            case 'C': v = 1; break;
            case 'G': v = 2; break;
            case 'T': v = 3; break;
            default: v = 4; break;  // 'N' (invalid bytes were rejected by validation)
          }
        } else if (c == n) {
          v = 4;
        }
        buf[b] = (uint8_t)(v * WF_CB);
      }
    }
    __syncwarp();
    uint32_t* dst = reinterpret_cast<uint32_t*>(codes + hc_off[h]);
    const int wpc = len >> 2;  // words per copy
    // copy k, word w = bytes [4w - k, 4w - k + 4) of copy 0 (PAD before byte 0)
    for (int k = 0; k < 4; ++k)
      for (int w = lane; w < wpc; w += 32) {
        const uint32_t lo = w > 0 ? buf32[w - 1] : kPadW, hi = buf32[w];
        dst[k * wpc + w] = __funnelshift_rc(lo, hi, 8 * (4 - k));
      }
  }
}

__global__ void k_hap_ncols(const int64_t* __restrict__ hoff, int64_t n_haps, int bucket, int64_t* __restrict__ nc) {
  for (int64_t h = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; h < n_haps; h += (int64_t)gridDim.x * blockDim.x) {
    const int64_t n = hoff[h + 1] - hoff[h];
    nc[h] = (n >= 1 && n <= kMaxHapLen) ? wf_hc_region((int)n, bucket) : 0;
  }
  if (blockIdx.x == 0 && threadIdx.x == 0) nc[n_haps] = 0;
}

// ---------------------------------------------------------------- coefficient tables
// Per table item (a read, or a rescued pair's read): nb = ceil((m+3)/K) blocks of K rows
//   [f >= 1 Z rows][R][read rows 1..m][S]          (phmm_common.cuh)
// One warp per item, lanes over its padded rows. The coefficients of the kernel's
// 5-op form of Eq. 6 (wavefront.cuh) are computed from a 128-entry
// Phred table (10^(-q/10), rounded once to T); each lane computes its row's storage
// scales and takes the row above's by __shfl_up_sync. Row i stores
//   M^ = a_i M, I^ = b_i I, D^ = d_i D,   a_i = k_i zeta_i, d_i = k_i, b_i = a_{i-1}/delta_i,
//   k_i = min(1, delta_{i+1}/zeta_i) (k_m = 1),   R row: a = delta_1, b = d = 1,
// so that no stored value exceeds its unscaled one (b_i <= 1, k_i <= 1) and
//   D^ = M^(left) + mu D^(left),  I^ = M^(up) + ep' I^(up),
//   M^ = T[code] * (M^(diag) + u I^(diag) + w D^(diag)).
constexpr int kTabThreads = 256;
// a / b in the table's precision: FP32 tables use the 2-ulp hardware division (7 divisions per
// row dominate the kernel; 2 ulp per coefficient is far inside the FP32 pass's 1e-3 log10
// tolerance), FP64 tables the correctly rounded one
__device__ __forceinline__ float tdiv(float a, float b) { return __fdividef(a, b); }
__device__ __forceinline__ double tdiv(double a, double b) { return a / b; }

template <typename T>
__global__ void __launch_bounds__(kTabThreads) k_build_table_wf(
    const int32_t* __restrict__ item_read, int64_t n_items, const int64_t* __restrict__ item_tab_off,
    const int64_t* __restrict__ roff, const uint8_t* __restrict__ rb, const uint8_t* __restrict__ q,
    const uint8_t* __restrict__ qi, const uint8_t* __restrict__ qd, const uint8_t* __restrict__ qg,
    TBlock<T>* __restrict__ tab) {
  // computed in the table's precision T: a few roundings per coefficient (FP32: well
  // inside the 1e-3 log10 tolerance; FP64: ~1e-16 per row)
  constexpr int K = WfT<T>::K;
  __shared__ T err[128];
  for (int i = threadIdx.x; i < 128; i += blockDim.x) err[i] = qual_err<T>((uint32_t)i);
  __syncthreads();
  const int lane = threadIdx.x & 31;
  const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t it = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5; it < n_items; it += nwarps) {
    const int64_t r = item_read ? item_read[it] : it;
    if (r < 0) continue;  // unused item (rescue pass, past the distinct reads)
    const int64_t r0 = roff[r];
    const int64_t m64 = roff[r + 1] - r0;
    // reads longer than kMaxReadLen bases have a 1-block reservation (k_item_nblocks) and no table:
    // a pair that uses one is rejected by k_pair_bins, an unused one must not be written
    if (m64 < 1 || m64 > kMaxReadLen) continue;
    const int m = (int)m64;
    const int nb = nblocks_of<K>(m);
    const int f = nb * K - (m + 2);  // >= 1 Z rows
    TBlock<T>* __restrict__ Tb = tab + item_tab_off[it];
    const T de1 = err[qi[r0] & 127];
    // storage scales (a, b, d) of the row above the lane's row, carried across iterations
    T ca = 1, cb = 1, cd = 1;
    for (int base = 0; base < nb * K; base += 32) {  // warp-uniform trip count
      const int row = base + lane;
      const int i = row - f;  // < 0 Z, 0 R, 1..m read rows, m+1 S
      const bool real = (i >= 1) && (i <= m);
      const int64_t x = r0 + (real ? i - 1 : 0);
      T ei = 0, ed = 0, eg = 0, eb = 0;
      uint8_t base_c = 'N';
      if (real) {
        ei = err[qi[x] & 127]; ed = err[qd[x] & 127]; eg = err[qg[x] & 127]; eb = err[q[x] & 127];
        base_c = rb[x];
      }
      // own a = k zeta, d = k with k = min(1, delta_{i+1}/zeta_i) (k_m = 1); R row: a = delta_1
      T a = 1, d = 1;
      if (i == 0) {
        a = de1;
      } else if (real) {
        const T k = (i < m) ? fmin((T)1, tdiv(err[qi[x + 1] & 127], ed)) : (T)1;
        a = k * ed;
        d = k;
      }
      T ap = __shfl_up_sync(0xffffffffu, a, 1);
      if (lane == 0) ap = ca;
      // b = a_{i-1} / delta_i (b_1 = 1)
      const T b = (real && i >= 2) ? tdiv(ap, ei) : (T)1;
      T bp = __shfl_up_sync(0xffffffffu, b, 1), dp = __shfl_up_sync(0xffffffffu, d, 1);
      if (lane == 0) { bp = cb; dp = cd; }
      ca = __shfl_sync(0xffffffffu, a, 31);
      cb = __shfl_sync(0xffffffffu, b, 31);
      cd = __shfl_sync(0xffffffffu, d, 31);
      if (row >= nb * K) continue;
      T uu = 0, ww = 0, ep = 0, mu = 0;
      T p5[5] = {0, 0, 0, 0, 0};
      if (i < 0) {
        // Z row: all zero (absorbs whatever finite values are above it)
      } else if (i == 0) {  // R row: D = d0 on every column
        mu = 1;
      } else if (real) {
        const T al = (T)1 - fmin(ei + ed, (T)1);  // > 0.0065 after validation (R16)
        const T be = (T)1 - eg;
        const T g = tdiv(be * ap, al);
        uu = tdiv(g, bp);
        ww = tdiv(g, dp);
        ep = tdiv(eg * b, bp);
        mu = eg;
        const T t = tdiv(a * al, ap);
        const T pm = t * ((T)1 - eb), px = t * tdiv(eb, (T)3);
        p5[0] = (base_c == 'A' || base_c == 'N') ? pm : px;
        p5[1] = (base_c == 'C' || base_c == 'N') ? pm : px;
        p5[2] = (base_c == 'G' || base_c == 'N') ? pm : px;
        p5[3] = (base_c == 'T' || base_c == 'N') ? pm : px;
        p5[4] = pm;  // haplotype 'N' matches everything
      } else {  // S: M^ = (M + I)(m, j-1), D^ = running sum (the L20@2262 termination)
        uu = tdiv(ap, bp);
        mu = 1;
        p5[0] = p5[1] = p5[2] = p5[3] = p5[4] = tdiv((T)1, ap);
      }
      TBlock<T>& B = Tb[row / K];
      const int t = row % K;
      B.coef[0][t] = uu; B.coef[1][t] = ww; B.coef[2][t] = ep; B.coef[3][t] = mu;
#pragma unroll
      for (int k = 0; k < 5; ++k) B.prior[k][t] = p5[k];
    }
  }
}

// ---------------------------------------------------------------- stable binning
// Pairs are radix-sorted by bin (stable: read-major input order survives inside a bin,
// the pairs of one read stay adjacent and its table is reused from L2), then each
// sorted pair gets a contiguous block range from an exclusive scan. Deterministic.
// sort keys: 2 * bin + (pair of <= 64 blocks): inside a bin the pass-padded pairs come first
// (padded_nb), so every one of them starts at a multiple of 64 blocks from any stream start
__global__ void k_iota_keys(const int32_t* __restrict__ pair_bin, const int32_t* __restrict__ pair_nb, int64_t n,
                            uint32_t* __restrict__ keys, int32_t* __restrict__ vals) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    keys[i] = 2u * (uint32_t)pair_bin[i] + (pair_nb[i] < kRescaleMinBlocks ? 1u : 0u);
    vals[i] = (int32_t)i;
  }
}

__global__ void k_sorted_nb(const int32_t* __restrict__ sorted_idx, const int32_t* __restrict__ pair_nb, int64_t n,
                            int64_t* __restrict__ nb_sorted) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    nb_sorted[i] = pair_nb[sorted_idx[i]];
  if (blockIdx.x == 0 && threadIdx.x == 0) nb_sorted[n] = 0;
}

// Block descriptors: one warp per 32 sorted entries, whose blocks are one contiguous range
// (blk_off is an exclusive scan in sorted order); the lanes write that range as consecutive
// 16-byte descriptors (coalesced), each finding its entry by a binary search over the 32
// entries' first blocks held in the lanes. Entry k of the pass is pair list[k] (or k when
// list == nullptr); its table item is pair_item[k] (or its read), its output slot k (list) or
// the pair id.
template <int K>
__global__ void k_alloc_blocks_wf(const int32_t* __restrict__ pairs, const int32_t* __restrict__ list,
                                  const int32_t* __restrict__ pair_item, const int32_t* __restrict__ sorted_idx,
                                  int64_t n, const int32_t* __restrict__ pair_nb, const int64_t* __restrict__ blk_off,
                                  const int64_t* __restrict__ roff, const int64_t* __restrict__ hoff,
                                  const int64_t* __restrict__ hc_off, const int64_t* __restrict__ item_tab_off,
                                  BlkDesc* __restrict__ blk) {
  const int lane = threadIdx.x & 31;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t base = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) & ~31ll; base < n; base += stride) {
    const int64_t i = base + lane;
    int nb = 0, nbr = 0, f = 0;
    int64_t g0 = INT64_MAX, slot = 0;
    uint32_t tab0 = 0, hap = 0;
    if (i < n) {
      const int64_t k = sorted_idx[i];
      const int64_t p = list ? list[k] : k;
      nb = pair_nb[k];  // blocks of the pair incl. fillers (padded_nb)
      const int32_t r = pairs[2 * p], h = pairs[2 * p + 1];
      const int m = (int)(roff[r + 1] - roff[r]);
      nbr = nblocks_of<K>(m);  // blocks with rows
      f = nbr * K - (m + 2);   // R row index within the pair's rows (f >= 1 Z rows before it)
      g0 = blk_off[i];
      tab0 = (uint32_t)item_tab_off[pair_item ? pair_item[k] : r];
      hap = (uint32_t)(hc_off[h] + WF_HC_FRONT);
      slot = list ? k : p;
    }
    const int cnt = (int)min((int64_t)32, n - base);
    const int64_t first = __shfl_sync(0xffffffffu, g0, 0);
    const int64_t last = __shfl_sync(0xffffffffu, g0, cnt - 1) + __shfl_sync(0xffffffffu, nb, cnt - 1);
    for (int64_t pos = first + lane; pos - lane < last; pos += 32) {
      // owner entry: the last of the (ascending) first blocks <= pos
      int e = 0;
#pragma unroll
      for (int st = 16; st > 0; st >>= 1) {
        const int cand = e + st;
        const int64_t gc = __shfl_sync(0xffffffffu, g0, cand & 31);
        if (cand < cnt && gc <= pos) e = cand;
      }
      const int64_t g0e = __shfl_sync(0xffffffffu, g0, e);
      const int nbe = __shfl_sync(0xffffffffu, nbr, e);
      const int fe = __shfl_sync(0xffffffffu, f, e);
      const int64_t slote = __shfl_sync(0xffffffffu, slot, e);
      const uint32_t tabe = __shfl_sync(0xffffffffu, tab0, e);
      const uint32_t hape = __shfl_sync(0xffffffffu, hap, e);
      if (pos < last) {
        const int j = (int)(pos - g0e);
        BlkDesc d;
        d.tab_blk = tabe + j;
        d.hap_off = hape;
        d.out_idx = (int32_t)slote;
        d.pad = 0;
        const int rrow = (fe / K == j) ? (fe % K) : WF_RROW_NONE;
        d.flags = (uint16_t)((j == nbe - 1 ? BLK_LAST : 0) | (j == 0 ? BLK_FIRST : 0) |
                             (nbe >= kRescaleMinBlocks ? BLK_RESC : 0) | (j >= nbe ? BLK_FILLER : 0) |
                             (rrow << WF_RROW_SHIFT));
        if (j >= nbe) d.out_idx = -1;
        blk[pos] = d;
      }
    }
  }
}

}  // namespace phmm
