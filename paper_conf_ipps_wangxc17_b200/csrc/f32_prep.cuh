// f32_prep.cuh -- prep kernels of the FP32 pass (haplotype code slots, per-read
// tables, block descriptors). Included only by phmm_lib.cu.
#pragma once
#include "wavefront_f32.cuh"

namespace phmm {

// ---------------------------------------------------------------- prep for the FP32 kernel

// Code slot of one haplotype: F32_HC_FRONT PAD codes, then columns
// c < N: base code 0..4; c == N: 4 ('N', matches all); c > N: PAD, up to the
// last column a lane can reach before its next switch event (its pass P).
// BlkDesc.hap_off points at column 0.
__host__ __device__ inline int f32_hc_slot(int n, int bucket) {
  const int nc = ncols_of(n, bucket);
  const int p = (nc + F32_G > F32_MIN_P) ? nc + F32_G : F32_MIN_P;
  return (int)F32_HC_FRONT + p + 8;
}
__global__ void k_hap_codes_f32(const uint8_t* __restrict__ hap, const int64_t* __restrict__ hoff, int64_t n_haps,
                                const int64_t* __restrict__ hc_off, int bucket, uint8_t* __restrict__ codes) {
  const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t h = warp; h < n_haps; h += nwarps) {
    const int64_t h0 = hoff[h];
    const int n = (int)(hoff[h + 1] - h0);
    if (n < 1 || n > kMaxHapLen) continue;
    const int slot = f32_hc_slot(n, bucket);
    uint8_t* dst = codes + hc_off[h];
    for (int c = lane - (int)F32_HC_FRONT; c < slot - (int)F32_HC_FRONT; c += 32) {
      uint8_t v = F32_PAD;
      if (c >= 0 && c < n) {
        switch (hap[h0 + c]) {
          case 'A': v = 0; break;
          case 'C': v = 1; break;
          case 'G': v = 2; break;
          case 'T': v = 3; break;
          default: v = 4; break;  // 'N' (invalid bytes were rejected by validation)
        }
      } else if (c == n) {
        v = 4;
      }
      dst[c + F32_HC_FRONT] = v;
    }
  }
}

__global__ void k_hap_ncols(const int64_t* __restrict__ hoff, int64_t n_haps, int bucket, int64_t* __restrict__ nc) {
  for (int64_t h = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; h < n_haps; h += (int64_t)gridDim.x * blockDim.x) {
    const int64_t n = hoff[h + 1] - hoff[h];
    nc[h] = (n >= 1 && n <= kMaxHapLen) ? f32_hc_slot((int)n, bucket) : 0;
  }
  if (blockIdx.x == 0 && threadIdx.x == 0) nc[n_haps] = 0;
}

// per-read FP32 tables: one thread per padded row (same row layout as k_build_table)
__global__ void k_build_table_f32(int64_t n_reads, const int64_t* __restrict__ item_tab_off,
                                  const int64_t* __restrict__ total_tab_blocks_dev, const int64_t* __restrict__ roff,
                                  const uint8_t* __restrict__ rb, const uint8_t* __restrict__ q,
                                  const uint8_t* __restrict__ qi, const uint8_t* __restrict__ qd,
                                  const uint8_t* __restrict__ qg, F32Block* __restrict__ tab) {
  constexpr int K = F32_K;
  const int64_t total_rows = (*total_tab_blocks_dev) * K;
  for (int64_t g = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; g < total_rows; g += (int64_t)gridDim.x * blockDim.x) {
    const int64_t b = g / K;
    const int t = (int)(g % K);
    int64_t lo = 0, hi = n_reads - 1;
    while (lo < hi) {
      const int64_t mid = (lo + hi + 1) >> 1;
      if (item_tab_off[mid] <= b) lo = mid; else hi = mid - 1;
    }
    const int64_t r = lo;
    const int64_t r0 = roff[r];
    const int m = (int)(roff[r + 1] - r0);
    const int nb = nblocks_of<K>(m);
    const int f = nb * K - (m + 3);
    const int row = (int)(b - item_tab_off[r]) * K + t;
    float al = 0, be = 0, de = 0, ep = 0, ze = 0, mu = 0;
    float pr[5] = {0, 0, 0, 0, 0};
    if (row < f) {
      // Z row: all zero
    } else if (row == f) {  // R row: D = d0 on every column
      mu = 1;
    } else if (row <= f + m) {
      const int64_t x = r0 + (row - f - 1);
      const float ei = qual_err<float>(qi[x]), ed = qual_err<float>(qd[x]), eg = qual_err<float>(qg[x]),
                  eb = qual_err<float>(q[x]);
      const float sum = ei + ed;
      al = 1.f - (sum < 1.f ? sum : 1.f);
      be = 1.f - eg;
      de = ei;
      ep = eg;
      ze = ed;
      mu = eg;
      const float pm = 1.f - eb, px = eb / 3.f;
      const uint8_t base = rb[x];
      const uint8_t codes[4] = {'A', 'C', 'G', 'T'};
#pragma unroll
      for (int k = 0; k < 4; ++k) pr[k] = (base == codes[k] || base == 'N') ? pm : px;
      pr[4] = pm;  // haplotype 'N' matches everything
    } else if (row == f + m + 1) {  // S1: I = M(m,j) + I(m,j)
      de = 1; ep = 1; mu = 1;
    } else {  // S2: M = I_S1(j-1), D = running sum
      be = 1; ze = 1; mu = 1;
      pr[0] = pr[1] = pr[2] = pr[3] = pr[4] = 1;
    }
    F32Block& B = tab[b];
    B.coef[0][t] = al; B.coef[1][t] = be; B.coef[2][t] = de;
    B.coef[3][t] = ep; B.coef[4][t] = ze; B.coef[5][t] = mu;
#pragma unroll
    for (int k = 0; k < 5; ++k) B.prior[k][t] = pr[k];
  }
}

// block descriptors for the FP32 pass (R row index in the flags, padded haplotype code offsets)
__global__ void k_alloc_blocks_f32(const int32_t* __restrict__ pairs, int64_t n_pairs,
                                   const int32_t* __restrict__ pair_bin, const int32_t* __restrict__ pair_nb,
                                   const unsigned long long* __restrict__ bin_start,
                                   unsigned long long* __restrict__ bin_cursor, const int64_t* __restrict__ roff,
                                   const int64_t* __restrict__ hoff, const int64_t* __restrict__ hc_off,
                                   const int64_t* __restrict__ item_tab_off, BlkDesc* __restrict__ blk) {
  constexpr int K = F32_K;
  for (int64_t p = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; p < n_pairs; p += (int64_t)gridDim.x * blockDim.x) {
    const int bin = pair_bin[p];
    if (bin < 0) continue;
    const int nb = pair_nb[p];
    const int32_t r = pairs[2 * p], h = pairs[2 * p + 1];
    const int m = (int)(roff[r + 1] - roff[r]);
    const int f = nb * K - (m + 3);  // R row index within the pair's rows
    const unsigned long long g0 = bin_start[bin] + atomicAdd(&bin_cursor[bin], (unsigned long long)nb);
    const uint32_t tab0 = (uint32_t)item_tab_off[r];
    const int nh = (int)(hoff[h + 1] - hoff[h]);
    for (int j = 0; j < nb; ++j) {
      BlkDesc d;
      d.tab_blk = tab0 + j;
      d.hap_off = (uint32_t)(hc_off[h] + F32_HC_FRONT);
      d.out_idx = (int32_t)p;
      d.n = (uint16_t)nh;
      const int rrow = (f / K == j) ? (f % K) : F32_RROW_NONE;
      d.flags = (uint16_t)((j == nb - 1 ? BLK_LAST : 0) | (j == 0 ? BLK_FIRST : 0) | (rrow << F32_RROW_SHIFT));
      blk[g0 + j] = d;
    }
  }
}

}  // namespace phmm
