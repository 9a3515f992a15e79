// sw.cuh -- batched Smith-Waterman (HaplotypeCaller variant) for sm_100a: the paper's
// second workload (Eq. 5, L16@3413; §IV-B).
//
// PRODUCT PATH (no oracle code). Included only by phmm_lib.cu.
//
// What is computed (readings R20-R25):
//   H(i,j) = max{0, H(i-1,j-1) + s(a_i,b_j), max_k H(i-k,j) + W_k, max_l H(i,j-l) + W_l},
//   W_k = open + (k-1)*extend, s = match / mismatch on byte equality, H(0,.) = H(.,0) = 0;
//   btrack(i,j) = 0 (diagonal), +k (vertical gap), -l (horizontal gap), STOP (0 term);
//   priorities diagonal > horizontal > vertical, longest gap on ties; the end cell is the
//   maximum of row M and column N (ties: smallest |i-j|, then largest i+j, then largest
//   i); the alignment is traced back from it until STOP or row/column 0.
//
// Design:
//  * one warp per task (persistent warps, atomic task counter); lane l owns K = SW_K
//    consecutive rows of a stripe of 32*K rows (stripes run one after the other) and
//    computes column j of its rows at step t = j + l of the stripe -- the paper's
//    row-per-thread mapping (L20@3179) with K rows per thread instead of one;
//  * the max over k and l uses the paper's running maxima "along each direction"
//    (L16@3800): per row a horizontal (best, length) pair in registers, per column the
//    vertical pair flows down the rows of the lane and to the next lane by __shfl_sync
//    (the shuffle design B of the paper, Listing 2b);
//  * lane 31's last row goes to lane 0 of the next stripe through a per-warp
//    shared-memory ring indexed by column;
//  * btrack is written as int16 per cell, step-major ([stripe][step][lane][K]), so a
//    warp's stores of one step are one contiguous 32*K*2-byte segment;
//  * the traceback is a second kernel, one thread per task.
#pragma once
#include <cuda_runtime.h>

#include <cstdint>

#include "phmm_common.cuh"

namespace phmm {

constexpr int SW_K = 8;                 // rows per lane
constexpr int SW_STRIPE = 32 * SW_K;    // rows per stripe
constexpr int SW_WARPS = 4;             // warps per CTA
constexpr int kSwMaxN = 4096;           // columns (the ring and the column bases live in smem)
constexpr int16_t SW_STOP = INT16_MIN;
constexpr int32_t SW_NEG = INT32_MIN / 4;

struct SwParams {
  int32_t match, mismatch, open, extend;
};

struct SwArgs {
  const uint8_t* ref;        // rows (sequence a)
  const int64_t* ref_off;
  const uint8_t* alt;        // columns (sequence b)
  const int64_t* alt_off;
  const int32_t* tasks;      // (ref_idx, alt_idx)
  const int32_t* order;      // processing order of the tasks (largest first)
  int64_t n_tasks;
  const int64_t* bt_off;     // per task: offset of its btrack (int16 elements)
  int16_t* bt;
  int32_t* res;              // n_tasks x 6: score, end_i, end_j, start_i, start_j, n_ops
  unsigned int* counter;
  SwParams p;
  int max_n;                 // ring / column-base capacity per warp
};

// end-cell candidate order (R23): higher score, then smaller |i-j|, larger i+j, larger i
__device__ __forceinline__ bool sw_better(int32_t s, int32_t i, int32_t j, int32_t bs, int32_t bi, int32_t bj) {
  if (s != bs) return s > bs;
  const int32_t d = abs(i - j), bd = abs(bi - bj);
  if (d != bd) return d < bd;
  if (i + j != bi + bj) return i + j > bi + bj;
  return i > bi;
}

__device__ __forceinline__ int64_t sw_steps(int n) { return (int64_t)n + 31; }

__global__ void __launch_bounds__(SW_WARPS * 32) k_sw_fill(SwArgs A) {
  extern __shared__ __align__(16) unsigned char smem_sw[];
  const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
  // per warp: ring of (H, best_v, len_v) for max_n + 1 columns, then the column bases
  const size_t per_warp = (size_t)(A.max_n + 1) * 12 + (size_t)((A.max_n + 15) & ~15);
  int32_t* ringH = reinterpret_cast<int32_t*>(smem_sw + per_warp * wib);
  int32_t* ringV = ringH + (A.max_n + 1);
  int32_t* ringK = ringV + (A.max_n + 1);
  uint8_t* bcol = reinterpret_cast<uint8_t*>(ringK + (A.max_n + 1));
  const SwParams p = A.p;
  while (true) {
    unsigned int it = 0;
    if (lane == 0) it = atomicAdd(A.counter, 1u);
    it = __shfl_sync(0xffffffffu, it, 0);
    if (it >= A.n_tasks) break;
    const int64_t task = A.order ? A.order[it] : it;
    const int32_t r = A.tasks[2 * task], c = A.tasks[2 * task + 1];
    const int64_t r0 = A.ref_off[r], c0 = A.alt_off[c];
    const int M = (int)(A.ref_off[r + 1] - r0), N = (int)(A.alt_off[c + 1] - c0);
    for (int j = lane; j < N; j += 32) bcol[j] = A.alt[c0 + j];
    for (int j = lane; j <= N; j += 32) { ringH[j] = 0; ringV[j] = SW_NEG; ringK[j] = 0; }
    __syncwarp();
    int16_t* __restrict__ bt = A.bt + A.bt_off[task];
    const int nstripe = (M + SW_STRIPE - 1) / SW_STRIPE;
    const int64_t T = sw_steps(N);
    // best end-cell candidate of this lane
    int32_t bs = INT32_MIN, bi = 0, bj = 0;
    for (int q = 0; q < nstripe; ++q) {
      const int row0 = q * SW_STRIPE + lane * SW_K;  // 0-based row of the lane's u = 0
      uint8_t a[SW_K];
#pragma unroll
      for (int u = 0; u < SW_K; ++u) a[u] = (row0 + u < M) ? A.ref[r0 + row0 + u] : (uint8_t)0;
      int32_t H[SW_K], bh[SW_K], kh[SW_K];
#pragma unroll
      for (int u = 0; u < SW_K; ++u) { H[u] = 0; bh[u] = SW_NEG; kh[u] = 0; }
      const int um = (M - 1) - row0;                 // row M's index in the lane, if it owns it
      const bool has_m = (um >= 0) && (um < SW_K);
      // row above the lane's rows: (H at column j-1 [diag], H / best_v / len_v at column j)
      int32_t upH = 0, upV = SW_NEG, upK = 0, dgH = 0;
      for (int64_t t = 0; t < T; ++t) {
        const int j = (int)t - lane;  // 0-based column of this step
        const bool act = (j >= 0) && (j < N);
        if (lane == 0 && act) {  // lane 0 reads the stripe above from the ring
          dgH = ringH[j];        // H(row0-1, j-1) lives at ring index j (index 0 = column 0)
          upH = ringH[j + 1];
          upV = ringV[j + 1];
          upK = ringK[j + 1];
        }
        int32_t oH = 0, oV = SW_NEG, oK = 0;  // this step's last row, for the lane below
        uint32_t cw[SW_K / 2];                // btrack codes of the step, two int16 per word
        if (act) {
          const uint8_t b = bcol[j];
          int32_t hd = dgH, hu = upH, vu = upV, ku = upK;  // row above at j-1 (diag) and j
#pragma unroll
          for (int u = 0; u < SW_K; ++u) {
            // branch-free cell (R22): values by max, the btrack code by selects
            const int32_t diag = hd + (a[u] == b ? p.match : p.mismatch);
            const int32_t ov = hu + p.open, ev = vu + p.extend;  // vertical: open below H(i-1,j) or extend
            const bool nv = ov > ev;                            // strictly better opens (longest gap on ties)
            const int32_t bv = max(ov, ev), kv = nv ? 1 : ku + 1;
            const int32_t oh = H[u] + p.open, eh = bh[u] + p.extend;  // horizontal, along the row
            const bool nh = oh > eh;
            bh[u] = max(oh, eh);
            kh[u] = nh ? 1 : kh[u] + 1;
            const int32_t h = max(diag, max(bh[u], bv));
            const bool dwin = (diag >= bh[u]) & (diag >= bv), rwin = bh[u] >= bv;
            int32_t cd = dwin ? 0 : (rwin ? -kh[u] : kv);
            cd = (h < 0) ? (int32_t)SW_STOP : cd;
            const int32_t h0 = max(h, 0);
            hd = H[u];  // H(i, j-1): the diagonal of row u+1
            H[u] = h0;
            if (u & 1) cw[u >> 1] = __byte_perm(cw[u >> 1], (uint32_t)cd, 0x5410);
            else cw[u >> 1] = (uint32_t)cd & 0xffffu;
            hu = h0; vu = bv; ku = kv;
          }
          oH = hu; oV = vu; oK = ku;
          // btrack of this step: one 16-byte store per lane, contiguous across the warp
          reinterpret_cast<uint4*>(bt)[((int64_t)q * T + t) * 32 + lane] = make_uint4(cw[0], cw[1], cw[2], cw[3]);
          // end-cell candidates (R23): column N (all rows of the lane, once per stripe) and row M
          if (j == N - 1) {
#pragma unroll
            for (int u = 0; u < SW_K; ++u) {
              const int i = row0 + u + 1;
              if (i <= M && sw_better(H[u], i, N, bs, bi, bj)) { bs = H[u]; bi = i; bj = N; }
            }
          }
          if (has_m) {
            int32_t hm = H[0];
#pragma unroll
            for (int u = 1; u < SW_K; ++u) hm = (u == um) ? H[u] : hm;
            if (sw_better(hm, M, j + 1, bs, bi, bj)) { bs = hm; bi = M; bj = j + 1; }
          }
          if (lane == 31) { ringH[j + 1] = oH; ringV[j + 1] = oV; ringK[j + 1] = oK; }
        }
        // next step: the row above comes from lane-1's last row (one column behind); its
        // diagonal is this step's row above, or the column-0 boundary on the first column
        const int32_t sH = __shfl_up_sync(0xffffffffu, oH, 1);
        const int32_t sV = __shfl_up_sync(0xffffffffu, oV, 1);
        const int32_t sK = __shfl_up_sync(0xffffffffu, oK, 1);
        if (lane > 0) {
          dgH = ((int)t + 1 - lane <= 0) ? 0 : upH;
          upH = sH; upV = sV; upK = sK;
        }
        __syncwarp();  // ring slots read by lane 0 / written by lane 31 stay in step order
      }
      __syncwarp();  // the ring row of this stripe is complete before the next reads it
    }
    // end cell: warp reduction of the per-lane candidates
    for (int o = 16; o > 0; o >>= 1) {
      const int32_t s2 = __shfl_xor_sync(0xffffffffu, bs, o), i2 = __shfl_xor_sync(0xffffffffu, bi, o),
                    j2 = __shfl_xor_sync(0xffffffffu, bj, o);
      if (sw_better(s2, i2, j2, bs, bi, bj)) { bs = s2; bi = i2; bj = j2; }
    }
    if (lane == 0) {
      int32_t* R = A.res + 6 * task;
      R[0] = bs; R[1] = bi; R[2] = bj;
    }
    __syncwarp();
  }
}

// Traceback, one thread per task: follows btrack from the end cell; writes the CIGAR
// runs (len << 4 | op, op 0 M, 1 I, 2 D) from start to end at ops + ops_off[task].
__global__ void k_sw_traceback(SwArgs A, const int64_t* __restrict__ ops_off, uint32_t* __restrict__ ops,
                               int64_t* __restrict__ nops_out) {
  for (int64_t task = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; task < A.n_tasks;
       task += (int64_t)gridDim.x * blockDim.x) {
    const int32_t r = A.tasks[2 * task], c = A.tasks[2 * task + 1];
    const int N = (int)(A.alt_off[c + 1] - A.alt_off[c]);
    (void)r;
    const int64_t T = sw_steps(N);
    const int16_t* __restrict__ bt = A.bt + A.bt_off[task];
    int32_t* R = A.res + 6 * task;
    int i = R[1], j = R[2];
    uint32_t* out = ops + ops_off[task];
    int64_t nops = 0;
    int last = -1;
    uint32_t run = 0;
    while (i > 0 && j > 0) {
      const int row = i - 1, q = row / SW_STRIPE, l = (row % SW_STRIPE) / SW_K, u = row % SW_K;
      const int64_t t = (int64_t)(j - 1) + l;
      const int16_t cd = bt[(((int64_t)q * T + t) * 32 + l) * SW_K + u];
      if (cd == SW_STOP) break;
      int op;
      uint32_t len;
      if (cd == 0) { op = 0; len = 1; --i; --j; }
      else if (cd < 0) { op = 1; len = (uint32_t)(-cd); j += cd; }
      else { op = 2; len = (uint32_t)cd; i -= cd; }
      if (op == last) run += len;
      else {
        if (last >= 0) out[nops++] = (run << 4) | (uint32_t)last;
        last = op;
        run = len;
      }
    }
    if (last >= 0) out[nops++] = (run << 4) | (uint32_t)last;
    for (int64_t x = 0, y = nops - 1; x < y; ++x, --y) { const uint32_t tmp = out[x]; out[x] = out[y]; out[y] = tmp; }
    R[3] = i + 1;
    R[4] = j + 1;
    R[5] = (int32_t)nops;
    nops_out[task] = nops;
  }
  if (blockIdx.x == 0 && threadIdx.x == 0) nops_out[A.n_tasks] = 0;
}

// Pack the CIGAR runs of all tasks back to back in task order (one warp per task).
__global__ void k_sw_compact(const uint32_t* __restrict__ ops_tmp, const int64_t* __restrict__ cap_off,
                             const int64_t* __restrict__ packed_off, int64_t n_tasks, uint32_t* __restrict__ ops) {
  const int lane = threadIdx.x & 31;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t t = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5; t < n_tasks; t += nw) {
    const int64_t n = packed_off[t + 1] - packed_off[t];
    for (int64_t k = lane; k < n; k += 32) ops[packed_off[t] + k] = ops_tmp[cap_off[t] + k];
  }
}

// Validation + per-task sizes: btrack elements (stripes * steps * 32 * K) and CIGAR
// capacity (M + N). Errors -> err bits.
__global__ void k_sw_sizes(const int32_t* __restrict__ tasks, int64_t n_tasks, const int64_t* __restrict__ ref_off,
                           int64_t n_refs, const int64_t* __restrict__ alt_off, int64_t n_alts,
                           int64_t* __restrict__ bt_size, int64_t* __restrict__ ops_cap, int64_t* __restrict__ cells,
                           int* __restrict__ max_n, uint32_t* err) {
  uint32_t e = 0;
  int64_t my_cells = 0;
  int my_max = 0;
  for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < n_tasks; t += (int64_t)gridDim.x * blockDim.x) {
    const int32_t r = tasks[2 * t], c = tasks[2 * t + 1];
    int64_t bs = 0, oc = 0;
    if (r < 0 || r >= n_refs || c < 0 || c >= n_alts) {
      e |= ERR_INDEX;
    } else {
      const int64_t M = ref_off[r + 1] - ref_off[r], N = alt_off[c + 1] - alt_off[c];
      if (M < 1 || N < 1) e |= ERR_EMPTY;
      else if (N > kSwMaxN || M > 32767) e |= ERR_ARG;  // gap lengths are stored as int16
      else {
        bs = (int64_t)((M + SW_STRIPE - 1) / SW_STRIPE) * (N + 31) * 32 * SW_K;
        oc = M + N;
        my_cells += M * N;
        my_max = max(my_max, (int)N);
      }
    }
    bt_size[t] = bs;
    ops_cap[t] = oc;
  }
  if (blockIdx.x == 0 && threadIdx.x == 0) { bt_size[n_tasks] = 0; ops_cap[n_tasks] = 0; }
  for (int o = 16; o > 0; o >>= 1) {
    e |= __shfl_xor_sync(0xffffffffu, e, o);
    my_cells += __shfl_xor_sync(0xffffffffu, my_cells, o);
    my_max = max(my_max, __shfl_xor_sync(0xffffffffu, my_max, o));
  }
  if ((threadIdx.x & 31) == 0) {
    if (e) atomicOr(err, e);
    if (my_cells) atomicAdd(reinterpret_cast<unsigned long long*>(cells), (unsigned long long)my_cells);
    if (my_max) atomicMax(max_n, my_max);
  }
}

// processing order: largest tasks (M*N) first, for the persistent warps' load balance
__global__ void k_sw_keys(const int32_t* __restrict__ tasks, int64_t n_tasks, const int64_t* __restrict__ ref_off,
                          const int64_t* __restrict__ alt_off, uint64_t* __restrict__ keys, int32_t* __restrict__ vals) {
  for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < n_tasks; t += (int64_t)gridDim.x * blockDim.x) {
    const int32_t r = tasks[2 * t], c = tasks[2 * t + 1];
    const uint64_t cells = (uint64_t)(ref_off[r + 1] - ref_off[r]) * (uint64_t)(alt_off[c + 1] - alt_off[c]);
    keys[t] = ~cells;  // ascending sort of ~cells = descending cells
    vals[t] = (int32_t)t;
  }
}

}  // namespace phmm
