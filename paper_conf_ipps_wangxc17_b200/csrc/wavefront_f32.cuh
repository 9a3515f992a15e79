// wavefront_f32.cuh -- the FP32 PairHMM wavefront kernel for sm_100a (the hot loop).
//
// PRODUCT PATH. Computes Eq. 6 of PAPER.md (L18@541) over "tall streams" of
// 4-row blocks (see phmm_device.cuh for the Z/R/S1/S2 pad-row layout that
// makes a pair's termination sum (L20@2262) fall out of the recurrence).
//
// The paper's PH2 kernel (L20@3509, Fig. 8) gives one warp one pair and lets
// each thread own consecutive rows, passing the row-above values by shuffle
// (its Design B, Listing 2b, L20@44). This kernel keeps the row ownership and
// the shuffle, and changes the rest for Blackwell:
//  * a warp streams through a long sequence of blocks of one length bin; the
//    warp has 64 VIRTUAL lanes v = 32h + l (h = 0: half A, h = 1: half B of
//    lane l), each owning one 4-row block per pass (blocks 64q + v);
//    virtual lane v processes column x of its block at step T_q + 1 + v + x.
//  * the two halves live in the two 32-bit halves of 64-bit register pairs, so
//    every FP op of Eq. 6 is one packed FFMA2/FMUL2/FADD2 for two independent
//    cells, including the eps*I + delta*M chain down the column (4 deep).
//    The FMA pipe still executes 8 FP32 ops per cell (the roofline).
//  * the emission prior P(i,j): each half keeps prior[code][row] in shared
//    memory (code = haplotype base A,C,G,T,N or 5 = PAD); 1 LDS.128 per half
//    per step replaces the per-cell compare/select.
//  * no per-lane "is this column real" branch: columns outside a block read
//    the PAD code (prior 0), and with the pad-row coefficients this makes an
//    idle virtual lane compute EXACTLY the boundary column (M = I = 0,
//    D = D(i,0)) before its block and freeze the S2 running sum after it
//    (DESIGN.md §4.4 proves both by induction down the lanes).
//  * virtual lanes switch blocks in groups of G = 8 (8 warp-divergent switch
//    events per pass instead of 64); a pass is P = max(ncols + G, 72) steps.
//  * row-above exchange: half A of lane l-1 -> half A of lane l and half B of
//    lane l-1 -> half B of lane l by __shfl_sync; lane 31 substitutes its half
//    A (virtual 31 -> virtual 32 = lane 0 half B) and the ring value
//    (virtual 63 of the previous pass -> virtual 0) into what it sends; the
//    ring is a per-warp shared-memory array indexed by column + 1 (slot 0 =
//    the boundary column), written by lane 31's half B.
#pragma once
#include <cuda_runtime.h>

#include <cstdint>

#include "phmm_common.cuh"

namespace phmm {

#if defined(PHMM_DBG_TRACE) && defined(PHMM_DEFINE_WF32)
// debug builds only: per-step row-3 state of the warp that runs work item 0
__device__ float g_trace[4096 * 32 * 2 * 3];
__device__ int g_trace_steps;
#endif

constexpr int F32_K = 4;      // rows per virtual lane (per half)
constexpr int F32_G = 8;      // virtual lanes per switch group
constexpr int F32_NCODE = 6;  // A C G T N PAD
constexpr int F32_PAD = 5;
constexpr int F32_WARPS = 4;   // warps per CTA
constexpr int F32_MIN_P = 72;  // ring delay: virtual lane 63 -> 0 needs P >= 72
constexpr int64_t F32_HC_FRONT = 16;  // PAD codes before every haplotype's code array

// per-block coefficient table: 6 transition fields + 5 prior codes, 4 rows each
struct alignas(16) F32Block {
  float coef[6][4];   // alpha, beta, delta, eps, zeta, mu
  float prior[5][4];  // P(row, code) for code = A, C, G, T, N
};
static_assert(sizeof(F32Block) == 176, "F32Block layout");

// BlkDesc.flags for the FP32 kernel: bit0 last, bit1 first, bits 8-11 R row (15 = none)
constexpr uint16_t F32_RROW_SHIFT = 8;
constexpr uint16_t F32_RROW_NONE = 15;

struct F32Args {
  const BlkDesc* blk;
  const F32Block* tab;
  const uint8_t* hcodes;                 // padded per-haplotype code arrays
  uint32_t pad_idx;                      // index of an all-PAD region (idle lanes)
  const unsigned long long* bin_start;   // [nbins+1]
  const unsigned long long* item_start;  // [nbins+1]
  int nbins;
  int bucket;
  int64_t chunk_blocks;
  unsigned int* item_counter;
  float* out;
  int ring_len;  // >= P + 4
};

// 64-bit register pair holding (half A, half B) FP32 values; all hot-loop math is
// packed f32x2 PTX so that ptxas keeps every pair in an aligned register pair.
typedef unsigned long long v2;
__device__ __forceinline__ v2 pk(float lo, float hi) {
  v2 r;
  asm("mov.b64 %0, {%1, %2};" : "=l"(r) : "f"(lo), "f"(hi));
  return r;
}
__device__ __forceinline__ float lo(v2 v) {
  float a, b;
  asm("mov.b64 {%0, %1}, %2;" : "=f"(a), "=f"(b) : "l"(v));
  return a;
}
__device__ __forceinline__ float hi(v2 v) {
  float a, b;
  asm("mov.b64 {%0, %1}, %2;" : "=f"(a), "=f"(b) : "l"(v));
  return b;
}
__device__ __forceinline__ v2 fma2(v2 a, v2 b, v2 c) {
  v2 d;
  asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(d) : "l"(a), "l"(b), "l"(c));
  return d;
}
__device__ __forceinline__ v2 mul2(v2 a, v2 b) {
  v2 d;
  asm("mul.rn.f32x2 %0, %1, %2;" : "=l"(d) : "l"(a), "l"(b));
  return d;
}
__device__ __forceinline__ v2 add2(v2 a, v2 b) {
  v2 d;
  asm("add.rn.f32x2 %0, %1, %2;" : "=l"(d) : "l"(a), "l"(b));
  return d;
}
template <int H>
__device__ __forceinline__ v2 set_half(v2 r, float v) {
  return H == 0 ? pk(v, hi(r)) : pk(lo(r), v);
}

// lane state: lo = half A (virtual lane l), hi = half B (virtual lane l + 32); index = row 0..3
struct F32Lane {
  v2 al[4], be[4], de[4], ep[4], ze[4], mu[4];
  v2 M[4], I[4], D[4];
};

// One column for both halves, in place. dg* = row above at column x-1, up* = row above at column x.
__device__ __forceinline__ void f32_column(F32Lane& L, const float4 pA, const float4 pB, const v2 dgM,
                                           const v2 dgI, const v2 dgD, const v2 upM, const v2 upI) {
  const float prA[4] = {pA.x, pA.y, pA.z, pA.w};
  const float prB[4] = {pB.x, pB.y, pB.z, pB.w};
  // M and D: rows descending so that row u-1's old values are intact when row u reads them
#pragma unroll
  for (int u = 3; u >= 0; --u) {
    const v2 md = (u == 0) ? dgM : L.M[u - 1];
    const v2 id = (u == 0) ? dgI : L.I[u - 1];
    const v2 dd = (u == 0) ? dgD : L.D[u - 1];
    // D(i,j) = zeta*M(i,j-1) + mu*D(i,j-1)
    L.D[u] = fma2(L.ze[u], L.M[u], mul2(L.mu[u], L.D[u]));
    // M(i,j) = P(i,j) * (alpha*M(i-1,j-1) + beta*(I(i-1,j-1) + D(i-1,j-1)))
    const v2 x = fma2(L.al[u], md, mul2(L.be[u], add2(id, dd)));
    L.M[u] = pk(prA[u] * lo(x), prB[u] * hi(x));
  }
  // I(i,j) = delta*M(i-1,j) + eps*I(i-1,j), rows ascending (a 4-deep FFMA2 chain)
  v2 m_up = upM, i_up = upI;
#pragma unroll
  for (int u = 0; u < 4; ++u) {
    const v2 ni = fma2(L.ep[u], i_up, mul2(L.de[u], m_up));
    m_up = L.M[u];
    i_up = ni;
    L.I[u] = ni;
  }
}

// Load a block (or nothing) into half H of a lane.
template <int H>
__device__ __forceinline__ void f32_load(const F32Args& A, F32Lane& L, float4* __restrict__ my_tab, bool have,
                                         const BlkDesc& d, float d0, uint32_t& idx, int& out_idx, int gi) {
  if (have) {
    const float4* __restrict__ s4 = reinterpret_cast<const float4*>(A.tab + d.tab_blk);
    float4 cw[6];
#pragma unroll
    for (int k = 0; k < 6; ++k) cw[k] = __ldg(s4 + k);
#pragma unroll
    for (int k = 0; k < 5; ++k) my_tab[k * 32] = __ldg(s4 + 6 + k);  // prior[code][row]
    const int rrow = (d.flags >> F32_RROW_SHIFT) & 15;
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      auto g = [&](int f) {
        const float4 v = cw[f];
        return u == 0 ? v.x : u == 1 ? v.y : u == 2 ? v.z : v.w;
      };
      L.al[u] = set_half<H>(L.al[u], g(0)); L.be[u] = set_half<H>(L.be[u], g(1));
      L.de[u] = set_half<H>(L.de[u], g(2)); L.ep[u] = set_half<H>(L.ep[u], g(3));
      L.ze[u] = set_half<H>(L.ze[u], g(4)); L.mu[u] = set_half<H>(L.mu[u], g(5));
      L.M[u] = set_half<H>(L.M[u], 0.f); L.I[u] = set_half<H>(L.I[u], 0.f);
      L.D[u] = set_half<H>(L.D[u], rrow == u ? d0 : 0.f);
    }
    idx = d.hap_off - (uint32_t)gi;  // = code index of column (-1 - gi) + 1
    out_idx = (d.flags & BLK_LAST) ? d.out_idx : -1;
  } else {
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      L.al[u] = set_half<H>(L.al[u], 0.f); L.be[u] = set_half<H>(L.be[u], 0.f);
      L.de[u] = set_half<H>(L.de[u], 0.f); L.ep[u] = set_half<H>(L.ep[u], 0.f);
      L.ze[u] = set_half<H>(L.ze[u], 0.f); L.mu[u] = set_half<H>(L.mu[u], 0.f);
      L.M[u] = set_half<H>(L.M[u], 0.f); L.I[u] = set_half<H>(L.I[u], 0.f);
      L.D[u] = set_half<H>(L.D[u], 0.f);
    }
    idx = A.pad_idx;
    out_idx = -1;
  }
}

// One warp streams through blocks [s, s+nblk) of one bin (ncols columns each).
__device__ __forceinline__ void f32_stream(const F32Args& A, float4* __restrict__ ptab, float4* __restrict__ ring,
                                           int lane, int64_t s, int nblk, int ncols, bool trace = false) {
  constexpr int G = F32_G;
  constexpr int NGRP = 64 / G;  // switch events per pass
  const int grp = lane / G, gi = lane % G;  // within a half
  const float d0 = ldexpf(1.0f, 120) / (float)ncols;  // virtual row 0
  const int P = max(ncols + G, F32_MIN_P);
  const int npass = (nblk + 63) >> 6;
  const uint8_t* __restrict__ const hc = A.hcodes;
  F32Lane L;
#pragma unroll
  for (int u = 0; u < 4; ++u) {
    L.al[u] = L.be[u] = L.de[u] = L.ep[u] = L.ze[u] = L.mu[u] = 0ull;
    L.M[u] = L.I[u] = L.D[u] = 0ull;
  }
  uint32_t idxA = A.pad_idx, idxB = A.pad_idx;  // code index of the next column
  int codeA_nx = F32_PAD, codeB_nx = F32_PAD;
  int outA = -1, outB = -1;
  v2 upM = 0ull, upI = 0ull, upD = 0ull, dgM = 0ull, dgI = 0ull, dgD = 0ull;
  float4* const tabA = ptab + lane;                   // [code][lane], half A
  float4* const tabB = ptab + F32_NCODE * 32 + lane;  // half B
  const int src = (lane + 31) & 31;
  const bool is0 = lane == 0, is31 = lane == 31;
  int c0 = -(1 << 20);    // (uniform) column of lane 0's half A
  int c31B = -(1 << 20);  // (uniform) column of lane 31's half B
  float* const ringf = reinterpret_cast<float*>(ring);
  const int rmax = A.ring_len - 1;
#ifdef PHMM_DBG_TRACE
  int tstep = 0;
#endif

  auto step = [&]() {
#ifdef PHMM_DBG_SYNC
    __syncwarp();
#endif
    // lane 31: the ring slot that virtual lane 0 needs next step (column c0 + 1)
    // (the ring is only ever accessed as float: one access type, no aliasing games)
    float rvM = 0.f, rvI = 0.f, rvD = 0.f;
    if (is31) {
      const float* r = ringf + 4 * min(c0 + 2, rmax);
      rvM = r[0]; rvI = r[1]; rvD = r[2];
    }
    const int codeA = codeA_nx, codeB = codeB_nx;
    codeA_nx = hc[idxA++];
    codeB_nx = hc[idxB++];
    const float4 pA = tabA[codeA * 32];
    const float4 pB = tabB[codeB * 32];
    f32_column(L, pA, pB, dgM, dgI, dgD, upM, upI);
    // what lane 31 sends: half A stream <- ring (for virtual lane 0), half B stream <- its half A
    const float m3a = lo(L.M[3]), i3a = lo(L.I[3]), d3a = lo(L.D[3]);
    const float m3b = hi(L.M[3]), i3b = hi(L.I[3]), d3b = hi(L.D[3]);
    const float sAM = is31 ? rvM : m3a;
    const float sAI = is31 ? rvI : i3a;
    const float sAD = is31 ? rvD : d3a;
    const float sBM = is31 ? m3a : m3b;
    const float sBI = is31 ? i3a : i3b;
    const float sBD = is31 ? d3a : d3b;
    if (is31 && (unsigned)(c31B + 1) <= (unsigned)ncols) {  // -1 <= c31B < ncols
      float* e = ringf + 4 * (c31B + 1);
      e[0] = m3b; e[1] = i3b; e[2] = d3b;
    }
    __syncwarp();
    dgM = upM; dgI = upI; dgD = upD;
    upM = pk(__shfl_sync(0xffffffffu, sAM, src), __shfl_sync(0xffffffffu, sBM, src));
    upI = pk(__shfl_sync(0xffffffffu, sAI, src), __shfl_sync(0xffffffffu, sBI, src));
    upD = pk(__shfl_sync(0xffffffffu, sAD, src), __shfl_sync(0xffffffffu, sBD, src));
#ifdef PHMM_DBG_TRACE
    if (trace && tstep < 4096) {
      float* t = g_trace + ((size_t)tstep * 32 + lane) * 6;
      t[0] = lo(L.M[3]); t[1] = lo(L.I[3]); t[2] = lo(L.D[3]);
      t[3] = hi(L.M[3]); t[4] = hi(L.I[3]); t[5] = hi(L.D[3]);
      if (lane == 0) g_trace_steps = tstep + 1;
    }
    ++tstep;
#endif
    ++c0;
    ++c31B;
  };

  for (int q = 0; q <= npass; ++q) {
#pragma unroll 1
    for (int e = 0; e < NGRP; ++e) {
      const int h = e / (NGRP / 2), g = e % (NGRP / 2);
      if (e == 0) {  // lane 0 half A starts its pass: column -1 next
        c0 = -1;
      }
      if (e == NGRP - 1) c31B = -1 - (G - 1);  // lane 31 half B
      if (grp == g) {  // switch event of virtual group (h, g): SIMT over its G lanes
        const int b = q * 64 + h * 32 + lane;
        const bool have = (q < npass) && (b < nblk);
        BlkDesc d;
        d.tab_blk = 0; d.hap_off = 0; d.out_idx = -1; d.n = 1; d.flags = 0;
        if (have) d = A.blk[s + b];
        if (h == 0) {
          if (outA >= 0) A.out[outA] = lo(L.D[3]);  // S2 row: the last-row M+I sum (L20@2262)
          f32_load<0>(A, L, tabA, have, d, d0, idxA, outA, gi);
          codeA_nx = F32_PAD;
          if (is0) {  // virtual lane 0: its column -1 needs the boundary slot of the ring
            upM = set_half<0>(upM, ringf[0]); upI = set_half<0>(upI, ringf[1]); upD = set_half<0>(upD, ringf[2]);
          }
        } else {
          if (outB >= 0) A.out[outB] = hi(L.D[3]);
          f32_load<1>(A, L, tabB, have, d, d0, idxB, outB, gi);
          codeB_nx = F32_PAD;
        }
      }
      const int nsteps = (e < NGRP - 1) ? G : (q < npass ? P - (NGRP - 1) * G : 0);
#ifndef PHMM_F32_UNROLL
#define PHMM_F32_UNROLL 2
#endif
#if PHMM_F32_UNROLL == 1
#pragma unroll 1
#else
#pragma unroll 2
#endif
      for (int k = 0; k < nsteps; ++k) step();
    }
  }
}

// The kernel is defined in wf32.cu (its own translation unit, compiled with
// -Xptxas -O1: ptxas -O2/-O3 mis-schedules this kernel -- results silently
// differ from the -O0/-O1 builds and from the CPU emulation of the schedule;
// DESIGN.md §4.6). phmm_lib.cu reaches it through these two host functions.
cudaError_t wf32_occupancy(size_t smem, int* blocks_per_sm);
cudaError_t wf32_launch(unsigned grid, size_t smem, cudaStream_t stream, const F32Args& args);

#ifdef PHMM_DEFINE_WF32
#ifndef PHMM_F32_MINB
#define PHMM_F32_MINB 4  // CTAs (of 4 warps) per SM the register budget must allow
#endif
__global__ void __launch_bounds__(F32_WARPS * 32, PHMM_F32_MINB) k_wavefront_f32(F32Args A) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  const int lane = threadIdx.x & 31;
  const int wib = threadIdx.x >> 5;
  // per warp: prior tables [2 halves][6 codes][32 lanes] float4 (6 KB), then the ring
  const int per_warp = 2 * F32_NCODE * 32 + A.ring_len;
  float4* ptab = reinterpret_cast<float4*>(smem_raw) + (size_t)wib * per_warp;
  float4* ring = ptab + 2 * F32_NCODE * 32;
  for (int i = lane; i < 2 * F32_NCODE * 32; i += 32) ptab[i] = make_float4(0.f, 0.f, 0.f, 0.f);
  for (int i = lane; i < 4 * A.ring_len; i += 32) reinterpret_cast<float*>(ring)[i] = 0.f;
  __syncwarp();
  const unsigned long long n_items = A.item_start[A.nbins];
  while (true) {
    unsigned int it = 0;
    if (lane == 0) it = atomicAdd(A.item_counter, 1u);
    it = __shfl_sync(0xffffffffu, it, 0);
    if (it >= n_items) break;
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
#ifdef PHMM_DBG_TRACE
    f32_stream(A, ptab, ring, lane, s, (int)(e - s), bin * A.bucket, it == 0);
#else
    f32_stream(A, ptab, ring, lane, s, (int)(e - s), bin * A.bucket);
#endif
    __syncwarp();
  }
}

#endif  // PHMM_DEFINE_WF32

}  // namespace phmm
