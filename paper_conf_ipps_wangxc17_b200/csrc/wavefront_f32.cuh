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

#ifndef PHMM_F32_K
#define PHMM_F32_K 8
#endif
constexpr int F32_K = PHMM_F32_K;  // rows per virtual lane (per half): 4 or 8
static_assert(F32_K == 4 || F32_K == 8, "F32_K must be 4 or 8");
constexpr int F32_KC = F32_K / 4;  // float4 chunks per row set
constexpr int F32_G = 8;      // virtual lanes per switch group
constexpr int F32_NCODE = 6;  // A C G T N PAD
constexpr int F32_PAD = 5;
constexpr int F32_WARPS = 4;   // warps per CTA
constexpr int F32_MIN_P = 72;  // ring delay: virtual lane 63 -> 0 needs P >= 72
constexpr int64_t F32_HC_FRONT = 16;  // PAD codes before every haplotype's code array

// per-block coefficient table: 6 transition fields + 5 prior codes, F32_K rows each
struct alignas(16) F32Block {
  float coef[6][F32_K];   // alpha, beta, delta, eps, zeta, mu
  float prior[5][F32_K];  // P(row, code) for code = A, C, G, T, N
};
static_assert(sizeof(F32Block) == 44 * F32_K, "F32Block layout");
// code byte in the haplotype code arrays: code * F32_CB; moved into bits 8..15 it is
// code * F32_K * 128 bytes = the stride of one code's rows in a lane's prior table
constexpr int F32_CB = F32_K / 2;

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

// lane state: lo = half A, hi = half B; index = row 0..F32_K-1
struct F32Lane {
  v2 al[F32_K], be[F32_K], de[F32_K], ep[F32_K], ze[F32_K], mu[F32_K];
  v2 M[F32_K], I[F32_K], D[F32_K];
};

// One column for both halves, in place. dg* = row above at column x-1, up* = row above at column x.
__device__ __forceinline__ void f32_column(F32Lane& L, const float (&prA)[F32_K], const float (&prB)[F32_K],
                                           const v2 dgM, const v2 dgI, const v2 dgD, const v2 upM, const v2 upI) {
  // M and D: rows descending so that row u-1's old values are intact when row u reads them
#pragma unroll
  for (int u = F32_K - 1; u >= 0; --u) {
    const v2 md = (u == 0) ? dgM : L.M[u - 1];
    const v2 id = (u == 0) ? dgI : L.I[u - 1];
    const v2 dd = (u == 0) ? dgD : L.D[u - 1];
    // D(i,j) = zeta*M(i,j-1) + mu*D(i,j-1)
    L.D[u] = fma2(L.ze[u], L.M[u], mul2(L.mu[u], L.D[u]));
    // M(i,j) = P(i,j) * (alpha*M(i-1,j-1) + beta*(I(i-1,j-1) + D(i-1,j-1)))
    const v2 x = fma2(L.al[u], md, mul2(L.be[u], add2(id, dd)));
    L.M[u] = pk(prA[u] * lo(x), prB[u] * hi(x));
  }
  // I(i,j) = delta*M(i-1,j) + eps*I(i-1,j), rows ascending (an F32_K-deep FFMA2 chain)
  v2 m_up = upM, i_up = upI;
#pragma unroll
  for (int u = 0; u < F32_K; ++u) {
    const v2 ni = fma2(L.ep[u], i_up, mul2(L.de[u], m_up));
    m_up = L.M[u];
    i_up = ni;
    L.I[u] = ni;
  }
}

// ---- shared-memory ring accessors (inline PTX, "memory" clobber: the ring is read
// and written through these only, so no compiler reordering or aliasing games)
__device__ __forceinline__ void ring_put3(uint32_t saddr, float a, float b, float c) {
  asm volatile("st.shared.f32 [%0], %1;\n\tst.shared.f32 [%0+4], %2;\n\tst.shared.f32 [%0+8], %3;"
               :: "r"(saddr), "f"(a), "f"(b), "f"(c) : "memory");
}
__device__ __forceinline__ void ring_get3(uint32_t saddr, float& a, float& b, float& c) {
  float d;
  asm volatile("ld.shared.v4.f32 {%0, %1, %2, %3}, [%4];" : "=f"(a), "=f"(b), "=f"(c), "=f"(d) : "r"(saddr) : "memory");
}
__device__ __forceinline__ uint32_t smem_addr(const void* p) {
  return (uint32_t)__cvta_generic_to_shared(p);
}

// Haplotype code slots (4 shifted copies per haplotype so that every lane reads its
// codes as aligned 32-bit words, 4 columns at a time). Byte = code * 32, the
// float4 index of that code's entry in a lane's prior table.
__host__ __device__ inline int f32_hc_copy_len(int ncols) {
  const int p = (ncols + F32_G > F32_MIN_P) ? ncols + F32_G : F32_MIN_P;
  return ((int)F32_HC_FRONT + p + 24 + 3) & ~3;  // + prefetch distance
}

// Load a block (or nothing) into half H of a lane. Returns the 32-bit-aligned code
// pointer for the lane's first step (column -1 - gi).
template <int H>
__device__ __forceinline__ const uint32_t* f32_load(const F32Args& A, F32Lane& L, float4* __restrict__ my_tab,
                                                    bool have, const BlkDesc& d, float d0, int& out_idx, int gi,
                                                    int copy_len) {
  if (have) {
    const float4* __restrict__ s4 = reinterpret_cast<const float4*>(A.tab + d.tab_blk);
    float4 cw[6 * F32_KC];
#pragma unroll
    for (int k = 0; k < 6 * F32_KC; ++k) cw[k] = __ldg(s4 + k);
#pragma unroll
    for (int k = 0; k < 5 * F32_KC; ++k) my_tab[k * 32] = __ldg(s4 + 6 * F32_KC + k);  // prior[code][chunk]
    const int rrow = (d.flags >> F32_RROW_SHIFT) & 15;
#pragma unroll
    for (int u = 0; u < F32_K; ++u) {
      auto g = [&](int f) {
        const float4 v = cw[f * F32_KC + (u >> 2)];
        return (u & 3) == 0 ? v.x : (u & 3) == 1 ? v.y : (u & 3) == 2 ? v.z : v.w;
      };
      L.al[u] = set_half<H>(L.al[u], g(0)); L.be[u] = set_half<H>(L.be[u], g(1));
      L.de[u] = set_half<H>(L.de[u], g(2)); L.ep[u] = set_half<H>(L.ep[u], g(3));
      L.ze[u] = set_half<H>(L.ze[u], g(4)); L.mu[u] = set_half<H>(L.mu[u], g(5));
      L.M[u] = set_half<H>(L.M[u], 0.f); L.I[u] = set_half<H>(L.I[u], 0.f);
      L.D[u] = set_half<H>(L.D[u], rrow == u ? d0 : 0.f);
    }
    out_idx = (d.flags & BLK_LAST) ? d.out_idx : -1;
    // copy k = (1 + gi) mod 4 has column 0 at hap_off + k*(copy_len + 1), so the byte
    // of column (-1 - gi) is 4-aligned
    const int k = (1 + gi) & 3;
    const uint32_t col0 = d.hap_off + (uint32_t)(k * (copy_len + 1));
    return reinterpret_cast<const uint32_t*>(A.hcodes + (col0 - 1u - (uint32_t)gi));
  }
#pragma unroll
  for (int u = 0; u < F32_K; ++u) {
    L.al[u] = set_half<H>(L.al[u], 0.f); L.be[u] = set_half<H>(L.be[u], 0.f);
    L.de[u] = set_half<H>(L.de[u], 0.f); L.ep[u] = set_half<H>(L.ep[u], 0.f);
    L.ze[u] = set_half<H>(L.ze[u], 0.f); L.mu[u] = set_half<H>(L.mu[u], 0.f);
    L.M[u] = set_half<H>(L.M[u], 0.f); L.I[u] = set_half<H>(L.I[u], 0.f);
    L.D[u] = set_half<H>(L.D[u], 0.f);
  }
  out_idx = -1;
  return reinterpret_cast<const uint32_t*>(A.hcodes + A.pad_idx);
}

// One warp streams through blocks [s, s+nblk) of one bin (ncols columns each).
// Virtual lane v = 2*lane + h (h = 0: half A = low 32 bits, h = 1: half B = high 32 bits),
// so half B's row above is its own lane's half A one step earlier (no shuffle) and
// half A's row above is lane-1's half B (one shuffle per value).
__device__ __forceinline__ void f32_stream(const F32Args& A, float4* __restrict__ ptab, float4* __restrict__ ring,
                                           int lane, int64_t s, int nblk, int ncols, bool trace = false) {
  constexpr int G = F32_G;            // virtual lanes per switch group
  constexpr int NGRP = 64 / G;        // switch events per pass
  constexpr int LPG = G / 2;          // physical lanes per group
  const int grp = lane / LPG;
  const int giA = 2 * (lane % LPG), giB = giA + 1;  // position of each half inside its group
  const float d0 = ldexpf(1.0f, 120) / (float)ncols;  // virtual row 0
  const int P = max(ncols + G, F32_MIN_P);           // multiple of 4 (ncols is)
  const int npass = (nblk + 63) >> 6;
  const int copy_len = f32_hc_copy_len(ncols);
  F32Lane L;
#pragma unroll
  for (int u = 0; u < F32_K; ++u) {
    L.al[u] = L.be[u] = L.de[u] = L.ep[u] = L.ze[u] = L.mu[u] = 0ull;
    L.M[u] = L.I[u] = L.D[u] = 0ull;
  }
  const uint32_t* pA = reinterpret_cast<const uint32_t*>(A.hcodes + A.pad_idx);  // next code word
  const uint32_t* pB = pA;
  constexpr uint32_t kPadW = (uint32_t)(F32_PAD * F32_CB) * 0x01010101u;  // four PAD codes
  // code words: current group, next group, the one after (prefetch distance 2 groups)
  uint32_t wA = kPadW, wB = kPadW, wA_nx = kPadW, wB_nx = kPadW, wA_nx2 = kPadW, wB_nx2 = kPadW;
  int outA = -1, outB = -1;
  v2 upM = 0ull, upI = 0ull, upD = 0ull, dgM = 0ull, dgI = 0ull, dgD = 0ull;
  const uint32_t tabA_s = smem_addr(ptab + lane);                            // [code][chunk][lane] float4
  const uint32_t tabB_s = smem_addr(ptab + F32_NCODE * F32_KC * 32 + lane);  // half B
  const uint32_t ring_s = smem_addr(ring);
  const int src = (lane + 31) & 31;
  const bool is0 = lane == 0, is31 = lane == 31;
  int c0 = -(1 << 20);    // (uniform) column of virtual lane 0 (lane 0, half A)
  int c31B = -(1 << 20);  // (uniform) column of virtual lane 63 (lane 31, half B)
  float rvM = 0.f, rvI = 0.f, rvD = 0.f;  // lane 31: ring slot for virtual lane 0's next column
  BlkDesc dnA, dnB;  // next pass's block descriptors (prefetched)
  dnA.tab_blk = 0; dnA.hap_off = 0; dnA.out_idx = -1; dnA.n = 1; dnA.flags = 0;
  dnB = dnA;
#ifdef PHMM_DBG_TRACE
  int tstep = 0;
#endif

  auto step = [&](const int r) {
    if (is31) ring_get3(ring_s + 16u * (uint32_t)(c0 + 2), rvM, rvI, rvD);
    // code byte r (= code*F32_CB) placed in byte 1 -> the code's rows in the table
    const uint32_t oA = __byte_perm(wA, 0, 0x4404 + (r << 4)), oB = __byte_perm(wB, 0, 0x4404 + (r << 4));
    float prA[F32_K], prB[F32_K];
#pragma unroll
    for (int ch = 0; ch < F32_KC; ++ch) {
      asm volatile("ld.shared.v4.f32 {%0, %1, %2, %3}, [%4];"
                   : "=f"(prA[4 * ch]), "=f"(prA[4 * ch + 1]), "=f"(prA[4 * ch + 2]), "=f"(prA[4 * ch + 3])
                   : "r"(tabA_s + oA + 512u * ch));
      asm volatile("ld.shared.v4.f32 {%0, %1, %2, %3}, [%4];"
                   : "=f"(prB[4 * ch]), "=f"(prB[4 * ch + 1]), "=f"(prB[4 * ch + 2]), "=f"(prB[4 * ch + 3])
                   : "r"(tabB_s + oB + 512u * ch));
    }
    f32_column(L, prA, prB, dgM, dgI, dgD, upM, upI);
    constexpr int LR = F32_K - 1;  // last row of a block
    const float m3a = lo(L.M[LR]), i3a = lo(L.I[LR]), d3a = lo(L.D[LR]);
    const float m3b = hi(L.M[LR]), i3b = hi(L.I[LR]), d3b = hi(L.D[LR]);
    // half B of lane-1 -> half A of lane; lane 31 sends the ring slot instead (virtual 63 -> 0)
    const float sM = is31 ? rvM : m3b;
    const float sI = is31 ? rvI : i3b;
    const float sD = is31 ? rvD : d3b;
    if (is31 && (unsigned)(c31B + 1) <= (unsigned)ncols)  // -1 <= c31B < ncols
      ring_put3(ring_s + 16u * (uint32_t)(c31B + 1), m3b, i3b, d3b);
    __syncwarp();
    dgM = upM; dgI = upI; dgD = upD;
    // next step: half A's row above = lane-1's half B; half B's row above = this lane's half A
    upM = pk(__shfl_sync(0xffffffffu, sM, src), m3a);
    upI = pk(__shfl_sync(0xffffffffu, sI, src), i3a);
    upD = pk(__shfl_sync(0xffffffffu, sD, src), d3a);
#ifdef PHMM_DBG_TRACE
    if (trace && tstep < 4096) {
      float* t = g_trace + ((size_t)tstep * 32 + lane) * 6;
      t[0] = lo(L.M[F32_K - 1]); t[1] = lo(L.I[F32_K - 1]); t[2] = lo(L.D[F32_K - 1]);
      t[3] = hi(L.M[F32_K - 1]); t[4] = hi(L.I[F32_K - 1]); t[5] = hi(L.D[F32_K - 1]);
      if (lane == 0) g_trace_steps = tstep + 1;
    }
    ++tstep;
#endif
    ++c0;
    ++c31B;
  };
  // 4 steps sharing one code word per half; the next words are prefetched
  auto group4 = [&]() {
    wA = wA_nx; wB = wB_nx;
    wA_nx = wA_nx2; wB_nx = wB_nx2;
    wA_nx2 = __ldg(pA); wB_nx2 = __ldg(pB);
    ++pA; ++pB;
    step(0); step(1); step(2); step(3);
  };

  for (int q = 0; q <= npass; ++q) {
#pragma unroll 1
    for (int e = 0; e < NGRP; ++e) {
      if (e == 0) c0 = -1;                      // virtual lane 0 starts its pass: column -1 next
      if (e == NGRP - 1) c31B = -1 - (G - 1);  // virtual lane 63
      if (grp == e) {  // switch event of virtual lanes 8e..8e+7 = lanes 4e..4e+3, both halves
        const int bA = q * 64 + 2 * lane, bB = bA + 1;
        const bool hA = (q < npass) && (bA < nblk), hB = (q < npass) && (bB < nblk);
        // this pass's descriptors were prefetched one pass ago (pass 0: loaded now);
        // prefetch the next pass's so their latency hides behind P steps
        BlkDesc dA = dnA, dB = dnB;
        if (q == 0) {
          if (hA) dA = A.blk[s + bA];
          if (hB) dB = A.blk[s + bB];
        }

        if (outA >= 0) A.out[outA] = lo(L.D[F32_K - 1]);  // S2 row: the last-row M+I sum (L20@2262)
        if (outB >= 0) A.out[outB] = hi(L.D[F32_K - 1]);
        pA = f32_load<0>(A, L, ptab + lane, hA, dA, d0, outA, giA, copy_len);
        pB = f32_load<1>(A, L, ptab + F32_NCODE * F32_KC * 32 + lane, hB, dB, d0, outB, giB, copy_len);
        wA_nx = __ldg(pA); wA_nx2 = __ldg(pA + 1); pA += 2;
        wB_nx = __ldg(pB); wB_nx2 = __ldg(pB + 1); pB += 2;
        // prefetch after this pass's loads are issued (a load issued before the
        // consumers of the previous prefetch would share their scoreboard)
        if (bA + 64 < nblk) dnA = A.blk[s + bA + 64];
        if (bB + 64 < nblk) dnB = A.blk[s + bB + 64];
        if (is0) {  // virtual lane 0: its column -1 needs the boundary slot of the ring
          float a, bb, c;
          ring_get3(ring_s, a, bb, c);
          upM = set_half<0>(upM, a); upI = set_half<0>(upI, bb); upD = set_half<0>(upD, c);
        }
      }
      const int ngroups = (e < NGRP - 1) ? G / 4 : (q < npass ? (P - (NGRP - 1) * G) / 4 : 0);
#pragma unroll 1
      for (int k = 0; k < ngroups; ++k) group4();
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
#define PHMM_F32_MINB 2  // CTAs (of 4 warps) per SM the register budget must allow (255 regs)
#endif
__global__ void __launch_bounds__(F32_WARPS * 32, PHMM_F32_MINB) k_wavefront_f32(F32Args A) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  const int lane = threadIdx.x & 31;
  const int wib = threadIdx.x >> 5;
  // per warp: prior tables [2 halves][6 codes][F32_KC chunks][32 lanes] float4, then the ring
  constexpr int kTab = 2 * F32_NCODE * F32_KC * 32;
  const int per_warp = kTab + A.ring_len;
  float4* ptab = reinterpret_cast<float4*>(smem_raw) + (size_t)wib * per_warp;
  float4* ring = ptab + kTab;
  for (int i = lane; i < kTab; i += 32) ptab[i] = make_float4(0.f, 0.f, 0.f, 0.f);
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
