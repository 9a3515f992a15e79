// wavefront.cuh -- the PairHMM wavefront kernel for sm_100a (the hot loop), FP32 and FP64.
//
// PRODUCT PATH. Computes Eq. 6 of PAPER.md (L18@541) over "tall streams" of
// K-row blocks (see phmm_common.cuh for the Z/R/S pad-row layout that makes
// a pair's termination sum (L20@2262) fall out of the recurrence).
//
// The paper's PH2 kernel (L20@3509, Fig. 8) gives one warp one pair and lets each
// thread own consecutive rows, passing the row-above values by shuffle (its Design
// B, Listing 2b, L20@44). This kernel keeps the row ownership and the shuffle and
// changes the rest for Blackwell:
//  * a warp streams through a long sequence of blocks of one length bin; it has 64
//    VIRTUAL lanes v = 2*lane + h (h = 0/1: the two halves of a register pair), each
//    owning one K-row block per pass (blocks 64q + v); virtual lane v computes column
//    x of its block at step T_q + 1 + v + x.
//  * FP32: the halves are the two floats of a 64-bit register, so every FP op of
//    Eq. 6 is one packed FFMA2/FMUL2/FADD2 for two independent cells (K = 8 rows).
//    FP64 (the rescue pass): the halves are two doubles, scalar DFMA (K = 4 rows).
//  * the emission prior P(i,j): a per-half table prior[code][row] in shared memory
//    (code = haplotype base A,C,G,T,N or PAD); 16-byte LDS per chunk of rows.
//  * no per-lane "is this column real" branch: columns outside a block read the PAD
//    code (prior 0); by induction down the lanes an idle virtual lane then computes
//    exactly the boundary column (M = I = 0, D = D(i,0)) before its block and freezes
//    the S running sum after it.
//  * virtual lanes switch blocks in groups of G = 8 (8 switch events per pass); a pass
//    is P = max(ncols + G, 72) steps.
//  * row above: half B of a lane takes its own half A one step later (no shuffle);
//    half A takes lane-1's half B by __shfl_sync; virtual lane 0 takes virtual lane
//    63 of the previous pass through a per-warp shared-memory ring indexed by column
//    + 1 (slot 0 = boundary column); lane 31 substitutes the ring slot into what it
//    shuffles.
#pragma once
#include <cuda_runtime.h>

#include <cstdint>

#include "phmm_common.cuh"

namespace phmm {

#ifndef PHMM_F32_K
#define PHMM_F32_K 8  // rows per half in the FP32 pass (8 or 4)
#endif
#ifndef PHMM_F32_MINB
#define PHMM_F32_MINB 2  // CTAs (of 4 warps) per SM the FP32 kernel's register budget must allow (2: 255 regs)
#endif
#ifndef PHMM_F64_K
#define PHMM_F64_K 4  // rows per half in the FP64 rescue pass (4 or 2)
#endif
#ifndef PHMM_F64_MINB
#define PHMM_F64_MINB 2
#endif
#ifndef PHMM_XCHG_SMEM
#define PHMM_XCHG_SMEM 0  // 1: design-A ablation build (row exchange through shared memory)
#endif

constexpr int WF_G = 8;           // virtual lanes per switch group
constexpr int WF_NCODE = 6;       // A C G T N PAD
constexpr int WF_PAD = 5;
#ifndef PHMM_WF_WARPS
#define PHMM_WF_WARPS 4
#endif
constexpr int WF_WARPS = PHMM_WF_WARPS;  // warps per CTA
#ifndef PHMM_TAIL_DIV
#define PHMM_TAIL_DIV 8
#endif
#ifndef PHMM_TAIL_SPLIT
#define PHMM_TAIL_SPLIT 8
#endif
constexpr int WF_TAIL_SPLIT = PHMM_TAIL_SPLIT;  // short items are 1/WF_TAIL_SPLIT of a full-size item
#ifndef PHMM_LPT
#define PHMM_LPT 1
#endif
constexpr int WF_LPT = PHMM_LPT;  // 1: longest-row bins first inside a launch
constexpr int WF_TAIL_DIV = PHMM_TAIL_DIV;  // last 1/WF_TAIL_DIV of a launch's blocks in short work items (0: none)
constexpr int WF_MIN_P = 72;      // ring delay: virtual lane 63 -> 0 needs P >= 72
// Staged switch events (both passes): a lane starts its next block wf_sh = 4 columns
// earlier (PAD: the code regions have 16 PAD columns in front), issues the block's table as
// cp.async copies at its switch event and commits the coefficients 4 steps later, before the
// first column whose result is used, so no instruction waits on the table loads; a pass is
// 4 steps longer. The FP64 pass packs its ring slots into 24 bytes to pay
// for the staging slots and stay at 8 warps per SM.
template <typename T> __host__ __device__ constexpr int wf_sh() { return 4; }
constexpr int64_t WF_HC_FRONT = 16;  // PAD codes before every haplotype's code array
constexpr int WF_KC32 = PHMM_F32_K / 4;  // 16-byte chunks per row set of the FP32 pass (K floats)
constexpr int WF_KC64 = PHMM_F64_K / 2;  // ... of the FP64 pass (K doubles)
// code byte in the haplotype code arrays = code * WF_CB; moved into bits 8..15 it is
// code * WF_KC32 * 512 bytes = the stride of one code's rows in a lane's FP32 prior table
// (the FP64 pass, which reads the same code arrays, scales it by WF_KC64 / WF_KC32)
constexpr int WF_CB = 2 * WF_KC32;

// BlkDesc.flags: bit0 last, bit1 first, bit2 BLK_RESC (pair of >= 65 blocks), bit3 BLK_FILLER,
// bits 8-11 R row (15 = none)
constexpr uint16_t WF_RROW_SHIFT = 8;
constexpr uint16_t WF_RROW_NONE = 15;

// ---------------------------------------------------------------- precision traits
typedef unsigned long long v2f;           // two floats in a 64-bit register pair
struct alignas(16) v2d { double a, b; };  // two doubles

template <typename T> struct WfT;
template <> struct WfT<float> {
  using V = v2f;
  static constexpr int K = PHMM_F32_K;
  static constexpr int KC = WF_KC32;
  static constexpr int MINB = PHMM_F32_MINB;  // CTAs per SM the register budget must allow
  static constexpr int kScaleExp = 120;
};
template <> struct WfT<double> {
  using V = v2d;
  static constexpr int K = PHMM_F64_K;
  static constexpr int KC = WF_KC64;
  static constexpr int MINB = PHMM_F64_MINB;
  static constexpr int kScaleExp = 1020;
};
static_assert(WfT<float>::K * 4 == WF_KC32 * 16 && WfT<double>::K * 8 == WF_KC64 * 16, "chunk layout");
static_assert(WF_KC64 % WF_KC32 == 0 || WF_KC32 % WF_KC64 == 0, "code stride");

__device__ __forceinline__ v2f pk(float lo, float hi) {
  v2f r;
  asm("mov.b64 %0, {%1, %2};" : "=l"(r) : "f"(lo), "f"(hi));
  return r;
}
__device__ __forceinline__ float lo(v2f v) {
  float a, b;
  asm("mov.b64 {%0, %1}, %2;" : "=f"(a), "=f"(b) : "l"(v));
  (void)b;
  return a;
}
__device__ __forceinline__ float hi(v2f v) {
  float a, b;
  asm("mov.b64 {%0, %1}, %2;" : "=f"(a), "=f"(b) : "l"(v));
  (void)a;
  return b;
}
__device__ __forceinline__ v2f fma2(v2f a, v2f b, v2f c) {
  v2f d;
  asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(d) : "l"(a), "l"(b), "l"(c));
  return d;
}
__device__ __forceinline__ v2f mul2(v2f a, v2f b) {
  v2f d;
  asm("mul.rn.f32x2 %0, %1, %2;" : "=l"(d) : "l"(a), "l"(b));
  return d;
}
__device__ __forceinline__ v2f add2(v2f a, v2f b) {
  v2f d;
  asm("add.rn.f32x2 %0, %1, %2;" : "=l"(d) : "l"(a), "l"(b));
  return d;
}
__device__ __forceinline__ v2d pk(double lo, double hi) { return v2d{lo, hi}; }
__device__ __forceinline__ double lo(v2d v) { return v.a; }
__device__ __forceinline__ double hi(v2d v) { return v.b; }
__device__ __forceinline__ v2d fma2(v2d a, v2d b, v2d c) { return v2d{fma(a.a, b.a, c.a), fma(a.b, b.b, c.b)}; }
__device__ __forceinline__ v2d mul2(v2d a, v2d b) { return v2d{a.a * b.a, a.b * b.b}; }
__device__ __forceinline__ v2d add2(v2d a, v2d b) { return v2d{a.a + b.a, a.b + b.b}; }

template <int H, typename V, typename S>
__device__ __forceinline__ V set_half(V r, S v) {
  return H == 0 ? pk(v, hi(r)) : pk(lo(r), v);
}
template <typename V> __device__ __forceinline__ V vzero();
template <> __device__ __forceinline__ v2f vzero<v2f>() { return 0ull; }
template <> __device__ __forceinline__ v2d vzero<v2d>() { return v2d{0.0, 0.0}; }

// per-block coefficient table: 4 transition fields + 5 prior codes, K rows each.
// The kernel evaluates Eq. 6 in a rescaled 5-op form: row i stores
// M^ = a_i M, I^ = b_i I, D^ = d_i D with per-row scales chosen so that the coefficient
// of M in the D update and of M(up) in the I update are exactly 1:
//   D^ = M^(i,j-1) + mu D^(i,j-1)                                    1 FFMA
//   I^ = M^(i-1,j) + ep' I^(i-1,j)                                   1 FFMA
//   M^ = T[code] * (M^(i-1,j-1) + u I^(i-1,j-1) + w D^(i-1,j-1))     2 FFMA + 1 FMUL
// (stream_prep.cuh k_build_table_wf has the scales; none exceeds the unscaled value).
constexpr int WF_NCOEF = 4;
template <typename T>
struct alignas(16) TBlock {
  T coef[WF_NCOEF][WfT<T>::K];  // u, w, ep', mu
  T prior[5][WfT<T>::K];        // T(row, code) for code = A, C, G, T, N
};
static_assert(sizeof(TBlock<float>) == 9 * WF_KC32 * 16 && sizeof(TBlock<double>) == 9 * WF_KC64 * 16, "TBlock");

template <typename T>
struct WfArgs2 {
  const BlkDesc* blk;
  const TBlock<T>* tab;
  const uint8_t* hcodes;                 // per-haplotype code regions (4 shifted copies)
  uint32_t pad_idx;                      // index of an all-PAD region (idle lanes)
  const unsigned long long* bin_start;   // [nbins+1] first block of each bin
  const unsigned long long* item_start;  // [nbins+1] first work item of each bin
  int bin_lo, bin_hi;                    // this launch runs the work items of bins [bin_lo, bin_hi)
  int bucket;
  int64_t chunk_blocks;                  // blocks per full-size work item
  int64_t chunk_small;                   // blocks per short work item (the tail of each bin)
  const unsigned long long* bin_nbig;    // [nbins] full-size items of each bin
  const unsigned long long* launch_items;  // [2]: this launch's work items are [launch_items[0], launch_items[1])
  int lpt;                               // 1: bins in descending order inside a launch (longest rows first)
  unsigned int* item_counter;
  T* out;
  int32_t* exp_out;  // FP32 pass: per output slot, the power of 2 the ring rescale applied
  int ring_len;  // slots, >= P + 4
};

template <typename T>
struct Lane {
  using V = typename WfT<T>::V;
  static constexpr int K = WfT<T>::K;
  V uu[K], ww[K], ep[K], mu[K];
  V M[K], I[K], D[K];
};

// One column for both halves, in place. dg* = row above at column x-1, up* = row above at column x.
template <typename T>
__device__ __forceinline__ void wf_column(Lane<T>& L, const T (&prA)[WfT<T>::K], const T (&prB)[WfT<T>::K],
                                          const typename WfT<T>::V dgM, const typename WfT<T>::V dgI,
                                          const typename WfT<T>::V dgD, const typename WfT<T>::V upM,
                                          const typename WfT<T>::V upI) {
  using V = typename WfT<T>::V;
  constexpr int K = WfT<T>::K;
  // M and D: rows descending so that row u-1's old values are intact when row u reads them
#pragma unroll
  for (int u = K - 1; u >= 0; --u) {
    const V md = (u == 0) ? dgM : L.M[u - 1];
    const V id = (u == 0) ? dgI : L.I[u - 1];
    const V dd = (u == 0) ? dgD : L.D[u - 1];
    // D^(i,j) = M^(i,j-1) + mu*D^(i,j-1)
    L.D[u] = fma2(L.mu[u], L.D[u], L.M[u]);
    // M^(i,j) = T(i, h_j) * (M^(i-1,j-1) + u*I^(i-1,j-1) + w*D^(i-1,j-1))
    const V x = fma2(L.ww[u], dd, fma2(L.uu[u], id, md));
    L.M[u] = pk(prA[u] * lo(x), prB[u] * hi(x));
  }
  // I^(i,j) = M^(i-1,j) + ep'*I^(i-1,j), rows ascending (a K-deep chain)
  V m_up = upM, i_up = upI;
#pragma unroll
  for (int u = 0; u < K; ++u) {
    const V ni = fma2(L.ep[u], i_up, m_up);
    m_up = L.M[u];
    i_up = ni;
    L.I[u] = ni;
  }
}

// ---- shared-memory accessors (inline PTX with "memory" clobbers: the ring and the prior
// tables are only touched through these, so no compiler reordering or aliasing games)
__device__ __forceinline__ uint32_t smem_addr(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void ring_put3(uint32_t a, float x, float y, float z) {
  asm volatile("st.shared.f32 [%0], %1;\n\tst.shared.f32 [%0+4], %2;\n\tst.shared.f32 [%0+8], %3;"
               :: "r"(a), "f"(x), "f"(y), "f"(z) : "memory");
}
__device__ __forceinline__ void ring_get3(uint32_t a, float& x, float& y, float& z) {
  float w;
  asm volatile("ld.shared.v4.f32 {%0, %1, %2, %3}, [%4];" : "=f"(x), "=f"(y), "=f"(z), "=f"(w) : "r"(a) : "memory");
  (void)w;
}
__device__ __forceinline__ void ring_put3(uint32_t a, double x, double y, double z) {
  asm volatile("st.shared.v2.f64 [%0], {%1, %2};\n\tst.shared.f64 [%0+16], %3;"
               :: "r"(a), "d"(x), "d"(y), "d"(z) : "memory");
}
__device__ __forceinline__ void ring_get3(uint32_t a, double& x, double& y, double& z) {
  asm volatile("ld.shared.v2.f64 {%0, %1}, [%3];\n\tld.shared.f64 %2, [%3+16];"
               : "=d"(x), "=d"(y), "=d"(z) : "r"(a) : "memory");
}
// ring slot: 16 / 32 bytes (one vector load); packed 24 bytes (three scalar loads) in the
// FP64 long-row kernel, where the ring limits occupancy (C4 rescue: 3 -> 4 warps per SM;
// packing the FP32 long-row ring measured slower)
template <typename T, bool kLong = false> __host__ __device__ constexpr bool ring_packed() {
  return sizeof(T) == 8;  // FP64: 24-byte slots pay for the staging slots (8 warps per SM)
}
template <typename T, bool kLong = false> __host__ __device__ constexpr uint32_t ring_slot_bytes() {
  return ring_packed<T, kLong>() ? 3u * (uint32_t)sizeof(T) : (sizeof(T) == 4 ? 16u : 32u);
}
template <typename T>
__device__ __forceinline__ void ring_get3p(uint32_t a, T& x, T& y, T& z) {
  if constexpr (sizeof(T) == 4)
    asm volatile("ld.shared.f32 %0, [%3];\n\tld.shared.f32 %1, [%3+4];\n\tld.shared.f32 %2, [%3+8];"
                 : "=f"(x), "=f"(y), "=f"(z) : "r"(a) : "memory");
  else
    asm volatile("ld.shared.f64 %0, [%3];\n\tld.shared.f64 %1, [%3+8];\n\tld.shared.f64 %2, [%3+16];"
                 : "=d"(x), "=d"(y), "=d"(z) : "r"(a) : "memory");
}
template <typename T>
__device__ __forceinline__ void ring_put3p(uint32_t a, T x, T y, T z) {
  if constexpr (sizeof(T) == 4)
    asm volatile("st.shared.f32 [%0], %1;\n\tst.shared.f32 [%0+4], %2;\n\tst.shared.f32 [%0+8], %3;"
                 :: "r"(a), "f"(x), "f"(y), "f"(z) : "memory");
  else
    asm volatile("st.shared.f64 [%0], %1;\n\tst.shared.f64 [%0+8], %2;\n\tst.shared.f64 [%0+16], %3;"
                 :: "r"(a), "d"(x), "d"(y), "d"(z) : "memory");
}
template <bool kPacked, typename T>
__device__ __forceinline__ void rget(uint32_t a, T& x, T& y, T& z) {
  if constexpr (kPacked) ring_get3p<T>(a, x, y, z); else ring_get3(a, x, y, z);
}
template <bool kPacked, typename T>
__device__ __forceinline__ void rput(uint32_t a, T x, T y, T z) {
  if constexpr (kPacked) ring_put3p<T>(a, x, y, z); else ring_put3(a, x, y, z);
}

// 16-byte shared load reinterpreted as 4 floats or 2 doubles
__device__ __forceinline__ void lds16(uint32_t a, float* v) {
  asm volatile("ld.shared.v4.f32 {%0, %1, %2, %3}, [%4];" : "=f"(v[0]), "=f"(v[1]), "=f"(v[2]), "=f"(v[3])
               : "r"(a) : "memory");
}
__device__ __forceinline__ void lds16(uint32_t a, double* v) {
  asm volatile("ld.shared.v2.f64 {%0, %1}, [%2];" : "=d"(v[0]), "=d"(v[1]) : "r"(a) : "memory");
}
__device__ __forceinline__ void sts16(uint32_t a, const uint4 v) {
  asm volatile("st.shared.v4.u32 [%0], {%1, %2, %3, %4};" :: "r"(a), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w)
               : "memory");
}

// Steps per pass: every virtual lane sweeps its ncols columns plus the G-step stagger of
// its switch group; P >= 72 keeps the ring slot of a column written (virtual lane 63)
// before it is read (virtual lane 0 of the next pass). Long rows (ncols >= WF_RESCALE_COLS)
// get 64 more steps, so that virtual lane 63 has finished its whole row when virtual lane
// 0 of the next pass starts: the ring rescale then sees the full ring row.
constexpr int WF_RESCALE_COLS = kRescaleCols;
template <typename T = float>
__host__ __device__ inline int wf_pass_len(int ncols) {
  constexpr int SH = wf_sh<T>();
  if (ncols >= WF_RESCALE_COLS) return ncols + WF_G + 64 + SH;
  return (ncols + WF_G + SH > WF_MIN_P) ? ncols + WF_G + SH : WF_MIN_P;
}
// Haplotype code regions: 4 shifted copies per haplotype so that every lane reads its
// codes as aligned 32-bit words, 4 columns at a time (sized for the longer of the two
// passes' P: the FP64 rescue reads the FP32 pass's regions).
__host__ __device__ inline int wf_hc_copy_len(int ncols) {
  const int P = wf_pass_len<float>(ncols) > wf_pass_len<double>(ncols) ? wf_pass_len<float>(ncols)
                                                                        : wf_pass_len<double>(ncols);
  return ((int)WF_HC_FRONT + P + 24 + 3) & ~3;  // + prefetch distance
}

// Value u of coefficient field f of a TBlock<T> held as 16-byte words w[f * KC + chunk]
// (FP32: 4 floats per word, FP64: 2 doubles per word).
template <typename T>
__device__ __forceinline__ T coef_of(const uint4* w, int f, int u);
template <>
__device__ __forceinline__ float coef_of<float>(const uint4* w, int f, int u) {
  const uint4 x = w[f * WF_KC32 + u / 4];
  const uint32_t b = (u & 3) == 0 ? x.x : (u & 3) == 1 ? x.y : (u & 3) == 2 ? x.z : x.w;
  return __uint_as_float(b);
}
template <>
__device__ __forceinline__ double coef_of<double>(const uint4* w, int f, int u) {
  const uint4 x = w[f * WF_KC64 + u / 2];
  return (u & 1) == 0 ? __hiloint2double((int)x.y, (int)x.x) : __hiloint2double((int)x.w, (int)x.z);
}

// The 32-bit-aligned code pointer of a block for a lane whose first step is column -1 - gi
// (the all-PAD region when there is no block): copy k = (1 + gi) mod 4 of the haplotype's
// code region has column 0 at hap_off + k*(copy_len + 1), so the byte of column (-1 - gi)
// is 4-aligned.
template <typename T>
__device__ __forceinline__ const uint32_t* wf_code_ptr(const WfArgs2<T>& A, bool have, const BlkDesc& d, int gi,
                                                       int copy_len) {
  if (!have) return reinterpret_cast<const uint32_t*>(A.hcodes + A.pad_idx);
  const int k = (1 + gi) & 3;
  const uint32_t col0 = d.hap_off + (uint32_t)(k * (copy_len + 1));
  return reinterpret_cast<const uint32_t*>(A.hcodes + (col0 - 1u - (uint32_t)gi));
}

// ---- staged switch: per-warp staging slots, the 4 lanes of a switch group x 2 halves,
// each [4*KC coefficient words][flags word]
template <typename T> __host__ __device__ constexpr uint32_t wf_stage_slot() {
  return 16u * (WF_NCOEF * WfT<T>::KC + 1);
}
__device__ __forceinline__ void cp_async16(uint32_t s, const void* g) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" :: "r"(s), "l"(g) : "memory");
}
__device__ __forceinline__ void cp_async_wait_all() { asm volatile("cp.async.wait_all;" ::: "memory"); }
__device__ __forceinline__ void sts32(uint32_t a, uint32_t v) {
  asm volatile("st.shared.u32 [%0], %1;" :: "r"(a), "r"(v) : "memory");
}
__device__ __forceinline__ uint32_t lds32(uint32_t a) {
  uint32_t v;
  asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(a) : "memory");
  return v;
}
__device__ __forceinline__ uint4 lds128(uint32_t a) {
  uint4 v;
  asm volatile("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(a)
               : "memory");
  return v;
}
constexpr uint32_t WF_STG_NONE = 0xffffu;  // staged flags: no block
// staging bytes of one warp: the 4 lanes of a switch group x 2 halves (a group commits before
// the next one switches)
template <typename T> __host__ __device__ constexpr uint32_t wf_stage_bytes() {
  return 8u * wf_stage_slot<T>();
}

// Switch event of half H (staged): the block's priors go straight into the lane's prior
// table and its coefficients into the staging slot, both by cp.async (no register waits on
// them); the R-row position (or "no block") as the slot's flags. The table rows A..N are not
// read again before column 0, wf_sh + 1 + gi steps later. Returns the code pointer of the
// lane's first step (column -1 - gi - wf_sh: one word of PAD).
template <int H, typename T>
__device__ __forceinline__ const uint32_t* wf_stage(const WfArgs2<T>& A, uint32_t tab_s, uint32_t stg_s, bool have,
                                                    const BlkDesc& d, int& out_idx, int gi, int copy_len) {
  constexpr int KC = WfT<T>::KC;
  if (have) {
    const uint4* s4 = reinterpret_cast<const uint4*>(A.tab + d.tab_blk);
#pragma unroll
    for (int k = 0; k < 5 * KC; ++k) cp_async16(tab_s + 512u * k, s4 + WF_NCOEF * KC + k);
#pragma unroll
    for (int k = 0; k < WF_NCOEF * KC; ++k) cp_async16(stg_s + 16u * k, s4 + k);
    sts32(stg_s + 16u * WF_NCOEF * KC, (uint32_t)((d.flags >> WF_RROW_SHIFT) & 15));
    out_idx = (d.flags & BLK_LAST) ? d.out_idx : -1;
    return wf_code_ptr(A, true, d, gi, copy_len) - wf_sh<T>() / 4;
  }
  sts32(stg_s + 16u * WF_NCOEF * KC, WF_STG_NONE);
  out_idx = -1;
  return reinterpret_cast<const uint32_t*>(A.hcodes + A.pad_idx);
}

// Commit of half H, 4 steps after its switch event: the staged coefficients into the lane's
// registers, M = I = 0 and D = the virtual row 0 on the R row.
template <int H, typename T>
__device__ __forceinline__ void wf_commit(Lane<T>& L, uint32_t stg_s, T d0) {
  constexpr int K = WfT<T>::K;
  constexpr int KC = WfT<T>::KC;
  cp_async_wait_all();
  const uint32_t fl = lds32(stg_s + 16u * WF_NCOEF * KC);
  const bool have = fl != WF_STG_NONE;
  uint4 cw[WF_NCOEF * KC];
#pragma unroll
  for (int k = 0; k < WF_NCOEF * KC; ++k) cw[k] = have ? lds128(stg_s + 16u * k) : make_uint4(0u, 0u, 0u, 0u);
  const int rrow = have ? (int)fl : -1;
#pragma unroll
  for (int u = 0; u < K; ++u) {
    L.uu[u] = set_half<H>(L.uu[u], coef_of<T>(cw, 0, u)); L.ww[u] = set_half<H>(L.ww[u], coef_of<T>(cw, 1, u));
    L.ep[u] = set_half<H>(L.ep[u], coef_of<T>(cw, 2, u)); L.mu[u] = set_half<H>(L.mu[u], coef_of<T>(cw, 3, u));
    L.M[u] = set_half<H>(L.M[u], (T)0); L.I[u] = set_half<H>(L.I[u], (T)0);
    L.D[u] = set_half<H>(L.D[u], rrow == u ? d0 : (T)0);
  }
}

#ifndef PHMM_RS_TARGET
#define PHMM_RS_TARGET 112  // ring rescale: a ring row whose max is below 2^PHMM_RS_TRIG is scaled to ~2^PHMM_RS_TARGET
#endif
#ifndef PHMM_RS_TRIG
#define PHMM_RS_TRIG 104
#endif
#ifndef PHMM_RS_CAP
#define PHMM_RS_CAP 126  // saturation of the scaled ring row (a saturated pair goes to the FP64 rescue)
#endif
// Ring rescale helpers, used once per rescaled pass by the non-inlined
// wf_ring_rescale, so they do not perturb the register allocation of the hot loop.
// Max of the ring row (slots [0, ncols]: M, I, D of every slot; NOT the 4th word of a 16-byte
// FP32 slot, which no store writes and which therefore holds whatever an earlier stream left
// there -- reading it made the rescale, and so a pair's rounding and rescue decision, depend on
// the warp's history, i.e. on the batch the pair ran in), reduced over the warp.
// (the ring addresses travel as 64-bit values: that is the code generation measured, §4.8)
template <typename T>
__device__ __forceinline__ T ring_ld1(uint64_t a) {
  T x;
  if constexpr (sizeof(T) == 4) asm volatile("ld.shared.f32 %0, [%1];" : "=f"(x) : "r"((uint32_t)a) : "memory");
  else asm volatile("ld.shared.f64 %0, [%1];" : "=d"(x) : "r"((uint32_t)a) : "memory");
  return x;
}
template <typename T>
__device__ __forceinline__ void ring_st1(uint64_t a, T x) {
  if constexpr (sizeof(T) == 4) asm volatile("st.shared.f32 [%0], %1;" :: "r"((uint32_t)a), "f"(x) : "memory");
  else asm volatile("st.shared.f64 [%0], %1;" :: "r"((uint32_t)a), "d"(x) : "memory");
}

template <typename T, bool kPacked>
__device__ __forceinline__ T wf_ring_max(uint64_t ring_a, int ncols, int lane) {
  constexpr uint32_t RS = kPacked ? 3u * (uint32_t)sizeof(T) : ring_slot_bytes<T, false>();
  T m = 0;
  __syncwarp();
  if constexpr (sizeof(T) == 4 && RS == 16) {
    // one 16-byte load per slot (consecutive lanes on consecutive slots: 4 wavefronts per warp
    // load, no conflicts), the three values of the slot
    for (int j = lane; j <= ncols; j += 32) {
      float x, y, z;
      ring_get3((uint32_t)ring_a + 16u * (uint32_t)j, x, y, z);
      m = fmax(m, fmax(x, fmax(y, z)));
    }
  } else {
    const int nw = (ncols + 1) * (int)(RS / sizeof(T));
    for (int k = lane; k < nw; k += 32) m = fmax(m, ring_ld1<T>(ring_a + (uint64_t)(k * (int)sizeof(T))));
  }
  for (int o = 16; o > 0; o >>= 1) m = fmax(m, __shfl_xor_sync(0xffffffffu, m, o));
  return m;
}

// Ring slots [0, ncols] *= 2^sh, saturating at 2^PHMM_RS_CAP; true if any value saturated
// (cannot happen with the exact row max; such a pair would go to the FP64 rescue).
template <typename T, bool kPacked>
__device__ __forceinline__ bool wf_ring_scale(uint64_t ring_a, int ncols, int lane, int sh) {
  constexpr uint32_t RS = kPacked ? 3u * (uint32_t)sizeof(T) : ring_slot_bytes<T, false>();
  const T f = (T)__int_as_float((127 + sh) << 23);
  const T cap = (T)__int_as_float((127 + PHMM_RS_CAP) << 23);
  bool sat = false;
  __syncwarp();
  if constexpr (sizeof(T) == 4 && RS == 16) {
    // slot-wise 16-byte loads and stores (the 4th word, padding, is written back unchanged)
    for (int j = lane; j <= ncols; j += 32) {
      const uint32_t a = (uint32_t)ring_a + 16u * (uint32_t)j;
      float v[4];
      lds16(a, v);
#pragma unroll
      for (int t = 0; t < 3; ++t) {
        v[t] *= f;
        sat |= v[t] > cap;
        v[t] = fmin(v[t], cap);
      }
      sts16(a, make_uint4(__float_as_uint(v[0]), __float_as_uint(v[1]), __float_as_uint(v[2]), __float_as_uint(v[3])));
    }
  } else {
    // the slots as a flat array of T: consecutive lanes on consecutive words, no bank conflicts
    const int nw = (ncols + 1) * (int)(RS / sizeof(T));
    for (int k = lane; k < nw; k += 32) {
      const uint64_t a = ring_a + (uint64_t)(k * (int)sizeof(T));
      T x = ring_ld1<T>(a);
      x *= f;
      sat |= x > cap;
      x = fmin(x, cap);
      ring_st1<T>(a, x);
    }
  }
  __syncwarp();
  return __any_sync(0xffffffffu, sat);
}

// The ring rescale decision of one pass, all lanes: if lane 0's block
// continues the pair of the ring row (`cont` of lane 0) and the row's max has decayed below
// 2^104 (but not below 2^-90), scale the row to 2^112 and add the power of 2 to the pair's
// exponent slot (lane 0; a saturated row marks the pair for the FP64 rescue). Not inlined,
// so that it leaves the hot loop's register allocation alone.
template <typename T, bool kPacked>
__device__ __noinline__ void wf_ring_rescale(uint64_t ring_a, int ncols, int lane, bool cont, int32_t* exp_slot) {
  if (!__shfl_sync(0xffffffffu, (int)cont, 0)) return;
  const float rm = (float)wf_ring_max<T, kPacked>(ring_a, ncols, lane);
  if (!(rm > 0.f && rm <= 3.0e38f)) return;
  const int E = ilogbf(rm);
  if (E < -90 || E >= PHMM_RS_TRIG) return;
  const int sh = min(PHMM_RS_TARGET - E, 126);
  const bool sat = wf_ring_scale<T, kPacked>(ring_a, ncols, lane, sh);
  if (lane == 0 && exp_slot) *exp_slot += sat ? -(1 << 24) : sh;
}

// Work item it of the launch -> its bin and pair-aligned block range [s, e) (all lanes; e <= s:
// empty). Bins by binary search in item_start (descending with LPT order).
template <typename T>
__device__ __forceinline__ void wf_item(const WfArgs2<T>& A, unsigned long long it, int lane, int& bin, int64_t& s,
                                        int64_t& e) {
  int lo_ = A.bin_lo, hi_ = A.bin_hi - 1;
  if (A.lpt) {  // item_start descending in the bin index: the smallest bin with item_start <= it
    while (lo_ < hi_) {
      const int mid = (lo_ + hi_) >> 1;
      if (A.item_start[mid] <= it) hi_ = mid; else lo_ = mid + 1;
    }
  } else {      // ascending: the largest bin with item_start <= it
    while (lo_ < hi_) {
      const int mid = (lo_ + hi_ + 1) >> 1;
      if (A.item_start[mid] <= it) lo_ = mid; else hi_ = mid - 1;
    }
  }
  bin = lo_;
  const int64_t b0 = (int64_t)A.bin_start[bin], b1 = (int64_t)A.bin_start[bin + 1];
  const int64_t k = (int64_t)(it - A.item_start[bin]);
  const int64_t nbig = (int64_t)A.bin_nbig[bin];
  if (k < nbig) {
    s = b0 + k * A.chunk_blocks;
    e = s + A.chunk_blocks;
  } else {
    s = b0 + nbig * A.chunk_blocks + (k - nbig) * A.chunk_small;
    e = s + A.chunk_small;
  }
  if (e > b1) e = b1;
  auto advance = [&](int64_t x) -> int64_t {  // first block of the first pair starting at or after x
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
}

template <typename T>
__device__ __forceinline__ unsigned long long wf_claim(const WfArgs2<T>& A, int lane) {
  unsigned long long it = 0;
  if (lane == 0) it = A.launch_items[0] + atomicAdd(A.item_counter, 1u);
  return __shfl_sync(0xffffffffu, it, 0);
}

// One warp streams through blocks [s, s+nblk) of one bin (ncols columns each). The stream's
// first block s lives in a per-warp shared-memory slot (read at switch events only), which
// keeps it out of the registers of the hot loop (212 instead of 218
// registers).
// kLong: the launch of the long-row bins (the only one with the ring rescale compiled in).
template <typename T, bool kLong>
__device__ __forceinline__ void wf_stream(const WfArgs2<T>& A, uint32_t ptab_s, uint32_t ring_base_s,
                                          uint32_t xbuf_s, uint32_t seg_s, uint32_t stg_s, int lane, int64_t s,
                                          int nblk, int bin) {
  const int ncols = bin * A.bucket;
  int64_t* seg = reinterpret_cast<int64_t*>(__cvta_shared_to_generic(seg_s));
  __syncwarp();
  if (lane == 0) seg[0] = s;
  __syncwarp();
  // FP32 long-row streams start LEAD idle virtual lanes late: the pass-padded (rescalable) pairs,
  // which sit at multiples of 64 blocks from every stream start (padded_nb, k_iota_keys), then
  // start half a pass into a pass, so a 1,000-row read crosses two pass boundaries (rows ~250 and
  // ~760) for its ring rescale, at the same rows in every batch (R14)
  constexpr int LEAD = (kLong && sizeof(T) == 4) ? 32 : 0;
  auto phys = [&](int b) -> int64_t { return seg[0] + b - LEAD; };  // b: virtual block index
  using V = typename WfT<T>::V;
  constexpr int K = WfT<T>::K;
  constexpr int PER = 16 / sizeof(T);
  constexpr int G = WF_G;            // virtual lanes per switch group
  constexpr int NGRP = 64 / G;       // switch events per pass
  constexpr int LPG = G / 2;         // physical lanes per group
  constexpr uint32_t RS = ring_slot_bytes<T, kLong>();
  // ring slot of column c = ring_s + RS * (c + 1); staged switches also read SH slots in
  // front (never written: zero) for the PAD columns before a block
  constexpr int SH = wf_sh<T>();
  const uint32_t ring_s = ring_base_s + RS * (uint32_t)SH;
  const int grp = lane / LPG;
  const int giA = 2 * (lane % LPG), giB = giA + 1;  // position of each half inside its group
  const T d0 = (T)ldexp(1.0, WfT<T>::kScaleExp) / (T)ncols;  // virtual row 0
  const int P = wf_pass_len<T>(ncols);                        // multiple of 4 (ncols is)
  int npass = (nblk + LEAD + 63) >> 6;
  const int copy_len = wf_hc_copy_len(ncols);
  Lane<T> L;
#pragma unroll
  for (int u = 0; u < K; ++u) {
    L.uu[u] = L.ww[u] = L.ep[u] = L.mu[u] = vzero<V>();
    L.M[u] = L.I[u] = L.D[u] = vzero<V>();
  }
  const uint32_t* pA = reinterpret_cast<const uint32_t*>(A.hcodes + A.pad_idx);  // next code word
  const uint32_t* pB = pA;
  constexpr uint32_t kPadW = (uint32_t)(WF_PAD * WF_CB) * 0x01010101u;  // four PAD codes
  // code words: current group, next group, the one after (prefetch distance 2 groups)
  uint32_t wA = kPadW, wB = kPadW, wA_nx = kPadW, wB_nx = kPadW, wA_nx2 = kPadW, wB_nx2 = kPadW;
  int outA = -1, outB = -1;
  V upM = vzero<V>(), upI = vzero<V>(), upD = vzero<V>(), dgM = vzero<V>(), dgI = vzero<V>(), dgD = vzero<V>();
  const uint32_t tabA_s = ptab_s + 16u * lane;                              // [code][chunk][lane] 16 B
  const uint32_t tabB_s = ptab_s + 16u * (WF_NCODE * WfT<T>::KC * 32 + lane);   // half B
  const int src = (lane + 31) & 31;
  const bool is31 = lane == 31;
  const uint32_t stgA_s = stg_s + wf_stage_slot<T>() * (uint32_t)(2 * (lane & 3));
  const uint32_t stgB_s = stgA_s + wf_stage_slot<T>();
  (void)stgA_s; (void)stgB_s;
  int c0 = -(1 << 20);    // (uniform) column of virtual lane 0 (lane 0, half A)
  int c31B = -(1 << 20);  // (uniform) column of virtual lane 63 (lane 31, half B)
  T rvM = 0, rvI = 0, rvD = 0;  // lane 31: ring slot for virtual lane 0's next column
  BlkDesc dnA, dnB;  // descriptors of the lane's next blocks (loaded one pass ahead)
  dnA.tab_blk = 0; dnA.hap_off = 0; dnA.out_idx = -1; dnA.pad = 0; dnA.flags = 0;
  dnB = dnA;
  if (2 * lane >= LEAD && 2 * lane < nblk + LEAD) dnA = A.blk[phys(2 * lane)];
  if (2 * lane + 1 >= LEAD && 2 * lane + 1 < nblk + LEAD) dnB = A.blk[phys(2 * lane + 1)];

  // Ring rescale (FP32 pass, long rows only): when a pair continues from
  // virtual lane 63 of one pass into virtual lane 0 of the next, its ring row (the row
  // above virtual lane 0, complete by then: wf_pass_len) is multiplied in place by 2^sh,
  // sh chosen from the row's max, so long reads stay inside the FP32 range; sh is added
  // to the pair's exponent slot. Costs nothing in the hot loop: the row max is read from the
  // ring itself once per pass.
#ifndef PHMM_RING_RESCALE
#define PHMM_RING_RESCALE 1
#endif
  constexpr bool rescale = kLong && PHMM_RING_RESCALE && sizeof(T) == 4;  // long-row launch: ncols >= WF_RESCALE_COLS

  auto step = [&](const int r, const uint32_t wA, const uint32_t wB) {
    if (is31) rget<ring_packed<T, kLong>()>(ring_s + RS * (uint32_t)(c0 + 2), rvM, rvI, rvD);
    // code byte r (= code*WF_CB) placed in byte 1 -> the code's rows in the table
    // code stride of this pass's table relative to the code byte's (powers of 2)
    constexpr int kKC = WfT<T>::KC;
    auto cs = [](uint32_t o) -> uint32_t {
      if constexpr (kKC == WF_KC32) return o;
      else if constexpr (kKC > WF_KC32) return o * (uint32_t)(kKC / WF_KC32);
      else return o / (uint32_t)(WF_KC32 / kKC);
    };
    const uint32_t oA = cs(__byte_perm(wA, 0, 0x4404 + (r << 4))), oB = cs(__byte_perm(wB, 0, 0x4404 + (r << 4)));
    T prA[K], prB[K];
#pragma unroll
    for (int ch = 0; ch < WfT<T>::KC; ++ch) {
      lds16(tabA_s + oA + 512u * ch, prA + PER * ch);
      lds16(tabB_s + oB + 512u * ch, prB + PER * ch);
    }
    wf_column<T>(L, prA, prB, dgM, dgI, dgD, upM, upI);
    constexpr int LR = K - 1;  // last row of a block
    const T m3a = lo(L.M[LR]), i3a = lo(L.I[LR]), d3a = lo(L.D[LR]);
    const T m3b = hi(L.M[LR]), i3b = hi(L.I[LR]), d3b = hi(L.D[LR]);
    // half B of lane-1 -> half A of lane; lane 31 sends the ring slot instead (virtual 63 -> 0)
    const T sM = is31 ? rvM : m3b;
    const T sI = is31 ? rvI : i3b;
    const T sD = is31 ? rvD : d3b;
    if (is31 && (unsigned)(c31B + 1) <= (unsigned)ncols)  // -1 <= c31B < ncols
      rput<ring_packed<T, kLong>()>(ring_s + RS * (uint32_t)(c31B + 1), m3b, i3b, d3b);
    dgM = upM; dgI = upI; dgD = upD;
    // next step: half A's row above = lane-1's half B; half B's row above = this lane's half A
#if PHMM_XCHG_SMEM
    // design A (Listing 2a, L20@44): write, synchronise, read through a
    // shared-memory line buffer (one slot per lane) instead of the shuffle
    rput<ring_packed<T, kLong>()>(xbuf_s + RS * (uint32_t)lane, sM, sI, sD);
    __syncwarp();
    T xM, xI, xD;
    rget<ring_packed<T, kLong>()>(xbuf_s + RS * (uint32_t)src, xM, xI, xD);
    __syncwarp();
    upM = pk(xM, m3a);
    upI = pk(xI, i3a);
    upD = pk(xD, d3a);
#else
    __syncwarp();
    upM = pk(__shfl_sync(0xffffffffu, sM, src), m3a);
    upI = pk(__shfl_sync(0xffffffffu, sI, src), i3a);
    upD = pk(__shfl_sync(0xffffffffu, sD, src), d3a);
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
    step(0, wA, wB); step(1, wA, wB); step(2, wA, wB); step(3, wA, wB);
  };
  // groups g, g+1, g+2 with the code words in three fixed registers: each word is loaded two
  // groups before the group that uses it and never moved (the rotation of group4 reads every
  // load one group after issuing it, which waits on it when it misses in L1). Used for the
  // long segment of a pass by the FP32 long-row kernel only: C4 kernel +5 %, while the
  // FP32 short-row kernel (-O1) loses 3 % on C2 and the FP64 kernel 1 % with it
  // (profiles/r02_ab_unroll3.txt).
#ifndef PHMM_UNROLL3_F64
#define PHMM_UNROLL3_F64 0
#endif
  constexpr bool kUnroll3 = (kLong && sizeof(T) == 4) || (PHMM_UNROLL3_F64 && sizeof(T) == 8);
  auto group12 = [&](uint32_t& a0, uint32_t& a1, uint32_t& a2, uint32_t& b0, uint32_t& b1, uint32_t& b2) {
    a2 = __ldg(pA); b2 = __ldg(pB); ++pA; ++pB;
    step(0, a0, b0); step(1, a0, b0); step(2, a0, b0); step(3, a0, b0);
    a0 = __ldg(pA); b0 = __ldg(pB); ++pA; ++pB;
    step(0, a1, b1); step(1, a1, b1); step(2, a1, b1); step(3, a1, b1);
    a1 = __ldg(pA); b1 = __ldg(pB); ++pA; ++pB;
    step(0, a2, b2); step(1, a2, b2); step(2, a2, b2); step(3, a2, b2);
  };

  // Staged switch events: group e switches at pass step 8e (its lanes start column
  // -1 - gi - SH), issuing the next block's table by cp.async, and commits the coefficients
  // and the initial state at pass step 8e + 4, before any column whose result is used (the
  // first is column -1 of gi = 0, at that step). Events every 4 steps: 2e switches group e,
  // 2e + 1 commits it; the last segment runs the rest of the pass.
  for (int q = 0; q <= npass; ++q) {
#pragma unroll 1
    for (int e2 = 0; e2 < 2 * NGRP; ++e2) {
      const int e = e2 >> 1;
      if (e2 == 0) {
        c0 = -1 - SH;  // virtual lane 0 starts its pass
        if constexpr (rescale) {
          const bool cont = (q < npass) && (q * 64 >= LEAD) && (q * 64 < nblk + LEAD) && !(dnA.flags & BLK_FIRST) &&
                            (dnA.flags & BLK_RESC) && ncols >= WF_RESCALE_COLS;
          wf_ring_rescale<T, ring_packed<T, kLong>()>((uint64_t)ring_s, ncols, lane, cont,
                                                      A.exp_out ? A.exp_out + dnA.out_idx : nullptr);
        }
      }
      if (e2 == 2 * NGRP - 2) c31B = -1 - (G - 1) - SH;  // virtual lane 63
      if (grp == e) {
        if (!(e2 & 1)) {  // switch event of virtual lanes 8e..8e+7 = lanes 4e..4e+3
          const int bA = q * 64 + 2 * lane, bB = bA + 1;
          const BlkDesc dA = dnA, dB = dnB;  // loaded one pass ago (pass 0: before the loop)
          // (a filler block after a pass-aligned pair is an idle lane)
          // (fillers only occur in long-row FP32 streams: the short-row kernel's code stays as it was,
          // its register allocation is sensitive even to switch-path changes)
          constexpr bool kFill = LEAD > 0;
          const bool hA = (q < npass) && (bA >= LEAD) && (bA < nblk + LEAD) && !(kFill && (dA.flags & BLK_FILLER));
          const bool hB = (q < npass) && (bB >= LEAD) && (bB < nblk + LEAD) && !(kFill && (dB.flags & BLK_FILLER));
          if (outA >= 0) A.out[outA] = lo(L.D[K - 1]);  // S row: the last-row M+I sum (L20@2262)
          if (outB >= 0) A.out[outB] = hi(L.D[K - 1]);
          pA = wf_stage<0, T>(A, tabA_s, stgA_s, hA, dA, outA, giA, copy_len);
          pB = wf_stage<1, T>(A, tabB_s, stgB_s, hB, dB, outB, giB, copy_len);
          // the first code word of a block (columns -1-gi-4 .. -2-gi) is PAD
          wA_nx = kPadW; wA_nx2 = __ldg(pA + 1); pA += 2;
          wB_nx = kPadW; wB_nx2 = __ldg(pB + 1); pB += 2;
          if (bA + 64 >= LEAD && bA + 64 < nblk + LEAD) dnA = A.blk[phys(bA + 64)];
          if (bB + 64 >= LEAD && bB + 64 < nblk + LEAD) dnB = A.blk[phys(bB + 64)];
        } else {  // commit of the group that switched 4 steps ago
          wf_commit<0, T>(L, stgA_s, d0);
          wf_commit<1, T>(L, stgB_s, d0);
        }
      }
      int ngroups = (e2 < 2 * NGRP - 1) ? 1 : (q < npass ? (P - (2 * NGRP - 1) * 4) / 4 : 0);
      if constexpr (kUnroll3) {
        if (ngroups >= 3) {
          uint32_t a0 = wA_nx, a1 = wA_nx2, a2, b0 = wB_nx, b1 = wB_nx2, b2;
#pragma unroll 1
          for (; ngroups >= 3; ngroups -= 3) group12(a0, a1, a2, b0, b1, b2);
          wA_nx = a0; wA_nx2 = a1; wB_nx = b0; wB_nx2 = b1;
        }
      }
#pragma unroll 1
      for (int k = 0; k < ngroups; ++k) group4();
    }
  }
}

// The kernels are defined in wf.cu (-Xptxas -O1) and wf_long32.cu (the FP32 long-row
// kernel, -O3): the optimisation level each is fastest at.
// phmm_lib.cu reaches them through these host functions.
// shared memory of one warp: its prior tables and its ring
template <typename T, bool kLong = false> __host__ __device__ size_t wf_warp_smem(int ring_len) {
  // prior tables, the staging slots, the ring (+ wf_sh front slots),
  // (design-A ablation only) the exchange line buffer; a multiple of 16 bytes so that every
  // warp's tables stay 16-byte aligned
  const size_t b = (size_t)2 * WF_NCODE * WfT<T>::KC * 32 * 16 + (size_t)wf_stage_bytes<T>() +
                   (size_t)(ring_len + wf_sh<T>() + (PHMM_XCHG_SMEM ? 32 : 0)) * ring_slot_bytes<T, kLong>() +
                   32;  // the stream's first block (wf_stream)
  return (b + 15) & ~(size_t)15;
}
template <typename T> cudaError_t wf_occupancy(bool long_rows, int warps, size_t smem, int* blocks_per_sm);
cudaError_t wf_set_max_smem(int smem_optin);
template <typename T>
cudaError_t wf_launch(bool long_rows, unsigned grid, int warps, size_t smem, cudaStream_t stream,
                      const WfArgs2<T>& args);

#ifdef PHMM_DEFINE_WF
template <typename T, bool kLong>
__global__ void __launch_bounds__(WF_WARPS * 32, WfT<T>::MINB) k_wavefront(WfArgs2<T> A) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  const int lane = threadIdx.x & 31;
  const int wib = threadIdx.x >> 5;
  // per warp: prior tables [2 halves][6 codes][KC chunks][32 lanes] x 16 B, then the ring
  constexpr uint32_t kTabBytes = 2 * WF_NCODE * WfT<T>::KC * 32 * 16;
  const uint32_t per_warp = (uint32_t)wf_warp_smem<T, kLong>(A.ring_len);
  unsigned char* base = smem_raw + (size_t)wib * per_warp;
  for (uint32_t i = 4 * lane; i < per_warp; i += 128) *reinterpret_cast<uint32_t*>(base + i) = 0u;
  __syncwarp();
  const uint32_t ptab_s = smem_addr(base), stg_s = ptab_s + kTabBytes, ring_s = stg_s + wf_stage_bytes<T>();
  const uint32_t xbuf_s = ring_s + (uint32_t)(A.ring_len + wf_sh<T>()) * ring_slot_bytes<T, kLong>();  // design A only
  const uint32_t seg_s = (ptab_s + per_warp - 32u) & ~7u;   // the stream's first block (last 32 B)
  // work items of the launch, claimed from an atomic counter
  const unsigned long long it1 = A.launch_items[1];
  while (true) {
    const unsigned long long it = wf_claim(A, lane);
    if (it >= it1) break;
    int bin;
    int64_t s, e;
    wf_item(A, it, lane, bin, s, e);
    if (e <= s) continue;
    wf_stream<T, kLong>(A, ptab_s, ring_s, xbuf_s, seg_s, stg_s, lane, s, (int)(e - s), bin);
    __syncwarp();
  }
}
#endif  // PHMM_DEFINE_WF

}  // namespace phmm
