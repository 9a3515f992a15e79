// phmm_common.cuh -- constants, descriptors and device helpers shared by the libphmm kernels (sm_100a).
//
// PRODUCT PATH. Shares no code with oracle/ (which is test infrastructure).
//
// What is computed: the PairHMM forward recurrence, Eq. 6 of PAPER.md
// (L18@541, §III-B), for every (read, haplotype) pair, terminated by the sum
// of the last row of M and I (L20@2262, §IV-C.1), with the GATK 3.6 Phred
// mapping (L22@4113) -- see include/phmm.h and DESIGN.md §2.
//
// How (DESIGN.md §4 -- differs from the paper's one-warp-per-pair PH2):
//  * "tall stream" layout: every pair is laid out as a whole number of K-row
//    BLOCKS: [Z..Z][R][read rows 1..m][S] (at least one Z row) where the pad rows
//    are plain rows of the same recurrence (the kernel's rescaled 5-op form,
//    wavefront.cuh) with special coefficients:
//      Z  (zero)   : T = u = w = ep' = mu = 0      -> M = D = 0 (I = M of the row
//                    above: finite garbage that the next Z/R row, with ep' = 0, drops)
//      R  (reset)  : T = 0, ep' = 0, mu = 1, boundary D(.,0) = s/ncols
//                    -> M = I = 0, D = s/ncols on every column: the virtual row 0
//                       of Eq. 6 (D(0,j) = 1/N, scaled by s)
//      S  (sum)    : T = 1/a_m, u = a_m/b_m, w = 0, mu = 1
//                    -> M(j) = M(m,j-1) + I(m,j-1) (unscaled), D(j) = sum_{j'<j} M(j'),
//                       so D_S(N+2) = sum_{j=1..N} M(m,j) + I(m,j)
//    The termination sum of L20@2262 therefore falls out of the recurrence
//    itself, read as D of the S row at column N+2 (0-based c = N+1), and
//    consecutive pairs can be stacked into one tall DP: a Z row followed by a
//    Z/R row ignores whatever (finite) values are above it. One warp streams
//    through a long sequence of blocks of equal column count (a length bin)
//    without draining between pairs.
//  * lane l of a warp owns one K-row block per "pass" (blocks l, l+32, ...),
//    processes one column per step (a K-row column tile), lags lane l-1 by
//    one step, receives the (M,I,D) of the row above by __shfl_sync
//    (the paper's Design B, Fig. 6b / Listing 2b, L20@44), and lane 31 hands
//    its last row to lane 0 of the next pass through a per-warp shared-memory
//    ring indexed by column (the stripe carry).
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace phmm {

// ---------------------------------------------------------------- constants
constexpr int kMinCols = 40;        // ring delay needs ncols > 32
constexpr int kMaxHapLen = 4094;    // FP32/FP64 ring in shared memory
constexpr int kMaxReadLen = 1 << 20;  // longest read a pair may use (include/phmm.h)
constexpr int kMaxBins = 4200;      // ncols / bucket <= kMaxBins
constexpr int kNcolsComplement = 1 << 20;  // > any column count: min(ncols) travels as max(this - ncols)

// error flag bits (device) -> phmm_status
enum : uint32_t {
  ERR_BASE = 1u, ERR_QUAL = 2u, ERR_EMPTY = 4u, ERR_INDEX = 8u, ERR_ARG = 16u
};

// base -> one-hot code; N matches everything; 0xff = invalid
__device__ __forceinline__ uint32_t base_code(uint8_t b) {
  switch (b) {
    case 'A': return 1u;
    case 'C': return 2u;
    case 'G': return 4u;
    case 'T': return 8u;
    case 'N': return 15u;
    default: return 0xffu;
  }
}

// Per-block descriptor in the bin-sorted block sequence (16 bytes).
struct BlkDesc {
  uint32_t tab_blk;   // block index in the coefficient table
  uint32_t hap_off;   // offset of the haplotype in the code array
  int32_t out_idx;    // output slot of the pair (valid on its last block)
  uint16_t pad;       // unused (keeps the descriptor 16 bytes)
  uint16_t flags;     // bit0: last block of its pair, bit1: first block of its pair
};
static_assert(sizeof(BlkDesc) == 16, "BlkDesc must be 16 bytes");
constexpr uint16_t BLK_LAST = 1, BLK_FIRST = 2;
// block of a pair of more than 64 blocks (FP32: reads of more than 509 bases), the only pairs the
// ring rescale of the long-row kernel may rescale: a pair that fits in one pass
// is never rescaled, so its result cannot depend on where the pass boundaries fall in it
constexpr uint16_t BLK_RESC = 4;
constexpr int kRescaleMinBlocks = 65;
// filler block after such a pair: the FP32 pass pads every rescalable pair of a long-row bin to a
// whole number of 64-block passes and sorts them to the front of their bin, so each starts a pass
// (virtual lane 0) in any stream and its pass boundaries fall at the same rows in every batch
// (R14); a filler is an idle lane (no table, PAD codes)
constexpr uint16_t BLK_FILLER = 8;
constexpr int kRescaleCols = 768;  // long-row kernel (ring rescale) from this many columns on
__host__ __device__ inline int padded_nb(int nb, int ncols, int align) {
  return (align && ncols >= kRescaleCols && nb >= kRescaleMinBlocks) ? ((nb + 63) & ~63) : nb;
}

__host__ __device__ constexpr int ceil_div(int64_t a, int64_t b) { return (int)((a + b - 1) / b); }

__host__ __device__ inline int ncols_of(int n, int bucket) {
  const int c = ((n + 2 + bucket - 1) / bucket) * bucket;
  const int lo = ((kMinCols + bucket - 1) / bucket) * bucket;
  return c < lo ? lo : c;
}
__host__ __device__ inline int bin_of_ncols(int ncols, int bucket) { return ncols / bucket; }
// rows: f >= 1 Z rows, R, m read rows, S  ->  nb*K >= m + 3
template <int K>
__host__ __device__ inline int nblocks_of(int m) { return (m + 3 + K - 1) / K; }

// Phred -> error probability, 10^(-q/10), in the table's precision.
template <typename T>
__device__ __forceinline__ T qual_err(uint32_t q);
template <>
__device__ __forceinline__ float qual_err<float>(uint32_t q) {
  return (float)exp10(-(double)q / 10.0);  // computed in double, rounded once
}
template <>
__device__ __forceinline__ double qual_err<double>(uint32_t q) {
  return exp10(-(double)q / 10.0);
}

}  // namespace phmm
