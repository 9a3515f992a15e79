// phmm_lib.cu -- host side of libphmm: the C ABI of include/phmm.h.
//
// PRODUCT PATH (no oracle code). Orchestrates, on one stream:
//   validate + haplotype codes -> per pass: bin pairs by column count,
//   per-read coefficient tables (the per-read precompute step),
//   block allocation per bin (the length-binned scheduler, §8a-3), the
//   wavefront kernel (§8a-4), finalize (§8a-5) and, for FP32, the FP64
//   rescue of underflowing pairs (§8a-6). See DESIGN.md §3-§5.
#include <cub/device/device_radix_sort.cuh>
#include <cub/device/device_scan.cuh>

#include <algorithm>
#include <chrono>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <condition_variable>
#include <deque>
#include <map>
#include <set>
#include <mutex>
#include <thread>
#include <vector>
#include <new>

#include <nvtx3/nvToolsExt.h>

#include "../../include/phmm.h"
#include "phmm_device.cuh"
#include "host_stage.h"
#include "stream_prep.cuh"
#include "sw.cuh"

using namespace phmm;

namespace {

enum BufId {
  B_READ_BASES, B_BQ, B_IQ, B_DQ, B_GQ, B_ROFF, B_HAP, B_HOFF, B_PAIRS,  // host-variant inputs
  B_HCODES, B_SCAL,                                                       // codes, scalars
  B_PAIR_BIN, B_PAIR_NB, B_BINS, B_ITEM_NB, B_ITEM_OFF, B_SCAN_TMP,
  B_TAB32, B_TAB64, B_BLK, B_OUT32, B_OUT64, B_RLIST, B_ITEM_READ, B_PAIR_ITEM,
  B_OUT_LOG10, B_OUT_STATUS, B_HNC, B_HC_OFF,
  B_SW_REF, B_SW_ROFF, B_SW_ALT, B_SW_AOFF, B_SW_TASKS, B_SW_RES, B_SW_OPS,  // SW host-variant staging
  B_SW_BTSZ, B_SW_BTOFF, B_SW_OPCAP, B_SW_OPOFF, B_SW_BT, B_SW_KEYS, B_SW_VALS, B_SW_OPTMP, B_SW_NOPS,
  B_SW_NOPOFF,
  B_SKEYS, B_SVALS, B_NBS, B_BLKOFF, B_SORT_TMP, B_EXP32,
  B_CH_ROFF, B_CH_HOFF, B_CH_PAIRS,            // chunked device call: one chunk's offsets / rebased pairs
  B_DEDUP,                                       // rescue pass: head flags + their scan (one table per read)
  B_CH_RANGES,                                   // chunked device call: read / haplotype index range per chunk
  B_UNDERFLOW,                                   // pairs of the call whose FP64 sum underflowed
  B_RLIST_CH,                                    // a chunk's own rescue list (per set: compute_one in a pipelined call)
  B_COUNT
};

struct Buf {
  void* p = nullptr;
  size_t n = 0;
};

struct AsyncQueue;

// NVTX range around a host phase of the path (a no-op unless a profiler is attached):
// "phmm:validate", "phmm:fp32_pass", "phmm:rescue", "phmm:fp64_pass", "phmm:chunk",
// "phmm:h2d", "phmm:d2h", "phmm:submit_run" show up on an Nsight timeline.
struct Nvtx {
  explicit Nvtx(const char* name) { nvtxRangePushA(name); }
  ~Nvtx() { nvtxRangePop(); }
};

// device scalars written by the prep kernels, read back in one D2H copy
struct Scalars {
  uint32_t err;
  int32_t max_ncols;
  int32_t min_ncols_c;  // kMinColsComplement - smallest column count (0-initialised max)
  unsigned long long cells;
  unsigned long long padded_cells;
  unsigned long long total_blocks;
  int64_t n_rescue;
  unsigned long long n_underflow;
  unsigned int item_counter[2];  // work-item counters of the (at most 2) wavefront launches
};

constexpr int kEvents = 11;
constexpr int kThreads = 256;
// device path: batches of more pairs than this run as consecutive chunks (compute_dev)
constexpr int64_t kDevChunkPairs = 1ll << 23;

struct PhaseMs {
  float prep, wf, fin, resc;
};

struct PassInfo {
  unsigned long long cells = 0, padded_cells = 0, total_blocks = 0;
  int max_ncols = 0, min_ncols = 0;
};


// one chunk of a pipelined host call (compute_host_pipe)
struct PipeChunk {
  int64_t p0, p1;       // pairs [p0, p1)
  int64_t rlo, rhi;     // read index range the chunk's pairs use
  int64_t hlo, hhi;     // haplotype index range
  int64_t rend, hend;   // reads [0, rend) and haplotypes [0, hend) are on the device before it runs
};

}  // namespace

struct phmm_ctx {
  int device = 0;
  cudaStream_t stream = nullptr;        // the stream calls enqueue on (phmm_set_stream)
  cudaStream_t owned_stream = nullptr;  // the context's own stream, if it made one
  phmm_precision prec = PHMM_PREC_FP32_RESCUE;
  uint32_t flags = 0;
  int bucket = 4;
  int nsm = 148;
  Buf buf[4 * B_COUNT];                  // [region][id]: 0 shared + chunk set 0, 1 chunk set 1, 2-3 async inputs
  int set = 0;                            // the buffer set the current chunk uses
  int iset = 0;                           // input buffers: 0 = the synchronous calls', 1 / 2 = async batches'
  cudaStream_t pf_stream = nullptr;       // async calls: the next batch's input prefetch
  cudaEvent_t pf_ev = nullptr;
  bool in_xjob = false;                   // the worker is running a no-copy batch (maybe_prefetch)
  uint32_t* gerr = nullptr;               // pipelined call: the call-wide device error word
  cudaStream_t stream2 = nullptr;         // pipelined call: the second chunk stream (odd chunks)
  int smem_per_sm = 0, smem_reserved = 0, smem_optin = 0;  // bytes (device attributes)
  Scalars* host_scal = nullptr;  // pinned
  int64_t* host_sizes = nullptr;  // pinned, 2 values
  int64_t sw_ops_cap = 0;         // last SW call: sum over tasks of M + N
  cudaEvent_t ev[kEvents] = {};
  Stager stage;                           // host variant: pinned staging of pageable buffers
  std::map<uint64_t, int> occ;            // wavefront occupancy per (precision, launch class, warps, smem)
  std::mutex run_mu;                      // one compute at a time (caller threads and the submit worker)
  AsyncQueue* aq = nullptr;               // phmm_submit / phmm_wait (created on first submit)
  size_t sw_smem_set = 0;                 // dynamic shared memory the SW fill kernel is allowed
  phmm_stats st{};
  PhaseMs acc{};                          // per-phase times summed over a call's chunks
  int launches = 0;
  int64_t chunk_pairs = kDevChunkPairs;   // PHMM_CHUNK_PAIRS=n overrides (tests)
  uint32_t* host_ranges = nullptr;        // pinned: per-chunk index ranges of a chunked call
  unsigned long long* host_underflow = nullptr;  // pinned: the call's FP64 underflow count (read at its end)
  bool timing_deferred = false;           // one-chunk call: phase times read after the final sync
  int64_t host_ranges_n = 0;
  Feeder* feeder = nullptr;               // pipelined host call: the copy thread + copy stream
  std::vector<cudaEvent_t> pipe_ev;       // ... its per-group events
  std::vector<CopyJob> pipe_jobs;
  std::vector<size_t> pipe_groups;
  std::vector<PipeChunk> pipe_chunks;
  std::vector<cudaEvent_t> pipe_gev;      // ... the events of the copy groups of one call
  bool pipe = true;                       // PHMM_PIPE=0: no pipelined host calls
  int64_t pipe_min = 1ll << 17;           // smallest pipelined batch (kPipeMinPairs; PHMM_PIPE_MIN: tests, sanitizer)
  bool pipe_trace = false;                // PHMM_PIPE_TRACE=1: per-chunk device timeline on stderr
  std::vector<cudaEvent_t> trace_ev;      // ... chunk start / end events
  std::vector<std::pair<const char*, double>> trace_host;  // ... host timestamps (us)
  std::chrono::steady_clock::time_point trace_t0;
};
static void trace_mark(phmm_ctx* c, const char* what) {
  if (c->pipe_trace)
    c->trace_host.emplace_back(what, std::chrono::duration<double, std::micro>(std::chrono::steady_clock::now() -
                                                                               c->trace_t0).count());
}

namespace {

void debug_cuda(cudaError_t e, const char* what, int line) {
  if (std::getenv("PHMM_DEBUG"))
    std::fprintf(stderr, "phmm: %s failed at line %d: %s\n", what, line, cudaGetErrorString(e));
}

#define CUDA_TRY(x)                   \
  do {                                \
    cudaError_t e_ = (x);             \
    if (e_ != cudaSuccess) {          \
      debug_cuda(e_, #x, __LINE__);   \
      cudaGetLastError();             \
      return PHMM_E_CUDA;             \
    }                                 \
  } while (0)

#define ST_TRY(x)                     \
  do {                                \
    phmm_status s_ = (x);             \
    if (s_ != PHMM_OK) return s_;     \
  } while (0)

#define LAUNCHED(c)                                   \
  do {                                                \
    ++(c)->launches;                                  \
    cudaError_t e_ = cudaGetLastError();              \
    if (e_ != cudaSuccess) {                          \
      debug_cuda(e_, "kernel launch", __LINE__);      \
      return PHMM_E_CUDA;                             \
    }                                                 \
  } while (0)

template <class X>
phmm_status ws(phmm_ctx* c, int id, size_t count, X** out) {
  size_t bytes = count * sizeof(X);
  if (bytes < 16) bytes = 16;
  // inputs, outputs and the call-wide lists are one per context; every per-chunk buffer has
  // one copy per set, so that two chunks can be in flight on two streams (compute_host_pipe)
  // (the async calls keep their inputs in regions 2 and 3, so that one batch's inputs can be
  // prefetched while another computes)
  const bool input = id <= B_PAIRS;
  const bool shared = input || id == B_OUT_LOG10 || id == B_OUT_STATUS || id == B_RLIST ||
                      id == B_UNDERFLOW || (id >= B_SW_REF && id <= B_SW_NOPOFF);
  Buf& b = c->buf[id + (input ? (c->iset ? (1 + c->iset) * B_COUNT : 0) : (shared ? 0 : c->set * B_COUNT))];
  if (b.n < bytes) {
    if (b.p) cudaFree(b.p);
    b.p = nullptr;
    b.n = 0;
    size_t want = bytes + bytes / 8;  // headroom for the next, slightly larger batch
    if (cudaMalloc(&b.p, want) != cudaSuccess) {
      cudaGetLastError();
      if (cudaMalloc(&b.p, bytes) != cudaSuccess) {
        cudaGetLastError();
        b.p = nullptr;
        return PHMM_E_OOM;
      }
      want = bytes;
    }
    b.n = want;
  }
  *out = reinterpret_cast<X*>(b.p);
  return PHMM_OK;
}

int grid_for(const phmm_ctx* c, int64_t n) {
  int64_t g = (n + kThreads - 1) / kThreads;
  const int64_t cap = (int64_t)c->nsm * 16;
  if (g > cap) g = cap;
  if (g < 1) g = 1;
  return (int)g;
}

// cudaMemsetAsync replacement (k_fill_bytes): value v in every byte of [p, p + n)
cudaError_t fill_async(phmm_ctx* c, void* p, int v, size_t n, cudaStream_t s) {
  if (n == 0) return cudaSuccess;
  const uint32_t b = (uint32_t)(v & 0xff);
  const int64_t work = (int64_t)(n / 16) + 1;
  int g = (int)std::min<int64_t>((work + kThreads - 1) / kThreads, (int64_t)c->nsm * 4);
  if (g < 1) g = 1;
  k_fill_bytes<<<g, kThreads, 0, s>>>(static_cast<uint8_t*>(p), b * 0x01010101u, (int64_t)n);
  ++c->launches;
  return cudaGetLastError();
}

phmm_status map_err(uint32_t e) {
  if (e & ERR_INDEX) return PHMM_E_INDEX;
  if (e & ERR_ARG) return PHMM_E_INVALID_ARG;
  if (e & ERR_EMPTY) return PHMM_E_EMPTY_SEQ;
  if (e & ERR_BASE) return PHMM_E_INVALID_BASE;
  if (e & ERR_QUAL) return PHMM_E_INVALID_QUAL;
  return PHMM_E_INVALID_ARG;
}

enum { EV_START, EV_H2D, EV_PREP, EV_WF0, EV_WF1, EV_RESC0, EV_RESC1, EV_FIN, EV_D2H, EV_END, EV_CH0 };

void ev_record(phmm_ctx* c, int i) {
  if (c->flags & PHMM_FLAG_TIMING) cudaEventRecord(c->ev[i], c->stream);
}
float ev_ms(phmm_ctx* c, int a, int b) {
  if (!(c->flags & PHMM_FLAG_TIMING)) return -1.f;
  float ms = -1.f;
  if (cudaEventElapsedTime(&ms, c->ev[a], c->ev[b]) != cudaSuccess) {
    cudaGetLastError();
    return -1.f;
  }
  return ms;
}

// device view of a batch
struct DevBatch {
  const uint8_t *rb, *q, *qi, *qd, *qg, *hap;
  const int64_t *roff, *hoff;
  const int32_t* pairs;
  int64_t n_reads, n_haps, n_pairs, n_rb, n_hb;
};


// Validation of the whole batch. Errors land in scal->err (read back by pass_prepare).
phmm_status run_validate(phmm_ctx* c, const DevBatch& d) {
  Nvtx nvtx_("phmm:validate");
  cudaStream_t s = c->stream;
  Scalars* scal;
  ST_TRY(ws(c, B_SCAL, 1, &scal));
  CUDA_TRY(fill_async(c, scal, 0, sizeof(Scalars), s));
  const int64_t work = std::max(std::max(d.n_hb, d.n_rb / 4), std::max(d.n_reads, d.n_haps) + 1);
  k_validate<<<grid_for(c, work), kThreads, 0, s>>>(d.hap, d.n_hb, d.rb, d.q, d.qi, d.qd, d.qg, d.n_rb, d.roff,
                                                    d.n_reads, d.hoff, d.n_haps, &scal->err);
  LAUNCHED(c);
  return PHMM_OK;
}

// While the worker runs a no-copy batch: copy the NEXT queued no-copy batch's inputs to the
// device now (called at the host round trips of the path, so the copy overlaps this batch).
void maybe_prefetch(phmm_ctx* c);

// Blocks per SM of a wavefront kernel configuration, cached per context (the occupancy
// calculator costs microseconds per query, a small batch asks a few times per call).
template <typename T>
cudaError_t occupancy(phmm_ctx* c, bool long_rows, int warps, size_t smem, int* bps) {
  const uint64_t key = ((uint64_t)smem << 16) | ((uint64_t)warps << 2) | ((uint64_t)long_rows << 1) |
                       (uint64_t)(sizeof(T) == 8);
  auto it = c->occ.find(key);
  if (it != c->occ.end()) {
    *bps = it->second;
    return cudaSuccess;
  }
  cudaError_t e = wf_occupancy<T>(long_rows, warps, smem, bps);
  if (e == cudaSuccess) c->occ[key] = *bps;
  return e;
}

// Part 1 of a pass: bin the pairs, size the coefficient table (and, with
// total_hcodes_out, the haplotype code regions). Ends with one D2H + sync (sizes for
// the allocations; input-content errors are reported here, before any output is written).
//   list == nullptr: all pairs, table items = reads, output slot = pair id
//   list != nullptr: the n listed pairs, one table item per listed pair,
//                    output slot = position in the list
template <typename T>
phmm_status pass_prepare(phmm_ctx* c, const DevBatch& d, const int32_t* list, int64_t n, PassInfo* pi,
                         int64_t* total_tab_out, int64_t* total_hcodes_out = nullptr) {
  constexpr int K = WfT<T>::K;
  cudaStream_t s = c->stream;
  Scalars* scal;
  ST_TRY(ws(c, B_SCAL, 1, &scal));
  const int nb1 = kMaxBins + 2;
  unsigned long long* bins;  // [blocks | pairs | nbig | start | item_start | launch items], nb1 each
  ST_TRY(ws(c, B_BINS, (size_t)6 * nb1, &bins));
  int32_t *pair_bin, *pair_nb;
  ST_TRY(ws(c, B_PAIR_BIN, (size_t)n, &pair_bin));
  ST_TRY(ws(c, B_PAIR_NB, (size_t)n, &pair_nb));
  trace_mark(c, "prep start");
  CUDA_TRY(fill_async(c, bins, 0, sizeof(unsigned long long) * 3 * nb1, s));
  // per-pass scalars (err is kept: it accumulates validation errors)
  CUDA_TRY(fill_async(c, &scal->max_ncols, 0, offsetof(Scalars, n_rescue) - offsetof(Scalars, max_ncols), s));

  const int pb_grid = (int)std::max<int64_t>(grid_for(c, (n + kPairBinsU - 1) / kPairBinsU),
                                              (n + kPairBinsPerCta - 1) / kPairBinsPerCta);
  k_pair_bins<K><<<pb_grid, kThreads, 0, s>>>(
      d.pairs, list, nullptr, n, d.roff, d.n_reads, d.hoff, d.n_haps, c->bucket, sizeof(T) == 4 ? 1 : 0, pair_bin,
      pair_nb, bins,
      bins + nb1, &scal->max_ncols, &scal->min_ncols_c, &scal->cells, &scal->padded_cells, &scal->total_blocks,
      c->gerr ? c->gerr : &scal->err);
  LAUNCHED(c);

  // table items and their block offsets (exclusive scan over n_items + 1)
  const int64_t n_items = list ? n : d.n_reads;
  int32_t* item_read = nullptr;
  if (list) {
    int32_t* pair_item;
    ST_TRY(ws(c, B_ITEM_READ, (size_t)n, &item_read));
    ST_TRY(ws(c, B_PAIR_ITEM, (size_t)n, &pair_item));
    // one table per distinct read of the listed pairs (the rescued pairs of a read share it):
    // radix sort of the read ids, head flags, inclusive scan -> item of every listed pair
    uint32_t* keys;
    int32_t *vals, *head, *incl;
    ST_TRY(ws(c, B_SKEYS, (size_t)2 * n, &keys));
    ST_TRY(ws(c, B_SVALS, (size_t)2 * n, &vals));
    ST_TRY(ws(c, B_DEDUP, (size_t)2 * n, &head));
    incl = head + n;
    k_rescue_read_keys<<<grid_for(c, n), kThreads, 0, s>>>(d.pairs, list, n, keys, vals);
    LAUNCHED(c);
    int end_bit = 1;
    while (end_bit < 32 && (1ll << end_bit) <= d.n_reads) ++end_bit;
    size_t sb = 0, cb = 0;
    CUDA_TRY(cub::DeviceRadixSort::SortPairs(nullptr, sb, keys, keys + n, vals, vals + n, n, 0, end_bit, s));
    CUDA_TRY(cub::DeviceScan::InclusiveSum(nullptr, cb, head, incl, n, s));
    unsigned char* tmp;
    ST_TRY(ws(c, B_SORT_TMP, std::max(sb, cb), &tmp));
    CUDA_TRY(cub::DeviceRadixSort::SortPairs(tmp, sb, keys, keys + n, vals, vals + n, n, 0, end_bit, s));
    k_rescue_head_flags<<<grid_for(c, n), kThreads, 0, s>>>(keys + n, n, head);
    LAUNCHED(c);
    CUDA_TRY(cub::DeviceScan::InclusiveSum(tmp, cb, head, incl, n, s));
    k_rescue_items_dedup<<<grid_for(c, n), kThreads, 0, s>>>(keys + n, vals + n, head, incl, n, item_read,
                                                             pair_item);
    LAUNCHED(c);
    c->launches += 2;
  }
  int64_t *item_nb, *item_off;
  ST_TRY(ws(c, B_ITEM_NB, (size_t)n_items + 1, &item_nb));
  ST_TRY(ws(c, B_ITEM_OFF, (size_t)n_items + 1, &item_off));
  k_item_nblocks<K><<<grid_for(c, n_items), kThreads, 0, s>>>(item_read, n_items, nullptr, d.roff, item_nb);
  LAUNCHED(c);
  size_t tmp_bytes = 0;
  CUDA_TRY(cub::DeviceScan::ExclusiveSum(nullptr, tmp_bytes, item_nb, item_off, (int64_t)(n_items + 1), s));
  size_t tb2 = 0;
  int64_t *hnc = nullptr, *hc_off = nullptr;
  if (total_hcodes_out) {
    ST_TRY(ws(c, B_HNC, (size_t)d.n_haps + 1, &hnc));
    ST_TRY(ws(c, B_HC_OFF, (size_t)d.n_haps + 1, &hc_off));
    CUDA_TRY(cub::DeviceScan::ExclusiveSum(nullptr, tb2, hnc, hc_off, (int64_t)(d.n_haps + 1), s));
  }
  unsigned char* tmp;
  ST_TRY(ws(c, B_SCAN_TMP, std::max(tmp_bytes, tb2), &tmp));
  CUDA_TRY(cub::DeviceScan::ExclusiveSum(tmp, tmp_bytes, item_nb, item_off, (int64_t)(n_items + 1), s));
  ++c->launches;
  // haplotype code regions (wf_hc_region bytes each)
  if (total_hcodes_out) {
    k_hap_ncols<<<grid_for(c, d.n_haps), kThreads, 0, s>>>(d.hoff, d.n_haps, c->bucket, hnc);
    LAUNCHED(c);
    CUDA_TRY(cub::DeviceScan::ExclusiveSum(tmp, tb2, hnc, hc_off, (int64_t)(d.n_haps + 1), s));
    ++c->launches;
  }
  // one small D2H: sizes + error flag
  CUDA_TRY(cudaMemcpyAsync(c->host_scal, scal, sizeof(Scalars), cudaMemcpyDeviceToHost, s));
  if (c->gerr) CUDA_TRY(cudaMemcpyAsync(&c->host_scal->err, c->gerr, sizeof(uint32_t), cudaMemcpyDeviceToHost, s));
  int64_t* hsz = c->host_sizes;
  hsz[0] = hsz[1] = 0;
  CUDA_TRY(cudaMemcpyAsync(&hsz[0], item_off + n_items, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
  if (hc_off) CUDA_TRY(cudaMemcpyAsync(&hsz[1], hc_off + d.n_haps, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
  trace_mark(c, "prep sync");
  maybe_prefetch(c);
  CUDA_TRY(cudaStreamSynchronize(s));
  trace_mark(c, "prep synced");
  if (c->host_scal->err) return map_err(c->host_scal->err);
  if (total_hcodes_out) *total_hcodes_out = hsz[1];
  pi->cells = c->host_scal->cells;
  pi->padded_cells = c->host_scal->padded_cells;
  pi->total_blocks = c->host_scal->total_blocks;
  pi->max_ncols = c->host_scal->max_ncols;
  pi->min_ncols = kNcolsComplement - c->host_scal->min_ncols_c;
  // block descriptors address tables and code regions with 32-bit offsets
  if (hsz[0] > 0xffffffffLL || pi->total_blocks > 0x7fffffffULL) return PHMM_E_INVALID_ARG;
  *total_tab_out = hsz[0];
  return PHMM_OK;
}

// Haplotype code regions of the whole batch (after pass_prepare with total_hcodes_out),
// followed by an all-PAD region for idle lanes. Returns the buffer and the PAD offset.
phmm_status build_hap_codes(phmm_ctx* c, const DevBatch& d, int64_t total_hc, int max_ncols, uint8_t** hc_out) {
  cudaStream_t s = c->stream;
  const int64_t pad_len = wf_hc_copy_len(max_ncols) + 64;
  if (total_hc + pad_len > 0xffffffffLL) return PHMM_E_INVALID_ARG;  // 32-bit code offsets
  int64_t* hc_off;
  uint8_t* hc;
  ST_TRY(ws(c, B_HC_OFF, (size_t)d.n_haps + 1, &hc_off));
  ST_TRY(ws(c, B_HCODES, (size_t)(total_hc + pad_len), &hc));
  CUDA_TRY(fill_async(c, hc + total_hc, WF_PAD * WF_CB, (size_t)pad_len, s));
  k_hap_codes_wf<<<grid_for(c, d.n_haps * 32), kThreads, 0, s>>>(d.hap, d.hoff, d.n_haps, hc_off, c->bucket, hc);
  LAUNCHED(c);
  *hc_out = hc;
  return PHMM_OK;
}

// Part 2 of a pass: coefficient tables, stable bin sort, block descriptors, wavefront.
// Writes out[slot] = scaled sum of the pair. The haplotype code regions
// (hc, pad region at total_hc) were built by build_hap_codes.
template <typename T>
phmm_status pass_run(phmm_ctx* c, const DevBatch& d, const int32_t* list, int64_t n, const PassInfo& pi,
                     int64_t total_tab, const uint8_t* hc, int64_t total_hc, T* out, bool timed,
                     int32_t* exp_out = nullptr) {
  constexpr int K = WfT<T>::K;
  cudaStream_t s = c->stream;
  Scalars* scal;
  ST_TRY(ws(c, B_SCAL, 1, &scal));
  const int nb1 = kMaxBins + 2;
  unsigned long long* bins;
  ST_TRY(ws(c, B_BINS, (size_t)6 * nb1, &bins));
  unsigned long long *bin_blocks = bins, *bin_nbig = bins + 2 * nb1, *bin_start = bins + 3 * nb1,
                     *item_start = bins + 4 * nb1, *launch_items = bins + 5 * nb1;
  int32_t *pair_bin, *pair_nb, *item_read = nullptr, *pair_item = nullptr;
  ST_TRY(ws(c, B_PAIR_BIN, (size_t)n, &pair_bin));
  ST_TRY(ws(c, B_PAIR_NB, (size_t)n, &pair_nb));
  const int64_t n_items = list ? n : d.n_reads;
  if (list) {
    ST_TRY(ws(c, B_ITEM_READ, (size_t)n, &item_read));
    ST_TRY(ws(c, B_PAIR_ITEM, (size_t)n, &pair_item));
  }
  int64_t *item_off, *hc_off;
  ST_TRY(ws(c, B_ITEM_OFF, (size_t)n_items + 1, &item_off));
  ST_TRY(ws(c, B_HC_OFF, (size_t)d.n_haps + 1, &hc_off));
  TBlock<T>* tab;
  BlkDesc* blk;
  ST_TRY(ws(c, sizeof(T) == 4 ? B_TAB32 : B_TAB64, (size_t)total_tab, &tab));
  ST_TRY(ws(c, B_BLK, (size_t)pi.total_blocks, &blk));
  if (total_tab > 0) {
    k_build_table_wf<T><<<grid_for(c, n_items * 32), kTabThreads, 0, s>>>(
        item_read, n_items, item_off, d.roff, d.rb, d.q, d.qi, d.qd, d.qg, tab);
    LAUNCHED(c);
  }

  // launch classes: bins whose ring fits at full occupancy, then (if any) the longer bins
  const int slot = (int)ring_slot_bytes<T>();
  auto P_of = [](int ncols) { return wf_pass_len<T>(ncols); };
  const int p_max = P_of(pi.max_ncols);
  int bps_full = 0;
  CUDA_TRY(occupancy<T>(c, false, WF_WARPS, wf_warp_smem<T>(wf_pass_len<T>(0) + 4) * WF_WARPS, &bps_full));
  if (bps_full < 1) return PHMM_E_CUDA;
  const int64_t cta_budget = (int64_t)c->smem_per_sm / bps_full - c->smem_reserved;
  const int ring_full = (int)std::min<int64_t>(
      (cta_budget / WF_WARPS - (int64_t)wf_warp_smem<T>(0)) / slot, (int64_t)(c->smem_optin / WF_WARPS) / slot);
  int bin_cut = kMaxBins + 1;  // bins < bin_cut run in the full-occupancy launch
  if (p_max + 4 > ring_full) {
    bin_cut = 0;
    while (bin_cut <= kMaxBins && P_of(bin_cut * c->bucket) + 4 <= ring_full) ++bin_cut;
  }
  // FP32: rows of >= WF_RESCALE_COLS columns run in the long launch (the kernel variant with
  // the ring rescale)
  if (sizeof(T) == 4 && pi.max_ncols >= WF_RESCALE_COLS)
    bin_cut = std::min(bin_cut, (WF_RESCALE_COLS + c->bucket - 1) / c->bucket);
  struct Launch { int bin_lo, bin_hi, warps, ring_len, bps; };
  Launch L[2];
  int nl = 0;
  L[nl++] = Launch{0, std::min(bin_cut, kMaxBins + 1), WF_WARPS, std::min(p_max + 4, ring_full), bps_full};
  if (bin_cut <= kMaxBins) {
    Launch lb{bin_cut, kMaxBins + 1, 0, p_max + 8, 0};  // global ring: prefetch reads up to slot P + 4
    int best = 0;
    for (int w = WF_WARPS; w >= 1; w >>= 1) {
      const size_t sm = wf_warp_smem<T, true>(lb.ring_len) * w;
      if (sm > (size_t)c->smem_optin) continue;
      int b = 0;
      CUDA_TRY(occupancy<T>(c, true, w, sm, &b));
      if (b * w > best) { best = b * w; lb.warps = w; lb.bps = b; }
    }
    if (best < 1) return PHMM_E_INVALID_ARG;  // cannot happen for ncols <= kMaxHapLen + 8
    L[nl++] = lb;
  }

  const int64_t nwarps = (int64_t)c->nsm * L[0].bps * L[0].warps;
  // work items: ~4 per warp for load balance; a small pass (e.g. the FP64 rescue list)
  // gets one item per warp instead of fewer, larger items that leave warps idle
  int64_t chunk = (int64_t)(pi.total_blocks / (unsigned long long)(nwarps * 4));
  int tail_div = WF_TAIL_DIV;
  if (chunk < 512) {
    chunk = std::max<int64_t>(64, ((int64_t)pi.total_blocks + nwarps - 1) / nwarps);
    tail_div = 0;  // one item per warp already
  }
  if (chunk > 65536) chunk = 65536;
  // the last 1/WF_TAIL_DIV of each launch's blocks in short items (guided self-scheduling)
  const int64_t chunk_s = std::max<int64_t>(64, chunk / WF_TAIL_SPLIT);
  const int nbins = kMaxBins + 1;
  k_scan_bins<<<1, 1024, 0, s>>>(bin_blocks, nbins, nl > 1 ? L[1].bin_lo : nbins, chunk, chunk_s, tail_div,
                                 WF_LPT, bin_start, item_start, bin_nbig, launch_items);
  LAUNCHED(c);
  // stable sort of the pass's pairs by bin, then contiguous block ranges by an exclusive scan
  uint32_t* keys;
  int32_t* vals;
  int64_t *nbs, *blk_off;
  ST_TRY(ws(c, B_SKEYS, (size_t)2 * n, &keys));
  ST_TRY(ws(c, B_SVALS, (size_t)2 * n, &vals));
  ST_TRY(ws(c, B_NBS, (size_t)n + 1, &nbs));
  ST_TRY(ws(c, B_BLKOFF, (size_t)n + 1, &blk_off));
  k_iota_keys<<<grid_for(c, n), kThreads, 0, s>>>(pair_bin, pair_nb, n, keys, vals);
  LAUNCHED(c);
  int end_bit = 1;
  while ((1 << end_bit) <= 2 * (kMaxBins + 1)) ++end_bit;  // keys 2 * bin + class (k_iota_keys)
  size_t sort_bytes = 0, scan_bytes = 0;
  // one length bin (every pair the same column count, e.g. C2): the stable sort is the identity
  // (not for a long-row bin, whose pass-padded pairs must come first)
  const bool one_bin = pi.min_ncols == pi.max_ncols && pi.max_ncols < kRescaleCols;
  const int32_t* sorted = one_bin ? vals : vals + n;
  if (!one_bin)
    CUDA_TRY(cub::DeviceRadixSort::SortPairs(nullptr, sort_bytes, keys, keys + n, vals, vals + n, n, 0, end_bit, s));
  CUDA_TRY(cub::DeviceScan::ExclusiveSum(nullptr, scan_bytes, nbs, blk_off, n + 1, s));
  unsigned char* tmp;
  ST_TRY(ws(c, B_SORT_TMP, std::max(sort_bytes, scan_bytes), &tmp));
  if (!one_bin) {
    CUDA_TRY(cub::DeviceRadixSort::SortPairs(tmp, sort_bytes, keys, keys + n, vals, vals + n, n, 0, end_bit, s));
    c->launches += 2;
  }
  k_sorted_nb<<<grid_for(c, n), kThreads, 0, s>>>(sorted, pair_nb, n, nbs);
  LAUNCHED(c);
  CUDA_TRY(cub::DeviceScan::ExclusiveSum(tmp, scan_bytes, nbs, blk_off, n + 1, s));
  ++c->launches;
  k_alloc_blocks_wf<K><<<grid_for(c, n), kThreads, 0, s>>>(d.pairs, list, pair_item, sorted, n, pair_nb, blk_off,
                                                           d.roff, d.hoff, hc_off, item_off, blk);
  LAUNCHED(c);

  WfArgs2<T> A;
  A.blk = blk;
  A.tab = tab;
  A.hcodes = hc;
  A.pad_idx = (uint32_t)total_hc;  // 4-aligned: every code region is a multiple of 4
  A.bin_start = bin_start;
  A.item_start = item_start;
  A.bucket = c->bucket;
  A.chunk_blocks = chunk;
  A.chunk_small = chunk_s;
  A.bin_nbig = bin_nbig;
  A.lpt = WF_LPT;
  A.out = out;
  A.exp_out = exp_out;
  CUDA_TRY(fill_async(c, scal->item_counter, 0, sizeof(scal->item_counter), s));
  if (timed) ev_record(c, EV_WF0);
  for (int i = 0; i < nl; ++i) {
    A.bin_lo = L[i].bin_lo;
    A.bin_hi = L[i].bin_hi;
    A.ring_len = L[i].ring_len;
    A.item_counter = &scal->item_counter[i];
    A.launch_items = launch_items + 2 * i;
    const size_t smem = (i == 1 ? wf_warp_smem<T, true>(L[i].ring_len) : wf_warp_smem<T>(L[i].ring_len)) * L[i].warps;
    CUDA_TRY(wf_launch<T>(i == 1, (unsigned)(c->nsm * L[i].bps), L[i].warps, smem, s, A));
    ++c->launches;
  }
  maybe_prefetch(c);
  if (timed) ev_record(c, EV_WF1);
  return PHMM_OK;
}

// The FP32 pass over a batch (all its pairs): per-read tables, binning, k_wavefront<float>,
// k_finalize_fp32 into dev_out / dev_status; pairs below the FP32 range are appended to rlist
// (as pair index + rbase) and counted in *n_rescue. Returns the haplotype code regions it built.
phmm_status fp32_pass(phmm_ctx* c, const DevBatch& d, double* dev_out, uint8_t* dev_status, int32_t* rlist,
                      int64_t rbase, int64_t* n_rescue, PassInfo* pi, uint8_t** hc, int64_t* total_hc, bool timed) {
  Nvtx nvtx_("phmm:fp32_pass");
  cudaStream_t s = c->stream;
  int64_t total_tab = 0;
  ST_TRY((pass_prepare<float>(c, d, nullptr, d.n_pairs, pi, &total_tab, total_hc)));
  ST_TRY(build_hap_codes(c, d, *total_hc, pi->max_ncols, hc));
  float* out32;
  ST_TRY(ws(c, B_OUT32, (size_t)d.n_pairs, &out32));
  int32_t* exp32;  // powers of 2 applied by the ring rescale of long pairs
  ST_TRY(ws(c, B_EXP32, (size_t)d.n_pairs, &exp32));
  CUDA_TRY(fill_async(c, exp32, 0, sizeof(int32_t) * (size_t)d.n_pairs, s));
  if (timed) ev_record(c, EV_PREP);
  ST_TRY(pass_run<float>(c, d, nullptr, d.n_pairs, *pi, total_tab, *hc, *total_hc, out32, timed, exp32));
  k_finalize_fp32<<<grid_for(c, d.n_pairs), kThreads, 0, s>>>(out32, exp32, d.n_pairs, d.pairs, d.hoff, c->bucket,
                                                                dev_out, dev_status, rlist, n_rescue,
                                                                dev_status != nullptr, rbase);
  LAUNCHED(c);
  c->st.cells += (int64_t)pi->cells;
  c->st.padded_cells += (int64_t)pi->padded_cells;
  return PHMM_OK;
}

// FP64 rescue of the nr listed pairs of batch d on the same kernel design. hc: the haplotype
// code regions of d (nullptr: build them here).
phmm_status rescue_pass(phmm_ctx* c, const DevBatch& d, double* dev_out, uint8_t* dev_status, const int32_t* rlist,
                        int64_t nr, const uint8_t* hc, int64_t total_hc, bool timed) {
  Nvtx nvtx_("phmm:rescue");
  cudaStream_t s = c->stream;
  Scalars* scal;
  ST_TRY(ws(c, B_SCAL, 1, &scal));
  PassInfo pr;
  int64_t tab_r = 0;
  if (hc) {
    ST_TRY((pass_prepare<double>(c, d, rlist, nr, &pr, &tab_r)));
  } else {
    uint8_t* hc_b;
    ST_TRY((pass_prepare<double>(c, d, rlist, nr, &pr, &tab_r, &total_hc)));
    ST_TRY(build_hap_codes(c, d, total_hc, pr.max_ncols, &hc_b));
    hc = hc_b;
  }
  double* out64;
  ST_TRY(ws(c, B_OUT64, (size_t)nr, &out64));
  ST_TRY((pass_run<double>(c, d, rlist, nr, pr, tab_r, hc, total_hc, out64, false)));
  unsigned long long* uf;
  ST_TRY(ws(c, B_UNDERFLOW, 1, &uf));
  k_finalize_fp64<<<grid_for(c, nr), kThreads, 0, s>>>(out64, rlist, nullptr, nr, d.pairs, d.hoff, c->bucket, dev_out,
                                                       dev_status, dev_status != nullptr, 1, uf);
  LAUNCHED(c);
  c->st.padded_cells += (int64_t)pr.padded_cells;
  if (timed) ev_record(c, EV_RESC1);
  return PHMM_OK;
}

// Per-phase times of one compute_one (PHMM_FLAG_TIMING), added to the call's totals once its
// last event completed.
void acc_phases(phmm_ctx* c) {
  if (!(c->flags & PHMM_FLAG_TIMING)) return;
  const bool fp64 = c->prec == PHMM_PREC_FP64;
  cudaEventSynchronize(c->ev[fp64 ? EV_FIN : EV_RESC1]);
  auto add = [&](float& acc, int a, int b) {
    const float ms = ev_ms(c, a, b);
    if (ms >= 0.f) acc += ms;
  };
  add(c->acc.prep, EV_CH0, EV_PREP);
  add(c->acc.wf, EV_WF0, EV_WF1);
  if (fp64) {
    add(c->acc.fin, EV_WF1, EV_FIN);
  } else {
    add(c->acc.fin, EV_WF1, EV_RESC0);
    add(c->acc.resc, EV_RESC0, EV_RESC1);
  }
}

// The whole path on one (validated) batch or chunk: the FP32 pass and the FP64 rescue of its
// underflowing pairs (or the FP64 pass), results into out / status (context scratch).
// Accumulates the call's statistics; ends synchronised.
phmm_status compute_one(phmm_ctx* c, const DevBatch& d, double* dev_out, uint8_t* dev_status) {
  Nvtx nvtx_("phmm:chunk");
  cudaStream_t s = c->stream;
  PassInfo pi;
  int64_t total_tab = 0, total_hc = 0;
  uint8_t* hc = nullptr;
  Scalars* scal;
  ST_TRY(ws(c, B_SCAL, 1, &scal));
  ev_record(c, EV_CH0);
  if (c->prec == PHMM_PREC_FP64) {
    ST_TRY((pass_prepare<double>(c, d, nullptr, d.n_pairs, &pi, &total_tab, &total_hc)));
    ST_TRY(build_hap_codes(c, d, total_hc, pi.max_ncols, &hc));
    double* out64;
    ST_TRY(ws(c, B_OUT64, (size_t)d.n_pairs, &out64));
    ev_record(c, EV_PREP);
    ST_TRY((pass_run<double>(c, d, nullptr, d.n_pairs, pi, total_tab, hc, total_hc, out64, true)));
    unsigned long long* uf;
    ST_TRY(ws(c, B_UNDERFLOW, 1, &uf));
    k_finalize_fp64<<<grid_for(c, d.n_pairs), kThreads, 0, s>>>(out64, nullptr, nullptr, d.n_pairs, d.pairs,
                                                                  d.hoff, c->bucket, dev_out,
                                                                  dev_status, dev_status != nullptr, 0, uf);
    LAUNCHED(c);
    ev_record(c, EV_FIN);
    c->st.cells += (int64_t)pi.cells;
    c->st.padded_cells += (int64_t)pi.padded_cells;
  } else {
    int32_t* rlist;  // per set: two chunks of a pipelined call may be in flight
    ST_TRY(ws(c, B_RLIST_CH, (size_t)d.n_pairs, &rlist));
    CUDA_TRY(fill_async(c, &scal->n_rescue, 0, sizeof(int64_t) + sizeof(unsigned long long), s));
    ST_TRY(fp32_pass(c, d, dev_out, dev_status, rlist, 0, &scal->n_rescue, &pi, &hc, &total_hc, true));
    ev_record(c, EV_RESC0);
    CUDA_TRY(cudaMemcpyAsync(c->host_scal, scal, sizeof(Scalars), cudaMemcpyDeviceToHost, s));
    maybe_prefetch(c);
    CUDA_TRY(cudaStreamSynchronize(s));
    const int64_t nr = c->host_scal->n_rescue;
    c->st.n_rescued += nr;
    if (nr > 0) ST_TRY(rescue_pass(c, d, dev_out, dev_status, rlist, nr, hc, total_hc, true));
    else ev_record(c, EV_RESC1);
  }
  if (!c->timing_deferred) acc_phases(c);
  ++c->st.n_chunks;
  return PHMM_OK;
}

// The whole path on device-resident inputs. Writes dev_out (+ dev_status), which are context
// scratch (the callers copy them to the caller's buffers after success).
// Batches of more than kDevChunkPairs pairs run as consecutive chunks of pairs, each an
// ordinary batch over the reads and haplotypes its pairs use (same results bit for bit:
// a pair's arithmetic does not depend on its batch, R14), so the per-read tables and block
// descriptors stay a few GB whatever the batch size (the 2^26-pair C5 at N = 1).
phmm_status compute_dev(phmm_ctx* c, const DevBatch& d, double* dev_out, uint8_t* dev_status) {
  cudaStream_t s = c->stream;
  c->st = phmm_stats{};
  c->acc = PhaseMs{};
  c->st.n_pairs = d.n_pairs;
  c->timing_deferred = false;
  if (d.n_pairs == 0) return PHMM_OK;
  ST_TRY(run_validate(c, d));
  unsigned long long* uf;
  ST_TRY(ws(c, B_UNDERFLOW, 1, &uf));
  CUDA_TRY(fill_async(c, uf, 0, sizeof(unsigned long long), s));
  const int64_t cp = c->chunk_pairs;
  // one chunk: the phase times and the underflow count are read after the call's final sync
  c->timing_deferred = d.n_pairs <= cp;
  if (d.n_pairs <= cp) return compute_one(c, d, dev_out, dev_status);
  // chunk k = pairs [k*cp, min((k+1)*cp, n)); its read / haplotype index ranges in one pass
  const int64_t nch = (d.n_pairs + cp - 1) / cp;
  Scalars* scal;
  uint32_t* rng;
  ST_TRY(ws(c, B_SCAL, 1, &scal));
  ST_TRY(ws(c, B_CH_RANGES, (size_t)4 * nch, &rng));
  CUDA_TRY(fill_async(c, rng, 0, sizeof(uint32_t) * 4 * nch, s));
  for (int64_t k = 0; k < nch; ++k) {  // minima start at UINT_MAX
    CUDA_TRY(fill_async(c, rng + 4 * k, 0xff, sizeof(uint32_t), s));
    CUDA_TRY(fill_async(c, rng + 4 * k + 2, 0xff, sizeof(uint32_t), s));
  }
  {
    const int bpc = (int)std::max<int64_t>(1, std::min<int64_t>((cp + kThreads - 1) / kThreads, 4 * c->nsm));
    k_chunk_ranges<<<dim3((unsigned)bpc, (unsigned)nch), kThreads, 0, s>>>(d.pairs, d.n_pairs, cp, d.n_reads,
                                                                              d.n_haps, rng, &scal->err);
    LAUNCHED(c);
  }
  uint32_t* hr = c->host_ranges;
  if (c->host_ranges_n < nch) {
    if (hr) cudaFreeHost(hr);
    c->host_ranges = nullptr;
    c->host_ranges_n = 0;
    if (cudaMallocHost(&hr, sizeof(uint32_t) * 4 * nch) != cudaSuccess) {
      cudaGetLastError();
      return PHMM_E_OOM;
    }
    c->host_ranges = hr;
    c->host_ranges_n = nch;
  }
  CUDA_TRY(cudaMemcpyAsync(hr, rng, sizeof(uint32_t) * 4 * nch, cudaMemcpyDeviceToHost, s));
  CUDA_TRY(cudaMemcpyAsync(c->host_scal, scal, sizeof(Scalars), cudaMemcpyDeviceToHost, s));
  CUDA_TRY(cudaStreamSynchronize(s));
  if (c->host_scal->err) return map_err(c->host_scal->err);
  int64_t *roff_c, *hoff_c;
  int32_t* pairs_c;
  for (int64_t k = 0; k < nch; ++k) {
    const int64_t p0 = k * cp, np = std::min(cp, d.n_pairs - p0);
    const int64_t rlo = hr[4 * k], nr = (int64_t)hr[4 * k + 1] + 1 - rlo;
    const int64_t hlo = hr[4 * k + 2], nh = (int64_t)hr[4 * k + 3] + 1 - hlo;
    ST_TRY(ws(c, B_CH_ROFF, (size_t)nr + 1, &roff_c));
    ST_TRY(ws(c, B_CH_HOFF, (size_t)nh + 1, &hoff_c));
    ST_TRY(ws(c, B_CH_PAIRS, (size_t)2 * np, &pairs_c));
    // the chunk's offsets keep their absolute values (the chunk addresses the batch's base
    // arrays); its pair indices become relative to rlo / hlo
    k_rebase_chunk<<<grid_for(c, std::max(std::max(nr, nh) + 1, np)), kThreads, 0, s>>>(
        d.roff, rlo, nr, roff_c, d.hoff, hlo, nh, hoff_c, d.pairs, p0, np, pairs_c, 0);
    LAUNCHED(c);
    DevBatch dk{d.rb, d.q, d.qi, d.qd, d.qg, d.hap, roff_c, hoff_c, pairs_c, nr, nh, np, d.n_rb, d.n_hb};
    ST_TRY(compute_one(c, dk, dev_out + p0, dev_status ? dev_status + p0 : nullptr));
  }
  return PHMM_OK;
}


// ============================================================ Smith-Waterman (§8f row 2)
struct SwDev {
  const uint8_t *ref, *alt;
  const int64_t *roff, *aoff;
  const int32_t* tasks;
  int64_t n_refs, n_alts, n_tasks, n_rb, n_ab;
};

phmm_status sw_check_args(const phmm_sw_batch* b, const phmm_sw_params* p) {
  if (!b || !p) return PHMM_E_INVALID_ARG;
  if (b->n_refs < 0 || b->n_alts < 0 || b->n_tasks < 0) return PHMM_E_INVALID_ARG;
  if (b->n_tasks > 0x7fffffffLL || b->n_refs > 0x7fffffffLL || b->n_alts > 0x7fffffffLL) return PHMM_E_INVALID_ARG;
  if (p->match <= 0 || p->mismatch > p->match || p->gap_extend > 0 || p->gap_open > p->gap_extend)
    return PHMM_E_INVALID_ARG;
  // |score| <= match * 4096 and gap totals stay far from int32 overflow
  if (p->match > (1 << 18) || p->mismatch < -(1 << 18) || p->gap_open < -(1 << 18)) return PHMM_E_INVALID_ARG;
  if (b->n_tasks == 0) return PHMM_OK;
  if (!b->tasks || !b->ref_offsets || !b->alt_offsets) return PHMM_E_INVALID_ARG;
  if (b->total_ref_bases < 0 || b->total_alt_bases < 0) return PHMM_E_INVALID_ARG;
  if (b->total_ref_bases > 0 && !b->ref_bases) return PHMM_E_INVALID_ARG;
  if (b->total_alt_bases > 0 && !b->alt_bases) return PHMM_E_INVALID_ARG;
  return PHMM_OK;
}

int64_t ops_total_cap(const phmm_ctx* c, const int64_t*, int64_t) { return c->sw_ops_cap; }

phmm_status sw_compute_dev(phmm_ctx* c, const SwDev& d, const phmm_sw_params* prm, int32_t* dev_res,
                           uint32_t* dev_ops) {
  cudaStream_t s = c->stream;
  c->st = phmm_stats{};
  c->st.n_pairs = d.n_tasks;
  if (d.n_tasks == 0) return PHMM_OK;
  Scalars* scal;
  ST_TRY(ws(c, B_SCAL, 1, &scal));
  CUDA_TRY(fill_async(c, scal, 0, sizeof(Scalars), s));
  if (d.n_rb > 0) {
    k_validate_haps<<<grid_for(c, d.n_rb), kThreads, 0, s>>>(d.ref, d.n_rb, &scal->err);
    LAUNCHED(c);
  }
  if (d.n_ab > 0) {
    k_validate_haps<<<grid_for(c, d.n_ab), kThreads, 0, s>>>(d.alt, d.n_ab, &scal->err);
    LAUNCHED(c);
  }
  k_validate_offsets<<<grid_for(c, d.n_refs + 1), kThreads, 0, s>>>(d.roff, d.n_refs, d.n_rb, &scal->err);
  LAUNCHED(c);
  k_validate_offsets<<<grid_for(c, d.n_alts + 1), kThreads, 0, s>>>(d.aoff, d.n_alts, d.n_ab, &scal->err);
  LAUNCHED(c);
  const int64_t n = d.n_tasks;
  int64_t *bt_sz, *bt_off, *op_cap, *op_off;
  ST_TRY(ws(c, B_SW_BTSZ, (size_t)n + 1, &bt_sz));
  ST_TRY(ws(c, B_SW_BTOFF, (size_t)n + 1, &bt_off));
  ST_TRY(ws(c, B_SW_OPCAP, (size_t)n + 1, &op_cap));
  ST_TRY(ws(c, B_SW_OPOFF, (size_t)n + 1, &op_off));
  k_sw_sizes<<<grid_for(c, n), kThreads, 0, s>>>(d.tasks, n, d.roff, d.n_refs, d.aoff, d.n_alts, bt_sz, op_cap,
                                                  reinterpret_cast<int64_t*>(&scal->cells), &scal->max_ncols,
                                                  &scal->err);
  LAUNCHED(c);
  size_t scan_bytes = 0, sort_bytes = 0;
  CUDA_TRY(cub::DeviceScan::ExclusiveSum(nullptr, scan_bytes, bt_sz, bt_off, n + 1, s));
  uint64_t* keys;
  int32_t* vals;
  ST_TRY(ws(c, B_SW_KEYS, (size_t)2 * n, &keys));
  ST_TRY(ws(c, B_SW_VALS, (size_t)2 * n, &vals));
  CUDA_TRY(cub::DeviceRadixSort::SortPairs(nullptr, sort_bytes, keys, keys + n, vals, vals + n, n, 0, 64, s));
  unsigned char* tmp;
  ST_TRY(ws(c, B_SORT_TMP, std::max(scan_bytes, sort_bytes), &tmp));
  CUDA_TRY(cub::DeviceScan::ExclusiveSum(tmp, scan_bytes, bt_sz, bt_off, n + 1, s));
  CUDA_TRY(cub::DeviceScan::ExclusiveSum(tmp, scan_bytes, op_cap, op_off, n + 1, s));
  c->launches += 2;
  CUDA_TRY(cudaMemcpyAsync(c->host_scal, scal, sizeof(Scalars), cudaMemcpyDeviceToHost, s));
  int64_t* hsz = c->host_sizes;
  CUDA_TRY(cudaMemcpyAsync(&hsz[0], bt_off + n, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
  CUDA_TRY(cudaMemcpyAsync(&hsz[1], op_off + n, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
  CUDA_TRY(cudaStreamSynchronize(s));
  if (c->host_scal->err) return map_err(c->host_scal->err);
  const int64_t total_bt = hsz[0];
  c->sw_ops_cap = hsz[1];
  const int max_n = c->host_scal->max_ncols;
  c->st.cells = (int64_t)c->host_scal->cells;
  int16_t* bt;
  ST_TRY(ws(c, B_SW_BT, (size_t)total_bt, &bt));
  // largest tasks first (persistent warps: the tail is the smallest tasks)
  k_sw_keys<<<grid_for(c, n), kThreads, 0, s>>>(d.tasks, n, d.roff, d.aoff, keys, vals);
  LAUNCHED(c);
  CUDA_TRY(cub::DeviceRadixSort::SortPairs(tmp, sort_bytes, keys, keys + n, vals, vals + n, n, 0, 64, s));
  ++c->launches;

  SwArgs A;
  A.ref = d.ref; A.ref_off = d.roff; A.alt = d.alt; A.alt_off = d.aoff; A.tasks = d.tasks;
  A.order = vals + n; A.n_tasks = n; A.bt_off = bt_off; A.bt = bt; A.res = dev_res;
  A.counter = &scal->item_counter[0];
  A.p = SwParams{prm->match, prm->mismatch, prm->gap_open, prm->gap_extend};
  A.max_n = max_n;
  const size_t per_warp = (size_t)(max_n + 1) * 12 + (size_t)((max_n + 15) & ~15);
  const size_t smem = per_warp * SW_WARPS;
  CUDA_TRY(cudaFuncSetAttribute(k_sw_fill, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  int bps = 0;
  CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, k_sw_fill, SW_WARPS * 32, smem));
  if (bps < 1) return PHMM_E_INVALID_ARG;
  CUDA_TRY(fill_async(c, A.counter, 0, sizeof(unsigned int), s));
  ev_record(c, EV_WF0);
  k_sw_fill<<<(unsigned)(c->nsm * bps), SW_WARPS * 32, smem, s>>>(A);
  LAUNCHED(c);
  ev_record(c, EV_WF1);
  // traceback into capacity-laid-out scratch, then pack the runs back to back
  uint32_t* ops_tmp;
  int64_t *nops, *nops_off;
  ST_TRY(ws(c, B_SW_OPTMP, (size_t)std::max<int64_t>(ops_total_cap(c, op_off, n), 1), &ops_tmp));
  ST_TRY(ws(c, B_SW_NOPS, (size_t)n + 1, &nops));
  ST_TRY(ws(c, B_SW_NOPOFF, (size_t)n + 1, &nops_off));
  k_sw_traceback<<<grid_for(c, n), 128, 0, s>>>(A, op_off, ops_tmp, nops);
  LAUNCHED(c);
  CUDA_TRY(cub::DeviceScan::ExclusiveSum(tmp, scan_bytes, nops, nops_off, n + 1, s));
  ++c->launches;
  k_sw_compact<<<grid_for(c, n * 32), kThreads, 0, s>>>(ops_tmp, op_off, nops_off, n, dev_ops);
  LAUNCHED(c);
  ev_record(c, EV_FIN);
  return PHMM_OK;
}

phmm_status check_batch_args(const phmm_batch* b) {
  if (!b) return PHMM_E_INVALID_ARG;
  if (b->n_reads < 0 || b->n_haps < 0 || b->n_pairs < 0) return PHMM_E_INVALID_ARG;
  if (b->n_pairs > 0x7fffffffLL || b->n_reads > 0x7fffffffLL || b->n_haps > 0x7fffffffLL) return PHMM_E_INVALID_ARG;
  if (b->n_pairs == 0) return PHMM_OK;
  if (!b->pairs || !b->read_offsets || !b->hap_offsets) return PHMM_E_INVALID_ARG;
  if (b->total_read_bases < 0 || b->total_hap_bases < 0) return PHMM_E_INVALID_ARG;
  if (b->total_read_bases > 0 &&
      (!b->read_bases || !b->base_quals || !b->ins_quals || !b->del_quals || !b->gcp_quals))
    return PHMM_E_INVALID_ARG;
  if (b->total_hap_bases > 0 && !b->hap_bases) return PHMM_E_INVALID_ARG;
  return PHMM_OK;
}

// Enqueue the read-back of the call's FP64 underflow count (before the call's final sync).
phmm_status enqueue_underflow_readback(phmm_ctx* c) {
  if (c->st.n_pairs == 0) return PHMM_OK;
  unsigned long long* uf;
  ST_TRY(ws(c, B_UNDERFLOW, 1, &uf));
  CUDA_TRY(cudaMemcpyAsync(c->host_underflow, uf, sizeof(unsigned long long), cudaMemcpyDeviceToHost, c->stream));
  return PHMM_OK;
}

// After the call's final sync: the statistics read at the end.
void finish_stats(phmm_ctx* c) {
  if (c->st.n_pairs > 0) c->st.n_fp64_underflow = (int64_t)*c->host_underflow;
  if (c->timing_deferred) {
    acc_phases(c);
    c->timing_deferred = false;
  }
  c->st.kernel_launches = c->launches;
  if (c->flags & PHMM_FLAG_TIMING) {
    cudaEventSynchronize(c->ev[EV_END]);
    c->st.ms_total = ev_ms(c, EV_START, EV_END);
    c->st.ms_prep = c->acc.prep;
    c->st.ms_wavefront = c->acc.wf;
    c->st.ms_finalize = c->acc.fin;
    c->st.ms_rescue = c->prec == PHMM_PREC_FP64 ? 0.f : c->acc.resc;
  } else {
    c->st.ms_total = c->st.ms_h2d = c->st.ms_prep = c->st.ms_wavefront = -1.f;
    c->st.ms_rescue = c->st.ms_finalize = c->st.ms_d2h = -1.f;
  }
}

// ---- pipelined host-buffer call (DESIGN.md §1 "Host buffers")
// A host batch of kPipeMinPairs .. chunk_pairs pairs whose pairs use reads and haplotypes in
// ascending index ranges (GATK order: region after region) runs as chunks of pairs of growing
// size (n/F, n/F, 2n/F, 4n/F, ...; F = kPipeFirstDiv): the copy thread (Feeder) moves chunk
// k's new input bytes to the device on a copy stream while chunk k-1 computes, so only the
// first chunk's copy is exposed. Consecutive chunks alternate between two streams and two
// buffer sets, so that chunk k's preparation kernels and wavefront start as soon as chunk
// k-1's wavefront drains. Every chunk is an ordinary batch over the reads /
// haplotypes it uses (the chunked device call's rebasing, R14: a pair's arithmetic does not
// depend on its batch), validated as its bytes arrive; the FP32 chunks append their
// underflowing pairs to one list and ONE FP64 rescue pass over the whole batch follows, so the
// call has one host round trip per chunk plus two. Results are bitwise those of the one-pass call.
constexpr int64_t kPipeMinPairs = 1ll << 17;
// chunk plans (measured on C2, profiles/r02_pipe_sweep.txt): n/8 + 7n/8 for page-locked and
// pageable inputs alike (with streaming-store staging the staging memcpy keeps up as well; more,
// smaller chunks cost more in chunk boundaries than they hide)
constexpr int kPipeFirstDivPinned = 8, kPipeMaxChPinned = 2;
constexpr int kPipeFirstDivPageable = 8, kPipeMaxChPageable = 2;


// Chunk boundaries of a pipelined call: sub-chunks of n/F pairs, chunk k = 1, 1, 2, 4, ...
// sub-chunks (the last one takes the rest, at most maxch chunks). Index ranges per sub-chunk:
// a page-locked pair list is NOT read on the host -- a CPU pass over a page-locked buffer right
// before its DMA slows that copy up to 10x on the GPU hosts (lines held in CPU caches,
// tools/h2d_probe4.py) -- so the device computes them (k_chunk_ranges) after the pair list
// arrived; a pageable pair list (which is staged through the context's slots anyway) is
// scanned by the copy pool (pipe_scan), so the copies start at once.
void pipe_chunks(int64_t n, bool pinned, int64_t cap, std::vector<PipeChunk>& ch, int64_t* sub) {
  int div = pinned ? kPipeFirstDivPinned : kPipeFirstDivPageable;
  if (const char* e = std::getenv("PHMM_PIPE_FIRST")) div = std::max(2, std::min(1024, std::atoi(e)));
  int maxch = pinned ? kPipeMaxChPinned : kPipeMaxChPageable;
  if (const char* e = std::getenv("PHMM_PIPE_MAXCH")) maxch = std::max(2, std::atoi(e));
  *sub = std::min<int64_t>(std::max<int64_t>(1, n / div), cap);
  ch.clear();
  for (int64_t p = 0, sz = *sub, k = 0; p < n; ++k) {
    // no runt chunk at the end; at most maxch chunks
    const int64_t e = (n - (p + sz) < *sub || k + 1 >= maxch) ? n : p + sz;
    // chunks of at most cap pairs (the device-call chunk size: per-chunk tables and descriptors
    // stay a few GB), as whole sub-chunks
    for (int64_t a = p; a < e;) {
      const int64_t z = (e - a > cap) ? a + std::max<int64_t>(*sub, cap / *sub * *sub) : e;
      ch.push_back(PipeChunk{a, z, 0, 0, 0, 0, 0, 0});
      a = z;
    }
    p = e;
    if (k >= 1) sz *= 2;
  }
}

// Host scan of a pageable pair list: rng[4t..4t+3] = min/max read index, min/max haplotype
// index of sub-chunk t (k_chunk_ranges' layout). PHMM_E_INDEX for an index out of range.
phmm_status pipe_scan(phmm_ctx* c, const phmm_batch* b, int64_t sub, int64_t nsub, uint32_t* rng) {
  std::vector<uint8_t> bad((size_t)nsub, 0);
  const int32_t* pr = b->pairs;
  const int64_t nr = b->n_reads, nh = b->n_haps;
  c->stage.pool->for_each((int)nsub, [&](int t) {
    const int64_t a = (int64_t)t * sub, z = std::min(b->n_pairs, a + sub);
    int64_t rmin = INT64_MAX, rmax = -1, hmin = INT64_MAX, hmax = -1;
    for (int64_t p = a; p < z; ++p) {
      const int64_t r = pr[2 * p], h = pr[2 * p + 1];
      rmin = std::min(rmin, r); rmax = std::max(rmax, r);
      hmin = std::min(hmin, h); hmax = std::max(hmax, h);
    }
    if (z > a && (rmin < 0 || rmax >= nr || hmin < 0 || hmax >= nh)) bad[(size_t)t] = 1;
    uint32_t* g = rng + 4 * t;
    g[0] = z > a ? (uint32_t)rmin : 0xffffffffu; g[1] = z > a ? (uint32_t)rmax : 0u;
    g[2] = z > a ? (uint32_t)hmin : 0xffffffffu; g[3] = z > a ? (uint32_t)hmax : 0u;
  });
  for (uint8_t x : bad)
    if (x) return PHMM_E_INDEX;
  return PHMM_OK;
}

// Index ranges of the chunks from the sub-chunk ranges rng (k_chunk_ranges, validated
// indices) and the byte ranges each chunk brings. *useful = false (run as one chunk) when the
// first chunk would need more than half of the input bytes or the host offsets are not
// ascending over the chunks (the device validation then reports the batch).
void pipe_ranges(const phmm_batch* b, std::vector<PipeChunk>& ch, int64_t sub, const uint32_t* rng, bool* useful) {
  const int nch = (int)ch.size();
  int64_t rend = 0, hend = 0;
  for (int k = 0; k < nch; ++k) {
    PipeChunk& x = ch[(size_t)k];
    x.rlo = x.hlo = INT64_MAX;
    x.rhi = x.hhi = -1;
    for (int64_t t = x.p0 / sub; t * sub < x.p1; ++t) {
      const uint32_t* g = rng + 4 * t;
      if (g[0] == 0xffffffffu) continue;  // empty sub-chunk
      x.rlo = std::min<int64_t>(x.rlo, g[0]); x.rhi = std::max<int64_t>(x.rhi, g[1]);
      x.hlo = std::min<int64_t>(x.hlo, g[2]); x.hhi = std::max<int64_t>(x.hhi, g[3]);
    }
    rend = std::max(rend, x.rhi + 1);
    hend = std::max(hend, x.hhi + 1);
    x.rend = (k == nch - 1) ? b->n_reads : rend;  // the last chunk brings every remaining byte (all validated)
    x.hend = (k == nch - 1) ? b->n_haps : hend;
  }
  int64_t pr_ = 0, ph_ = 0;
  for (const PipeChunk& x : ch) {
    const int64_t r1 = b->read_offsets[x.rend], h1 = b->hap_offsets[x.hend];
    if (r1 < pr_ || r1 > b->total_read_bases || h1 < ph_ || h1 > b->total_hap_bases) {
      *useful = false;
      return;
    }
    pr_ = r1;
    ph_ = h1;
  }
  const int64_t rb = b->read_offsets[ch[0].rend], hb = b->hap_offsets[ch[0].hend];
  *useful = nch > 1 && 2 * (rb * 5 + hb) < b->total_read_bases * 5 + b->total_hap_bases;
}

phmm_status compute_host_pipe(phmm_ctx* c, const phmm_batch* b, double* out_log10, uint8_t* out_status) {
  cudaStream_t s = c->stream;
  if (!c->feeder) {
    c->feeder = new (std::nothrow) Feeder();
    if (!c->feeder) return PHMM_E_OOM;
    if (c->feeder->init(c->device) != cudaSuccess) {
      cudaGetLastError();
      delete c->feeder;
      c->feeder = nullptr;
      return PHMM_E_CUDA;
    }
  }
  std::vector<PipeChunk>& ch = c->pipe_chunks;
  int64_t sub = 0;
  const bool pinned = Stager::is_pinned(b->read_bases) && Stager::is_pinned(b->pairs);
  pipe_chunks(b->n_pairs, pinned, c->chunk_pairs, ch, &sub);
  // batches larger than one device chunk: every chunk runs its own FP64 rescue (compute_one), as
  // in the chunked device call (one rescue over all of them would outgrow the 32-bit code-region
  // offsets); otherwise one rescue pass over the whole batch at the end
  const bool chunk_rescue = b->n_pairs > c->chunk_pairs;
  const int64_t nsub = (b->n_pairs + sub - 1) / sub;
  const int nmax = (int)ch.size();
  while ((int)c->pipe_ev.size() < nmax + 4) {
    cudaEvent_t e;
    CUDA_TRY(cudaEventCreate(&e));  // timed: PHMM_PIPE_TRACE reads the copy timeline
    c->pipe_ev.push_back(e);
  }
  while (c->pipe_trace && (int)c->trace_ev.size() < 2 * nmax) {
    cudaEvent_t e;
    CUDA_TRY(cudaEventCreate(&e));
    c->trace_ev.push_back(e);
  }
  if (c->host_ranges_n < nsub) {
    if (c->host_ranges) cudaFreeHost(c->host_ranges);
    c->host_ranges = nullptr;
    c->host_ranges_n = 0;
    if (cudaMallocHost(&c->host_ranges, sizeof(uint32_t) * 4 * nsub) != cudaSuccess) {
      cudaGetLastError();
      c->host_ranges = nullptr;
      return PHMM_E_OOM;
    }
    c->host_ranges_n = nsub;
  }
  Feeder& F = *c->feeder;
  const cudaStream_t cs = F.stream();
  uint8_t *rb, *q, *qi, *qd, *qg, *hap;
  int64_t *roff, *hoff;
  int32_t* pairs;
  double* out;
  uint8_t* status = nullptr;
  const size_t nr = (size_t)b->total_read_bases, nh = (size_t)b->total_hap_bases;
  ST_TRY(ws(c, B_READ_BASES, nr, &rb));
  ST_TRY(ws(c, B_BQ, nr, &q));
  ST_TRY(ws(c, B_IQ, nr, &qi));
  ST_TRY(ws(c, B_DQ, nr, &qd));
  ST_TRY(ws(c, B_GQ, nr, &qg));
  ST_TRY(ws(c, B_HAP, nh, &hap));
  ST_TRY(ws(c, B_ROFF, (size_t)b->n_reads + 1, &roff));
  ST_TRY(ws(c, B_HOFF, (size_t)b->n_haps + 1, &hoff));
  ST_TRY(ws(c, B_PAIRS, (size_t)b->n_pairs * 2, &pairs));
  ST_TRY(ws(c, B_OUT_LOG10, (size_t)b->n_pairs, &out));
  if (out_status) ST_TRY(ws(c, B_OUT_STATUS, (size_t)b->n_pairs, &status));
  int32_t* rlist = nullptr;
  if (c->prec == PHMM_PREC_FP32_RESCUE) ST_TRY(ws(c, B_RLIST, (size_t)b->n_pairs, &rlist));
  Scalars *scal, *scal1;
  unsigned long long* uf;
  uint32_t* rng;
  ST_TRY(ws(c, B_SCAL, 1, &scal));
  ST_TRY(ws(c, B_UNDERFLOW, 1, &uf));
  ST_TRY(ws(c, B_CH_RANGES, (size_t)4 * nsub, &rng));
  c->set = 1;
  const phmm_status s1 = ws(c, B_SCAL, 1, &scal1);
  c->set = 0;
  ST_TRY(s1);
  // odd chunks run on a second stream with the second buffer set, so that chunk k + 1's
  // preparation and wavefront start while chunk k's wavefront drains
  if (!c->stream2) CUDA_TRY(cudaStreamCreateWithFlags(&c->stream2, cudaStreamNonBlocking));
  const cudaStream_t sk[2] = {s, c->stream2};
  Stager& S = c->stage;
  S.staged_bytes = 0;
  c->st = phmm_stats{};
  c->acc = PhaseMs{};
  c->st.n_pairs = b->n_pairs;
  c->timing_deferred = true;  // no per-chunk phase events (finish_stats overrides them)
  c->trace_host.clear();
  c->trace_t0 = std::chrono::steady_clock::now();
  ev_record(c, EV_START);
  cudaEvent_t ev_start = c->pipe_ev[nmax + 1], ev_s1 = c->pipe_ev[nmax + 2], ev_s1_end = c->pipe_ev[nmax + 3];
  cudaEvent_t ev_pre = c->pipe_ev[0];
  int nch = nmax;
  bool fed = false;
  // every exit from here on drains the copy stream (and stops the feeder) first
  auto run = [&]() -> phmm_status {
    // the copies start after whatever the compute stream ran before the call
    CUDA_TRY(cudaEventRecord(ev_start, s));
    CUDA_TRY(cudaStreamWaitEvent(cs, ev_start, 0));
    CUDA_TRY(fill_async(c, scal, 0, sizeof(Scalars), s));
    CUDA_TRY(fill_async(c, scal1, 0, sizeof(Scalars), s));
    CUDA_TRY(fill_async(c, uf, 0, sizeof(unsigned long long), s));
    c->gerr = &scal->err;  // validation and binning errors of every chunk
    if (pinned) {
      // step 1: offsets and pair list (this thread), the sub-chunks' index ranges on the device
      CUDA_TRY(S.h2d(roff, b->read_offsets, sizeof(int64_t) * (size_t)(b->n_reads + 1), cs));
      CUDA_TRY(S.h2d(hoff, b->hap_offsets, sizeof(int64_t) * (size_t)(b->n_haps + 1), cs));
      CUDA_TRY(S.h2d(pairs, b->pairs, sizeof(int32_t) * 2 * (size_t)b->n_pairs, cs));
      CUDA_TRY(cudaEventRecord(ev_pre, cs));
      k_ranges_init<<<grid_for(c, 4 * nsub), kThreads, 0, s>>>(rng, nsub);
      LAUNCHED(c);
      CUDA_TRY(cudaStreamWaitEvent(s, ev_pre, 0));
      const int bpc = (int)std::max<int64_t>(1, std::min<int64_t>((sub + kThreads - 1) / kThreads, 2 * c->nsm / nsub + 1));
      k_chunk_ranges<<<dim3((unsigned)bpc, (unsigned)nsub), kThreads, 0, s>>>(pairs, b->n_pairs, sub, b->n_reads,
                                                                                 b->n_haps, rng, c->gerr);
      LAUNCHED(c);
      CUDA_TRY(cudaMemcpyAsync(c->host_ranges, rng, sizeof(uint32_t) * 4 * (size_t)nsub, cudaMemcpyDeviceToHost, s));
      CUDA_TRY(cudaMemcpyAsync(&c->host_scal->err, c->gerr, sizeof(uint32_t), cudaMemcpyDeviceToHost, s));
      CUDA_TRY(cudaStreamSynchronize(s));
      trace_mark(c, "ranges");
      if (c->host_scal->err) return map_err(c->host_scal->err);  // index errors: nothing computed
    } else {
      ST_TRY(pipe_scan(c, b, sub, nsub, c->host_ranges));
      trace_mark(c, "ranges");
    }
    bool useful = false;
    pipe_ranges(b, ch, sub, c->host_ranges, &useful);
    if (!useful) {  // one chunk over the whole batch
      ch.assign(1, PipeChunk{0, b->n_pairs, 0, b->n_reads - 1, 0, b->n_haps - 1, b->n_reads, b->n_haps});
      if (b->n_reads == 0 || b->n_haps == 0) return PHMM_E_INDEX;  // cannot happen: ranges validated
    }
    nch = (int)ch.size();
    // step 2: chunk k's new input bytes, one event per chunk, by the copy thread
    std::vector<CopyJob>& J = c->pipe_jobs;
    std::vector<size_t>& G = c->pipe_groups;
    std::vector<cudaEvent_t>& E = c->pipe_gev;
    J.clear();
    G.clear();
    E.clear();
    const int g0 = pinned ? 0 : 1;  // pageable: the copy thread also stages offsets + pair list first
    if (!pinned) {
      J.push_back(CopyJob{roff, b->read_offsets, sizeof(int64_t) * (size_t)(b->n_reads + 1)});
      J.push_back(CopyJob{hoff, b->hap_offsets, sizeof(int64_t) * (size_t)(b->n_haps + 1)});
      J.push_back(CopyJob{pairs, b->pairs, sizeof(int32_t) * 2 * (size_t)b->n_pairs});
      G.push_back(J.size());
      E.push_back(ev_pre);
    }
    int64_t r0 = 0, h0 = 0;
    for (int i = 0; i < nch; ++i) {
      const PipeChunk& k = ch[(size_t)i];
      const int64_t r1 = b->read_offsets[k.rend], h1 = b->hap_offsets[k.hend];
      if (h1 > h0) J.push_back(CopyJob{hap + h0, b->hap_bases + h0, (size_t)(h1 - h0)});
      if (r1 > r0) {
        J.push_back(CopyJob{rb + r0, b->read_bases + r0, (size_t)(r1 - r0)});
        J.push_back(CopyJob{q + r0, b->base_quals + r0, (size_t)(r1 - r0)});
        J.push_back(CopyJob{qi + r0, b->ins_quals + r0, (size_t)(r1 - r0)});
        J.push_back(CopyJob{qd + r0, b->del_quals + r0, (size_t)(r1 - r0)});
        J.push_back(CopyJob{qg + r0, b->gcp_quals + r0, (size_t)(r1 - r0)});
      }
      G.push_back(J.size());
      E.push_back(c->pipe_ev[i + 1]);
      r0 = std::max(r0, r1);
      h0 = std::max(h0, h1);
    }
    F.trace = c->pipe_trace;
    F.job_us.clear();
    F.start(&S, &J, &G, &E);
    fed = true;
    // the offsets' validation (once they are on the device)
    if (!pinned) {
      CUDA_TRY(F.wait_group(0));
      CUDA_TRY(cudaStreamWaitEvent(s, ev_pre, 0));
    }
    k_validate_offsets<<<grid_for(c, b->n_reads + 1), kThreads, 0, s>>>(roff, b->n_reads, (int64_t)nr, c->gerr);
    LAUNCHED(c);
    k_validate_offsets<<<grid_for(c, b->n_haps + 1), kThreads, 0, s>>>(hoff, b->n_haps, (int64_t)nh, c->gerr);
    LAUNCHED(c);
    CUDA_TRY(cudaEventRecord(ev_s1, s));
    CUDA_TRY(cudaStreamWaitEvent(sk[1], ev_s1, 0));
    int64_t vr = 0, vh = 0;  // bytes validated so far
    for (int i = 0; i < nch; ++i) {
      const PipeChunk& k = ch[(size_t)i];
      const cudaStream_t si = sk[i & 1];
      c->set = i & 1;
      c->stream = si;
      trace_mark(c, "wait_group");
      CUDA_TRY(F.wait_group(i + g0));
      trace_mark(c, "group ready");
      CUDA_TRY(cudaStreamWaitEvent(si, c->pipe_ev[i + 1], 0));
      if (c->pipe_trace) CUDA_TRY(cudaEventRecord(c->trace_ev[2 * i], si));
      const int64_t r1 = b->read_offsets[k.rend], h1 = b->hap_offsets[k.hend];
      if (r1 > vr || h1 > vh) {
        const int64_t nrb = std::max<int64_t>(0, r1 - vr), nhb = std::max<int64_t>(0, h1 - vh);
        k_validate<<<grid_for(c, std::max(nhb, nrb / 4)), kThreads, 0, si>>>(
            hap + vh, nhb, rb + vr, q + vr, qi + vr, qd + vr, qg + vr, nrb, nullptr, -1, nullptr, -1, c->gerr);
        LAUNCHED(c);
        vr = std::max(vr, r1);
        vh = std::max(vh, h1);
      }
      const int64_t np = k.p1 - k.p0, nrk = k.rhi + 1 - k.rlo, nhk = k.hhi + 1 - k.hlo;
      int64_t *roff_c, *hoff_c;
      int32_t* pairs_c;
      ST_TRY(ws(c, B_CH_ROFF, (size_t)nrk + 1, &roff_c));
      ST_TRY(ws(c, B_CH_HOFF, (size_t)nhk + 1, &hoff_c));
      ST_TRY(ws(c, B_CH_PAIRS, (size_t)2 * np, &pairs_c));
      k_rebase_chunk<<<grid_for(c, std::max(std::max(nrk, nhk) + 1, np)), kThreads, 0, si>>>(
          roff, k.rlo, nrk, roff_c, hoff, k.hlo, nhk, hoff_c, pairs, k.p0, np, pairs_c, 0);
      LAUNCHED(c);
      trace_mark(c, "rebased");
      DevBatch dk{rb, q, qi, qd, qg, hap, roff_c, hoff_c, pairs_c, nrk, nhk, np, (int64_t)nr, (int64_t)nh};
      double* o = out + k.p0;
      uint8_t* st = status ? status + k.p0 : nullptr;
      if (c->prec == PHMM_PREC_FP64 || chunk_rescue) {
        ST_TRY(compute_one(c, dk, o, st));
      } else {
        PassInfo pi;
        uint8_t* hc = nullptr;
        int64_t total_hc = 0;
        ST_TRY(fp32_pass(c, dk, o, st, rlist, k.p0, &scal->n_rescue, &pi, &hc, &total_hc, false));
        ++c->st.n_chunks;
      }
      if (c->pipe_trace) CUDA_TRY(cudaEventRecord(c->trace_ev[2 * i + 1], si));
      trace_mark(c, "chunk issued");
    }
    c->set = 0;
    c->stream = s;
    c->gerr = nullptr;
    CUDA_TRY(cudaEventRecord(ev_s1_end, sk[1]));
    CUDA_TRY(cudaStreamWaitEvent(s, ev_s1_end, 0));
    const DevBatch d{rb, q, qi, qd, qg, hap, roff, hoff, pairs, b->n_reads, b->n_haps, b->n_pairs,
                     (int64_t)nr, (int64_t)nh};
    // the call's errors (validation of every chunk's bytes, binning), then the FP64 rescue
    CUDA_TRY(cudaMemcpyAsync(c->host_scal, scal, sizeof(Scalars), cudaMemcpyDeviceToHost, s));
    CUDA_TRY(cudaStreamSynchronize(s));
    if (c->host_scal->err) return map_err(c->host_scal->err);
    if (c->prec == PHMM_PREC_FP32_RESCUE && !chunk_rescue) {
      const int64_t n_resc = c->host_scal->n_rescue;
      c->st.n_rescued += n_resc;
      if (n_resc > 0) ST_TRY(rescue_pass(c, d, out, status, rlist, n_resc, nullptr, 0, false));
    }
    return PHMM_OK;
  };
  phmm_status st = run();
  c->set = 0;
  c->stream = s;
  c->gerr = nullptr;
  if (st != PHMM_OK && fed) F.cancel();
  const cudaError_t fe = fed ? F.wait_all() : cudaStreamSynchronize(cs);
  if (st == PHMM_OK && fe != cudaSuccess) st = PHMM_E_CUDA;
  if (st != PHMM_OK) {
    cudaStreamSynchronize(sk[1]);
    cudaStreamSynchronize(s);
    cudaGetLastError();
    return st;
  }
  ST_TRY(enqueue_underflow_readback(c));
  ev_record(c, EV_D2H);
  {
    Nvtx nv("phmm:d2h");
    CUDA_TRY(S.d2h(out_log10, out, sizeof(double) * b->n_pairs, s, false));  // synchronised below
    if (out_status) CUDA_TRY(S.d2h(out_status, status, b->n_pairs, s));
  }
  ev_record(c, EV_END);
  CUDA_TRY(cudaStreamSynchronize(s));
  finish_stats(c);
  if (c->pipe_trace) {
    auto t = [&](cudaEvent_t e) {
      float ms = -1.f;
      if (cudaEventElapsedTime(&ms, c->ev[EV_START], e) != cudaSuccess) cudaGetLastError();
      return ms;
    };
    std::fprintf(stderr, "phmm pipe: %d chunks, offsets + pairs copied %.3f ms\n", nch, t(ev_pre));
    for (int i = 0; i < nch; ++i)
      std::fprintf(stderr, "  chunk %d pairs [%lld, %lld): copied %.3f, compute %.3f .. %.3f ms\n", i,
                   (long long)ch[(size_t)i].p0, (long long)ch[(size_t)i].p1, t(c->pipe_ev[i + 1]),
                   t(c->trace_ev[2 * i]), t(c->trace_ev[2 * i + 1]));
    std::fprintf(stderr, "  rescue + d2h from %.3f, end %.3f ms\n", t(c->trace_ev[2 * nch - 1]), t(c->ev[EV_END]));
    std::fprintf(stderr, "  host:");
    for (auto& h : c->trace_host) std::fprintf(stderr, " %s %.0f,", h.first, h.second);
    std::fprintf(stderr, "\n");
  }
  // per-phase times are not split out in a pipelined call (chunks overlap the copies)
  c->st.ms_h2d = c->st.ms_prep = c->st.ms_wavefront = c->st.ms_rescue = c->st.ms_finalize = -1.f;
  c->st.ms_d2h = ev_ms(c, EV_D2H, EV_END);
  c->st.staged_bytes = S.staged_bytes;
  return PHMM_OK;
}

phmm_status compute_host(phmm_ctx* c, const phmm_batch* b, double* out_log10, uint8_t* out_status) {
  ST_TRY(check_batch_args(b));
  if (b->n_pairs > 0 && !out_log10) return PHMM_E_INVALID_ARG;
  if (cudaSetDevice(c->device) != cudaSuccess) {
    cudaGetLastError();
    return PHMM_E_CUDA;
  }
  c->launches = 0;
  if (b->n_pairs == 0) {
    c->st = phmm_stats{};
    return PHMM_OK;
  }
  // host-side size checks that need the host offsets
  if (b->read_offsets[b->n_reads] != b->total_read_bases || b->hap_offsets[b->n_haps] != b->total_hap_bases)
    return PHMM_E_INVALID_ARG;
  if (b->n_pairs >= c->pipe_min && c->pipe)
    return compute_host_pipe(c, b, out_log10, out_status);
  cudaStream_t s = c->stream;
  uint8_t *rb, *q, *qi, *qd, *qg, *hap;
  int64_t *roff, *hoff;
  int32_t* pairs;
  double* out;
  uint8_t* status = nullptr;
  const size_t nr = (size_t)b->total_read_bases, nh = (size_t)b->total_hap_bases;
  ST_TRY(ws(c, B_READ_BASES, nr, &rb));
  ST_TRY(ws(c, B_BQ, nr, &q));
  ST_TRY(ws(c, B_IQ, nr, &qi));
  ST_TRY(ws(c, B_DQ, nr, &qd));
  ST_TRY(ws(c, B_GQ, nr, &qg));
  ST_TRY(ws(c, B_HAP, nh, &hap));
  ST_TRY(ws(c, B_ROFF, (size_t)b->n_reads + 1, &roff));
  ST_TRY(ws(c, B_HOFF, (size_t)b->n_haps + 1, &hoff));
  ST_TRY(ws(c, B_PAIRS, (size_t)b->n_pairs * 2, &pairs));
  ST_TRY(ws(c, B_OUT_LOG10, (size_t)b->n_pairs, &out));
  if (out_status) ST_TRY(ws(c, B_OUT_STATUS, (size_t)b->n_pairs, &status));
  // H2D: page-locked caller buffers directly, pageable ones through the context's pinned
  // staging ring (host_stage.h); the small arrays first
  Stager& S = c->stage;
  S.staged_bytes = 0;
  ev_record(c, EV_START);
  {
    Nvtx nv("phmm:h2d");
    CUDA_TRY(S.h2d(roff, b->read_offsets, sizeof(int64_t) * (b->n_reads + 1), s));
    CUDA_TRY(S.h2d(hoff, b->hap_offsets, sizeof(int64_t) * (b->n_haps + 1), s));
    CUDA_TRY(S.h2d(pairs, b->pairs, sizeof(int32_t) * 2 * b->n_pairs, s));
    CUDA_TRY(S.h2d(hap, b->hap_bases, nh, s));
    CUDA_TRY(S.h2d(rb, b->read_bases, nr, s));
    CUDA_TRY(S.h2d(q, b->base_quals, nr, s));
    CUDA_TRY(S.h2d(qi, b->ins_quals, nr, s));
    CUDA_TRY(S.h2d(qd, b->del_quals, nr, s));
    CUDA_TRY(S.h2d(qg, b->gcp_quals, nr, s));
  }
  ev_record(c, EV_H2D);
  DevBatch d{rb, q, qi, qd, qg, hap, roff, hoff, pairs, b->n_reads, b->n_haps, b->n_pairs, (int64_t)nr, (int64_t)nh};
  phmm_status st = compute_dev(c, d, out, status);
  if (st != PHMM_OK) {
    cudaStreamSynchronize(s);
    cudaGetLastError();
    return st;
  }
  ST_TRY(enqueue_underflow_readback(c));
  ev_record(c, EV_D2H);
  {
    Nvtx nv("phmm:d2h");
    CUDA_TRY(S.d2h(out_log10, out, sizeof(double) * b->n_pairs, s, false));  // synchronised below
    if (out_status) CUDA_TRY(S.d2h(out_status, status, b->n_pairs, s));
  }
  ev_record(c, EV_END);
  CUDA_TRY(cudaStreamSynchronize(s));
  finish_stats(c);
  c->st.ms_h2d = ev_ms(c, EV_START, EV_H2D);
  c->st.ms_d2h = ev_ms(c, EV_D2H, EV_END);
  c->st.staged_bytes = S.staged_bytes;
  return PHMM_OK;
}


// ------------------------------------------------------------ phmm_submit / phmm_wait
// Region-sized batches (~189 pairs in the paper, L24@575) cost ~0.6 ms per synchronous call
// however small they are (launches and size read-backs), so the library offers a submission
// queue: phmm_submit appends a batch to a host ARENA (inputs gathered back to back, offsets
// and pair indices rebased) and returns a ticket at once; a worker thread takes the whole
// arena whenever it is idle and runs it as ONE batch (compute_host), while later submissions
// fill the other arena; then it copies each batch's results to its caller's buffers. Results
// are bitwise those of separate calls (a pair's arithmetic never depends on its batch, R14).
// If the coalesced run fails (an input-content error in one of the batches), every batch of
// that run is re-run on its own, so each ticket gets its own status.
struct AsyncJob {
  uint64_t ticket;
  int64_t p0, np, r0, nr, h0, nh, rb0, nrb, hb0, nhb;  // the batch's place in its arena
  double* out;
  uint8_t* status;
};

// Growable host byte buffer of an arena. Plain (pageable) memory: growing it costs a
// realloc, not a page-locking allocation (which takes milliseconds and serialises with the
// driver); compute_host stages it to the device through the context's pinned ring.
struct HostVec {
  uint8_t* p = nullptr;
  size_t n = 0, cap = 0;
  bool reserve(size_t want) {
    if (want <= cap) return true;
    const size_t c2 = std::max(want, cap * 2 + ((size_t)1 << 20));
    void* q = std::realloc(p, c2);
    if (!q) return false;
    p = static_cast<uint8_t*>(q);
    cap = c2;
    return true;
  }
  void release() {
    std::free(p);
    p = nullptr;
    n = cap = 0;
  }
};

struct Arena {
  HostVec rb, q, qi, qd, qg, hb, roff, hoff, pairs, out, st;
  std::vector<AsyncJob> jobs;
  int64_t n_reads = 0, n_haps = 0, n_pairs = 0;
  bool any_status = false;
  void clear() {
    for (HostVec* v : {&rb, &q, &qi, &qd, &qg, &hb, &roff, &hoff, &pairs, &out, &st}) v->n = 0;
    jobs.clear();
    n_reads = n_haps = n_pairs = 0;
    any_status = false;
  }
  void release() {
    for (HostVec* v : {&rb, &q, &qi, &qd, &qg, &hb, &roff, &hoff, &pairs, &out, &st}) v->release();
  }
};

// A no-copy batch (phmm_compute_batch_async): the caller's pointers, valid until phmm_wait.
struct XJob {
  uint64_t ticket;
  phmm_batch b;
  double* out;
  uint8_t* status;
  int iset;        // its async input region
  bool prefetched; // its inputs were copied to that region while the previous batch computed
  bool tried;      // a prefetch was attempted
};

struct AsyncQueue {
  std::mutex mu;
  std::condition_variable cv, done_cv;
  Arena arena[2];
  int fill = 0;              // the arena submissions append to
  bool stop = false, busy = false;
  uint64_t next_ticket = 1;
  std::map<uint64_t, phmm_status> done;  // finished tickets not yet waited for
  std::set<uint64_t> outstanding;        // submitted tickets not yet waited for
  std::thread worker;
  std::deque<XJob> xjobs;                // phmm_compute_batch_async: no-copy batches, in order
  int xset = 1;                          // the async input region (1 / 2) of the next no-copy batch
};

void run_arena(phmm_ctx* c, Arena& A) {
  Nvtx nvtx_("phmm:submit_run");
  std::vector<phmm_status> st(A.jobs.size(), PHMM_OK);
  auto batch_of = [&](int64_t r0, int64_t nr, int64_t h0, int64_t nh, int64_t p0, int64_t np, int64_t rb0,
                      int64_t hb0, std::vector<int64_t>* ro, std::vector<int64_t>* ho, std::vector<int32_t>* pr) {
    phmm_batch b{};
    const int64_t* aro = reinterpret_cast<const int64_t*>(A.roff.p);
    const int64_t* aho = reinterpret_cast<const int64_t*>(A.hoff.p);
    const int32_t* apr = reinterpret_cast<const int32_t*>(A.pairs.p);
    ro->resize(nr + 1);
    ho->resize(nh + 1);
    pr->resize(2 * np);
    for (int64_t i = 0; i <= nr; ++i) (*ro)[i] = aro[r0 + i] - rb0;
    for (int64_t i = 0; i <= nh; ++i) (*ho)[i] = aho[h0 + i] - hb0;
    for (int64_t i = 0; i < np; ++i) {
      (*pr)[2 * i] = apr[2 * (p0 + i)] - (int32_t)r0;
      (*pr)[2 * i + 1] = apr[2 * (p0 + i) + 1] - (int32_t)h0;
    }
    b.read_bases = A.rb.p + rb0; b.base_quals = A.q.p + rb0; b.ins_quals = A.qi.p + rb0;
    b.del_quals = A.qd.p + rb0; b.gcp_quals = A.qg.p + rb0; b.hap_bases = A.hb.p + hb0;
    b.read_offsets = ro->data(); b.hap_offsets = ho->data(); b.pairs = pr->data();
    b.n_reads = nr; b.n_haps = nh; b.n_pairs = np;
    b.total_read_bases = (*ro)[nr];
    b.total_hap_bases = (*ho)[nh];
    return b;
  };
  phmm_status all = PHMM_OK;
  {
    phmm_batch b{};
    b.read_bases = A.rb.p; b.base_quals = A.q.p; b.ins_quals = A.qi.p; b.del_quals = A.qd.p; b.gcp_quals = A.qg.p;
    b.read_offsets = reinterpret_cast<const int64_t*>(A.roff.p); b.n_reads = A.n_reads;
    b.hap_bases = A.hb.p; b.hap_offsets = reinterpret_cast<const int64_t*>(A.hoff.p); b.n_haps = A.n_haps;
    b.pairs = reinterpret_cast<const int32_t*>(A.pairs.p); b.n_pairs = A.n_pairs;
    b.total_read_bases = (int64_t)A.rb.n; b.total_hap_bases = (int64_t)A.hb.n;
    std::lock_guard<std::mutex> g(c->run_mu);
    all = compute_host(c, &b, reinterpret_cast<double*>(A.out.p), A.any_status ? A.st.p : nullptr);
  }
  if (all != PHMM_OK) {  // attribute the failure: every batch of the run on its own
    std::vector<int64_t> ro, ho;
    std::vector<int32_t> pr;
    for (size_t k = 0; k < A.jobs.size(); ++k) {
      const AsyncJob& j = A.jobs[k];
      phmm_batch b = batch_of(j.r0, j.nr, j.h0, j.nh, j.p0, j.np, j.rb0, j.hb0, &ro, &ho, &pr);
      std::lock_guard<std::mutex> g(c->run_mu);
      st[k] = compute_host(c, &b, reinterpret_cast<double*>(A.out.p) + j.p0, A.any_status ? A.st.p + j.p0 : nullptr);
    }
  }
  for (size_t k = 0; k < A.jobs.size(); ++k) {
    const AsyncJob& j = A.jobs[k];
    if (st[k] != PHMM_OK || j.np == 0) continue;
    std::memcpy(j.out, reinterpret_cast<double*>(A.out.p) + j.p0, sizeof(double) * (size_t)j.np);
    if (j.status) std::memcpy(j.status, A.st.p + j.p0, (size_t)j.np);
  }
  AsyncQueue* q = c->aq;
  std::lock_guard<std::mutex> g(q->mu);
  for (size_t k = 0; k < A.jobs.size(); ++k) q->done[A.jobs[k].ticket] = st[k];
  q->done_cv.notify_all();
}

// Copy every input array of an all-page-locked no-copy batch into its async input region on the
// prefetch stream (ends with pf_ev). false: not prefetchable (a pageable array) or a copy failed.
bool prefetch_inputs(phmm_ctx* c, XJob& j) {
  const phmm_batch& b = j.b;
  const void* arrs[9] = {b.read_bases, b.base_quals, b.ins_quals, b.del_quals, b.gcp_quals, b.hap_bases,
                         b.read_offsets, b.hap_offsets, b.pairs};
  for (const void* a : arrs)
    if (a && !Stager::is_pinned(a)) return false;
  if (!c->pf_stream && cudaStreamCreateWithFlags(&c->pf_stream, cudaStreamNonBlocking) != cudaSuccess) {
    cudaGetLastError();
    c->pf_stream = nullptr;
    return false;
  }
  if (!c->pf_ev && cudaEventCreateWithFlags(&c->pf_ev, cudaEventDisableTiming) != cudaSuccess) {
    cudaGetLastError();
    c->pf_ev = nullptr;
    return false;
  }
  const int keep = c->iset;
  c->iset = j.iset;
  const size_t nr = (size_t)b.total_read_bases, nh = (size_t)b.total_hap_bases;
  uint8_t* d[6];
  int64_t *roff, *hoff;
  int32_t* pairs;
  bool ok = ws(c, B_READ_BASES, nr, &d[0]) == PHMM_OK && ws(c, B_BQ, nr, &d[1]) == PHMM_OK &&
            ws(c, B_IQ, nr, &d[2]) == PHMM_OK && ws(c, B_DQ, nr, &d[3]) == PHMM_OK &&
            ws(c, B_GQ, nr, &d[4]) == PHMM_OK && ws(c, B_HAP, nh, &d[5]) == PHMM_OK &&
            ws(c, B_ROFF, (size_t)b.n_reads + 1, &roff) == PHMM_OK &&
            ws(c, B_HOFF, (size_t)b.n_haps + 1, &hoff) == PHMM_OK &&
            ws(c, B_PAIRS, (size_t)b.n_pairs * 2, &pairs) == PHMM_OK;
  c->iset = keep;
  if (!ok) return false;
  cudaStream_t s = c->pf_stream;
  const size_t sz[6] = {nr, nr, nr, nr, nr, nh};
  for (int i = 0; i < 6 && ok; ++i)
    ok = sz[i] == 0 || cudaMemcpyAsync(d[i], arrs[i], sz[i], cudaMemcpyHostToDevice, s) == cudaSuccess;
  ok = ok && cudaMemcpyAsync(roff, b.read_offsets, 8 * (size_t)(b.n_reads + 1), cudaMemcpyHostToDevice, s) == cudaSuccess;
  ok = ok && cudaMemcpyAsync(hoff, b.hap_offsets, 8 * (size_t)(b.n_haps + 1), cudaMemcpyHostToDevice, s) == cudaSuccess;
  ok = ok && cudaMemcpyAsync(pairs, b.pairs, 8 * (size_t)b.n_pairs, cudaMemcpyHostToDevice, s) == cudaSuccess;
  ok = ok && cudaEventRecord(c->pf_ev, s) == cudaSuccess;
  if (!ok) {
    cudaGetLastError();
    cudaStreamSynchronize(s);
  }
  return ok;
}

void maybe_prefetch(phmm_ctx* c) {
  if (!c->in_xjob || !c->aq) return;
  AsyncQueue* q = c->aq;
  std::lock_guard<std::mutex> g(q->mu);
  if (q->xjobs.size() > 1 && !q->xjobs[1].prefetched && !q->xjobs[1].tried) {
    q->xjobs[1].tried = true;
    q->xjobs[1].prefetched = prefetch_inputs(c, q->xjobs[1]);
  }
}

// One no-copy batch. Prefetched: its inputs are in its async region (after pf_ev): the device
// path on them, then the results to the caller's buffers; otherwise the host-buffer call with
// that region as its input buffers. Bitwise phmm_compute_batch (R14).
phmm_status run_xjob(phmm_ctx* c, XJob& j) {
  Nvtx nvtx_("phmm:async_batch");
  const phmm_batch* b = &j.b;
  c->iset = j.iset;
  phmm_status st = PHMM_OK;
  if (!j.prefetched) {
    st = compute_host(c, b, j.out, j.status);
    c->iset = 0;
    return st;
  }
  auto run = [&]() -> phmm_status {
    c->launches = 0;
    if (b->n_pairs == 0) {
      c->st = phmm_stats{};
      return PHMM_OK;
    }
    uint8_t *rb, *q, *qi, *qd, *qg, *hap;
    int64_t *roff, *hoff;
    int32_t* pairs;
    double* out;
    uint8_t* status = nullptr;
    const size_t nr = (size_t)b->total_read_bases, nh = (size_t)b->total_hap_bases;
    ST_TRY(ws(c, B_READ_BASES, nr, &rb));
    ST_TRY(ws(c, B_BQ, nr, &q));
    ST_TRY(ws(c, B_IQ, nr, &qi));
    ST_TRY(ws(c, B_DQ, nr, &qd));
    ST_TRY(ws(c, B_GQ, nr, &qg));
    ST_TRY(ws(c, B_HAP, nh, &hap));
    ST_TRY(ws(c, B_ROFF, (size_t)b->n_reads + 1, &roff));
    ST_TRY(ws(c, B_HOFF, (size_t)b->n_haps + 1, &hoff));
    ST_TRY(ws(c, B_PAIRS, (size_t)b->n_pairs * 2, &pairs));
    ST_TRY(ws(c, B_OUT_LOG10, (size_t)b->n_pairs, &out));
    if (j.status) ST_TRY(ws(c, B_OUT_STATUS, (size_t)b->n_pairs, &status));
    cudaStream_t s = c->stream;
    ev_record(c, EV_START);
    CUDA_TRY(cudaStreamWaitEvent(s, c->pf_ev, 0));
    ev_record(c, EV_H2D);
    DevBatch d{rb, q, qi, qd, qg, hap, roff, hoff, pairs, b->n_reads, b->n_haps, b->n_pairs, (int64_t)nr, (int64_t)nh};
    phmm_status e = compute_dev(c, d, out, status);
    if (e != PHMM_OK) {
      cudaStreamSynchronize(s);
      cudaGetLastError();
      return e;
    }
    ST_TRY(enqueue_underflow_readback(c));
    ev_record(c, EV_D2H);
    CUDA_TRY(c->stage.d2h(j.out, out, sizeof(double) * b->n_pairs, s, false));  // synchronised below
    if (j.status) CUDA_TRY(c->stage.d2h(j.status, status, b->n_pairs, s));
    ev_record(c, EV_END);
    CUDA_TRY(cudaStreamSynchronize(s));
    finish_stats(c);
    c->st.ms_h2d = -1.f;  // the prefetch overlapped the previous batch
    c->st.ms_d2h = ev_ms(c, EV_D2H, EV_END);
    c->st.staged_bytes = c->stage.staged_bytes;
    return PHMM_OK;
  };
  c->stage.staged_bytes = 0;
  st = run();
  c->iset = 0;
  return st;
}

void async_worker(phmm_ctx* c) {
  AsyncQueue* q = c->aq;
  cudaSetDevice(c->device);
  while (true) {
    int k;
    // no-copy batches first (in their submission order); the next one's inputs are prefetched
    // while this one computes
    {
      std::unique_lock<std::mutex> lk(q->mu);
      q->cv.wait(lk, [&] { return q->stop || !q->arena[q->fill].jobs.empty() || !q->xjobs.empty(); });
      if (!q->xjobs.empty()) {
        XJob j = q->xjobs.front();
        q->busy = true;
        lk.unlock();
        phmm_status st;
        {
          std::lock_guard<std::mutex> g(c->run_mu);
          // the next batch (its region differs from this one's: regions alternate) is prefetched
          // at this batch's first host round trip (maybe_prefetch), after its first kernels are
          // queued, not before them
          c->in_xjob = true;
          st = run_xjob(c, j);
          c->in_xjob = false;
        }
        lk.lock();
        q->xjobs.pop_front();
        q->done[j.ticket] = st;
        q->busy = false;
        q->done_cv.notify_all();
        continue;
      }
      if (q->arena[q->fill].jobs.empty()) return;  // stop, nothing left
      k = q->fill;
      q->fill ^= 1;  // submissions go to the other arena while this one runs
      q->busy = true;
    }
    run_arena(c, q->arena[k]);
    std::lock_guard<std::mutex> g(q->mu);
    q->arena[k].clear();
    q->busy = false;
    q->done_cv.notify_all();
  }
}

void async_stop(phmm_ctx* c) {
  AsyncQueue* q = c->aq;
  if (!q) return;
  {
    std::lock_guard<std::mutex> g(q->mu);
    q->stop = true;
  }
  q->cv.notify_all();
  if (q->worker.joinable()) q->worker.join();
  q->arena[0].release();
  q->arena[1].release();
  delete q;
  c->aq = nullptr;
}

// host-side checks of a submitted batch (the device checks the contents when it runs)
phmm_status submit_checks(const phmm_batch* b) {
  ST_TRY(check_batch_args(b));
  if (b->n_pairs == 0) return PHMM_OK;
  const int64_t* ro = b->read_offsets;
  const int64_t* ho = b->hap_offsets;
  if (ro[0] != 0 || ho[0] != 0 || ro[b->n_reads] != b->total_read_bases || ho[b->n_haps] != b->total_hap_bases)
    return PHMM_E_INVALID_ARG;
  for (int64_t i = 0; i < b->n_reads; ++i)
    if (ro[i + 1] < ro[i]) return PHMM_E_INVALID_ARG;
  for (int64_t i = 0; i < b->n_haps; ++i)
    if (ho[i + 1] < ho[i]) return PHMM_E_INVALID_ARG;
  for (int64_t p = 0; p < b->n_pairs; ++p) {
    const int32_t r = b->pairs[2 * p], h = b->pairs[2 * p + 1];
    if (r < 0 || r >= b->n_reads || h < 0 || h >= b->n_haps) return PHMM_E_INDEX;
  }
  return PHMM_OK;
}

}  // namespace

extern "C" {

int phmm_abi_version(void) { return PHMM_ABI_VERSION; }



const char* phmm_status_string(phmm_status s) {
  switch (s) {
    case PHMM_OK: return "ok";
    case PHMM_E_INVALID_ARG: return "invalid argument";
    case PHMM_E_INVALID_BASE: return "invalid base (expected A, C, G, T or N)";
    case PHMM_E_INVALID_QUAL: return "invalid quality (> 127)";
    case PHMM_E_EMPTY_SEQ: return "empty read or haplotype";
    case PHMM_E_INDEX: return "pair index out of range";
    case PHMM_E_CUDA: return "CUDA error";
    case PHMM_E_OOM: return "out of memory";
  }
  return "unknown status";
}

phmm_status phmm_create(phmm_ctx** out, const phmm_config* cfg) {
  if (!out) return PHMM_E_INVALID_ARG;
  *out = nullptr;
  phmm_config def{};
  def.device = 0;
  def.precision = PHMM_PREC_FP32_RESCUE;
  def.cuda_stream = nullptr;
  def.flags = 0;
  def.col_bucket = 0;
  if (!cfg) cfg = &def;
  if (cfg->precision != PHMM_PREC_FP64 && cfg->precision != PHMM_PREC_FP32_RESCUE) return PHMM_E_INVALID_ARG;
  if (cfg->col_bucket < 0 || cfg->col_bucket > 64) return PHMM_E_INVALID_ARG;
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess) {
    cudaGetLastError();
    return PHMM_E_CUDA;
  }
  if (cfg->device < 0 || cfg->device >= ndev) return PHMM_E_INVALID_ARG;
  phmm_ctx* c = new (std::nothrow) phmm_ctx();
  if (!c) return PHMM_E_OOM;
  c->device = cfg->device;
  c->prec = cfg->precision;
  c->flags = cfg->flags;
  c->bucket = cfg->col_bucket > 0 ? cfg->col_bucket : 4;
  auto fail = [&](phmm_status s) {
    phmm_destroy(c);
    return s;
  };
  if (cudaSetDevice(c->device) != cudaSuccess) return fail(PHMM_E_CUDA);
  if (cudaDeviceGetAttribute(&c->nsm, cudaDevAttrMultiProcessorCount, c->device) != cudaSuccess ||
      cudaDeviceGetAttribute(&c->smem_per_sm, cudaDevAttrMaxSharedMemoryPerMultiprocessor, c->device) !=
          cudaSuccess ||
      cudaDeviceGetAttribute(&c->smem_reserved, cudaDevAttrReservedSharedMemoryPerBlock, c->device) !=
          cudaSuccess ||
      cudaDeviceGetAttribute(&c->smem_optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, c->device) != cudaSuccess)
    return fail(PHMM_E_CUDA);
  if (wf_set_max_smem(c->smem_optin) != cudaSuccess) return fail(PHMM_E_CUDA);
  if (cfg->cuda_stream) {
    c->stream = reinterpret_cast<cudaStream_t>(cfg->cuda_stream);
  } else {
    if (cudaStreamCreateWithFlags(&c->owned_stream, cudaStreamNonBlocking) != cudaSuccess) {
      c->owned_stream = nullptr;
      return fail(PHMM_E_CUDA);
    }
    c->stream = c->owned_stream;
  }
  if (cudaMallocHost(&c->host_scal, sizeof(Scalars)) != cudaSuccess) {
    c->host_scal = nullptr;
    return fail(PHMM_E_OOM);
  }
  if (cudaMallocHost(&c->host_sizes, 2 * sizeof(int64_t)) != cudaSuccess) {
    c->host_sizes = nullptr;
    return fail(PHMM_E_OOM);
  }
  if (cudaMallocHost(&c->host_underflow, sizeof(unsigned long long)) != cudaSuccess) {
    c->host_underflow = nullptr;
    return fail(PHMM_E_OOM);
  }
  *c->host_underflow = 0;
  for (int i = 0; i < kEvents; ++i)
    if (cudaEventCreate(&c->ev[i]) != cudaSuccess) return fail(PHMM_E_CUDA);
  {
    int threads = (int)std::min(8u, std::max(1u, std::thread::hardware_concurrency() / 2));
    if (const char* e = std::getenv("PHMM_STAGE_THREADS")) threads = std::max(1, std::min(64, std::atoi(e)));
    if (c->stage.init(threads) != cudaSuccess) {
      cudaGetLastError();
      return fail(PHMM_E_OOM);
    }
  }
  if (const char* e = std::getenv("PHMM_PIPE")) c->pipe = std::atoi(e) != 0;
  if (const char* e = std::getenv("PHMM_PIPE_MIN")) c->pipe_min = std::max<int64_t>(16, std::atoll(e));
  if (const char* e = std::getenv("PHMM_PIPE_TRACE")) c->pipe_trace = std::atoi(e) != 0;
  if (const char* e = std::getenv("PHMM_CHUNK_PAIRS")) c->chunk_pairs = std::max<int64_t>(64, std::atoll(e));
  *out = c;
  return PHMM_OK;
}

void phmm_destroy(phmm_ctx* c) {
  if (!c) return;
  async_stop(c);  // finishes every submitted batch first
  cudaSetDevice(c->device);
  if (c->stream) cudaStreamSynchronize(c->stream);
  for (int i = 0; i < B_COUNT; ++i)
    if (c->buf[i].p) cudaFree(c->buf[i].p);
  for (int i = B_COUNT; i < 4 * B_COUNT; ++i)
    if (c->buf[i].p) cudaFree(c->buf[i].p);
  if (c->pf_stream) {
    cudaStreamSynchronize(c->pf_stream);
    cudaStreamDestroy(c->pf_stream);
  }
  if (c->pf_ev) cudaEventDestroy(c->pf_ev);
  if (c->stream2) {
    cudaStreamSynchronize(c->stream2);
    cudaStreamDestroy(c->stream2);
  }
  for (int i = 0; i < kEvents; ++i)
    if (c->ev[i]) cudaEventDestroy(c->ev[i]);
  delete c->feeder;  // joins the copy thread, drains its stream
  c->feeder = nullptr;
  for (cudaEvent_t e : c->pipe_ev) cudaEventDestroy(e);
  c->pipe_ev.clear();
  for (cudaEvent_t e : c->trace_ev) cudaEventDestroy(e);
  c->trace_ev.clear();
  c->stage.release();
  if (c->host_scal) cudaFreeHost(c->host_scal);
  if (c->host_sizes) cudaFreeHost(c->host_sizes);
  if (c->host_ranges) cudaFreeHost(c->host_ranges);
  if (c->host_underflow) cudaFreeHost(c->host_underflow);
  if (c->owned_stream) {
    cudaStreamSynchronize(c->owned_stream);
    cudaStreamDestroy(c->owned_stream);
  }
  cudaGetLastError();
  delete c;
}

phmm_status phmm_get_stats(const phmm_ctx* c, phmm_stats* out) {
  if (!c || !out) return PHMM_E_INVALID_ARG;
  *out = c->st;
  return PHMM_OK;
}

phmm_status phmm_set_stream(phmm_ctx* c, void* stream) {
  if (!c) return PHMM_E_INVALID_ARG;
  std::lock_guard<std::mutex> g_(c->run_mu);
  if (cudaSetDevice(c->device) != cudaSuccess) {
    cudaGetLastError();
    return PHMM_E_CUDA;
  }
  cudaStream_t s = stream ? reinterpret_cast<cudaStream_t>(stream) : c->owned_stream;
  if (!s) {  // created on a caller's stream: make a private one for the NULL case
    if (cudaStreamCreateWithFlags(&c->owned_stream, cudaStreamNonBlocking) != cudaSuccess) {
      cudaGetLastError();
      c->owned_stream = nullptr;
      return PHMM_E_CUDA;
    }
    s = c->owned_stream;
  }
  c->stream = s;
  return PHMM_OK;
}


phmm_status phmm_submit(phmm_ctx* c, const phmm_batch* b, double* out_log10, uint8_t* out_status, uint64_t* ticket) {
  if (!c || !ticket) return PHMM_E_INVALID_ARG;
  ST_TRY(submit_checks(b));
  if (b->n_pairs > 0 && !out_log10) return PHMM_E_INVALID_ARG;
  if (!c->aq) {
    c->aq = new (std::nothrow) AsyncQueue();
    if (!c->aq) return PHMM_E_OOM;
    c->aq->worker = std::thread(async_worker, c);
  }
  AsyncQueue* q = c->aq;
  std::lock_guard<std::mutex> g(q->mu);
  if (q->stop) return PHMM_E_INVALID_ARG;
  Arena& A = q->arena[q->fill];
  const int64_t np = b->n_pairs, nr = b->n_reads, nh = b->n_haps;
  if (A.n_pairs + np > 0x7fffffffLL || A.n_reads + nr > 0x7fffffffLL || A.n_haps + nh > 0x7fffffffLL)
    return PHMM_E_INVALID_ARG;  // wait for some tickets first
  AsyncJob j{q->next_ticket, A.n_pairs, np, A.n_reads, nr, A.n_haps, nh, (int64_t)A.rb.n, b->total_read_bases,
             (int64_t)A.hb.n, b->total_hap_bases, out_log10, out_status};
  const size_t nrb = (size_t)b->total_read_bases, nhb = (size_t)b->total_hap_bases;
  const bool first = A.jobs.empty();
  // the arena's offset arrays hold n + 1 entries (a leading 0)
  if (!A.rb.reserve(A.rb.n + nrb) || !A.q.reserve(A.q.n + nrb) || !A.qi.reserve(A.qi.n + nrb) ||
      !A.qd.reserve(A.qd.n + nrb) || !A.qg.reserve(A.qg.n + nrb) || !A.hb.reserve(A.hb.n + nhb) ||
      !A.roff.reserve(A.roff.n + 8 * (size_t)(nr + 1)) || !A.hoff.reserve(A.hoff.n + 8 * (size_t)(nh + 1)) ||
      !A.pairs.reserve(A.pairs.n + 8 * (size_t)np) || !A.out.reserve(8 * (size_t)(A.n_pairs + np)) ||
      !A.st.reserve((size_t)(A.n_pairs + np)))
    return PHMM_E_OOM;
  auto app = [](HostVec& v, const void* src, size_t n) {
    if (n) std::memcpy(v.p + v.n, src, n);
    v.n += n;
  };
  app(A.rb, b->read_bases, nrb); app(A.q, b->base_quals, nrb); app(A.qi, b->ins_quals, nrb);
  app(A.qd, b->del_quals, nrb); app(A.qg, b->gcp_quals, nrb); app(A.hb, b->hap_bases, nhb);
  if (first) {
    const int64_t zero = 0;
    app(A.roff, &zero, 8);
    app(A.hoff, &zero, 8);
  }
  int64_t* ro = reinterpret_cast<int64_t*>(A.roff.p + A.roff.n);
  for (int64_t i = 1; i <= nr; ++i) ro[i - 1] = b->read_offsets[i] + j.rb0;
  A.roff.n += 8 * (size_t)nr;
  int64_t* ho = reinterpret_cast<int64_t*>(A.hoff.p + A.hoff.n);
  for (int64_t i = 1; i <= nh; ++i) ho[i - 1] = b->hap_offsets[i] + j.hb0;
  A.hoff.n += 8 * (size_t)nh;
  int32_t* pr = reinterpret_cast<int32_t*>(A.pairs.p + A.pairs.n);
  for (int64_t p = 0; p < np; ++p) {
    pr[2 * p] = b->pairs[2 * p] + (int32_t)j.r0;
    pr[2 * p + 1] = b->pairs[2 * p + 1] + (int32_t)j.h0;
  }
  A.pairs.n += 8 * (size_t)np;
  A.n_pairs += np;
  A.n_reads += nr;
  A.n_haps += nh;
  A.any_status |= out_status != nullptr;
  A.jobs.push_back(j);
  q->outstanding.insert(j.ticket);
  *ticket = q->next_ticket++;
  q->cv.notify_one();
  return PHMM_OK;
}

phmm_status phmm_compute_batch_async(phmm_ctx* c, const phmm_batch* b, double* out_log10, uint8_t* out_status,
                                     uint64_t* ticket) {
  if (!c || !ticket) return PHMM_E_INVALID_ARG;
  ST_TRY(check_batch_args(b));
  if (b->n_pairs > 0 && !out_log10) return PHMM_E_INVALID_ARG;
  if (b->n_pairs > 0 &&
      (b->read_offsets[b->n_reads] != b->total_read_bases || b->hap_offsets[b->n_haps] != b->total_hap_bases))
    return PHMM_E_INVALID_ARG;
  if (!c->aq) {
    c->aq = new (std::nothrow) AsyncQueue();
    if (!c->aq) return PHMM_E_OOM;
    c->aq->worker = std::thread(async_worker, c);
  }
  AsyncQueue* q = c->aq;
  std::lock_guard<std::mutex> g(q->mu);
  if (q->stop) return PHMM_E_INVALID_ARG;
  XJob j{q->next_ticket, *b, out_log10, out_status, q->xset, false, false};
  q->xset = 3 - q->xset;  // regions alternate 1, 2
  q->xjobs.push_back(j);
  q->outstanding.insert(j.ticket);
  *ticket = q->next_ticket++;
  q->cv.notify_one();
  return PHMM_OK;
}

phmm_status phmm_wait(phmm_ctx* c, uint64_t ticket) {
  if (!c || !c->aq) return PHMM_E_INVALID_ARG;
  AsyncQueue* q = c->aq;
  std::unique_lock<std::mutex> lk(q->mu);
  if (!q->outstanding.count(ticket)) return PHMM_E_INVALID_ARG;  // unknown, or waited for before
  q->done_cv.wait(lk, [&] { return q->done.count(ticket) > 0; });
  auto it = q->done.find(ticket);
  const phmm_status st = it->second;
  q->done.erase(it);
  q->outstanding.erase(ticket);
  return st;
}

phmm_status phmm_compute_batch(phmm_ctx* c, const phmm_batch* b, double* out_log10, uint8_t* out_status) {
  if (!c) return PHMM_E_INVALID_ARG;
  std::lock_guard<std::mutex> g(c->run_mu);
  return compute_host(c, b, out_log10, out_status);
}

phmm_status phmm_compute_batch_dev(phmm_ctx* c, const phmm_batch* b, double* dev_out, uint8_t* dev_status) {
  if (!c) return PHMM_E_INVALID_ARG;
  std::lock_guard<std::mutex> g(c->run_mu);
  ST_TRY(check_batch_args(b));
  if (b->n_pairs > 0 && !dev_out) return PHMM_E_INVALID_ARG;
  if (cudaSetDevice(c->device) != cudaSuccess) {
    cudaGetLastError();
    return PHMM_E_CUDA;
  }
  c->launches = 0;
  DevBatch d{b->read_bases, b->base_quals, b->ins_quals, b->del_quals, b->gcp_quals, b->hap_bases,
             b->read_offsets, b->hap_offsets, b->pairs, b->n_reads, b->n_haps, b->n_pairs,
             b->total_read_bases, b->total_hap_bases};
  // results go to context scratch first and reach the caller's buffers only after the
  // whole path (FP32 pass and FP64 rescue) succeeded: outputs stay untouched on error
  double* out = nullptr;
  uint8_t* status = nullptr;
  if (b->n_pairs > 0) {
    ST_TRY(ws(c, B_OUT_LOG10, (size_t)b->n_pairs, &out));
    if (dev_status) ST_TRY(ws(c, B_OUT_STATUS, (size_t)b->n_pairs, &status));
  }
  ev_record(c, EV_START);
  ev_record(c, EV_H2D);
  phmm_status st = compute_dev(c, d, out, status);
  if (st != PHMM_OK) {
    cudaStreamSynchronize(c->stream);
    cudaGetLastError();
    return st;
  }
  if (b->n_pairs > 0) {
    CUDA_TRY(cudaMemcpyAsync(dev_out, out, sizeof(double) * (size_t)b->n_pairs, cudaMemcpyDeviceToDevice,
                             c->stream));
    if (dev_status)
      CUDA_TRY(cudaMemcpyAsync(dev_status, status, (size_t)b->n_pairs, cudaMemcpyDeviceToDevice, c->stream));
  }
  ST_TRY(enqueue_underflow_readback(c));
  ev_record(c, EV_END);
  if (cudaStreamSynchronize(c->stream) != cudaSuccess) {
    cudaGetLastError();
    return PHMM_E_CUDA;
  }
  finish_stats(c);
  c->st.ms_h2d = 0.f;
  c->st.ms_d2h = 0.f;
  return PHMM_OK;
}

phmm_status phmm_sw_align_batch_dev(phmm_ctx* c, const phmm_sw_batch* b, const phmm_sw_params* p, int32_t* dev_res,
                                    uint32_t* dev_ops) {
  if (!c) return PHMM_E_INVALID_ARG;
  std::lock_guard<std::mutex> g_(c->run_mu);
  ST_TRY(sw_check_args(b, p));
  if (b->n_tasks > 0 && (!dev_res || !dev_ops)) return PHMM_E_INVALID_ARG;
  if (cudaSetDevice(c->device) != cudaSuccess) {
    cudaGetLastError();
    return PHMM_E_CUDA;
  }
  c->launches = 0;
  SwDev d{b->ref_bases, b->alt_bases, b->ref_offsets, b->alt_offsets, b->tasks, b->n_refs, b->n_alts, b->n_tasks,
          b->total_ref_bases, b->total_alt_bases};
  ev_record(c, EV_START);
  ev_record(c, EV_H2D);
  phmm_status st = sw_compute_dev(c, d, p, dev_res, dev_ops);
  if (st != PHMM_OK) {
    cudaStreamSynchronize(c->stream);
    cudaGetLastError();
    return st;
  }
  ev_record(c, EV_END);
  CUDA_TRY(cudaStreamSynchronize(c->stream));
  c->st.kernel_launches = c->launches;
  c->st.ms_total = ev_ms(c, EV_START, EV_END);
  c->st.ms_wavefront = ev_ms(c, EV_WF0, EV_WF1);
  c->st.ms_finalize = ev_ms(c, EV_WF1, EV_FIN);
  c->st.ms_prep = ev_ms(c, EV_H2D, EV_WF0);
  c->st.ms_h2d = c->st.ms_d2h = 0.f;
  return PHMM_OK;
}

phmm_status phmm_sw_align_batch(phmm_ctx* c, const phmm_sw_batch* b, const phmm_sw_params* p, int32_t* out_res,
                                uint32_t* out_ops) {
  if (!c) return PHMM_E_INVALID_ARG;
  std::lock_guard<std::mutex> g_(c->run_mu);
  ST_TRY(sw_check_args(b, p));
  if (b->n_tasks > 0 && (!out_res || !out_ops)) return PHMM_E_INVALID_ARG;
  if (cudaSetDevice(c->device) != cudaSuccess) {
    cudaGetLastError();
    return PHMM_E_CUDA;
  }
  c->launches = 0;
  if (b->n_tasks == 0) {
    c->st = phmm_stats{};
    return PHMM_OK;
  }
  if (b->ref_offsets[b->n_refs] != b->total_ref_bases || b->alt_offsets[b->n_alts] != b->total_alt_bases)
    return PHMM_E_INVALID_ARG;
  // output capacity: sum over tasks of M + N (indices checked here, lengths on the device)
  int64_t ops_total = 0;
  for (int64_t t = 0; t < b->n_tasks; ++t) {
    const int32_t r = b->tasks[2 * t], a = b->tasks[2 * t + 1];
    if (r < 0 || r >= b->n_refs || a < 0 || a >= b->n_alts) return PHMM_E_INDEX;
    ops_total += (b->ref_offsets[r + 1] - b->ref_offsets[r]) + (b->alt_offsets[a + 1] - b->alt_offsets[a]);
  }
  cudaStream_t s = c->stream;
  uint8_t *ref, *alt;
  int64_t *roff, *aoff;
  int32_t *tasks, *res;
  uint32_t* ops;
  const size_t nr = (size_t)b->total_ref_bases, na = (size_t)b->total_alt_bases;
  ST_TRY(ws(c, B_SW_REF, nr, &ref));
  ST_TRY(ws(c, B_SW_ALT, na, &alt));
  ST_TRY(ws(c, B_SW_ROFF, (size_t)b->n_refs + 1, &roff));
  ST_TRY(ws(c, B_SW_AOFF, (size_t)b->n_alts + 1, &aoff));
  ST_TRY(ws(c, B_SW_TASKS, (size_t)b->n_tasks * 2, &tasks));
  ST_TRY(ws(c, B_SW_RES, (size_t)b->n_tasks * 6, &res));
  ST_TRY(ws(c, B_SW_OPS, (size_t)std::max<int64_t>(ops_total, 1), &ops));
  Stager& S = c->stage;
  S.staged_bytes = 0;
  ev_record(c, EV_START);
  CUDA_TRY(S.h2d(ref, b->ref_bases, nr, s));
  CUDA_TRY(S.h2d(alt, b->alt_bases, na, s));
  CUDA_TRY(S.h2d(roff, b->ref_offsets, sizeof(int64_t) * (b->n_refs + 1), s));
  CUDA_TRY(S.h2d(aoff, b->alt_offsets, sizeof(int64_t) * (b->n_alts + 1), s));
  CUDA_TRY(S.h2d(tasks, b->tasks, sizeof(int32_t) * 2 * b->n_tasks, s));
  ev_record(c, EV_H2D);
  SwDev d{ref, alt, roff, aoff, tasks, b->n_refs, b->n_alts, b->n_tasks, (int64_t)nr, (int64_t)na};
  phmm_status st = sw_compute_dev(c, d, p, res, ops);
  if (st != PHMM_OK) {
    cudaStreamSynchronize(s);
    cudaGetLastError();
    return st;
  }
  ev_record(c, EV_D2H);
  CUDA_TRY(S.d2h(out_res, res, sizeof(int32_t) * 6 * b->n_tasks, s));
  int64_t used = 0;  // packed runs: only these travel back
  for (int64_t t = 0; t < b->n_tasks; ++t) used += out_res[6 * t + 5];
  if (used > 0) CUDA_TRY(S.d2h(out_ops, ops, sizeof(uint32_t) * used, s));
  ev_record(c, EV_END);
  CUDA_TRY(cudaStreamSynchronize(s));
  c->st.kernel_launches = c->launches;
  c->st.ms_total = ev_ms(c, EV_START, EV_END);
  c->st.ms_h2d = ev_ms(c, EV_START, EV_H2D);
  c->st.ms_prep = ev_ms(c, EV_H2D, EV_WF0);
  c->st.ms_wavefront = ev_ms(c, EV_WF0, EV_WF1);
  c->st.ms_finalize = ev_ms(c, EV_WF1, EV_FIN);
  c->st.ms_d2h = ev_ms(c, EV_D2H, EV_END);
  return PHMM_OK;
}

}  // extern "C"
