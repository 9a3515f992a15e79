/*
 * phmm.h -- C ABI of the B200-native batched PairHMM forward library
 * (libphmm.so, sm_100a). No C++ types, exceptions or torch types cross it.
 *
 * Operation (J. Wang, X. Xie, J. Cong, "Communication Optimization on GPU:
 * A Case Study of Sequence Alignment Algorithms", IPDPS 2017, PAPER.md):
 *   A task is "a pair of sequences" (L22@4659, §V-B); tasks are batched per
 *   region, one batch per launch (L24@575). For every (read, haplotype) pair
 *   the library evaluates the PairHMM forward recurrence of Eq. 6
 *   (L18@541, §III-B):
 *     M(i,j) = P(i,j) * (alpha*M(i-1,j-1) + beta*I(i-1,j-1) + gamma*D(i-1,j-1))
 *     I(i,j) = delta*M(i-1,j) + eps*I(i-1,j)
 *     D(i,j) = zeta*M(i,j-1) + mu*D(i,j-1)
 *   read = rows i = 1..m, haplotype = columns j = 1..N, and returns "one
 *   single number" per pair (L18@1062): log10 of the sum of the last row of
 *   M and I (L20@2262, §IV-C.1; reading R1).
 *   The Phred -> probability mapping of alpha..mu and P(i,j), and the initial
 *   row D(0,j) = 1/N, follow GATK 3.6 (L22@4113; readings R2-R6):
 *     e(Q) = 10^(-Q/10); alpha = 1 - min(1, e(qi)+e(qd)); beta = gamma = 1 - e(qg);
 *     delta = e(qi); eps = mu = e(qg); zeta = e(qd);
 *     P = 1 - e(q) if bases match or either is 'N', else e(q)/3.
 *   Precision (reading R7): PHMM_PREC_FP32_RESCUE computes in FP32 with the
 *   initial row scaled by 2^120 and re-runs, in FP64 scaled by 2^1020, every
 *   pair whose scaled FP32 sum is < 1e-28 or not finite; PHMM_PREC_FP64 runs
 *   every pair in FP64.
 *
 * Ownership: the caller owns every input and output buffer. The library reads
 * the inputs during the call (the host variant copies them to the device),
 * keeps no pointer to them after return, and writes only out_log10 /
 * out_status. Device workspace is owned by the context and reused across
 * calls (grown on demand).
 *
 * Errors: every call validates its arguments and inputs before any output is
 * written; on error it returns a negative status and leaves the outputs
 * untouched (both variants compute into context scratch and copy the results
 * to the caller's buffers only after the whole path, FP64 rescue included,
 * succeeded). Input-content errors (bad base, bad quality, empty sequence,
 * pair index out of range, length caps) are detected on the device in the
 * same pass that reads the data; the call then returns the error without
 * writing outputs. CUDA failures return PHMM_E_CUDA (the context stays usable
 * after a recoverable one). A context is bound to one device, is not
 * thread-safe, and holds no global state: use one context per host thread.
 *
 * Input limits (each violation -> the status named, outputs untouched):
 *   - bases: 'A','C','G','T','N' only (uppercase)          -> PHMM_E_INVALID_BASE
 *   - every quality <= 127                                  -> PHMM_E_INVALID_QUAL
 *   - every read base with e(qi) + e(qd) <= 1, i.e. no base
 *     with qi or qd <= 3 whose two gap-open probabilities
 *     sum above 1 (reading R16: the transitions
 *     out of M must be a distribution; checked on EVERY
 *     read of the batch, used by a pair or not)            -> PHMM_E_INVALID_QUAL
 *   - a read or haplotype used by a pair has length >= 1   -> PHMM_E_EMPTY_SEQ
 *   - pair indices inside [0, n_reads) x [0, n_haps)       -> PHMM_E_INDEX
 *   - a haplotype used by a pair has N <= 4094 bases and a
 *     read used by a pair has m <= 2^20 bases (unused
 *     sequences may be longer)                             -> PHMM_E_INVALID_ARG
 *   - n_pairs, n_reads, n_haps <= 2^31 - 1                 -> PHMM_E_INVALID_ARG
 *
 * Synchronisation: every compute call returns only when its results are in
 * the caller's buffers (the path reads device-computed sizes back to the host
 * a few times per call, so it cannot be captured in a CUDA graph). Work is
 * issued on the context's stream: the cuda_stream of phmm_config, or the one
 * set by phmm_set_stream, or (NULL) a stream the context owns.
 */
#ifndef PHMM_H_
#define PHMM_H_

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define PHMM_ABI_VERSION 4

typedef struct phmm_ctx phmm_ctx; /* opaque */

typedef enum {
  PHMM_OK = 0,
  PHMM_E_INVALID_ARG = -1,  /* NULL pointer, negative count, bad offsets, bad config, length caps */
  PHMM_E_INVALID_BASE = -2, /* a base outside 'A','C','G','T','N' (uppercase only) */
  PHMM_E_INVALID_QUAL = -3, /* a quality > 127, or e(qi) + e(qd) > 1 (reading R16) */
  PHMM_E_EMPTY_SEQ = -4,    /* a read or haplotype of length 0 used by a pair */
  PHMM_E_INDEX = -5,        /* a pair's read or haplotype index out of range */
  PHMM_E_CUDA = -6,         /* a CUDA runtime error */
  PHMM_E_OOM = -7           /* device or pinned-host allocation failed */
} phmm_status;

typedef enum {
  PHMM_PREC_FP64 = 0,        /* every pair in FP64 (scale 2^1020) */
  PHMM_PREC_FP32_RESCUE = 1  /* FP32 (scale 2^120) + FP64 re-run of underflowing pairs */
} phmm_precision;

/* per-pair status byte written to out_status */
enum { PHMM_PAIR_OK = 0, PHMM_PAIR_RESCUED = 1, PHMM_PAIR_FP64_UNDERFLOW = 2 };

/* config flags */
#define PHMM_FLAG_TIMING 1u /* record CUDA events around each phase; see phmm_get_timing */

typedef struct {
  int device;               /* CUDA device ordinal */
  phmm_precision precision; /* default PHMM_PREC_FP32_RESCUE */
  void* cuda_stream;        /* cudaStream_t to run on; NULL = a context-owned stream */
  uint32_t flags;           /* PHMM_FLAG_* */
  int32_t col_bucket;       /* haplotype-length bin width in columns (0 = default 4) */
} phmm_config;

/*
 * A batch. Reads and their four quality arrays share one layout: read r is
 * bytes [read_offsets[r], read_offsets[r+1]) of each array. Haplotype h is
 * bytes [hap_offsets[h], hap_offsets[h+1]) of hap_bases. Offsets are int64,
 * non-decreasing, start at 0. pairs[2p] = read index, pairs[2p+1] = haplotype
 * index of pair p. Bases are ASCII 'A','C','G','T','N'; qualities are raw
 * Phred integers 0..127 (NOT ASCII+33). For phmm_compute_batch every pointer
 * is a host pointer; for phmm_compute_batch_dev every array pointer is a
 * device pointer (the struct itself lives on the host).
 */
typedef struct {
  const uint8_t* read_bases;
  const uint8_t* base_quals; /* per read base: base quality q_i */
  const uint8_t* ins_quals;  /* per read base: insertion (gap-open) quality qi_i */
  const uint8_t* del_quals;  /* per read base: deletion (gap-open) quality qd_i */
  const uint8_t* gcp_quals;  /* per read base: gap-continuation quality qg_i */
  const int64_t* read_offsets; /* n_reads + 1 */
  int64_t n_reads;
  const uint8_t* hap_bases;
  const int64_t* hap_offsets;  /* n_haps + 1 */
  int64_t n_haps;
  const int32_t* pairs;        /* 2 * n_pairs: (read_idx, hap_idx) */
  int64_t n_pairs;
  int64_t total_read_bases;    /* = read_offsets[n_reads] (required by the _dev variant) */
  int64_t total_hap_bases;     /* = hap_offsets[n_haps]  (required by the _dev variant) */
} phmm_batch;

/* Create a context on cfg->device (cfg may be NULL: device 0, FP32+rescue). */
phmm_status phmm_create(phmm_ctx** out, const phmm_config* cfg);

/*
 * Host-buffer variant. Copies the batch to the device on the context stream,
 * runs the whole path, copies the results back and returns when out_log10
 * (n_pairs doubles, caller-owned host memory) and, if non-NULL, out_status
 * (n_pairs bytes) are written.
 * out_log10[p] = log10 P(read | hap) of pair p; -inf when P underflows even
 * the FP64 rescue or is exactly 0 (Q0 inputs).
 * Copies: a buffer that is page-locked (cudaMallocHost / cudaHostRegister) is
 * copied by one cudaMemcpyAsync; a pageable buffer goes through the context's
 * pinned staging ring (4 x 8 MiB, filled by a pool of host threads while the
 * previous piece is in flight; phmm_stats.staged_bytes counts these bytes). The
 * number of host threads is min(8, cores / 2), or PHMM_STAGE_THREADS when the
 * context is created.
 * Pipelining: a batch of >= 2^17 pairs runs as chunks of pairs (n/8 and 7n/8, at most 2^23
 * pairs each): a context-owned copy thread moves chunk k+1's new input bytes to the device
 * on a copy stream while chunk k computes, chunks alternate between two compute streams,
 * and one FP64 rescue pass over the whole batch follows (batches above 2^23 pairs: a rescue
 * per chunk). Fills of device scratch are kernels, not cudaMemsetAsync (which would queue
 * behind the copy stream's transfers). Results are bitwise those of the unpipelined call
 * (PHMM_PIPE=0 at context creation disables it), as for any change of batch composition
 * (reading R14). Pairs that use
 * reads and haplotypes in ascending index ranges (region after region, as GATK emits them)
 * overlap best; a batch whose first chunk would need more than half of the input bytes
 * runs as one chunk.
 * Either way the call returns only when the outputs are written, and the caller's
 * buffers are not touched after it returns.
 */
phmm_status phmm_compute_batch(phmm_ctx* ctx, const phmm_batch* b, double* out_log10,
                               uint8_t* out_status);

/*
 * Device-buffer variant (for torch tensors): every array in *b, dev_out_log10
 * (n_pairs doubles) and dev_out_status (optional, n_pairs bytes) are device
 * pointers on the context's device. Work is enqueued on the context stream,
 * which must be ordered after whatever produced the inputs (the Python binding
 * sets it to torch's current stream with phmm_set_stream before each call);
 * the call synchronises that stream before returning, so outputs are final
 * when it returns PHMM_OK.
 */
phmm_status phmm_compute_batch_dev(phmm_ctx* ctx, const phmm_batch* b, double* dev_out_log10,
                                   uint8_t* dev_out_status);

/*
 * Make later calls on ctx enqueue their work on `cuda_stream` (a cudaStream_t of
 * the context's device; NULL = the context's own stream, created on demand).
 * The caller keeps ownership of the stream and must keep it alive while the
 * context uses it. Returns PHMM_E_INVALID_ARG for a NULL ctx, PHMM_E_CUDA if a
 * stream cannot be created.
 */
phmm_status phmm_set_stream(phmm_ctx* ctx, void* cuda_stream);

/*
 * Asynchronous submission of host-buffer batches (for region-sized batches: a synchronous
 * call costs ~0.6 ms whatever the batch size, PAPER.md's batches average 189 pairs,
 * L24@575). phmm_submit checks the batch on the host (offsets, pair indices, sizes),
 * copies it into the context's host queue and returns at once with a ticket; a worker
 * thread of the context runs everything queued so far as ONE batch whenever it is idle
 * (so batches submitted while a run is in flight are coalesced into the next run) and
 * writes each batch's results to its own out_log10 / out_status, which must stay valid
 * until phmm_wait returns for that ticket (the inputs are copied: they may be reused as
 * soon as phmm_submit returns). Results are bitwise those of phmm_compute_batch on the same
 * batch. phmm_wait blocks until the ticket's results are written and returns the batch's
 * status: PHMM_OK, or the error that batch alone raises (a coalesced run that fails is
 * re-run batch by batch; the outputs of a failed batch are untouched). A ticket can be
 * waited for once. Other calls on the context wait while a run is in progress (the
 * context serialises its work); phmm_destroy completes every submitted batch first.
 * Returns PHMM_E_INVALID_ARG (NULL arguments, bad sizes or offsets, too many pairs
 * queued), PHMM_E_INDEX, PHMM_E_OOM (host queue) from phmm_submit; PHMM_E_INVALID_ARG
 * for an unknown or already-waited ticket from phmm_wait.
 */
phmm_status phmm_submit(phmm_ctx* ctx, const phmm_batch* b, double* out_log10, uint8_t* out_status,
                        uint64_t* ticket);
phmm_status phmm_wait(phmm_ctx* ctx, uint64_t ticket);

/*
 * Asynchronous host-buffer call WITHOUT an input copy (for large batches streamed one after
 * another): returns at once with a ticket; the library reads the caller's input arrays and
 * writes out_log10 / out_status until phmm_wait(ctx, ticket) returns, so the caller keeps all
 * of them valid and the inputs unchanged until then. Batches of this call run one at a time in
 * their submission order on the context's worker thread (the phmm_submit queue's); while one
 * batch computes, the worker already copies the NEXT submitted batch's inputs to the device
 * (two device input regions, used alternately), when all of that batch's arrays are page-locked
 * -- so a caller that keeps two batches in flight overlaps one batch's host->device copy with
 * the other's compute. A batch that was not prefetched runs as phmm_compute_batch. Results are
 * bitwise those of phmm_compute_batch; phmm_wait returns the batch's status (input errors as
 * for phmm_compute_batch, outputs then untouched). Returns PHMM_E_INVALID_ARG (NULL
 * arguments, bad sizes) or PHMM_E_OOM at submission.
 */
phmm_status phmm_compute_batch_async(phmm_ctx* ctx, const phmm_batch* b, double* out_log10, uint8_t* out_status,
                                     uint64_t* ticket);

/* Release the context and its device workspace. NULL-safe, idempotent per pointer. */
void phmm_destroy(phmm_ctx* ctx);

/* Static string for a status code. */
const char* phmm_status_string(phmm_status s);

/*
 * Statistics of the last successful compute call on ctx.
 * timing fields are filled only with PHMM_FLAG_TIMING (milliseconds, CUDA
 * events on the context stream), else set to -1.
 */
typedef struct {
  int64_t n_pairs;
  int64_t cells;            /* sum of m*N over pairs (the paper's cell count, L22@1416) */
  int64_t padded_cells;     /* cells the wavefront kernels actually computed (pad rows/cols) */
  int64_t n_rescued;        /* pairs re-run in FP64 */
  int64_t n_fp64_underflow; /* pairs whose FP64 sum was 0 or subnormal */
  int32_t n_chunks;         /* pair chunks the call ran as (batches > 2^23 pairs run in chunks) */
  int32_t kernel_launches;  /* kernels launched by the call */
  float ms_total;           /* whole call on the stream (device side) */
  float ms_h2d;             /* host->device copies (host variant only) */
  float ms_prep;            /* validation, per-read tables, binning */
  float ms_wavefront;       /* main wavefront kernel (FP32 or FP64 mode) */
  float ms_rescue;          /* FP64 rescue pass (prep + wavefront) */
  float ms_finalize;        /* log10 + scatter */
  float ms_d2h;             /* device->host copy (host variant only) */
  int64_t staged_bytes;     /* host variant: bytes copied through the pinned staging buffers */
} phmm_stats;

phmm_status phmm_get_stats(const phmm_ctx* ctx, phmm_stats* out);

/* ABI version of the loaded library (PHMM_ABI_VERSION). */
int phmm_abi_version(void);

/* ======================================================================
 * Smith-Waterman, HaplotypeCaller variant (the paper's second workload,
 * PAPER.md Eq. 5, L16@3413, §III-B; readings R20-R25 in
 * DESIGN.md §12). Integer scores:
 *   H(i,0) = H(0,j) = 0,
 *   H(i,j) = max{0, H(i-1,j-1) + s(a_i,b_j), max_k H(i-k,j) + W_k, max_l H(i,j-l) + W_l}
 * for rows i = 1..M of the "ref" sequence a and columns j = 1..N of the "alt"
 * sequence b; s = match if the bytes are equal else mismatch; W_k = gap_open +
 * (k-1)*gap_extend. Ties: diagonal, then horizontal, then vertical; within a
 * direction the longest gap; H = 0 from the 0 term when every other term is
 * negative (the traceback stops there). The end cell is the maximum of row M and
 * column N ("the cell with the maximal value in the last row and column",
 * L16@3960; ties: smallest |i-j|, then largest i+j, then largest i); the alignment
 * is traced back from it until a 0-term cell or row/column 0.
 * ====================================================================== */
typedef struct {
  int32_t match;       /* > 0 */
  int32_t mismatch;    /* <= match */
  int32_t gap_open;    /* W_1, <= gap_extend */
  int32_t gap_extend;  /* <= 0 */
} phmm_sw_params;      /* HaplotypeCaller: {200, -150, -260, -11} */

typedef struct {
  const uint8_t* ref_bases;    /* concatenated rows sequences, 'A','C','G','T','N' */
  const int64_t* ref_offsets;  /* n_refs + 1; 1 <= M <= 32767 per task */
  int64_t n_refs;
  const uint8_t* alt_bases;    /* concatenated column sequences */
  const int64_t* alt_offsets;  /* n_alts + 1; 1 <= N <= 4096 per task */
  int64_t n_alts;
  const int32_t* tasks;        /* 2 * n_tasks: (ref_idx, alt_idx) */
  int64_t n_tasks;
  int64_t total_ref_bases;     /* = ref_offsets[n_refs] */
  int64_t total_alt_bases;     /* = alt_offsets[n_alts] */
} phmm_sw_batch;

/*
 * Align every task. out_res: n_tasks x 6 int32 per task, in task order:
 *   score, end_i, end_j (1-based end cell), start_i, start_j (first aligned cell;
 *   end + 1 for an empty alignment), n_ops.
 * out_ops: CIGAR runs (len << 4 | op; op 0 = 'M', 1 = 'I' (gap in the ref row
 * sequence: consumes alt bases), 2 = 'D' (consumes ref bases)), from start to end,
 * the tasks' runs back to back in task order: task t's start at element
 * sum_{t' < t} n_ops[t']. Capacity: sum_t (M_t + N_t) uint32 always suffices.
 * Host variant: caller-owned host buffers, returns when they are written. Errors: PHMM_E_INVALID_ARG (NULL pointers, sizes, parameters
 * outside the ranges above, M or N too long), PHMM_E_INVALID_BASE, PHMM_E_EMPTY_SEQ,
 * PHMM_E_INDEX, PHMM_E_CUDA, PHMM_E_OOM; outputs are untouched on error.
 */
phmm_status phmm_sw_align_batch(phmm_ctx* ctx, const phmm_sw_batch* b, const phmm_sw_params* p,
                                int32_t* out_res, uint32_t* out_ops);
/* Device-buffer variant: every array in *b, dev_res and dev_ops are device pointers. */
phmm_status phmm_sw_align_batch_dev(phmm_ctx* ctx, const phmm_sw_batch* b, const phmm_sw_params* p,
                                    int32_t* dev_res, uint32_t* dev_ops);

#ifdef __cplusplus
}
#endif
#endif /* PHMM_H_ */
