/* sw_oracle.c -- plain CPU oracle for the Smith-Waterman kernel of the paper
 * (HaplotypeCaller variant).
 *
 * TEST INFRASTRUCTURE ONLY: used by tests/, never by the product path; shares no code
 * with the CUDA path (csrc/sw*.cu*).
 *
 * What is computed (PAPER.md L16@3413, §III-B, Eq. 5; readings R20-R25 in DESIGN.md §12):
 *
 *   H(i,0) = H(0,j) = 0
 *   H(i,j) = max{ 0,
 *                 H(i-1,j-1) + s(a_i, b_j),
 *                 max_{k>=1} H(i-k,j) + W_k,          (vertical: a gap in b, CIGAR 'D')
 *                 max_{l>=1} H(i,j-l) + W_l }         (horizontal: a gap in a, CIGAR 'I')
 *   for 1 <= i <= M (rows, sequence a = s1) and 1 <= j <= N (columns, sequence b = s2),
 *   s(x,y) = match if x == y else mismatch, W_k = open + (k-1)*extend   (R20, R21)
 *
 * btrack(i,j) records the chosen term (R22): 0 for the diagonal, +k for a vertical gap of
 * length k, -l for a horizontal gap of length l, BT_STOP when every non-zero term is < 0
 * (H = 0 from the first term). Priorities on equal scores: diagonal, then horizontal, then
 * vertical; within one direction the longest gap.
 *
 * "After the computation, we will locate the cell with the maximal value in the last row
 * and column of the score matrix H, and retrieve the optimal alignment of two sequences
 * back from this position using the matrix btrack" (L16@3960): the end cell is the
 * maximum over row M and column N (ties: smallest |i-j|, then largest i+j, then largest
 * i; R23); the traceback follows btrack until a BT_STOP cell or row/column 0 (R24).
 *
 * Two forms of the recurrence:
 *   sw_fill_literal  -- Eq. 5 as written, the max over k and l by explicit loops
 *                       (O(M N (M+N)), for small cases and to pin the other one);
 *   sw_fill_running  -- the paper's "two buffers holding the local maximum along each
 *                       direction so that each time only the left and up neighbors need to
 *                       be accessed" (L16@3800): best_v(i,j) = max(best_v(i-1,j) + extend,
 *                       H(i-1,j) + open), valid because W is linear in k (O(M N)).
 */
#include <limits.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#define BT_STOP INT32_MIN

typedef struct {
  int32_t match, mismatch, open, extend;
} sw_params;

static int32_t score_of(uint8_t x, uint8_t y, const sw_params* p) { return x == y ? p->match : p->mismatch; }

/* Choose among the three terms with the R22 priorities; returns H and writes btrack. */
static int32_t choose(int32_t diag, int32_t right, int32_t kh, int32_t down, int32_t kv, int32_t* bt) {
  int32_t h;
  if (diag >= right && diag >= down) {
    h = diag;
    *bt = 0;
  } else if (right >= down) {
    h = right;
    *bt = -kh;
  } else {
    h = down;
    *bt = kv;
  }
  if (h < 0) {
    *bt = BT_STOP;
    h = 0;
  }
  return h;
}

/* H and btrack are (M+1) x (N+1), row-major. */
void sw_fill_literal(int64_t M, int64_t N, const uint8_t* a, const uint8_t* b, const sw_params* p, int32_t* H,
                     int32_t* bt) {
  const int64_t W = N + 1;
  for (int64_t j = 0; j <= N; ++j) { H[j] = 0; bt[j] = BT_STOP; }
  for (int64_t i = 1; i <= M; ++i) {
    H[i * W] = 0;
    bt[i * W] = BT_STOP;
    for (int64_t j = 1; j <= N; ++j) {
      const int32_t diag = H[(i - 1) * W + j - 1] + score_of(a[i - 1], b[j - 1], p);
      /* max_k H(i-k,j) + W_k, ties -> largest k */
      int32_t down = INT32_MIN / 2, kv = 0;
      for (int64_t k = 1; k <= i; ++k) {
        const int32_t c = H[(i - k) * W + j] + p->open + (int32_t)(k - 1) * p->extend;
        if (c >= down) { down = c; kv = (int32_t)k; }
      }
      /* max_l H(i,j-l) + W_l, ties -> largest l */
      int32_t right = INT32_MIN / 2, kh = 0;
      for (int64_t l = 1; l <= j; ++l) {
        const int32_t c = H[i * W + j - l] + p->open + (int32_t)(l - 1) * p->extend;
        if (c >= right) { right = c; kh = (int32_t)l; }
      }
      H[i * W + j] = choose(diag, right, kh, down, kv, &bt[i * W + j]);
    }
  }
}

void sw_fill_running(int64_t M, int64_t N, const uint8_t* a, const uint8_t* b, const sw_params* p, int32_t* H,
                     int32_t* bt) {
  const int64_t W = N + 1;
  int32_t* best_v = (int32_t*)malloc(sizeof(int32_t) * (size_t)W);
  int32_t* size_v = (int32_t*)malloc(sizeof(int32_t) * (size_t)W);
  for (int64_t j = 0; j <= N; ++j) { H[j] = 0; bt[j] = BT_STOP; best_v[j] = INT32_MIN / 2; size_v[j] = 0; }
  for (int64_t i = 1; i <= M; ++i) {
    int32_t best_h = INT32_MIN / 2, size_h = 0;
    H[i * W] = 0;
    bt[i * W] = BT_STOP;
    for (int64_t j = 1; j <= N; ++j) {
      const int32_t diag = H[(i - 1) * W + j - 1] + score_of(a[i - 1], b[j - 1], p);
      /* vertical: open a new gap below H(i-1,j) or extend the best one (strictly better opens) */
      const int32_t open_v = H[(i - 1) * W + j] + p->open;
      best_v[j] += p->extend;
      if (open_v > best_v[j]) { best_v[j] = open_v; size_v[j] = 1; } else { size_v[j] += 1; }
      /* horizontal */
      const int32_t open_h = H[i * W + j - 1] + p->open;
      best_h += p->extend;
      if (open_h > best_h) { best_h = open_h; size_h = 1; } else { size_h += 1; }
      H[i * W + j] = choose(diag, best_h, size_h, best_v[j], size_v[j], &bt[i * W + j]);
    }
  }
  free(best_v);
  free(size_v);
}

/* End cell (R23) and traceback (R24). ops: run-length CIGAR from start to end,
 * encoded (len << 4) | op with op 0 = 'M', 1 = 'I' (horizontal), 2 = 'D' (vertical);
 * capacity >= M + N. Returns the number of ops; writes score, end and start cells
 * (1-based; start = first aligned cell, end_i = end_j = 0 and no ops when M or N is 0). */
int64_t sw_result(int64_t M, int64_t N, const int32_t* H, const int32_t* bt, int32_t* score, int32_t* end_i,
                  int32_t* end_j, int32_t* start_i, int32_t* start_j, uint32_t* ops) {
  const int64_t W = N + 1;
  int64_t bi = 0, bj = 0;
  int32_t best = INT32_MIN;
  for (int64_t pass = 0; pass < 2; ++pass) {
    const int64_t n = pass == 0 ? M : N;
    for (int64_t t = 1; t <= n; ++t) {
      const int64_t i = pass == 0 ? t : M, j = pass == 0 ? N : t;
      const int32_t v = H[i * W + j];
      int better = 0;
      if (v > best) better = 1;
      else if (v == best) {
        const int64_t di = llabs(i - j), db = llabs(bi - bj);
        if (di < db) better = 1;
        else if (di == db && (i + j > bi + bj || (i + j == bi + bj && i > bi))) better = 1;
      }
      if (better) { best = v; bi = i; bj = j; }
    }
  }
  *score = (bi > 0) ? best : 0;
  *end_i = (int32_t)bi;
  *end_j = (int32_t)bj;
  /* walk back; collect moves in reverse */
  int64_t i = bi, j = bj, nops = 0;
  int last_op = -1;
  uint32_t run = 0;
  uint32_t* rev = ops;  /* reversed runs, flipped at the end */
  while (i > 0 && j > 0) {
    const int32_t c = bt[i * W + j];
    if (c == BT_STOP) break;
    int op;
    uint32_t len;
    if (c == 0) { op = 0; len = 1; i -= 1; j -= 1; }
    else if (c < 0) { op = 1; len = (uint32_t)(-c); j += c; }
    else { op = 2; len = (uint32_t)c; i -= c; }
    if (op == last_op) run += len;
    else {
      if (last_op >= 0) rev[nops++] = (run << 4) | (uint32_t)last_op;
      last_op = op;
      run = len;
    }
  }
  if (last_op >= 0) rev[nops++] = (run << 4) | (uint32_t)last_op;
  for (int64_t x = 0, y = nops - 1; x < y; ++x, --y) { uint32_t t = rev[x]; rev[x] = rev[y]; rev[y] = t; }
  *start_i = (int32_t)(i + 1);
  *start_j = (int32_t)(j + 1);
  return nops;
}

/* One pair, both fills available (literal != 0 -> Eq. 5 loops). Returns nops or -1. */
int64_t sw_align(int64_t M, int64_t N, const uint8_t* a, const uint8_t* b, const sw_params* p, int literal,
                 int32_t* H, int32_t* bt, int32_t* res5, uint32_t* ops) {
  if (literal) sw_fill_literal(M, N, a, b, p, H, bt);
  else sw_fill_running(M, N, a, b, p, H, bt);
  return sw_result(M, N, H, bt, &res5[0], &res5[1], &res5[2], &res5[3], &res5[4], ops);
}

/* Batch in the ABI layout (ref = rows, alt = columns), OpenMP over tasks.
 * res: n_tasks x 6 int32 (score, end_i, end_j, start_i, start_j, n_ops);
 * ops: task t's runs at ops_off[t] (= prefix sum of M_t + N_t). */
int sw_batch(const uint8_t* ref, const int64_t* ref_off, const uint8_t* alt, const int64_t* alt_off,
             const int32_t* tasks, int64_t n_tasks, const sw_params* p, int32_t* res, uint32_t* ops,
             const int64_t* ops_off, int nthreads) {
  int err = 0;
#pragma omp parallel for schedule(dynamic, 4) num_threads(nthreads > 0 ? nthreads : 1) reduction(| : err)
  for (int64_t t = 0; t < n_tasks; ++t) {
    const int32_t r = tasks[2 * t], s = tasks[2 * t + 1];
    const int64_t M = ref_off[r + 1] - ref_off[r], N = alt_off[s + 1] - alt_off[s];
    int32_t* H = (int32_t*)malloc(sizeof(int32_t) * (size_t)((M + 1) * (N + 1)));
    int32_t* bt = (int32_t*)malloc(sizeof(int32_t) * (size_t)((M + 1) * (N + 1)));
    if (!H || !bt) { err |= 1; free(H); free(bt); continue; }
    const int64_t n = sw_align(M, N, ref + ref_off[r], alt + alt_off[s], p, 0, H, bt, res + 6 * t,
                               ops + ops_off[t]);
    res[6 * t + 5] = (int32_t)n;
    free(H);
    free(bt);
  }
  return err ? -1 : 0;
}
