/*
 * phmm_oracle.c -- the PairHMM forward ORACLE (plain C, double precision).
 *
 * TEST INFRASTRUCTURE ONLY. Only tests/, __graft_entry__.smoke() and the
 * cpu_baseline / --impl reference legs of bench.py may load or call this
 * code. The product path (paper_conf_ipps_wangxc17_b200/ and its CUDA
 * library) never includes, links or calls anything under oracle/, and this
 * file shares no code, header, table or constant with it.
 *
 * What it computes -- J. Wang, X. Xie, J. Cong, IPDPS 2017, PAPER.md:
 *   Eq. 6 (L18@541, §III-B), the three PairHMM matrices
 *     M(i,j) = P(i,j) * ( alpha*M(i-1,j-1) + beta*I(i-1,j-1) + gamma*D(i-1,j-1) )
 *     I(i,j) = delta*M(i-1,j) + eps*I(i-1,j)
 *     D(i,j) = zeta*M(i,j-1) + mu*D(i,j-1)
 *   over the dependence graph of Fig. 4 (L16@2004) / Fig. 5 (L16@2878);
 *   termination: the sum of the last row of M and I ("accumulating the
 *   results of cells in matrix match and insertion", L20@2262, §IV-C.1;
 *   DESIGN.md reading R1), one number per pair (L18@1062).
 * The paper gives alpha..mu and P(i,j) only symbolically (L18@327, L18@674);
 * their Phred mapping and the initial row follow GATK 3.6, from which the
 * paper extracts the algorithm (L22@4113) -- DESIGN.md readings R2..R6:
 *   e(Q)      = 10^(-Q/10)
 *   alpha_i   = 1 - min(1, e(qi_i) + e(qd_i))          (M->M)
 *   beta_i    = gamma_i = 1 - e(qg_i)                   (I->M, D->M)
 *   delta_i   = e(qi_i),  eps_i = e(qg_i)               (M->I, I->I)
 *   zeta_i    = e(qd_i),  mu_i  = e(qg_i)               (M->D, D->D)
 *   P(i,j)    = 1 - e(q_i)  if r_i == h_j or r_i == 'N' or h_j == 'N'
 *             = e(q_i)/3    otherwise
 *   M(0,j) = I(0,j) = 0, D(0,j) = 1/N (j = 0..N); M(i,0)=I(i,0)=D(i,0)=0, i>=1
 *   log10 P(read|hap) = log10( sum_{j=1..N} M(m,j) + I(m,j) )
 *
 * Numerics (reading R7): plain double arithmetic in the order the
 * recurrence is written, no fixed scale. After row i is COMPLETE (D(i,j)
 * reads M(i,j-1)), the whole row is multiplied by 2^-E where E is the binary
 * exponent of the row's largest value (frexp/ldexp: exact), and E is
 * accumulated. The final answer is log10(sum) + Etot*log10(2). Power-of-two
 * scaling is exact, so the result equals the unscaled double DP wherever
 * that one does not underflow, and never underflows itself.
 *
 * Three entry points (all pure functions, no global state):
 *   oracle_prob_parts  probability-domain core: per-row alpha..mu and a
 *                      full m x N emission matrix P(i,j); returns the M part
 *                      and the I part of the last-row sum as (log10) values.
 *   oracle_phred_log10 the Phred wrapper for one (read, haplotype) pair.
 *   oracle_batch       a batch in the C-ABI layout (concatenated bytes +
 *                      offsets + pair list), OpenMP over pairs.
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

#define LOG10_2 0.30102999566398119521

/* e(Q) = 10^(-Q/10)  [EXT GATK QualityUtils.qualToErrorProb] */
static double phred_to_err(int q) { return pow(10.0, -(double)q / 10.0); }

/*
 * Probability-domain core. Row-major emission matrix prior[(i-1)*N + (j-1)]
 * for i = 1..m, j = 1..N. Transition arrays are indexed by the destination
 * row i = 1..m at position i-1 (reading R3).
 * Outputs: *log10_m = log10 sum_j M(m,j), *log10_i = log10 sum_j I(m,j),
 *          *log10_p = log10 of their sum. -inf when the sum is 0.
 * Returns 0 on success, -1 on bad sizes / allocation failure.
 */
int oracle_prob_parts(int64_t m, int64_t n,
                      const double* alpha, const double* beta, const double* gamma,
                      const double* delta, const double* eps, const double* zeta,
                      const double* mu, const double* prior,
                      double* log10_m, double* log10_i, double* log10_p) {
  if (m < 1 || n < 1) return -1;
  /* two rows of each matrix, columns 0..n */
  double* Mp = (double*)calloc((size_t)(n + 1), sizeof(double));
  double* Ip = (double*)calloc((size_t)(n + 1), sizeof(double));
  double* Dp = (double*)calloc((size_t)(n + 1), sizeof(double));
  double* Mc = (double*)calloc((size_t)(n + 1), sizeof(double));
  double* Ic = (double*)calloc((size_t)(n + 1), sizeof(double));
  double* Dc = (double*)calloc((size_t)(n + 1), sizeof(double));
  if (!Mp || !Ip || !Dp || !Mc || !Ic || !Dc) {
    free(Mp); free(Ip); free(Dp); free(Mc); free(Ic); free(Dc);
    return -1;
  }
  /* row 0: M = I = 0, D = 1/N for j = 0..N */
  for (int64_t j = 0; j <= n; ++j) Dp[j] = 1.0 / (double)n;
  int64_t etot = 0; /* accumulated binary exponent: true value = stored * 2^etot */

  for (int64_t i = 1; i <= m; ++i) {
    const double a = alpha[i - 1], b = beta[i - 1], g = gamma[i - 1];
    const double d = delta[i - 1], e = eps[i - 1], z = zeta[i - 1], u = mu[i - 1];
    const double* pr = prior + (i - 1) * n;
    Mc[0] = 0.0; Ic[0] = 0.0; Dc[0] = 0.0;
    for (int64_t j = 1; j <= n; ++j) {
      Mc[j] = pr[j - 1] * (a * Mp[j - 1] + b * Ip[j - 1] + g * Dp[j - 1]);
      Ic[j] = d * Mp[j] + e * Ip[j];
      Dc[j] = z * Mc[j - 1] + u * Dc[j - 1];
    }
    /* renormalise the finished row by an exact power of two */
    double mx = 0.0;
    for (int64_t j = 0; j <= n; ++j) {
      if (Mc[j] > mx) mx = Mc[j];
      if (Ic[j] > mx) mx = Ic[j];
      if (Dc[j] > mx) mx = Dc[j];
    }
    if (mx > 0.0 && isfinite(mx)) {
      int ex = 0;
      frexp(mx, &ex);
      for (int64_t j = 0; j <= n; ++j) {
        Mc[j] = ldexp(Mc[j], -ex);
        Ic[j] = ldexp(Ic[j], -ex);
        Dc[j] = ldexp(Dc[j], -ex);
      }
      etot += ex;
    }
    double* t;
    t = Mp; Mp = Mc; Mc = t;
    t = Ip; Ip = Ic; Ic = t;
    t = Dp; Dp = Dc; Dc = t;
  }
  /* termination: sum of the last row of M and I (L20@2262) */
  double sm = 0.0, si = 0.0;
  for (int64_t j = 1; j <= n; ++j) { sm += Mp[j]; si += Ip[j]; }
  const double off = (double)etot * LOG10_2;
  if (log10_m) *log10_m = log10(sm) + off;
  if (log10_i) *log10_i = log10(si) + off;
  if (log10_p) *log10_p = log10(sm + si) + off;
  free(Mp); free(Ip); free(Dp); free(Mc); free(Ic); free(Dc);
  return 0;
}

/* base match rule with the 'N' wildcard (reading R5) */
static int bases_match(uint8_t r, uint8_t h) { return r == h || r == 'N' || h == 'N'; }

/*
 * Phred wrapper for one pair. read/quals have length m, hap length n.
 * Qualities are raw Phred integers (not ASCII+33). Returns 0 / -1.
 * *log10_m and *log10_i may be NULL.
 */
int oracle_phred_parts(const uint8_t* read, const uint8_t* q, const uint8_t* qi,
                       const uint8_t* qd, const uint8_t* qg, int64_t m,
                       const uint8_t* hap, int64_t n,
                       double* log10_m, double* log10_i, double* log10_p) {
  if (m < 1 || n < 1) return -1;
  double* tr = (double*)malloc(sizeof(double) * (size_t)(7 * m));
  double* prior = (double*)malloc(sizeof(double) * (size_t)(m * n));
  if (!tr || !prior) { free(tr); free(prior); return -1; }
  double *alpha = tr, *beta = tr + m, *gamma = tr + 2 * m, *delta = tr + 3 * m,
         *eps = tr + 4 * m, *zeta = tr + 5 * m, *mu = tr + 6 * m;
  for (int64_t i = 0; i < m; ++i) {
    const double ei = phred_to_err(qi[i]), ed = phred_to_err(qd[i]), eg = phred_to_err(qg[i]);
    const double s = ei + ed;
    alpha[i] = 1.0 - (s < 1.0 ? s : 1.0);
    beta[i] = 1.0 - eg;
    gamma[i] = 1.0 - eg;
    delta[i] = ei;
    eps[i] = eg;
    zeta[i] = ed;
    mu[i] = eg;
    const double eb = phred_to_err(q[i]);
    for (int64_t j = 0; j < n; ++j)
      prior[i * n + j] = bases_match(read[i], hap[j]) ? 1.0 - eb : eb / 3.0;
  }
  int rc = oracle_prob_parts(m, n, alpha, beta, gamma, delta, eps, zeta, mu, prior,
                             log10_m, log10_i, log10_p);
  free(tr);
  free(prior);
  return rc;
}

double oracle_phred_log10(const uint8_t* read, const uint8_t* q, const uint8_t* qi,
                          const uint8_t* qd, const uint8_t* qg, int64_t m,
                          const uint8_t* hap, int64_t n) {
  double p = NAN;
  if (oracle_phred_parts(read, q, qi, qd, qg, m, hap, n, NULL, NULL, &p) != 0) return NAN;
  return p;
}

/*
 * Batch in the library's layout (include/phmm.h documents it; this file does
 * not include that header): reads and their four quality arrays concatenated
 * with int64 offsets (n_reads+1), haplotypes likewise (n_haps+1), pairs as
 * int32 (read_idx, hap_idx). Writes out[p] = log10 P for every pair.
 * nthreads <= 0 uses the OpenMP default. Returns 0, or -1 on a bad index.
 */
int oracle_batch(const uint8_t* read_bases, const uint8_t* base_q, const uint8_t* ins_q,
                 const uint8_t* del_q, const uint8_t* gcp_q, const int64_t* read_off,
                 int64_t n_reads, const uint8_t* hap_bases, const int64_t* hap_off,
                 int64_t n_haps, const int32_t* pairs, int64_t n_pairs, double* out,
                 int nthreads) {
  for (int64_t p = 0; p < n_pairs; ++p) {
    if (pairs[2 * p] < 0 || pairs[2 * p] >= n_reads) return -1;
    if (pairs[2 * p + 1] < 0 || pairs[2 * p + 1] >= n_haps) return -1;
  }
#ifdef _OPENMP
  if (nthreads > 0) omp_set_num_threads(nthreads);
#pragma omp parallel for schedule(dynamic, 4)
#endif
  for (int64_t p = 0; p < n_pairs; ++p) {
    const int64_t r = pairs[2 * p], h = pairs[2 * p + 1];
    const int64_t r0 = read_off[r], m = read_off[r + 1] - r0;
    const int64_t h0 = hap_off[h], n = hap_off[h + 1] - h0;
    out[p] = oracle_phred_log10(read_bases + r0, base_q + r0, ins_q + r0, del_q + r0,
                                gcp_q + r0, m, hap_bases + h0, n);
  }
  return 0;
}

int oracle_max_threads(void) {
#ifdef _OPENMP
  return omp_get_max_threads();
#else
  return 1;
#endif
}
