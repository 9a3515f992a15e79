/*
 * synth_gen.c -- the seeded synthetic batch generator (native, OpenMP over regions).
 *
 * It only DRAWS inputs: no transition probability, prior or likelihood is computed
 * here (the quality-bin error rates below are the chance that the simulated
 * sequencer mis-called a base, a data-synthesis constant). Both the CUDA path's
 * tests / bench and the oracle's tests take their inputs from it through
 * paper_conf_ipps_wangxc17_b200/synth.py ("Input recipe").
 *
 * Workload shape (PAPER.md L22@4659: a task is a pair of sequences;
 * L24@575: PairHMM tasks come in batches of ~189 per HaplotypeCaller region):
 * per region
 *   1. a reference segment of iid uniform ACGT with ~5 % of its positions inside
 *      homopolymer runs of 4-10 bases;
 *   2. H haplotypes: haplotype 0 is the reference, the others carry SNPs at snp_rate
 *      and 1-5 bp indels at indel_rate per position; each is cut (or padded with random
 *      bases) to its target length N;
 *   3. R reads copied from a random haplotype at a uniform start (extended with random
 *      bases when the haplotype is shorter), decoy_frac of them random sequence, with
 *      per-base substitution errors drawn with the error rate of the base's quality bin;
 *   4. base qualities from {Q37 85 %, Q23 9 %, Q12 4 %, Q6 2 %} (or one fixed quality),
 *      n_rate of the read bases set to 'N' with Q6;
 *   5. insertion / deletion qualities in [iq_lo, iq_hi] (constant when equal), gap
 *      continuation quality gcp;
 *   6. pairs = all R x H combinations, read-major.
 *
 * Randomness is counter-based: every region has two independent streams derived from
 * (seed, region) -- stream 0 draws the region's SHAPE (H, R, lengths), stream 1 its
 * CONTENT -- so synth_shapes() can size a batch of any region range without
 * generating it, synth_fill() can fill regions in any order on any thread, and a rank
 * generates its own shard (seed, region id) with no communication.
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

typedef struct {
  int32_t h_lo, h_hi;       /* haplotypes per region */
  int32_t r_lo, r_hi;       /* reads per region */
  int32_t m_lo, m_hi;       /* read length of the region */
  int32_t n_lo, n_hi;       /* haplotype length (use_factor == 0) */
  int32_t use_factor;       /* 1: N ~ U{ceil(f_lo*m) .. floor(f_hi*m)} */
  double f_lo, f_hi;
  double short_frac;        /* fraction of reads with length U{s_lo..s_hi} */
  int32_t s_lo, s_hi;
  double snp_rate, indel_rate, decoy_frac, n_rate;
  int32_t iq_lo, iq_hi;     /* insertion / deletion quality range */
  int32_t gcp;              /* gap-continuation quality */
  int32_t fixed_q;          /* >= 0: every base quality = fixed_q, error rate fixed_err */
  double fixed_err;
} synth_spec;

enum { MAX_H = 64 };

/* ---------------------------------------------------------------- counter-based RNG */
static uint64_t mix64(uint64_t z) {
  z += 0x9e3779b97f4a7c15ull;
  z = (z ^ (z >> 30)) * 0xbf58476d1ce4e5b9ull;
  z = (z ^ (z >> 27)) * 0x94d049bb133111ebull;
  return z ^ (z >> 31);
}
typedef struct { uint64_t key, ctr; } rng_t;
static rng_t rng_make(uint64_t seed, int64_t region, uint64_t stream) {
  rng_t r;
  r.key = mix64(mix64(mix64(seed) ^ (uint64_t)region) ^ (stream + 0x632be59bd9b4e019ull));
  r.ctr = 0;
  return r;
}
static uint64_t rng_u64(rng_t* r) { return mix64(r->key ^ mix64(r->ctr++)); }
static double rng_unif(rng_t* r) { return (double)(rng_u64(r) >> 11) * (1.0 / 9007199254740992.0); }
/* uniform integer in [lo, hi] */
static int64_t rng_int(rng_t* r, int64_t lo, int64_t hi) {
  if (hi <= lo) return lo;
  const uint64_t span = (uint64_t)(hi - lo) + 1u;
  return lo + (int64_t)(rng_u64(r) % span);
}

static const uint8_t BASES[4] = {'A', 'C', 'G', 'T'};
static const uint8_t QBIN[4] = {37, 23, 12, 6};
static const double QBIN_CUM[4] = {0.85, 0.94, 0.98, 1.0};
static const double QBIN_ERR[4] = {1.9952623e-4, 5.0118723e-3, 6.3095734e-2, 2.5118864e-1};

static int base_idx(uint8_t b) {
  switch (b) {
    case 'A': return 0;
    case 'C': return 1;
    case 'G': return 2;
    default: return 3;
  }
}

/* ---------------------------------------------------------------- region shape */
typedef struct {
  int H, R, m_region;
  int n_h[MAX_H];
  int64_t read_bases, hap_bases, cells;
} shape_t;

/* Draws the shape of a region from stream 0; read lengths are written to m_out
   (R entries, may be NULL: then only the totals). */
static void region_shape(const synth_spec* sp, uint64_t seed, int64_t region, shape_t* s, int32_t* m_out) {
  rng_t r = rng_make(seed, region, 0);
  s->H = (int)rng_int(&r, sp->h_lo, sp->h_hi);
  if (s->H > MAX_H) s->H = MAX_H;
  s->R = (int)rng_int(&r, sp->r_lo, sp->r_hi);
  s->m_region = (int)rng_int(&r, sp->m_lo, sp->m_hi);
  s->hap_bases = 0;
  for (int h = 0; h < s->H; ++h) {
    int n;
    if (sp->use_factor) {
      const int lo = (int)ceil(sp->f_lo * s->m_region), hi = (int)floor(sp->f_hi * s->m_region);
      n = (int)rng_int(&r, lo, hi);
    } else {
      n = (int)rng_int(&r, sp->n_lo, sp->n_hi);
    }
    if (n < 1) n = 1;
    s->n_h[h] = n;
    s->hap_bases += n;
  }
  s->read_bases = 0;
  s->cells = 0;
  for (int k = 0; k < s->R; ++k) {
    int m = s->m_region;
    if (sp->short_frac > 0 && rng_unif(&r) < sp->short_frac) m = (int)rng_int(&r, sp->s_lo, sp->s_hi);
    if (m < 1) m = 1;
    if (m_out) m_out[k] = m;
    s->read_bases += m;
    s->cells += (int64_t)m * s->hap_bases;
  }
}

/* counts[5*i + ...] = R, H, read bases, haplotype bases, cells (sum of m*N) of region
   region0 + i. Returns 0, or -1 on a bad spec. */
int synth_shapes(const synth_spec* sp, uint64_t seed, int64_t region0, int64_t n_regions, int64_t* counts) {
  if (!sp || !counts || n_regions < 0 || sp->h_hi > MAX_H || sp->h_lo < 1 || sp->r_lo < 0) return -1;
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < n_regions; ++i) {
    shape_t s;
    region_shape(sp, seed, region0 + i, &s, NULL);
    counts[5 * i + 0] = s.R;
    counts[5 * i + 1] = s.H;
    counts[5 * i + 2] = s.read_bases;
    counts[5 * i + 3] = s.hap_bases;
    counts[5 * i + 4] = s.cells;
  }
  return 0;
}

/* reference of `len` bases with ~5 % of the positions in homopolymer runs of 4..10 */
static void make_reference(rng_t* r, uint8_t* ref, int len) {
  for (int i = 0; i < len; ++i) ref[i] = BASES[rng_int(r, 0, 3)];
  const int target = (int)(0.05 * len);
  int covered = 0;
  while (covered < target && len > 10) {
    const int run = (int)rng_int(r, 4, 10);
    const int st = (int)rng_int(r, 0, len - run - 1);
    const uint8_t b = BASES[rng_int(r, 0, 3)];
    for (int k = 0; k < run; ++k) ref[st + k] = b;
    covered += run;
  }
}

/* haplotype h != 0: SNPs and 1-5 bp indels applied to ref, then cut / padded to n */
static void make_haplotype(rng_t* r, const synth_spec* sp, const uint8_t* ref, int len, uint8_t* out, int n) {
  int o = 0;
  for (int i = 0; i < len && o < n;) {
    if (sp->indel_rate > 0 && rng_unif(r) < sp->indel_rate) {
      const int ln = (int)rng_int(r, 1, 5);
      if (rng_unif(r) < 0.5) {  /* insertion of ln random bases before position i */
        for (int k = 0; k < ln && o < n; ++k) out[o++] = BASES[rng_int(r, 0, 3)];
        if (o >= n) break;
      } else {                  /* deletion of ln reference bases */
        i += ln;
        continue;
      }
    }
    uint8_t b = ref[i++];
    if (rng_unif(r) < sp->snp_rate) b = BASES[(base_idx(b) + rng_int(r, 1, 3)) & 3];
    out[o++] = b;
  }
  while (o < n) out[o++] = BASES[rng_int(r, 0, 3)];
}

/*
 * Fill regions region0 .. region0 + n_regions - 1 into one batch (the layout of
 * include/phmm.h). For region i, read_base0[i] / hap_base0[i] are its first read /
 * haplotype INDEX in the batch, rb0[i] / hb0[i] its first read / haplotype BYTE, pair0[i]
 * its first pair (all from prefix sums of synth_shapes' counts). Writes roff[read] and
 * hoff[hap] (the caller sets the final offsets), every byte of the region's reads,
 * qualities and haplotypes, and its R x H pairs. Returns 0, or -1 on a bad spec.
 */
int synth_fill(const synth_spec* sp, uint64_t seed, int64_t region0, int64_t n_regions, const int64_t* read0,
               const int64_t* hap0, const int64_t* rb0, const int64_t* hb0, const int64_t* pair0, uint8_t* rb,
               uint8_t* q, uint8_t* qi, uint8_t* qd, uint8_t* qg, int64_t* roff, uint8_t* hb, int64_t* hoff,
               int32_t* pairs) {
  if (!sp || n_regions < 0 || sp->h_hi > MAX_H || sp->h_lo < 1) return -1;
  int bad = 0;
#pragma omp parallel reduction(| : bad)
  {
    int32_t* mlen = NULL;
    int mcap = 0;
    uint8_t* ref = NULL;
    int rcap = 0;
#pragma omp for schedule(dynamic, 16)
    for (int64_t i = 0; i < n_regions; ++i) {
      const int64_t region = region0 + i;
      shape_t s;
      region_shape(sp, seed, region, &s, NULL);
      if (s.R > mcap) {
        free(mlen);
        mcap = s.R;
        mlen = (int32_t*)malloc(sizeof(int32_t) * (size_t)mcap);
      }
      region_shape(sp, seed, region, &s, mlen);
      int nmax = 0;
      for (int h = 0; h < s.H; ++h) nmax = s.n_h[h] > nmax ? s.n_h[h] : nmax;
      const int rlen = nmax + 64;
      if (rlen > rcap) {
        free(ref);
        rcap = rlen;
        ref = (uint8_t*)malloc((size_t)rcap);
      }
      if ((s.R && !mlen) || !ref) {
        bad = 1;
        continue;
      }
      rng_t r = rng_make(seed, region, 1);
      make_reference(&r, ref, rlen);
      /* haplotypes */
      int64_t ho = hb0[i];
      for (int h = 0; h < s.H; ++h) {
        hoff[hap0[i] + h] = ho;
        uint8_t* out = hb + ho;
        if (h == 0) {
          memcpy(out, ref, (size_t)s.n_h[0]);
        } else {
          make_haplotype(&r, sp, ref, rlen, out, s.n_h[h]);
        }
        ho += s.n_h[h];
      }
      /* reads */
      int64_t ro = rb0[i];
      for (int k = 0; k < s.R; ++k) {
        const int m = mlen[k];
        roff[read0[i] + k] = ro;
        uint8_t *rd = rb + ro, *bq = q + ro;
        const int src = (int)rng_int(&r, 0, s.H - 1);
        const uint8_t* sh = hb + hb0[i];
        for (int h = 0; h < src; ++h) sh += s.n_h[h];
        const int sn = s.n_h[src];
        if (rng_unif(&r) < sp->decoy_frac) {
          for (int x = 0; x < m; ++x) rd[x] = BASES[rng_int(&r, 0, 3)];
        } else if (sn >= m) {
          const int st = (int)rng_int(&r, 0, sn - m);
          memcpy(rd, sh + st, (size_t)m);
        } else {
          memcpy(rd, sh, (size_t)sn);
          for (int x = sn; x < m; ++x) rd[x] = BASES[rng_int(&r, 0, 3)];
        }
        for (int x = 0; x < m; ++x) {
          double err;
          if (sp->fixed_q >= 0) {
            bq[x] = (uint8_t)sp->fixed_q;
            err = sp->fixed_err;
          } else {
            const double u = rng_unif(&r);
            int b = 0;
            while (b < 3 && u >= QBIN_CUM[b]) ++b;
            bq[x] = QBIN[b];
            err = QBIN_ERR[b];
          }
          if (rng_unif(&r) < err) rd[x] = BASES[(base_idx(rd[x]) + rng_int(&r, 1, 3)) & 3];
          if (sp->n_rate > 0 && rng_unif(&r) < sp->n_rate) {
            rd[x] = 'N';
            bq[x] = 6;
          }
          if (sp->iq_lo == sp->iq_hi) {
            qi[ro + x] = qd[ro + x] = (uint8_t)sp->iq_lo;
          } else {
            qi[ro + x] = (uint8_t)rng_int(&r, sp->iq_lo, sp->iq_hi);
            qd[ro + x] = (uint8_t)rng_int(&r, sp->iq_lo, sp->iq_hi);
          }
          qg[ro + x] = (uint8_t)sp->gcp;
        }
        ro += m;
      }
      /* pairs: all R x H, read-major */
      int32_t* pp = pairs + 2 * pair0[i];
      for (int k = 0; k < s.R; ++k)
        for (int h = 0; h < s.H; ++h) {
          *pp++ = (int32_t)(read0[i] + k);
          *pp++ = (int32_t)(hap0[i] + h);
        }
    }
    free(mlen);
    free(ref);
  }
  return bad ? -1 : 0;
}

int synth_max_threads(void) {
#ifdef _OPENMP
  return omp_get_max_threads();
#else
  return 1;
#endif
}
