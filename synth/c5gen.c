/* synth/c5gen.c — seeded synthetic generator for config C5 (circuit/LP-like, 50M rows).
 *
 * INPUT GENERATION ONLY.  This file holds none of the SpMV method's arithmetic: it
 * produces a CSR matrix (sorted, distinct columns per row) and nothing else.  It is
 * shared by the oracle side (tests) and the product side (bench) as the prompt allows.
 *
 * Recipe (shape of Circuit5M):
 *   row i: the diagonal, plus Poisson(lambda) off-diagonals, each with probability
 *   p_local uniform within +-band of i (wrapped into [0,N)), else uniform over [0,N).
 *   n_net "net" rows (positions and lengths drawn from the seed) hold L distinct uniform
 *   columns, L log-uniform in [2^16, 2^21].  Duplicates are merged, so the structure of
 *   every row is a deterministic function of (seed, i) only: any row range can be
 *   generated independently (the matrix is identical for every rank count P).
 *
 * Counter-based RNG: splitmix64 finaliser over (seed, domain, row, k).
 * Value kinds: 0 = positive U(0,1] off-diagonal, diag = 1 + sum(row);
 *              1 = signed U[-1,1) everywhere;  2 = integers in {-2..2}.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <math.h>

static inline uint64_t mix64(uint64_t z) {
  z += 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}
static inline uint64_t draw(uint64_t seed, uint64_t dom, uint64_t row, uint64_t k) {
  return mix64(mix64(mix64(seed ^ (dom * 0xD1B54A32D192ED03ull)) ^ row) + k);
}
static inline double u01(uint64_t r) { return (double)(r >> 11) * (1.0 / 9007199254740992.0); }

typedef struct {
  int64_t n;          /* rows == cols */
  double lambda;      /* Poisson mean of off-diagonals */
  double p_local;
  int64_t band;
  int32_t n_net;
  int32_t net_lo_log2, net_hi_log2;
  uint64_t seed;
} c5_params;

#define MAXPOIS 128
static void pois_cdf(double lam, double* cdf) {
  double p = exp(-lam), c = p;
  cdf[0] = c;
  for (int k = 1; k < MAXPOIS; ++k) { p *= lam / k; c += p; cdf[k] = c; }
  cdf[MAXPOIS - 1] = 2.0;
}

static int cmp_i64(const void* a, const void* b) {
  int64_t x = *(const int64_t*)a, y = *(const int64_t*)b;
  return (x > y) - (x < y);
}

/* net rows: positions r_j and lengths L_j for j < n_net (sorted by position) */
static void net_rows(const c5_params* P, int64_t* pos, int64_t* len) {
  for (int j = 0; j < P->n_net; ++j) {
    pos[j] = (int64_t)(draw(P->seed, 7, (uint64_t)j, 0) % (uint64_t)P->n);
    double e = P->net_lo_log2 + (P->net_hi_log2 - P->net_lo_log2) * u01(draw(P->seed, 7, (uint64_t)j, 1));
    len[j] = (int64_t)floor(pow(2.0, e));
    if (len[j] > P->n) len[j] = P->n;
  }
  /* sort by position (insertion sort; n_net is tiny), drop duplicate positions */
  for (int a = 1; a < P->n_net; ++a)
    for (int b = a; b > 0 && pos[b - 1] > pos[b]; --b) {
      int64_t t = pos[b]; pos[b] = pos[b - 1]; pos[b - 1] = t;
      t = len[b]; len[b] = len[b - 1]; len[b - 1] = t;
    }
}

/* generate the sorted distinct columns of row i into buf (capacity cap); returns count */
static int64_t gen_row(const c5_params* P, const double* cdf, const int64_t* npos, const int64_t* nlen,
                       int64_t i, int64_t* buf, int64_t cap) {
  int64_t cnt = 0;
  int64_t L = -1;
  for (int j = 0; j < P->n_net; ++j) if (npos[j] == i) { L = nlen[j]; break; }
  buf[cnt++] = i;
  if (L >= 0) {
    for (int64_t k = 0; k < L && cnt < cap; ++k)
      buf[cnt++] = (int64_t)(draw(P->seed, 3, (uint64_t)i, (uint64_t)k) % (uint64_t)P->n);
  } else {
    double u = u01(draw(P->seed, 1, (uint64_t)i, 0));
    int k = 0;
    while (k < MAXPOIS - 1 && u > cdf[k]) ++k;
    for (int q = 0; q < k && cnt < cap; ++q) {
      uint64_t r = draw(P->seed, 2, (uint64_t)i, (uint64_t)q);
      double v = u01(r);
      uint64_t r2 = draw(P->seed, 4, (uint64_t)i, (uint64_t)q);
      int64_t c;
      if (v < P->p_local) {
        int64_t off = (int64_t)(r2 % (uint64_t)(2 * P->band + 1)) - P->band;
        c = i + off;
        c %= P->n; if (c < 0) c += P->n;
      } else {
        c = (int64_t)(r2 % (uint64_t)P->n);
      }
      buf[cnt++] = c;
    }
  }
  qsort(buf, (size_t)cnt, sizeof(int64_t), cmp_i64);
  int64_t w = 0;
  for (int64_t q = 0; q < cnt; ++q) if (w == 0 || buf[w - 1] != buf[q]) buf[w++] = buf[q];
  return w;
}

static double val_of(const c5_params* P, int kind, int64_t i, int64_t c) {
  uint64_t r = draw(P->seed, 5, (uint64_t)i, (uint64_t)c);
  if (kind == 0) return 1.0 - u01(r);               /* U(0,1] */
  if (kind == 1) return 2.0 * u01(r) - 1.0;         /* U[-1,1) */
  return (double)((int64_t)(r % 5) - 2);            /* {-2..2} */
}

static int64_t max_row_len(const c5_params* P, const int64_t* nlen) {
  int64_t m = 1 + MAXPOIS;
  for (int j = 0; j < P->n_net; ++j) if (nlen[j] + 1 > m) m = nlen[j] + 1;
  return m;
}

/* Pass 1: row lengths of rows [r0, r1) into counts[r1-r0]. */
int c5_count(const c5_params* P, int64_t r0, int64_t r1, int64_t* counts) {
  double cdf[MAXPOIS];
  pois_cdf(P->lambda, cdf);
  int64_t npos[64], nlen[64];
  if (P->n_net > 64) return -1;
  net_rows(P, npos, nlen);
  int64_t cap = max_row_len(P, nlen);
  int err = 0;
#pragma omp parallel
  {
    int64_t* buf = (int64_t*)malloc((size_t)cap * sizeof(int64_t));
    if (!buf) err = 1;
#pragma omp for schedule(dynamic, 4096)
    for (int64_t i = r0; i < r1; ++i)
      if (buf) counts[i - r0] = gen_row(P, cdf, npos, nlen, i, buf, cap);
    free(buf);
  }
  return err ? -2 : 0;
}

/* Pass 2: fill CSR rows [r0, r1).  row_ptr[0..r1-r0] must hold the local exclusive
 * prefix of counts (row_ptr[0] == 0).  vals is float (dtype 0) or double (dtype 1). */
int c5_fill(const c5_params* P, int64_t r0, int64_t r1, const int64_t* row_ptr, int32_t* col,
            void* vals, int dtype, int kind) {
  double cdf[MAXPOIS];
  pois_cdf(P->lambda, cdf);
  int64_t npos[64], nlen[64];
  if (P->n_net > 64) return -1;
  net_rows(P, npos, nlen);
  int64_t cap = max_row_len(P, nlen);
  int err = 0;
#pragma omp parallel
  {
    int64_t* buf = (int64_t*)malloc((size_t)cap * sizeof(int64_t));
    if (!buf) err = 1;
#pragma omp for schedule(dynamic, 4096)
    for (int64_t i = r0; i < r1; ++i) {
      if (!buf) continue;
      int64_t n = gen_row(P, cdf, npos, nlen, i, buf, cap);
      int64_t base = row_ptr[i - r0];
      double offsum = 0.0;
      int64_t dpos = -1;
      for (int64_t q = 0; q < n; ++q) {
        col[base + q] = (int32_t)buf[q];
        double v;
        if (buf[q] == i) { dpos = q; v = 0.0; }
        else { v = val_of(P, kind, i, buf[q]); offsum += fabs(v); }
        if (dtype == 0) ((float*)vals)[base + q] = (float)v;
        else ((double*)vals)[base + q] = v;
      }
      double dv = (kind == 0) ? 1.0 + offsum : val_of(P, kind, i, i);
      if (kind == 0 && dtype == 0) {
        /* positive variant in fp32: diagonal from the fp32-rounded entries */
        double s = 0.0;
        for (int64_t q = 0; q < n; ++q) if (q != dpos) s += (double)((float*)vals)[base + q];
        dv = 1.0 + s;
      }
      if (dtype == 0) ((float*)vals)[base + dpos] = (float)dv;
      else ((double*)vals)[base + dpos] = dv;
    }
    free(buf);
  }
  return err ? -2 : 0;
}

/* net row positions/lengths (for reporting and for sampling long rows in tests) */
int c5_net_rows(const c5_params* P, int64_t* pos, int64_t* len) {
  if (P->n_net > 64) return -1;
  net_rows(P, pos, len);
  return 0;
}
