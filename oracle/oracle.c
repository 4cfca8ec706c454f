/* oracle.c — plain CPU oracle (TEST INFRASTRUCTURE ONLY; see oracle.h for who may load it).
 *
 * Written from the paper (/root/reference/PAPER.md, "P:L<n>") and the readings of SURVEY.md §8(c)
 * (restated in DESIGN.md §"Readings").  Single-threaded plain loops; no blocking, fusion or
 * reordering beyond the definitions.  Integer features are exact; each float feature is one fixed
 * fp64 expression of exact integers (int128 intermediates, IEEE division and sqrt).
 * Parity pins: tests/test_oracle_*.py (closed forms, brute force from dense, invariants).
 */
#include "oracle.h"

#include <math.h>
#include <stdlib.h>
#include <string.h>
#include <time.h>

typedef __int128 i128;
static double i2d(i128 v) { return (double)v; } /* round-to-nearest int -> double */

void or_default_opts(or_opts *o) {
  o->max_fill = 3.0;
  o->fill_slack = (int64_t)1 << 20;
  o->hyb_rel_speed = 3.0;
  o->hyb_breakeven = 4096;
  o->csr_warps = 148 * 64;
}

/* Q16: rp[0] = 0, rp non-decreasing, rp[m] = z, 0 <= col < n, columns strictly increasing per row. */
int or_validate(int64_t m, int64_t n, int64_t z, const int32_t *rp, const int32_t *col) {
  if (m < 1 || n < 1 || z < 0) return 1;
  if (rp[0] != 0) return 2;
  for (int64_t r = 0; r < m; r++)
    if (rp[r + 1] < rp[r]) return 3;
  if (rp[m] != z) return 4;
  for (int64_t r = 0; r < m; r++)
    for (int64_t k = rp[r]; k < rp[r + 1]; k++) {
      if (col[k] < 0 || col[k] >= n) return 5;
      if (k > rp[r] && col[k] <= col[k - 1]) return 6;
    }
  return 0;
}

/* Q6 (HYB width, CUSP-style rule): smallest k in [1, max] such that the number R(k) of rows
   longer than k satisfies rel_speed * R(k) < m or R(k) < breakeven.  max = 0 gives K = 0. */
static int64_t hyb_width(int64_t m, const int32_t *rp, int64_t mx, const or_opts *o) {
  if (mx == 0) return 0;
  int64_t *hist = (int64_t *)calloc((size_t)mx + 1, sizeof(int64_t));
  for (int64_t r = 0; r < m; r++) hist[rp[r + 1] - rp[r]]++;
  int64_t K = mx;
  int64_t rows = m - hist[0]; /* R(0) */
  for (int64_t k = 1; k <= mx; k++) {
    rows -= hist[k]; /* R(k) = rows with length > k */
    if (o->hyb_rel_speed * (double)rows < (double)m || rows < o->hyb_breakeven) {
      K = k;
      break;
    }
  }
  free(hist);
  return K;
}

/* Q4 csr_max: simulate the CSR vector kernel's row -> warp mapping.  Threads per vector TPV from
   floor(z/m); vector v handles rows v, v+V, v+2V, ... with V = warps * (32/TPV); warp = v/(32/TPV). */
static int64_t csr_max_sim(int64_t m, int64_t z, int64_t warps) {
  int64_t avg = z / m, tpv;
  if (avg <= 2) tpv = 2; else if (avg <= 4) tpv = 4; else if (avg <= 8) tpv = 8; else if (avg <= 16) tpv = 16; else tpv = 32;
  int64_t vpw = 32 / tpv, V = warps * vpw;
  int64_t *cnt = (int64_t *)calloc((size_t)warps, sizeof(int64_t));
  for (int64_t r = 0; r < m; r++) cnt[(r % V) / vpw]++;
  int64_t mx = 0;
  for (int64_t w = 0; w < warps; w++) if (cnt[w] > mx) mx = cnt[w];
  free(cnt);
  return mx;
}

int or_features_compute(int64_t m, int64_t n, const int32_t *rp, const int32_t *col, const or_opts *o,
                        or_features *f) {
  memset(f, 0, sizeof(*f));
  const int64_t z = rp[m];
  /* 1. exact integer aggregates over rows */
  int64_t mn = -1, mx = 0, S2 = 0, cL = 0, s1L = 0, s2L = 0, cH = 0, s1H = 0, s2H = 0;
  for (int64_t r = 0; r < m; r++) {
    int64_t len = rp[r + 1] - rp[r];
    if (mn < 0 || len < mn) mn = len;
    if (len > mx) mx = len;
    S2 += len * len;
    if (len * m < z) { cL++; s1L += len; s2L += len * len; }      /* len < nnz_mu (Q3, strict) */
    else if (len * m > z) { cH++; s1H += len; s2H += len * len; } /* len > nnz_mu */
  }
  /* 2. diagonals: distinct offsets c - r over stored entries (Q9) */
  char *seen = (char *)calloc((size_t)(m + n - 1), 1);
  for (int64_t r = 0; r < m; r++)
    for (int64_t k = rp[r]; k < rp[r + 1]; k++) seen[col[k] - r + m - 1] = 1;
  int64_t nd = 0;
  for (int64_t d = 0; d < m + n - 1; d++) nd += seen[d];
  free(seen);
  /* 3. HYB */
  int64_t K = hyb_width(m, rp, mx, o), hcoo = 0;
  for (int64_t r = 0; r < m; r++) {
    int64_t len = rp[r + 1] - rp[r];
    if (len > K) hcoo += len - K;
  }
  const i128 M = m, Z = z;
  f->nrows = m; f->ncols = n; f->nnz = z;
  f->nnz_min = mn; f->nnz_max = mx;
  f->csr_max = csr_max_sim(m, z, o->csr_warps);
  f->ell_size = m * mx;
  f->hyb_k = K; f->hyb_ell_size = m * K; f->hyb_coo = hcoo; f->hyb_ell_nnz = z - hcoo;
  f->diagonals = nd; f->dia_size = nd * m;
  f->nnz_frac = i2d(Z) / i2d(M * (i128)n);                       /* Q1 fraction */
  f->nnz_mu = i2d(Z) / i2d(M);
  f->nnz_sig = sqrt(i2d(M * (i128)S2 - Z * Z) / i2d(M * M));      /* Q2 population std */
  f->max_mu = i2d((i128)mx * M - Z) / i2d(M);                     /* Q5 */
  f->mu_min = i2d(Z - (i128)mn * M) / i2d(M);
  f->sig_lower = cL == 0 ? 0.0 : sqrt(i2d(M * M * (i128)s2L - 2 * M * Z * (i128)s1L + (i128)cL * Z * Z) / i2d((i128)cL * M * M));
  f->sig_higher = cH == 0 ? 0.0 : sqrt(i2d(M * M * (i128)s2H - 2 * M * Z * (i128)s1H + (i128)cH * Z * Z) / i2d((i128)cH * M * M));
  f->hyb_ell_frac = z == 0 ? 0.0 : i2d(Z - hcoo) / i2d(Z);       /* Q7 */
  f->dia_frac = f->dia_size == 0 ? 0.0 : i2d(Z) / i2d((i128)f->dia_size);
  f->ell_frac = f->ell_size == 0 ? 0.0 : i2d(Z) / i2d((i128)f->ell_size);
  /* Q11 admissibility: CSR, COO, HYB always; ELL / DIA by padded-slot guard */
  int64_t lim = (int64_t)(o->max_fill * (double)z);
  if (lim < o->fill_slack) lim = o->fill_slack;
  f->admissible_mask = (1u << OR_CSR) | (1u << OR_COO) | (1u << OR_HYB);
  if (f->ell_size <= lim) f->admissible_mask |= 1u << OR_ELL;
  if (f->dia_size <= lim) f->admissible_mask |= 1u << OR_DIA;
  return 0;
}

/* ------------------------------------------------------------------ conversions */

void or_csr_to_coo(int64_t m, const int32_t *rp, const int32_t *col, const double *val, int32_t *row_out,
                   int32_t *col_out, double *val_out) {
  for (int64_t r = 0; r < m; r++)
    for (int64_t k = rp[r]; k < rp[r + 1]; k++) {
      row_out[k] = (int32_t)r;
      col_out[k] = col[k];
      val_out[k] = val[k];
    }
}

void or_csr_to_ell(int64_t m, const int32_t *rp, const int32_t *col, const double *val, int64_t K,
                   int32_t *ecol, double *eval) {
  for (int64_t r = 0; r < m; r++)
    for (int64_t j = 0; j < K; j++) {
      int64_t k = rp[r] + j;
      if (k < rp[r + 1]) { ecol[r * K + j] = col[k]; eval[r * K + j] = val[k]; }
      else { ecol[r * K + j] = -1; eval[r * K + j] = 0.0; } /* Q10 padding */
    }
}

void or_csr_to_hyb(int64_t m, const int32_t *rp, const int32_t *col, const double *val, int64_t K,
                   int32_t *ecol, double *eval, int32_t *crow, int32_t *ccol, double *cval) {
  int64_t c = 0;
  for (int64_t r = 0; r < m; r++) {
    for (int64_t j = 0; j < K; j++) {
      int64_t k = rp[r] + j;
      if (k < rp[r + 1]) { ecol[r * K + j] = col[k]; eval[r * K + j] = val[k]; }
      else { ecol[r * K + j] = -1; eval[r * K + j] = 0.0; }
    }
    for (int64_t k = rp[r] + K; k < rp[r + 1]; k++) {
      crow[c] = (int32_t)r; ccol[c] = col[k]; cval[c] = val[k]; c++;
    }
  }
}

int64_t or_dia_offsets(int64_t m, int64_t n, const int32_t *rp, const int32_t *col, int32_t *offs) {
  char *seen = (char *)calloc((size_t)(m + n - 1), 1);
  for (int64_t r = 0; r < m; r++)
    for (int64_t k = rp[r]; k < rp[r + 1]; k++) seen[col[k] - r + m - 1] = 1;
  int64_t nd = 0;
  for (int64_t d = 0; d < m + n - 1; d++)
    if (seen[d]) { if (offs) offs[nd] = (int32_t)(d - (m - 1)); nd++; }
  free(seen);
  return nd;
}

void or_csr_to_dia(int64_t m, const int32_t *rp, const int32_t *col, const double *val, int64_t nd,
                   const int32_t *offs, double *dval) {
  for (int64_t i = 0; i < nd * m; i++) dval[i] = 0.0;
  for (int64_t r = 0; r < m; r++)
    for (int64_t k = rp[r]; k < rp[r + 1]; k++) {
      int64_t off = (int64_t)col[k] - r, d = 0;
      while (offs[d] != off) d++; /* linear search: plain, slow, obvious */
      dval[d * m + r] = val[k];
    }
}

/* ------------------------------------------------------------------ SpMV, long double */

static void finish(int64_t m, const long double *acc, const long double *aacc, double *y, double *absy) {
  for (int64_t r = 0; r < m; r++) {
    y[r] = (double)acc[r];
    if (absy) absy[r] = (double)aacc[r];
  }
}

void or_spmv_csr(int64_t m, const int32_t *rp, const int32_t *col, const double *val, const double *x,
                 double *y, double *absy) {
  long double *acc = (long double *)calloc((size_t)m, sizeof(long double));
  long double *aacc = (long double *)calloc((size_t)m, sizeof(long double));
  for (int64_t r = 0; r < m; r++)
    for (int64_t k = rp[r]; k < rp[r + 1]; k++) {
      acc[r] += (long double)val[k] * (long double)x[col[k]];
      aacc[r] += fabsl((long double)val[k] * (long double)x[col[k]]);
    }
  finish(m, acc, aacc, y, absy);
  free(acc); free(aacc);
}

void or_spmv_coo(int64_t m, int64_t z, const int32_t *row, const int32_t *col, const double *val,
                 const double *x, double *y, double *absy) {
  long double *acc = (long double *)calloc((size_t)m, sizeof(long double));
  long double *aacc = (long double *)calloc((size_t)m, sizeof(long double));
  for (int64_t k = 0; k < z; k++) {
    acc[row[k]] += (long double)val[k] * (long double)x[col[k]];
    aacc[row[k]] += fabsl((long double)val[k] * (long double)x[col[k]]);
  }
  finish(m, acc, aacc, y, absy);
  free(acc); free(aacc);
}

void or_spmv_ell(int64_t m, int64_t K, const int32_t *ecol, const double *eval, const double *x, double *y,
                 double *absy) {
  long double *acc = (long double *)calloc((size_t)m, sizeof(long double));
  long double *aacc = (long double *)calloc((size_t)m, sizeof(long double));
  for (int64_t r = 0; r < m; r++)
    for (int64_t j = 0; j < K; j++) {
      int32_t c = ecol[r * K + j];
      if (c < 0) continue;
      acc[r] += (long double)eval[r * K + j] * (long double)x[c];
      aacc[r] += fabsl((long double)eval[r * K + j] * (long double)x[c]);
    }
  finish(m, acc, aacc, y, absy);
  free(acc); free(aacc);
}

void or_spmv_hyb(int64_t m, int64_t K, const int32_t *ecol, const double *eval, int64_t nc, const int32_t *crow,
                 const int32_t *ccol, const double *cval, const double *x, double *y, double *absy) {
  long double *acc = (long double *)calloc((size_t)m, sizeof(long double));
  long double *aacc = (long double *)calloc((size_t)m, sizeof(long double));
  for (int64_t r = 0; r < m; r++)
    for (int64_t j = 0; j < K; j++) {
      int32_t c = ecol[r * K + j];
      if (c < 0) continue;
      acc[r] += (long double)eval[r * K + j] * (long double)x[c];
      aacc[r] += fabsl((long double)eval[r * K + j] * (long double)x[c]);
    }
  for (int64_t k = 0; k < nc; k++) {
    acc[crow[k]] += (long double)cval[k] * (long double)x[ccol[k]];
    aacc[crow[k]] += fabsl((long double)cval[k] * (long double)x[ccol[k]]);
  }
  finish(m, acc, aacc, y, absy);
  free(acc); free(aacc);
}

void or_spmv_dia(int64_t m, int64_t n, int64_t nd, const int32_t *offs, const double *dval, const double *x,
                 double *y, double *absy) {
  long double *acc = (long double *)calloc((size_t)m, sizeof(long double));
  long double *aacc = (long double *)calloc((size_t)m, sizeof(long double));
  for (int64_t d = 0; d < nd; d++)
    for (int64_t r = 0; r < m; r++) {
      int64_t c = r + offs[d];
      if (c < 0 || c >= n) continue;
      acc[r] += (long double)dval[d * m + r] * (long double)x[c];
      aacc[r] += fabsl((long double)dval[d * m + r] * (long double)x[c]);
    }
  finish(m, acc, aacc, y, absy);
  free(acc); free(aacc);
}

/* ------------------------------------------------------------------ label rule (Q14) */

int32_t or_label(const double *t, uint32_t mask) {
  int32_t best = -1;
  for (int32_t f = 0; f < OR_NFMT; f++) {
    if (!(mask & (1u << f))) continue;
    if (best < 0 || t[f] < t[best]) best = f; /* strict: ties keep the lower id */
  }
  return best;
}

static double now_s(void) {
  struct timespec ts;
  clock_gettime(CLOCK_MONOTONIC, &ts);
  return (double)ts.tv_sec + 1e-9 * (double)ts.tv_nsec;
}

int32_t or_label_matrix(int64_t m, int64_t n, const int32_t *rp, const int32_t *col, const double *val,
                        const double *x, const or_opts *o, int32_t reps, uint32_t formats_mask,
                        or_features *f, double *t_spmv, double *t_conv) {
  or_features_compute(m, n, rp, col, o, f);
  const int64_t z = f->nnz;
  double *y = (double *)malloc(sizeof(double) * (size_t)m);
  uint32_t mask = f->admissible_mask & formats_mask;
  for (int i = 0; i < OR_NFMT; i++) { t_spmv[i] = 0.0; t_conv[i] = 0.0; }
  if (reps < 1) reps = 1;
  double t0;
  if (mask & (1u << OR_CSR)) {
    t0 = now_s();
    for (int i = 0; i < reps; i++) or_spmv_csr(m, rp, col, val, x, y, NULL);
    t_spmv[OR_CSR] = (now_s() - t0) / reps;
  }
  if (mask & (1u << OR_COO)) {
    int32_t *r = malloc(sizeof(int32_t) * (size_t)(z + 1)), *c = malloc(sizeof(int32_t) * (size_t)(z + 1));
    double *v = malloc(sizeof(double) * (size_t)(z + 1));
    t0 = now_s();
    or_csr_to_coo(m, rp, col, val, r, c, v);
    t_conv[OR_COO] = now_s() - t0;
    t0 = now_s();
    for (int i = 0; i < reps; i++) or_spmv_coo(m, z, r, c, v, x, y, NULL);
    t_spmv[OR_COO] = (now_s() - t0) / reps;
    free(r); free(c); free(v);
  }
  if (mask & (1u << OR_ELL)) {
    int64_t K = f->nnz_max;
    int32_t *ec = malloc(sizeof(int32_t) * (size_t)(m * K + 1));
    double *ev = malloc(sizeof(double) * (size_t)(m * K + 1));
    t0 = now_s();
    or_csr_to_ell(m, rp, col, val, K, ec, ev);
    t_conv[OR_ELL] = now_s() - t0;
    t0 = now_s();
    for (int i = 0; i < reps; i++) or_spmv_ell(m, K, ec, ev, x, y, NULL);
    t_spmv[OR_ELL] = (now_s() - t0) / reps;
    free(ec); free(ev);
  }
  if (mask & (1u << OR_HYB)) {
    int64_t K = f->hyb_k, nc = f->hyb_coo;
    int32_t *ec = malloc(sizeof(int32_t) * (size_t)(m * K + 1));
    double *ev = malloc(sizeof(double) * (size_t)(m * K + 1));
    int32_t *cr = malloc(sizeof(int32_t) * (size_t)(nc + 1)), *cc = malloc(sizeof(int32_t) * (size_t)(nc + 1));
    double *cv = malloc(sizeof(double) * (size_t)(nc + 1));
    t0 = now_s();
    or_csr_to_hyb(m, rp, col, val, K, ec, ev, cr, cc, cv);
    t_conv[OR_HYB] = now_s() - t0;
    t0 = now_s();
    for (int i = 0; i < reps; i++) or_spmv_hyb(m, K, ec, ev, nc, cr, cc, cv, x, y, NULL);
    t_spmv[OR_HYB] = (now_s() - t0) / reps;
    free(ec); free(ev); free(cr); free(cc); free(cv);
  }
  if (mask & (1u << OR_DIA)) {
    int64_t nd = f->diagonals;
    int32_t *offs = malloc(sizeof(int32_t) * (size_t)(nd + 1));
    double *dv = malloc(sizeof(double) * (size_t)(nd * m + 1));
    t0 = now_s();
    or_dia_offsets(m, n, rp, col, offs);
    or_csr_to_dia(m, rp, col, val, nd, offs, dv);
    t_conv[OR_DIA] = now_s() - t0;
    t0 = now_s();
    for (int i = 0; i < reps; i++) or_spmv_dia(m, n, nd, offs, dv, x, y, NULL);
    t_spmv[OR_DIA] = (now_s() - t0) / reps;
    free(offs); free(dv);
  }
  free(y);
  return or_label(t_spmv, mask);
}
