/* gen.c — seeded synthetic CSR generators (TEST / BENCH INPUT ONLY; see sfsgen.h).
 *
 * Recipe: SURVEY.md Appendix B, restated in DESIGN.md §"Input recipe".  The structure classes
 * stand in for the SuiteSparse classes of PAPER.md L194 (§5.1).  Nothing here computes a
 * feature, a conversion or a product: only (row, col, value) draws.
 */
#include "sfsgen.h"

#include <math.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

uint64_t sfsgen_splitmix64(uint64_t x) {
  x += 0x9E3779B97F4A7C15ULL;
  uint64_t z = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ULL;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
  return z ^ (z >> 31);
}

uint64_t sfsgen_hash(uint64_t seed, uint64_t a, uint64_t b) {
  return sfsgen_splitmix64(seed ^ sfsgen_splitmix64(a ^ sfsgen_splitmix64(b ^ 0x243F6A8885A308D3ULL)));
}

static inline double U(uint64_t h) { return (double)(h >> 11) * (1.0 / 9007199254740992.0); }
static inline double U1(uint64_t h) { return 1.0 - U(h); }

/* value v(seed, r, c): random sign, magnitude in [0.5, 1). Never 0 (so DIA round trips hold). */
static inline double value_of(uint64_t seed, int64_t r, int64_t c) {
  double mag = 0.5 + 0.5 * U(sfsgen_hash(seed ^ 0xA5ULL, (uint64_t)r, (uint64_t)c));
  return (sfsgen_hash(seed, (uint64_t)r, (uint64_t)c) & 1ULL) ? -mag : mag;
}

int sfsgen_threads(void) {
#ifdef _OPENMP
  return omp_get_max_threads();
#else
  return 1;
#endif
}

int sfsgen_dims(const sfsgen_spec *s, int64_t *m, int64_t *n) {
  switch (s->cls) {
    case SFSGEN_RMAT: *m = *n = (int64_t)1 << s->ia; return 0;
    case SFSGEN_ST2D5: *m = *n = s->ia * s->ia; return 0;
    case SFSGEN_ST3D7:
    case SFSGEN_ST3D27: *m = *n = s->ia * s->ia * s->ia; return 0;
    case SFSGEN_BAND:
    case SFSGEN_BLOCKDIAG:
    case SFSGEN_UNIFORM:
    case SFSGEN_POWERLAW: *m = s->m; *n = s->n; return (s->m >= 1 && s->n >= 1) ? 0 : -1;
    default: return -1;
  }
}

/* ---------------------------------------------------------------- per-row generation */

typedef struct {
  const sfsgen_spec *s;
  int64_t m, n;
  const double *plaw_T; /* power-law thresholds T[L] = (2/L)^(alpha-1), L = 0..cap (T[0],T[1] unused) */
  int64_t plaw_cap;
  int64_t max_row;      /* upper bound on any row length (scratch size) */
} genctx;

static int cmp_i64(const void *a, const void *b) {
  int64_t x = *(const int64_t *)a, y = *(const int64_t *)b;
  return (x > y) - (x < y);
}

static int64_t sort_dedup(int64_t *c, int64_t len) {
  if (len <= 1) return len;
  if (len <= 32) { /* insertion sort */
    for (int64_t i = 1; i < len; i++) {
      int64_t v = c[i], j = i - 1;
      while (j >= 0 && c[j] > v) { c[j + 1] = c[j]; j--; }
      c[j + 1] = v;
    }
  } else {
    qsort(c, (size_t)len, sizeof(int64_t), cmp_i64);
  }
  int64_t w = 1;
  for (int64_t i = 1; i < len; i++)
    if (c[i] != c[w - 1]) c[w++] = c[i];
  return w;
}

/* Emit the column list of row r into cols (sorted, distinct). Returns its length. */
static int64_t gen_row(const genctx *g, int64_t r, int64_t *cols) {
  const sfsgen_spec *s = g->s;
  const uint64_t seed = s->seed;
  const int64_t n = g->n;
  int64_t len = 0;
  switch (s->cls) {
    case SFSGEN_BAND: {
      int64_t b = s->ia, lo = r - b < 0 ? 0 : r - b, hi = r + b > n - 1 ? n - 1 : r + b;
      for (int64_t c = lo; c <= hi; c++)
        if (c == r || U(sfsgen_hash(seed, (uint64_t)r, (uint64_t)c)) < s->pa) cols[len++] = c;
      return len;
    }
    case SFSGEN_BLOCKDIAG: {
      int64_t B = s->ia, q = r / B, lo = q * B, hi = (q + 1) * B < n ? (q + 1) * B : n;
      for (int64_t c = lo; c < hi; c++)
        if (c == r || U(sfsgen_hash(seed, (uint64_t)r, (uint64_t)c)) < s->pa) cols[len++] = c;
      return len;
    }
    case SFSGEN_UNIFORM: {
      int64_t len0 = (int64_t)floor(s->pa * (0.5 + U(sfsgen_hash(seed, (uint64_t)r, 1ULL << 40))));
      if (len0 < 1) len0 = 1;
      for (int64_t k = 0; k < len0; k++) cols[k] = (int64_t)(sfsgen_hash(seed, (uint64_t)r, (uint64_t)k) % (uint64_t)n);
      return sort_dedup(cols, len0);
    }
    case SFSGEN_POWERLAW: {
      double u = U1(sfsgen_hash(seed, (uint64_t)r, 1ULL << 40));
      /* len0 = largest L in [2, cap] with u <= T[L] (T decreasing, T[2] = 1). */
      int64_t lo = 2, hi = g->plaw_cap;
      if (hi < 2) hi = 2;
      while (lo < hi) {
        int64_t mid = lo + (hi - lo + 1) / 2;
        if (u <= g->plaw_T[mid]) lo = mid; else hi = mid - 1;
      }
      int64_t len0 = lo < n ? lo : n;
      if (len0 <= n / 8) {
        for (int64_t k = 0; k < len0; k++) cols[k] = (int64_t)(sfsgen_hash(seed, (uint64_t)r, (uint64_t)k) % (uint64_t)n);
        return sort_dedup(cols, len0);
      }
      double thr = (double)len0 / (double)n;
      for (int64_t c = 0; c < n; c++)
        if (U(sfsgen_hash(seed, (uint64_t)r, (uint64_t)c)) < thr) cols[len++] = c;
      return len;
    }
    case SFSGEN_ST2D5: {
      int64_t N = s->ia, i = r / N, j = r % N;
      static const int d[5][2] = {{-1, 0}, {0, -1}, {0, 0}, {0, 1}, {1, 0}};
      for (int t = 0; t < 5; t++) {
        int64_t ii = i + d[t][0], jj = j + d[t][1];
        if (ii >= 0 && ii < N && jj >= 0 && jj < N) cols[len++] = ii * N + jj;
      }
      return len;
    }
    case SFSGEN_ST3D7:
    case SFSGEN_ST3D27: {
      int64_t N = s->ia, i = r / (N * N), j = (r / N) % N, k = r % N;
      for (int di = -1; di <= 1; di++)
        for (int dj = -1; dj <= 1; dj++)
          for (int dk = -1; dk <= 1; dk++) {
            if (s->cls == SFSGEN_ST3D7 && (di != 0) + (dj != 0) + (dk != 0) > 1) continue;
            int64_t ii = i + di, jj = j + dj, kk = k + dk;
            if (ii >= 0 && ii < N && jj >= 0 && jj < N && kk >= 0 && kk < N) cols[len++] = (ii * N + jj) * N + kk;
          }
      return len;
    }
  }
  return 0;
}

static double entry_value(const sfsgen_spec *s, int64_t r, int64_t c) {
  switch (s->cls) {
    case SFSGEN_ST2D5: return r == c ? 4.0 : -1.0;
    case SFSGEN_ST3D7: return r == c ? 6.0 : -1.0;
    case SFSGEN_ST3D27: return r == c ? 26.0 : -1.0;
    default: return value_of(s->seed, r, c);
  }
}

static int alloc_out(sfsgen_csr *out, int64_t m, int64_t n, int64_t nnz, int32_t dtype) {
  out->m = m; out->n = n; out->nnz = nnz; out->dtype = dtype;
  out->rp = (int32_t *)malloc(sizeof(int32_t) * (size_t)(m + 1));
  out->col = (int32_t *)malloc(sizeof(int32_t) * (size_t)(nnz > 0 ? nnz : 1));
  out->val = malloc((dtype ? 8 : 4) * (size_t)(nnz > 0 ? nnz : 1));
  return (out->rp && out->col && out->val) ? 0 : -1;
}

/* ---------------------------------------------------------------- R-MAT (Graph500 A/B/C/D) */

static int gen_rmat(const sfsgen_spec *s, sfsgen_csr *out) {
  const int scale = (int)s->ia;
  const int64_t ef = s->ib > 0 ? s->ib : 16;
  const int64_t nv = (int64_t)1 << scale, ne = nv * ef;
  const uint64_t seed = s->seed;
  /* inner hash of the level index is a constant per level */
  uint64_t lev[128];
  for (int l = 0; l < 2 * scale; l++) lev[l] = sfsgen_splitmix64((uint64_t)l ^ 0x243F6A8885A308D3ULL);
  const double tb = 0.19 / 0.24, ta = 0.57 / 0.76;
  int32_t *er = (int32_t *)malloc(sizeof(int32_t) * (size_t)ne);
  int32_t *ec = (int32_t *)malloc(sizeof(int32_t) * (size_t)ne);
  if (!er || !ec) { free(er); free(ec); return -1; }
#pragma omp parallel for schedule(static)
  for (int64_t e = 0; e < ne; e++) {
    int64_t r = 0, c = 0;
    for (int l = 0; l < scale; l++) {
      double u1 = U(sfsgen_splitmix64(seed ^ sfsgen_splitmix64((uint64_t)e ^ lev[2 * l])));
      double u2 = U(sfsgen_splitmix64(seed ^ sfsgen_splitmix64((uint64_t)e ^ lev[2 * l + 1])));
      int rb = u1 >= 0.76;
      int cb = rb ? (u2 >= tb) : (u2 >= ta);
      r |= (int64_t)rb << l;
      c |= (int64_t)cb << l;
    }
    er[e] = (int32_t)r;
    ec[e] = (int32_t)c;
  }
  /* bucket by row (counting sort), then sort + dedup each row */
  int64_t *cnt = (int64_t *)calloc((size_t)nv + 1, sizeof(int64_t));
  for (int64_t e = 0; e < ne; e++) cnt[er[e] + 1]++;
  for (int64_t r = 0; r < nv; r++) cnt[r + 1] += cnt[r];
  int64_t *pos = (int64_t *)malloc(sizeof(int64_t) * (size_t)nv);
  memcpy(pos, cnt, sizeof(int64_t) * (size_t)nv);
  int64_t *bucket = (int64_t *)malloc(sizeof(int64_t) * (size_t)ne);
  for (int64_t e = 0; e < ne; e++) bucket[pos[er[e]]++] = ec[e];
  free(er); free(ec); free(pos);
  int64_t *ulen = (int64_t *)malloc(sizeof(int64_t) * (size_t)nv);
#pragma omp parallel for schedule(dynamic, 1024)
  for (int64_t r = 0; r < nv; r++) ulen[r] = sort_dedup(bucket + cnt[r], cnt[r + 1] - cnt[r]);
  int64_t nnz = 0;
  for (int64_t r = 0; r < nv; r++) nnz += ulen[r];
  if (alloc_out(out, nv, nv, nnz, s->dtype)) { free(cnt); free(bucket); free(ulen); return -1; }
  out->rp[0] = 0;
  for (int64_t r = 0; r < nv; r++) out->rp[r + 1] = (int32_t)(out->rp[r] + ulen[r]);
#pragma omp parallel for schedule(dynamic, 1024)
  for (int64_t r = 0; r < nv; r++) {
    int64_t o = out->rp[r];
    for (int64_t k = 0; k < ulen[r]; k++) {
      int64_t c = bucket[cnt[r] + k];
      out->col[o + k] = (int32_t)c;
      double v = value_of(seed, r, c);
      if (s->dtype) ((double *)out->val)[o + k] = v; else ((float *)out->val)[o + k] = (float)v;
    }
  }
  free(cnt); free(bucket); free(ulen);
  return 0;
}

/* ---------------------------------------------------------------- generic two-pass build */

int sfsgen_generate(const sfsgen_spec *s, sfsgen_csr *out) {
  memset(out, 0, sizeof(*out));
  if (s->cls == SFSGEN_RMAT) {
    if (s->ia < 1 || s->ia > 30) return -1;
    return gen_rmat(s, out);
  }
  genctx g;
  memset(&g, 0, sizeof(g));
  g.s = s;
  if (sfsgen_dims(s, &g.m, &g.n)) return -1;
  const int64_t m = g.m, n = g.n;
  double *T = NULL;
  switch (s->cls) {
    case SFSGEN_BAND: g.max_row = 2 * s->ia + 1; break;
    case SFSGEN_BLOCKDIAG: g.max_row = s->ia; break;
    case SFSGEN_UNIFORM: g.max_row = (int64_t)(1.5 * s->pa) + 2; break;
    case SFSGEN_POWERLAW: {
      int64_t cap = n < ((int64_t)1 << 17) ? n : ((int64_t)1 << 17);
      if (cap < 2) cap = 2;
      T = (double *)malloc(sizeof(double) * (size_t)(cap + 1));
      T[0] = T[1] = 1.0;
      for (int64_t L = 2; L <= cap; L++) T[L] = pow(2.0 / (double)L, s->pa - 1.0);
      g.plaw_T = T;
      g.plaw_cap = cap;
      g.max_row = n > cap ? n : cap;
      break;
    }
    case SFSGEN_ST2D5: g.max_row = 5; break;
    case SFSGEN_ST3D7: g.max_row = 7; break;
    case SFSGEN_ST3D27: g.max_row = 27; break;
    default: return -1;
  }
  if (g.max_row < 1) g.max_row = 1;
  int32_t *len = (int32_t *)malloc(sizeof(int32_t) * (size_t)m);
  int fail = 0;
#pragma omp parallel
  {
    int64_t *scratch = (int64_t *)malloc(sizeof(int64_t) * (size_t)g.max_row);
    if (!scratch) fail = 1;
#pragma omp for schedule(dynamic, 256)
    for (int64_t r = 0; r < m; r++) len[r] = scratch ? (int32_t)gen_row(&g, r, scratch) : 0;
    free(scratch);
  }
  int64_t nnz = 0;
  for (int64_t r = 0; r < m; r++) nnz += len[r];
  if (fail || nnz >= ((int64_t)1 << 31) || alloc_out(out, m, n, nnz, s->dtype)) {
    free(len); free(T); sfsgen_free(out); return -1;
  }
  out->rp[0] = 0;
  for (int64_t r = 0; r < m; r++) out->rp[r + 1] = out->rp[r] + len[r];
  free(len);
#pragma omp parallel
  {
    int64_t *scratch = (int64_t *)malloc(sizeof(int64_t) * (size_t)g.max_row);
#pragma omp for schedule(dynamic, 256)
    for (int64_t r = 0; r < m; r++) {
      int64_t l = gen_row(&g, r, scratch), o = out->rp[r];
      for (int64_t k = 0; k < l; k++) {
        out->col[o + k] = (int32_t)scratch[k];
        double v = entry_value(s, r, scratch[k]);
        if (s->dtype) ((double *)out->val)[o + k] = v; else ((float *)out->val)[o + k] = (float)v;
      }
    }
    free(scratch);
  }
  free(T);
  return 0;
}

void sfsgen_free(sfsgen_csr *c) {
  if (!c) return;
  free(c->rp); free(c->col); free(c->val);
  c->rp = NULL; c->col = NULL; c->val = NULL;
}

void sfsgen_vector(uint64_t seed, int64_t n, int32_t dtype, void *out) {
#pragma omp parallel for schedule(static)
  for (int64_t j = 0; j < n; j++) {
    double x = 2.0 * U(sfsgen_hash(seed ^ 0x78ULL, (uint64_t)j, 0)) - 1.0;
    if (dtype) ((double *)out)[j] = x; else ((float *)out)[j] = (float)x;
  }
}

/* ---------------------------------------------------------------- corpora (BASELINE configs) */

static double draw(uint64_t seed_i, int k) { return U(sfsgen_hash(seed_i, 0, (uint64_t)k)); }

int sfsgen_corpus_spec(int32_t corpus, int64_t i, sfsgen_spec *o) {
  memset(o, 0, sizeof(*o));
  const uint64_t seed_i = sfsgen_splitmix64(0x5EEDULL ^ (uint64_t)i);
  o->seed = seed_i;
  double d0 = draw(seed_i, 0), d1 = draw(seed_i, 1), d2 = draw(seed_i, 2), d3 = draw(seed_i, 3),
         d4 = draw(seed_i, 4), d5 = draw(seed_i, 5);
  if (corpus == 200) {
    /* configs[1]: 200 matrices, classes banded / uniform / block-diagonal / power-law,
       10K-1M rows, fp32 and fp64 (half each). */
    static const int cls_of[4] = {SFSGEN_BAND, SFSGEN_UNIFORM, SFSGEN_BLOCKDIAG, SFSGEN_POWERLAW};
    o->cls = cls_of[i % 4];
    o->dtype = ((i >> 2) & 1) ? 0 : 1;
    o->m = o->n = (int64_t)floor(1e4 * pow(100.0, d0));
    switch (o->cls) {
      case SFSGEN_BAND: o->ia = (int64_t)floor(pow(33.0, d1)); if (o->ia > 32) o->ia = 32; if (o->ia < 1) o->ia = 1; o->pa = 0.5 + 0.5 * d2; break;
      case SFSGEN_UNIFORM: o->pa = 4.0 * pow(16.0, d1); break;
      case SFSGEN_BLOCKDIAG: o->ia = (int64_t)floor(4.0 * pow(16.0, d1)); if (o->ia > 64) o->ia = 64; o->pa = 0.5 + 0.5 * d2; break;
      case SFSGEN_POWERLAW: o->pa = 2.1 + 0.9 * d1; break;
    }
    return 0;
  }
  if (corpus == 2000) {
    /* configs[4]: SuiteSparse-shaped, target nnz logU[1e4, 5e7]; 30% banded/stencil,
       25% uniform, 20% block-diagonal, 25% power-law/R-MAT; fp64. */
    double zt = floor(1e4 * pow(5000.0, d0));
    o->dtype = 1;
    int64_t m;
    if (d1 < 0.30) {
      if (d2 < 0.5) {
        o->cls = SFSGEN_BAND;
        o->ia = (int64_t)floor(pow(33.0, d4)); if (o->ia > 32) o->ia = 32; if (o->ia < 1) o->ia = 1;
        o->pa = 0.5 + 0.5 * d5;
        m = (int64_t)(zt / (1.0 + 2.0 * (double)o->ia * o->pa));
      } else {
        int kind = (int)floor(3.0 * d3);
        o->cls = kind == 0 ? SFSGEN_ST2D5 : (kind == 1 ? SFSGEN_ST3D7 : SFSGEN_ST3D27);
        double pts = kind == 0 ? 5.0 : (kind == 1 ? 7.0 : 27.0);
        o->ia = (int64_t)llround(pow(zt / pts, kind == 0 ? 0.5 : 1.0 / 3.0));
        if (o->ia < 4) o->ia = 4;
        return 0;
      }
    } else if (d1 < 0.55) {
      o->cls = SFSGEN_UNIFORM;
      o->pa = 4.0 * pow(16.0, d4);
      m = (int64_t)(zt / o->pa);
    } else if (d1 < 0.75) {
      o->cls = SFSGEN_BLOCKDIAG;
      o->ia = (int64_t)floor(4.0 * pow(16.0, d4)); if (o->ia > 64) o->ia = 64;
      o->pa = 0.5 + 0.5 * d5;
      m = (int64_t)(zt / ((double)o->ia * o->pa));
    } else if (d2 < 0.5) {
      o->cls = SFSGEN_POWERLAW;
      o->pa = 2.1 + 0.9 * d4;
      m = (int64_t)(zt / (2.0 * (o->pa - 1.0) / (o->pa - 2.0)));
    } else {
      o->cls = SFSGEN_RMAT;
      int64_t sc = (int64_t)llround(log2(zt / 16.0));
      o->ia = sc < 12 ? 12 : (sc > 21 ? 21 : sc);
      o->ib = 16;
      return 0;
    }
    if (m < 1000) m = 1000;
    if (m > ((int64_t)1 << 24)) m = (int64_t)1 << 24;
    o->m = o->n = m;
    return 0;
  }
  return -1;
}
