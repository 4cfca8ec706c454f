/* oracle.h — plain, slow, obviously-correct CPU oracle of the labelling/featurisation path.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference leg may load this library.  It shares no code, header, table or constant
 * generator with the CUDA path (paper_conf_icppw_dhandhaniadpbl21_b200/), and neither includes the
 * other.  Everything is fp64 (SpMV accumulates in x86 80-bit long double, rounded once).
 *
 * Paper: Dhandhania et al., "Explaining the Performance of Supervised and Semi-Supervised Methods
 * for Automated Sparse Matrix Format Selection", ICPP Workshops '21 = /root/reference/PAPER.md (P:L<n>).
 * Readings where the paper is silent: SURVEY.md §8(c) Q1-Q18, restated in DESIGN.md §"Readings".
 */
#ifndef SFS_ORACLE_H
#define SFS_ORACLE_H
#include <stdint.h>

enum { OR_CSR = 0, OR_COO = 1, OR_ELL = 2, OR_HYB = 3, OR_DIA = 4, OR_NFMT = 5 };

typedef struct {
  double max_fill;      /* Q11: ELL/DIA admissible iff padded slots <= max(trunc(max_fill*z), fill_slack) */
  int64_t fill_slack;
  double hyb_rel_speed; /* Q6: HYB width rule parameters */
  int64_t hyb_breakeven;
  int64_t csr_warps;    /* Q4: warps of the CSR vector kernel grid (csr_max) */
} or_opts;

typedef struct {
  /* Table 1 */
  int64_t nrows, ncols, nnz, nnz_min, nnz_max, csr_max, ell_size, hyb_k, hyb_ell_size, hyb_coo,
      hyb_ell_nnz, diagonals, dia_size;
  double nnz_frac, nnz_mu, nnz_sig, max_mu, mu_min, sig_lower, sig_higher, hyb_ell_frac, dia_frac,
      ell_frac;
  uint32_t admissible_mask; /* bit f set iff format f is admissible (Q11) */
} or_features;

/* Q16 canonical CSR check: 0 = valid, else a nonzero code. */
int or_validate(int64_t m, int64_t n, int64_t z, const int32_t *rp, const int32_t *col);

void or_default_opts(or_opts *o);
/* Table-1 features + HYB width (Q6) + admissibility (Q11). */
int or_features_compute(int64_t m, int64_t n, const int32_t *rp, const int32_t *col, const or_opts *o,
                        or_features *f);

/* Conversions (§2.1; step (ii) of P:L331).  Oracle layouts are its own, row-major:
 *   ELL : ecol[r*K + j], eval[r*K + j]   (pad col = -1, val = +0.0)          K = nnz_max
 *   HYB : ELL part as ELL with K = hyb_k; COO part crow/ccol/cval (hyb_coo entries, (r,j) order)
 *   DIA : offs[d] ascending, dval[d*m + r] = A[r, r+offs[d]] or +0.0                          */
void or_csr_to_coo(int64_t m, const int32_t *rp, const int32_t *col, const double *val, int32_t *row_out,
                   int32_t *col_out, double *val_out);
void or_csr_to_ell(int64_t m, const int32_t *rp, const int32_t *col, const double *val, int64_t K,
                   int32_t *ecol, double *eval);
void or_csr_to_hyb(int64_t m, const int32_t *rp, const int32_t *col, const double *val, int64_t K,
                   int32_t *ecol, double *eval, int32_t *crow, int32_t *ccol, double *cval);
int64_t or_dia_offsets(int64_t m, int64_t n, const int32_t *rp, const int32_t *col, int32_t *offs);
void or_csr_to_dia(int64_t m, const int32_t *rp, const int32_t *col, const double *val, int64_t nd,
                   const int32_t *offs, double *dval);

/* Per-format y = A x, each over its own format arrays.  Optional absy = |A||x|. */
void or_spmv_csr(int64_t m, const int32_t *rp, const int32_t *col, const double *val, const double *x,
                 double *y, double *absy);
void or_spmv_coo(int64_t m, int64_t z, const int32_t *row, const int32_t *col, const double *val,
                 const double *x, double *y, double *absy);
void or_spmv_ell(int64_t m, int64_t K, const int32_t *ecol, const double *eval, const double *x, double *y,
                 double *absy);
void or_spmv_hyb(int64_t m, int64_t K, const int32_t *ecol, const double *eval, int64_t nc, const int32_t *crow,
                 const int32_t *ccol, const double *cval, const double *x, double *y, double *absy);
void or_spmv_dia(int64_t m, int64_t n, int64_t nd, const int32_t *offs, const double *dval, const double *x,
                 double *y, double *absy);

/* Label decision rule (Q14): argmin of mean times over admissible formats in `mask`,
   exact ties to the lowest format id.  -1 if the mask is empty. */
int32_t or_label(const double *t, uint32_t mask);

/* The whole oracle labelling pass for one matrix (the cpu_baseline): features, every admissible
   conversion, `reps` timed SpMVs per format, argmin.  t_spmv[f] in seconds (mean), t_conv[f]. */
int32_t or_label_matrix(int64_t m, int64_t n, const int32_t *rp, const int32_t *col, const double *val,
                        const double *x, const or_opts *o, int32_t reps, uint32_t formats_mask,
                        or_features *f, double *t_spmv, double *t_conv);
#endif
