/* semisup.c — plain CPU oracle of the paper's semi-supervised format predictor.
 *
 * TEST INFRASTRUCTURE ONLY (see oracle.h for who may load it).  Written from PAPER.md §4:
 *   feature transform: "a log transform or a square root transform is applied to all features which
 *     have a sparse distribution", then "minmax scaling ... to a range of [0, 1]", then "Principal
 *     Component Analysis (PCA) to decompose the features to a feature vector of size 8";
 *   K-Means on those points, the format of a new matrix = the label of the cluster
 *     whose centroid is closest;
 *   purity(c) = max_f count(c, f) / |c|;
 *   cluster labels by majority vote over the benchmarked members, with the worked
 *     example of P:L169 (82% / 68% / 96% / 78%).
 * Readings where the paper is silent (transform per feature, PCA sign, K-Means initialisation and
 * stopping, vote ties, unbenchmarked clusters) are DESIGN.md §"Readings" F1–F7.
 *
 * Every floating-point expression is evaluated in a fixed order with IEEE +, -, *, /, sqrt only
 * (compiled without FP contraction), so an independent implementation that follows the same
 * definitions reproduces the results bit for bit.
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#define OR_NFEAT 21

/* F1: Table-1 order of the 21 features.  Kind 0: log1p (counts, sizes, moments);
   kind 1: sqrt (fractions in [0, 1]). */
static const int kind_of[OR_NFEAT] = {
    0, /* nrows */ 0, /* ncols */ 0, /* nnz */ 1, /* nnz_frac */ 0, /* nnz_mu */ 0, /* nnz_min */
    0, /* nnz_max */ 0, /* nnz_sig */ 0, /* max_mu */ 0, /* mu_min */ 0, /* csr_max */
    0, /* sig_lower */ 0, /* sig_higher */ 0, /* hyb_ell_size */ 0, /* hyb_coo */ 1, /* hyb_ell_frac */
    0, /* diagonals */ 0, /* dia_size */ 1, /* dia_frac */ 1, /* ell_frac */ 0 /* ell_size */};

int or_ss_feature_kind(int j) { return kind_of[j]; }

/* F1 + F2: transform then min-max scale each column over the n rows (constant column -> 0). */
void or_ss_preprocess(int64_t n, const double *raw, double *out, double *mins, double *maxs) {
  for (int j = 0; j < OR_NFEAT; j++) {
    for (int64_t i = 0; i < n; i++) {
      double v = raw[i * OR_NFEAT + j];
      out[i * OR_NFEAT + j] = kind_of[j] == 0 ? log1p(v) : sqrt(v);
    }
    double lo = out[j], hi = out[j];
    for (int64_t i = 1; i < n; i++) {
      double v = out[i * OR_NFEAT + j];
      if (v < lo) lo = v;
      if (v > hi) hi = v;
    }
    mins[j] = lo;
    maxs[j] = hi;
    for (int64_t i = 0; i < n; i++) {
      double v = out[i * OR_NFEAT + j];
      out[i * OR_NFEAT + j] = hi > lo ? (v - lo) / (hi - lo) : 0.0;
    }
  }
}

/* F3: PCA.  Population covariance of the scaled points, cyclic Jacobi eigendecomposition (rows p < q
   in order, fixed number of sweeps or until every off-diagonal entry is exactly 0), eigenvalues sorted
   descending (stable), each eigenvector's sign chosen so its largest-magnitude entry (first on ties) is
   positive.  basis is k x d (row = component). */
void or_ss_pca(int64_t n, int d, const double *X, int k, double *mean, double *basis, double *eigval) {
  double *C = (double *)calloc((size_t)d * d, sizeof(double));
  double *V = (double *)calloc((size_t)d * d, sizeof(double));
  for (int j = 0; j < d; j++) {
    double s = 0.0;
    for (int64_t i = 0; i < n; i++) s = s + X[i * d + j];
    mean[j] = s / (double)n;
  }
  for (int a = 0; a < d; a++)
    for (int b = a; b < d; b++) {
      double s = 0.0;
      for (int64_t i = 0; i < n; i++) {
        double u = X[i * d + a] - mean[a], w = X[i * d + b] - mean[b];
        s = s + u * w;
      }
      C[a * d + b] = C[b * d + a] = s / (double)n;
    }
  for (int a = 0; a < d; a++) V[a * d + a] = 1.0;
  for (int sweep = 0; sweep < 64; sweep++) {
    int rotated = 0;
    for (int p = 0; p < d; p++)
      for (int q = p + 1; q < d; q++) {
        double apq = C[p * d + q];
        if (apq == 0.0) continue;
        double app = C[p * d + p], aqq = C[q * d + q];
        double theta = (aqq - app) / (2.0 * apq);
        double t = 1.0 / (fabs(theta) + sqrt(theta * theta + 1.0));
        if (theta < 0.0) t = -t;
        double c = 1.0 / sqrt(t * t + 1.0), s = t * c;
        /* if the rotation changes nothing representable, treat the entry as converged */
        if (s == 0.0) { C[p * d + q] = C[q * d + p] = 0.0; continue; }
        rotated = 1;
        for (int r = 0; r < d; r++) { /* C <- C J (columns p, q) */
          double crp = C[r * d + p], crq = C[r * d + q];
          C[r * d + p] = c * crp - s * crq;
          C[r * d + q] = s * crp + c * crq;
        }
        for (int r = 0; r < d; r++) { /* C <- J^T C (rows p, q) */
          double cpr = C[p * d + r], cqr = C[q * d + r];
          C[p * d + r] = c * cpr - s * cqr;
          C[q * d + r] = s * cpr + c * cqr;
        }
        C[p * d + q] = C[q * d + p] = 0.0;
        for (int r = 0; r < d; r++) { /* V <- V J */
          double vrp = V[r * d + p], vrq = V[r * d + q];
          V[r * d + p] = c * vrp - s * vrq;
          V[r * d + q] = s * vrp + c * vrq;
        }
      }
    if (!rotated) break;
  }
  int *order = (int *)malloc(sizeof(int) * d);
  for (int a = 0; a < d; a++) order[a] = a;
  for (int a = 1; a < d; a++) { /* stable insertion sort, descending eigenvalue */
    int o = order[a], b = a - 1;
    while (b >= 0 && C[order[b] * d + order[b]] < C[o * d + o]) { order[b + 1] = order[b]; b--; }
    order[b + 1] = o;
  }
  for (int c = 0; c < k; c++) {
    int col = order[c];
    eigval[c] = C[col * d + col];
    int big = 0;
    for (int r = 1; r < d; r++)
      if (fabs(V[r * d + col]) > fabs(V[big * d + col])) big = r;
    double sg = V[big * d + col] < 0.0 ? -1.0 : 1.0;
    for (int r = 0; r < d; r++) basis[c * d + r] = sg * V[r * d + col];
  }
  free(order);
  free(C);
  free(V);
}

/* Y[i, c] = sum_r (X[i, r] - mean[r]) * basis[c, r], summed over r in order. */
void or_ss_project(int64_t n, int d, const double *X, const double *mean, int k, const double *basis, double *Y) {
  for (int64_t i = 0; i < n; i++)
    for (int c = 0; c < k; c++) {
      double s = 0.0;
      for (int r = 0; r < d; r++) s = s + (X[i * d + r] - mean[r]) * basis[c * d + r];
      Y[i * k + c] = s;
    }
}

static double dist2(const double *a, const double *b, int k) {
  double s = 0.0;
  for (int c = 0; c < k; c++) {
    double t = a[c] - b[c];
    s = s + t * t;
  }
  return s;
}

/* Nearest centroid, ties to the lowest cluster id. */
void or_ss_assign(int64_t n, int k, const double *Y, int nc, const double *cent, int32_t *assign) {
  for (int64_t i = 0; i < n; i++) {
    int best = 0;
    double bd = dist2(Y + i * k, cent, k);
    for (int c = 1; c < nc; c++) {
      double dd = dist2(Y + i * k, cent + (int64_t)c * k, k);
      if (dd < bd) { bd = dd; best = c; }
    }
    assign[i] = best;
  }
}

/* F4: K-Means (Lloyd).  Centroids start at the points init_idx[0..nc) (drawn by the caller from a
   seeded generator); each iteration assigns every point to its nearest centroid, then sets each
   centroid to the mean of its members summed in increasing point order (an empty cluster keeps its
   centroid); stops when no assignment changes or after max_iter iterations.  Returns iterations. */
int or_ss_kmeans(int64_t n, int k, const double *Y, int nc, const int32_t *init_idx, int max_iter, double *cent,
                 int32_t *assign) {
  for (int c = 0; c < nc; c++)
    for (int j = 0; j < k; j++) cent[(int64_t)c * k + j] = Y[(int64_t)init_idx[c] * k + j];
  for (int64_t i = 0; i < n; i++) assign[i] = -1;
  int32_t *na = (int32_t *)malloc(sizeof(int32_t) * (size_t)(n > 0 ? n : 1));
  double *sum = (double *)malloc(sizeof(double) * (size_t)nc * k);
  int64_t *cnt = (int64_t *)malloc(sizeof(int64_t) * (size_t)nc);
  int it = 0;
  for (; it < max_iter; it++) {
    or_ss_assign(n, k, Y, nc, cent, na);
    int changed = 0;
    for (int64_t i = 0; i < n; i++)
      if (na[i] != assign[i]) { changed = 1; assign[i] = na[i]; }
    if (!changed) break;
    for (int64_t q = 0; q < (int64_t)nc * k; q++) sum[q] = 0.0;
    for (int c = 0; c < nc; c++) cnt[c] = 0;
    for (int64_t i = 0; i < n; i++) {
      int c = assign[i];
      cnt[c]++;
      for (int j = 0; j < k; j++) sum[(int64_t)c * k + j] = sum[(int64_t)c * k + j] + Y[i * k + j];
    }
    for (int c = 0; c < nc; c++)
      if (cnt[c] > 0)
        for (int j = 0; j < k; j++) cent[(int64_t)c * k + j] = sum[(int64_t)c * k + j] / (double)cnt[c];
  }
  free(na);
  free(sum);
  free(cnt);
  return it;
}

/* F5/F6: cluster label = majority of the benchmarked members' labels (labels[i] < 0: not benchmarked),
   ties to the lowest format id (Q14); a cluster with no benchmarked member takes the majority label of
   all benchmarked matrices (-1 if there is none). */
void or_ss_vote(int64_t n, const int32_t *assign, const int32_t *labels, int nc, int nfmt, int32_t *cluster_label) {
  int64_t *h = (int64_t *)calloc((size_t)nc * nfmt, sizeof(int64_t));
  int64_t *g = (int64_t *)calloc((size_t)nfmt, sizeof(int64_t));
  for (int64_t i = 0; i < n; i++)
    if (labels[i] >= 0) { h[(int64_t)assign[i] * nfmt + labels[i]]++; g[labels[i]]++; }
  int gl = -1;
  for (int f = 0; f < nfmt; f++)
    if (g[f] > 0 && (gl < 0 || g[f] > g[gl])) gl = f;
  for (int c = 0; c < nc; c++) {
    int best = -1;
    for (int f = 0; f < nfmt; f++)
      if (h[(int64_t)c * nfmt + f] > 0 && (best < 0 || h[(int64_t)c * nfmt + f] > h[(int64_t)c * nfmt + best])) best = f;
    cluster_label[c] = best >= 0 ? best : gl;
  }
  free(h);
  free(g);
}

/* purity of every cluster (0 for an empty cluster) and the size-weighted mean purity. */
double or_ss_purity(int64_t n, const int32_t *assign, const int32_t *labels, int nc, int nfmt, double *purity) {
  int64_t *h = (int64_t *)calloc((size_t)nc * nfmt, sizeof(int64_t));
  int64_t *sz = (int64_t *)calloc((size_t)nc, sizeof(int64_t));
  for (int64_t i = 0; i < n; i++) { h[(int64_t)assign[i] * nfmt + labels[i]]++; sz[assign[i]]++; }
  int64_t num = 0;
  for (int c = 0; c < nc; c++) {
    int64_t mx = 0;
    for (int f = 0; f < nfmt; f++)
      if (h[(int64_t)c * nfmt + f] > mx) mx = h[(int64_t)c * nfmt + f];
    purity[c] = sz[c] ? (double)mx / (double)sz[c] : 0.0;
    num += mx;
  }
  free(h);
  free(sz);
  return n ? (double)num / (double)n : 0.0;
}

/* The worked example of P:L169: a cluster whose members' best formats have counts[f]; `draws`
   members are benchmarked, drawn independently with replacement, and the cluster takes their majority
   label (ties to the lowest format id).  Returns the expected fraction of the cluster classified
   correctly, sum over outcomes of P(outcome) * counts[label(outcome)] / |c|; p_label (nfmt) receives
   the probability that each format is chosen.  Brute force over all nfmt^draws ordered outcomes. */
double or_ss_vote_expected_accuracy(const int64_t *counts, int nfmt, int draws, double *p_label) {
  int64_t total = 0;
  for (int f = 0; f < nfmt; f++) { total += counts[f]; p_label[f] = 0.0; }
  if (total == 0 || draws < 1) return 0.0;
  int64_t outcomes = 1;
  for (int d = 0; d < draws; d++) outcomes *= nfmt;
  int *h = (int *)malloc(sizeof(int) * nfmt);
  double acc = 0.0;
  for (int64_t o = 0; o < outcomes; o++) {
    int64_t t = o;
    double pr = 1.0;
    for (int f = 0; f < nfmt; f++) h[f] = 0;
    for (int d = 0; d < draws; d++) {
      int f = (int)(t % nfmt);
      t /= nfmt;
      h[f]++;
      pr = pr * ((double)counts[f] / (double)total);
    }
    int best = 0;
    for (int f = 1; f < nfmt; f++)
      if (h[f] > h[best]) best = f;
    p_label[best] += pr;
    acc += pr * ((double)counts[best] / (double)total);
  }
  free(h);
  return acc;
}

/* Scale new matrices with the fitted ranges (prediction path): transform, then
   (v - lo) / (hi - lo) per column (0 for a constant training column). */
void or_ss_scale(int64_t n, const double *raw, const double *mins, const double *maxs, double *out) {
  for (int64_t i = 0; i < n; i++)
    for (int j = 0; j < OR_NFEAT; j++) {
      double v = raw[i * OR_NFEAT + j];
      double t = kind_of[j] == 0 ? log1p(v) : sqrt(v);
      out[i * OR_NFEAT + j] = maxs[j] > mins[j] ? (t - mins[j]) / (maxs[j] - mins[j]) : 0.0;
    }
}
