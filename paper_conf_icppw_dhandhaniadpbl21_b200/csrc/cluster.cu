// cluster.cu — the paper's semi-supervised format predictor on top of the race output
// (§4): Table-1 features -> log1p / sqrt transform -> min-max
// to [0, 1] -> PCA(8) -> K-Means -> majority vote of the benchmarked members per cluster -> nearest
// centroid for new matrices.  Readings F1–F7: DESIGN.md.
//
// Work split: the per-element transform (glibc log1p / sqrt) and the 21x21 symmetric eigensolver
// (eigen.cpp: Householder + implicit QL) run on the host; everything that scales with the corpus (min/max, covariance, projection, every K-Means
// assignment and update, votes, prediction) runs in the kernels below.  All device arithmetic uses
// explicitly rounded intrinsics (__dadd_rn / __dmul_rn / __dsub_rn / __ddiv_rn: never contracted into
// FMAs) in the fixed orders of the definitions, so results are reproducible bit for bit.
#include <math.h>
#include <string.h>

#include <vector>

#include "common.cuh"
#include "internal.h"

namespace sfs {
namespace {

constexpr int kF = 21;  // Table-1 features

// F1: Table-1 order; 1 = fraction in [0, 1] (sqrt), 0 = count / size / moment (log1p).
constexpr int kFraction[kF] = {0, 0, 0, 1, 0, 0, 0, 0, 0, 0, 0, 0, 0, 0, 0, 1, 0, 0, 1, 1, 0};

__global__ void k_minmax_scale(double* __restrict__ X, long long n, double* __restrict__ mins,
                               double* __restrict__ maxs, int fit) {
  // one CTA per feature column; min / max are order-independent (exact)
  const int j = blockIdx.x;
  __shared__ double s_lo[256], s_hi[256];
  double lo = INFINITY, hi = -INFINITY;
  if (fit) {
    for (long long i = threadIdx.x; i < n; i += blockDim.x) {
      const double v = X[i * kF + j];
      lo = v < lo ? v : lo;
      hi = v > hi ? v : hi;
    }
    s_lo[threadIdx.x] = lo;
    s_hi[threadIdx.x] = hi;
    __syncthreads();
    for (int o = blockDim.x / 2; o > 0; o >>= 1) {
      if (threadIdx.x < o) {
        s_lo[threadIdx.x] = s_lo[threadIdx.x + o] < s_lo[threadIdx.x] ? s_lo[threadIdx.x + o] : s_lo[threadIdx.x];
        s_hi[threadIdx.x] = s_hi[threadIdx.x + o] > s_hi[threadIdx.x] ? s_hi[threadIdx.x + o] : s_hi[threadIdx.x];
      }
      __syncthreads();
    }
    if (threadIdx.x == 0) { mins[j] = s_lo[0]; maxs[j] = s_hi[0]; }
    __syncthreads();
  }
  lo = mins[j];
  hi = maxs[j];
  for (long long i = threadIdx.x; i < n; i += blockDim.x) {
    const double v = X[i * kF + j];
    X[i * kF + j] = hi > lo ? __ddiv_rn(__dsub_rn(v, lo), __dsub_rn(hi, lo)) : 0.0;
  }
}

// column means (thread per column, sequential over rows)
__global__ void k_col_mean(const double* __restrict__ X, long long n, double* __restrict__ mean) {
  const int j = threadIdx.x;
  if (j >= kF) return;
  double s = 0.0;
  for (long long i = 0; i < n; i++) s = __dadd_rn(s, X[i * kF + j]);
  mean[j] = __ddiv_rn(s, (double)n);
}

// population covariance, one thread per (a <= b), sequential over rows
__global__ void k_covariance(const double* __restrict__ X, long long n, const double* __restrict__ mean,
                             double* __restrict__ C) {
  const int t = blockIdx.x * blockDim.x + threadIdx.x;
  int a = 0, rem = t;
  while (a < kF && rem >= kF - a) { rem -= kF - a; a++; }
  if (a >= kF) return;
  const int b = a + rem;
  double s = 0.0;
  for (long long i = 0; i < n; i++) {
    const double u = __dsub_rn(X[i * kF + a], mean[a]), w = __dsub_rn(X[i * kF + b], mean[b]);
    s = __dadd_rn(s, __dmul_rn(u, w));
  }
  C[a * kF + b] = C[b * kF + a] = __ddiv_rn(s, (double)n);
}

// Y[i, c] = sum_r (X[i, r] - mean[r]) * basis[c, r]
__global__ void k_project(const double* __restrict__ X, long long n, const double* __restrict__ mean,
                          const double* __restrict__ basis, int k, double* __restrict__ Y) {
  const long long t = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  if (t >= n * k) return;
  const long long i = t / k;
  const int c = (int)(t % k);
  double s = 0.0;
  for (int r = 0; r < kF; r++) s = __dadd_rn(s, __dmul_rn(__dsub_rn(X[i * kF + r], mean[r]), basis[c * kF + r]));
  Y[t] = s;
}

__device__ __forceinline__ double dist2(const double* a, const double* b, int k) {
  double s = 0.0;
  for (int c = 0; c < k; c++) {
    const double t = __dsub_rn(a[c], b[c]);
    s = __dadd_rn(s, __dmul_rn(t, t));
  }
  return s;
}

// nearest centroid (ties to the lowest id), thread per point; centroids staged in shared memory
__global__ void k_assign(const double* __restrict__ Y, long long n, int k, const double* __restrict__ cent, int nc,
                         int* __restrict__ assign, int* __restrict__ changed) {
  extern __shared__ double s_cent[];
  for (int i = threadIdx.x; i < nc * k; i += blockDim.x) s_cent[i] = cent[i];
  __syncthreads();
  const long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  double y[16];
  for (int c = 0; c < k; c++) y[c] = Y[i * k + c];
  int best = 0;
  double bd = dist2(y, s_cent, k);
  for (int c = 1; c < nc; c++) {
    const double dd = dist2(y, s_cent + c * k, k);
    if (dd < bd) { bd = dd; best = c; }
  }
  if (changed) {
    if (assign[i] != best) { assign[i] = best; *changed = 1; }
  } else {
    assign[i] = best;
  }
}

// centroid update: thread per (cluster, dim), members summed in increasing point order; an empty
// cluster keeps its centroid
__global__ void k_update(const double* __restrict__ Y, long long n, int k, const int* __restrict__ assign, int nc,
                         double* __restrict__ cent) {
  const long long t = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  if (t >= (long long)nc * k) return;
  const int c = (int)(t / k), j = (int)(t % k);
  double s = 0.0;
  long long cnt = 0;
  for (long long i = 0; i < n; i++)
    if (assign[i] == c) { s = __dadd_rn(s, Y[i * k + j]); cnt++; }
  if (cnt > 0) cent[t] = __ddiv_rn(s, (double)cnt);
}

// F5/F6: majority of the benchmarked members per cluster (ties to the lowest format id); empty ->
// global majority (-1 if nothing is benchmarked).  One thread per cluster.
__global__ void k_vote(const int* __restrict__ assign, const int* __restrict__ labels, long long n, int nc,
                       int* __restrict__ out) {
  const int c = blockIdx.x * blockDim.x + threadIdx.x;
  if (c >= nc) return;
  long long h[SFS_NFMT] = {0, 0, 0, 0, 0}, g[SFS_NFMT] = {0, 0, 0, 0, 0};
  for (long long i = 0; i < n; i++) {
    const int l = labels[i];
    if (l < 0 || l >= SFS_NFMT) continue;
    g[l]++;
    if (assign[i] == c) h[l]++;
  }
  int best = -1, gl = -1;
  for (int f = 0; f < SFS_NFMT; f++) {
    if (h[f] > 0 && (best < 0 || h[f] > h[best])) best = f;
    if (g[f] > 0 && (gl < 0 || g[f] > g[gl])) gl = f;
  }
  out[c] = best >= 0 ? best : gl;
}

void transform_host(const double* raw, long long n, std::vector<double>& out) {
  out.resize((size_t)n * kF);
  for (long long i = 0; i < n; i++)
    for (int j = 0; j < kF; j++) {
      const double v = raw[i * kF + j];
      out[(size_t)i * kF + j] = kFraction[j] ? sqrt(v) : log1p(v);
    }
}

}  // namespace

struct ClusterModel {
  int nc = 0, k = 0, iters = 0;
  long long n = 0;
  double mins[kF], maxs[kF], mean[kF];
  std::vector<double> basis, eigval, cent;  // host copies
  std::vector<int> assign;
  double* d_cent = nullptr;   // device centroids (nc x k)
  double* d_param = nullptr;  // device mins | maxs | mean | basis
  cudaStream_t stream = nullptr;
};

static inline unsigned blocks_for(long long n, int t) { return (unsigned)((n + t - 1) / t); }

cudaError_t cluster_fit(const double* raw, long long n, const int* init_idx, int nc, int k, int max_iter,
                        ClusterModel* M, cudaStream_t s) {
  M->nc = nc;
  M->k = k;
  M->n = n;
  M->stream = s;
  std::vector<double> X;
  transform_host(raw, n, X);
  const size_t bx = sizeof(double) * X.size();
  double* dX = (double*)dalloc(bx, s);
  double* dY = (double*)dalloc(sizeof(double) * (size_t)n * k, s);
  double* dP = (double*)dalloc(sizeof(double) * (3 * kF + (size_t)k * kF), s);
  double* dC = (double*)dalloc(sizeof(double) * kF * kF, s);
  int* dA = (int*)dalloc(sizeof(int) * (size_t)n + 2 * sizeof(int), s);
  M->d_cent = (double*)dalloc(sizeof(double) * (size_t)nc * k, s);
  M->d_param = dP;
  if (!dX || !dY || !dP || !dC || !dA || !M->d_cent) return cudaErrorMemoryAllocation;
  int* dChanged = dA + n;
  double *dmin = dP, *dmax = dP + kF, *dmean = dP + 2 * kF, *dbasis = dP + 3 * kF;
  cudaError_t e;
  if ((e = cudaMemcpyAsync(dX, X.data(), bx, cudaMemcpyHostToDevice, s)) != cudaSuccess) return e;
  k_minmax_scale<<<kF, 256, 0, s>>>(dX, n, dmin, dmax, 1);
  k_col_mean<<<1, 32, 0, s>>>(dX, n, dmean);
  k_covariance<<<1, 256, 0, s>>>(dX, n, dmean, dC);
  count_launch(3);
  double C[kF * kF];
  if ((e = cudaMemcpyAsync(C, dC, sizeof(C), cudaMemcpyDeviceToHost, s)) != cudaSuccess) return e;
  if ((e = cudaMemcpyAsync(M->mins, dmin, sizeof(double) * kF, cudaMemcpyDeviceToHost, s)) != cudaSuccess) return e;
  if ((e = cudaMemcpyAsync(M->maxs, dmax, sizeof(double) * kF, cudaMemcpyDeviceToHost, s)) != cudaSuccess) return e;
  if ((e = cudaMemcpyAsync(M->mean, dmean, sizeof(double) * kF, cudaMemcpyDeviceToHost, s)) != cudaSuccess) return e;
  if ((e = cudaStreamSynchronize(s)) != cudaSuccess) return e;
  M->basis.resize((size_t)k * kF);
  M->eigval.resize(k);
  // F3: Householder tridiagonalisation + implicit QL (eigen.cpp; independent of the oracle's Jacobi)
  if (!sym_eigen_basis(kF, C, k, M->basis.data(), M->eigval.data())) return cudaErrorUnknown;
  if ((e = cudaMemcpyAsync(dbasis, M->basis.data(), sizeof(double) * k * kF, cudaMemcpyHostToDevice, s)) != cudaSuccess)
    return e;
  k_project<<<blocks_for(n * k, 256), 256, 0, s>>>(dX, n, dmean, dbasis, k, dY);
  count_launch();
  // F4: K-Means from the caller's initial points
  std::vector<double> c0((size_t)nc * k);
  std::vector<double> Yh((size_t)n * k);
  if ((e = cudaMemcpyAsync(Yh.data(), dY, sizeof(double) * Yh.size(), cudaMemcpyDeviceToHost, s)) != cudaSuccess) return e;
  if ((e = cudaStreamSynchronize(s)) != cudaSuccess) return e;
  for (int c = 0; c < nc; c++)
    for (int j = 0; j < k; j++) c0[(size_t)c * k + j] = Yh[(size_t)init_idx[c] * k + j];
  if ((e = cudaMemcpyAsync(M->d_cent, c0.data(), sizeof(double) * c0.size(), cudaMemcpyHostToDevice, s)) != cudaSuccess)
    return e;
  if ((e = cudaMemsetAsync(dA, 0xff, sizeof(int) * (size_t)n, s)) != cudaSuccess) return e;  // -1
  const size_t smem = sizeof(double) * (size_t)nc * k;
  if (smem > 200 * 1024) return cudaErrorInvalidValue;
  if (smem > 48 * 1024) cudaFuncSetAttribute(k_assign, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  int it = 0;
  for (; it < max_iter; it++) {
    int changed = 0;
    if ((e = cudaMemsetAsync(dChanged, 0, sizeof(int), s)) != cudaSuccess) return e;
    k_assign<<<blocks_for(n, 256), 256, smem, s>>>(dY, n, k, M->d_cent, nc, dA, dChanged);
    count_launch();
    if ((e = cudaMemcpyAsync(&changed, dChanged, sizeof(int), cudaMemcpyDeviceToHost, s)) != cudaSuccess) return e;
    if ((e = cudaStreamSynchronize(s)) != cudaSuccess) return e;
    if (!changed) break;
    k_update<<<blocks_for((long long)nc * k, 128), 128, 0, s>>>(dY, n, k, dA, nc, M->d_cent);
    count_launch();
  }
  M->iters = it;
  M->cent.resize((size_t)nc * k);
  M->assign.resize((size_t)n);
  if ((e = cudaMemcpyAsync(M->cent.data(), M->d_cent, sizeof(double) * M->cent.size(), cudaMemcpyDeviceToHost, s)) !=
      cudaSuccess)
    return e;
  if ((e = cudaMemcpyAsync(M->assign.data(), dA, sizeof(int) * (size_t)n, cudaMemcpyDeviceToHost, s)) != cudaSuccess)
    return e;
  if ((e = cudaStreamSynchronize(s)) != cudaSuccess) return e;
  dfree(dX, s);
  dfree(dY, s);
  dfree(dC, s);
  dfree(dA, s);
  return cudaGetLastError();
}

cudaError_t cluster_vote(const ClusterModel* M, const int* labels, int* out, cudaStream_t s) {
  const long long n = M->n;
  int* dA = (int*)dalloc(sizeof(int) * (size_t)(2 * n + M->nc), s);
  if (!dA) return cudaErrorMemoryAllocation;
  cudaError_t e;
  if ((e = cudaMemcpyAsync(dA, M->assign.data(), sizeof(int) * n, cudaMemcpyHostToDevice, s)) != cudaSuccess) return e;
  if ((e = cudaMemcpyAsync(dA + n, labels, sizeof(int) * n, cudaMemcpyHostToDevice, s)) != cudaSuccess) return e;
  k_vote<<<blocks_for(M->nc, 128), 128, 0, s>>>(dA, dA + n, n, M->nc, dA + 2 * n);
  count_launch();
  if ((e = cudaMemcpyAsync(out, dA + 2 * n, sizeof(int) * M->nc, cudaMemcpyDeviceToHost, s)) != cudaSuccess) return e;
  if ((e = cudaStreamSynchronize(s)) != cudaSuccess) return e;
  dfree(dA, s);
  return cudaGetLastError();
}

cudaError_t cluster_predict(const ClusterModel* M, const double* raw, long long q, int* cluster, cudaStream_t s) {
  const int k = M->k;
  std::vector<double> X;
  transform_host(raw, q, X);
  double* dX = (double*)dalloc(sizeof(double) * X.size(), s);
  double* dY = (double*)dalloc(sizeof(double) * (size_t)q * k, s);
  int* dA = (int*)dalloc(sizeof(int) * (size_t)q, s);
  if (!dX || !dY || !dA) return cudaErrorMemoryAllocation;
  cudaError_t e;
  if ((e = cudaMemcpyAsync(dX, X.data(), sizeof(double) * X.size(), cudaMemcpyHostToDevice, s)) != cudaSuccess) return e;
  double *dmin = M->d_param, *dmax = M->d_param + kF, *dmean = M->d_param + 2 * kF, *dbasis = M->d_param + 3 * kF;
  k_minmax_scale<<<kF, 256, 0, s>>>(dX, q, dmin, dmax, 0);  // scale with the fitted ranges
  k_project<<<blocks_for(q * k, 256), 256, 0, s>>>(dX, q, dmean, dbasis, k, dY);
  const size_t smem = sizeof(double) * (size_t)M->nc * k;
  k_assign<<<blocks_for(q, 256), 256, smem, s>>>(dY, q, k, M->d_cent, M->nc, dA, nullptr);
  count_launch(3);
  if ((e = cudaMemcpyAsync(cluster, dA, sizeof(int) * q, cudaMemcpyDeviceToHost, s)) != cudaSuccess) return e;
  if ((e = cudaStreamSynchronize(s)) != cudaSuccess) return e;
  dfree(dX, s);
  dfree(dY, s);
  dfree(dA, s);
  return cudaGetLastError();
}

ClusterModel* cluster_new() { return new ClusterModel(); }

void cluster_info(const ClusterModel* M, sfs_cluster_info* out) {
  out->n = M->n;
  out->nc = M->nc;
  out->pcs = M->k;
  out->iters = M->iters;
  out->assign = M->assign.data();
  out->centroids = M->cent.data();
  out->basis = M->basis.data();
  out->eigval = M->eigval.data();
  out->mins = M->mins;
  out->maxs = M->maxs;
  out->mean = M->mean;
}

void cluster_free(ClusterModel* M) {
  if (!M) return;
  dfree(M->d_cent, M->stream);
  dfree(M->d_param, M->stream);
  delete M;
}

}  // namespace sfs
