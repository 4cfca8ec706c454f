// internal.h — host-side internals of libsfs (not part of the ABI).
#pragma once
#include <cuda_runtime.h>
#include <stddef.h>
#include <stdint.h>

#include <atomic>
#include <string>

#include "sfs.h"
#include "shape.h"

namespace sfs {

// ---------------------------------------------------------------- errors
void set_error(const std::string& msg);
#define SFS_CUDA_TRY(expr)                                                                          \
  do {                                                                                              \
    cudaError_t _e = (expr);                                                                        \
    if (_e != cudaSuccess) {                                                                        \
      ::sfs::set_error(std::string(#expr) + ": " + cudaGetErrorString(_e) + " @" + __FILE__ + ":" + \
                       std::to_string(__LINE__));                                                   \
      return _e == cudaErrorMemoryAllocation ? SFS_ERR_OOM : SFS_ERR_CUDA;                          \
    }                                                                                               \
  } while (0)

// ---------------------------------------------------------------- memory
constexpr int kMaxDevices = 64;              // per-device state (memory pools, function attributes)
void* dalloc(size_t bytes, cudaStream_t s);  // nullptr on failure
void dfree(void* p, cudaStream_t s);

// kernels launched by this library (sfs_launch_count)
extern std::atomic<int64_t> g_launches;
inline void count_launch(int64_t n = 1) { g_launches.fetch_add(n, std::memory_order_relaxed); }

// ---------------------------------------------------------------- feature pass (features.cu)
constexpr int kHistCap = 4096;  // exact row-length histogram bins [0, 4095]; bin 4096 = ">= 4096"

struct DevAggr {                // zeroed by memset; every field updated with atomics
  unsigned long long flags;     // validation error bits (Q16)
  unsigned long long min_inv;   // max over rows of (INT32_MAX - len)
  unsigned long long max_len;
  unsigned long long S2, cL, s1L, s2L, cH, s1H, s2H;
  unsigned long long ndiag;
  unsigned long long big_cnt, big_sum;  // rows with len >= kHistCap
  long long hyb_k;                      // -1: order statistic beyond the histogram, host refines
  long long hyb_coo;
  long long empty_rows;                 // rows of length 0 (hist[0]; csr variant choice, Q17)
  long long pad[1];
};

enum : unsigned long long {
  FLAG_RP0 = 1, FLAG_RP_DECREASE = 2, FLAG_RP_END = 4, FLAG_COL_RANGE = 8, FLAG_COL_ORDER = 16
};

struct FeatWork {
  void* base = nullptr;
  size_t bytes = 0;
  DevAggr* aggr = nullptr;
  unsigned* hist = nullptr;    // kHistCap + 1
  unsigned* bitmap = nullptr;  // words
  long long words = 0;         // ceil((m + n - 1) / 32)
};

size_t feat_work_bytes(long long m, long long n);
void feat_work_bind(FeatWork& w, void* base, long long m, long long n);
// memset + row stats + nnz pass + diag count + HYB select (4 kernels + 1 memset)
cudaError_t launch_features(const int* rp, const int* col, long long m, long long n, long long z, long long rmax,
                            const FeatWork& w, DevAggr* host_out, cudaStream_t s);
// refine pass of the HYB order statistic: histogram of lengths in [lo, hi] with bin width wdt
cudaError_t launch_len_hist_range(const int* rp, long long m, long long lo, long long hi, long long wdt,
                                  unsigned* hist, cudaStream_t s);
cudaError_t launch_hyb_coo(const int* rp, long long m, long long K, long long* out, cudaStream_t s);

// ---------------------------------------------------------------- scans (scan.cu)
// exclusive scan of transformed per-row values; out has m+1 entries (out[m] = total)
size_t scan_work_bytes(long long m);
cudaError_t launch_overflow_scan(const int* rp, long long m, int K, int* out, void* work, cudaStream_t s);
cudaError_t launch_popc_scan(const unsigned* words, long long nw, int* out, void* work, cudaStream_t s);
// pos[r] = number of non-empty rows before r (out[m] = non-empty rows): the CSR tile kernel's row map
cudaError_t launch_nonempty_scan(const int* rp, long long m, int* out, void* work, cudaStream_t s);

// ---------------------------------------------------------------- conversions (convert.cu)
cudaError_t launch_csr2coo(int dtype, const int* rp, const int* col, const void* val, long long m, long long z,
                           int* orow, int* ocol, void* oval, cudaStream_t s);
// ELL slab (and the ELL part of HYB): width K, pitch P
cudaError_t launch_csr2ell(int dtype, const int* rp, const int* col, const void* val, long long m, long long P,
                           int K, int* ecol, void* eval, cudaStream_t s);
// COO part of HYB: entries j >= K of each row, placed at ovf[r] + j - K
cudaError_t launch_hyb_coo_part(int dtype, const int* rp, const int* col, const void* val, long long m,
                                long long z, int K, const int* ovf, int* crow, int* ccol, void* cval,
                                cudaStream_t s);
cudaError_t launch_dia_offsets(const unsigned* bitmap, long long nw, const int* wprefix, long long m, int* offs,
                               cudaStream_t s);
cudaError_t launch_csr2dia(int dtype, const int* rp, const int* col, const void* val, long long m,
                           long long P, const unsigned* bitmap, const int* wprefix, void* dval, cudaStream_t s);

// ---------------------------------------------------------------- SpMV (spmv.cu)
struct Matrix;
int spmv_kernels_per_call(const Matrix* A);
cudaError_t launch_spmv(const Matrix* A, const void* x, void* y, cudaStream_t s);
size_t csr_merge_work_bytes(long long m, long long z, int dtype);
cudaError_t launch_csr_merge_prepare(const int* rp, long long m, long long z, void* work, cudaStream_t s);
size_t csr_tile_work_bytes(long long m, long long z, int bitmap);
cudaError_t launch_csr_tile_prepare(const int* rp, long long m, long long z, void* work, int bitmap, cudaStream_t s);
int csr_vector_tpv(long long m, long long z);
int hyb_rowwise(long long nnz_max, long long K, long long coo_nnz, long long z);
cudaError_t launch_fill(int dtype, void* p, long long n, double v, cudaStream_t s);
// dst[i] = src[idx[i]], i < n (exchange.cu: halo send buffers of the row-partitioned SpMV)
cudaError_t launch_gather(int dtype, const void* src, const int* idx, long long n, void* dst, cudaStream_t s);
cudaError_t launch_l2_flush(const void* buf, size_t bytes, cudaStream_t s);
// fused SpMV + halo push (sfs_spmv_push) and the push alone (sfs_halo_push); `p` validated by the caller
cudaError_t launch_spmv_push(const Matrix* A, const void* x, void* y, const sfs_push_t& p, cudaStream_t s);
cudaError_t launch_halo_push(int dtype, const void* src, long long nrows, const sfs_push_t& p, cudaStream_t s);

// ---------------------------------------------------------------- semi-supervised predictor (cluster.cu)
struct ClusterModel;
cudaError_t cluster_fit(const double* raw, long long n, const int* init_idx, int nc, int k, int max_iter,
                        ClusterModel* M, cudaStream_t s);
cudaError_t cluster_vote(const ClusterModel* M, const int* labels, int* out, cudaStream_t s);
cudaError_t cluster_predict(const ClusterModel* M, const double* raw, long long q, int* cluster, cudaStream_t s);
ClusterModel* cluster_new();
// eigen.cpp: leading k eigenpairs of a symmetric n x n matrix, descending, sign-normalised (F3)
bool sym_eigen_basis(int n, const double* C, int k, double* basis, double* eigval);
void cluster_free(ClusterModel* M);
void cluster_info(const ClusterModel* M, sfs_cluster_info* out);

// ---------------------------------------------------------------- matrix handle
struct Matrix {
  int fmt = 0, dtype = 0;
  long long m = 0, n = 0, nnz = 0, pitch = 0, width = 0, ndiag = 0, coo_nnz = 0;
  const void* ptr[6] = {nullptr, nullptr, nullptr, nullptr, nullptr, nullptr};
  void* owned[8] = {nullptr};  // buffers to free
  int n_owned = 0;
  long long bytes = 0;
  int variant = 0;             // CSR: 0 vector, 1 merge, 2 stream, 3 tile, 4 tile + row-start bitmap,
                               // 5 tile + bitmap over the non-empty rows + row map;
                               // HYB: 1 = one launch (ptr[5] = ovf)
  bool banded = false;         // DIA-admissible pattern (columns near the diagonal): the TMA ELL kernel
                               // streams its slots while x reads hit L1 (gather-bound patterns keep LDG)
  void* work = nullptr;        // CSR merge / tile partition and carries
  cudaStream_t stream = nullptr;
  void (*user_free)(void*, void*) = nullptr;  // allocator hook at creation (nullptr: the library's pool)
};

}  // namespace sfs
