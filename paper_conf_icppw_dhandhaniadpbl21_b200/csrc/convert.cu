// convert.cu — CSR -> COO / ELL / HYB / DIA (§2.1; step (ii) of L331 §5.4).
//
// Layouts (include/sfs.h, sfs_layout_t):
//   COO : row/col/val, nnz each, CSR order.
//   ELL : column-major slab of width K and pitch P = ceil(m/32)*32: entry (r, j) at j*P + r, so a warp
//         reading slot j of 32 consecutive rows touches one contiguous 128 B line of col (coalesced).
//         Padding col = -1, val = +0 (Q10).  Rows [m, P) are padding too.
//   HYB : ELL slab of width K_hyb + COO part (entries j >= K_hyb of each row, (r, j) order).
//   DIA : offsets ascending + slab val[d*P + r] (+0 where the entry is absent).
#include "common.cuh"
#include <mutex>

#include "internal.h"

namespace sfs {
namespace {

constexpr int kTileThreads = 256;
constexpr int kTileIPT = 8;
constexpr int kTile = kTileThreads * kTileIPT;

// Shared setup of a merge-path tile: stage the row_ptr window and return the tile coordinates.
__device__ __forceinline__ void tile_begin(const int* __restrict__ rp, long long m, long long z, int* s_rp,
                                           int* s_coord, long long& d0, long long& d1) {
  const long long total = m + z;
  d0 = (long long)blockIdx.x * kTile;
  d1 = d0 + kTile < total ? d0 + kTile : total;
  if (threadIdx.x < 64) {  // warp 0 finds the tile start, warp 1 its end
    const int wsel = threadIdx.x >> 5;
    int x, y;
    merge_path_search_warp(wsel == 0 ? d0 : d1, rp + 1, (int)m, (int)z, x, y);
    if ((threadIdx.x & 31) == 0) {
      s_coord[wsel * 2] = x;
      s_coord[wsel * 2 + 1] = y;
    }
  }
  __syncthreads();
  const int r0 = s_coord[0], r1 = s_coord[2];
  for (int i = threadIdx.x; i <= r1 - r0 + 1 && r0 + i <= m; i += blockDim.x) s_rp[i] = rp[r0 + i];
  __syncthreads();
}

// COO: row index of every nnz via the merge walk, staged in smem, then coalesced writes of row/col/val.
template <typename T>
__global__ void __launch_bounds__(kTileThreads) k_csr2coo(const int* __restrict__ rp, const int* __restrict__ col,
                                                          const T* __restrict__ val, long long m, long long z,
                                                          int* __restrict__ orow, int* __restrict__ ocol,
                                                          T* __restrict__ oval) {
  dep_wait();
  __shared__ int s_rp[kTile + 2];
  __shared__ int s_row[kTile];
  __shared__ int s_coord[4];
  long long d0, d1;
  tile_begin(rp, m, z, s_rp, s_coord, d0, d1);
  const int r0 = s_coord[0], k0 = s_coord[1], r1 = s_coord[2], k1 = s_coord[3];
  const int ld = threadIdx.x * kTileIPT, items_all = (int)(d1 - d0);
  if (ld < items_all) {
    int r, k;
    merge_local_search(s_rp, r1 - r0, k0, k1, ld, r0, r, k);
    const int items = items_all - ld < kTileIPT ? items_all - ld : kTileIPT;
    for (int it = 0; it < items; it++) {
      if (r < m && s_rp[r - r0 + 1] <= k) { r++; continue; }
      if (k >= k1) break;
      s_row[k - k0] = r;
      k++;
    }
  }
  __syncthreads();
  for (int i = threadIdx.x; i < k1 - k0; i += blockDim.x) {
    orow[k0 + i] = s_row[i];
    ocol[k0 + i] = col[k0 + i];
    oval[k0 + i] = val[k0 + i];
  }
  dep_trigger();
}

// ELL slab (also the ELL part of HYB).  A CTA owns 128 consecutive rows; their CSR segment is
// contiguous, so it is staged in shared memory with coalesced loads, then written slot by slot
// (coalesced).  The staging capacity follows the slab width (128 * K entries, 2048..8192: dynamic
// shared memory), so rows of up to K entries stay on the staged path; a CTA whose segment is larger
// still reads its rows from global memory.
constexpr int kEllRows = 128;
constexpr int kSegCapMin = 2048;
constexpr int kSegCapMax = 8192;

template <typename T>
__global__ void __launch_bounds__(kEllRows) k_csr2ell(const int* __restrict__ rp, const int* __restrict__ col,
                                                      const T* __restrict__ val, long long m, long long P, int K,
                                                      int cap, int* __restrict__ ecol, T* __restrict__ eval) {
  dep_wait();
  extern __shared__ __align__(16) unsigned char s_seg[];
  T* s_val = (T*)s_seg;                          // [cap]
  int* s_col = (int*)(s_seg + sizeof(T) * cap);  // [cap]
  const long long r0 = (long long)blockIdx.x * kEllRows;
  const long long r = r0 + threadIdx.x;
  const long long rend = r0 + kEllRows < m ? r0 + kEllRows : m;
  int seg0 = 0, seg1 = 0, st = 0, len = 0;
  if (r0 < m) { seg0 = rp[r0]; seg1 = rp[rend]; }
  if (r < m) { st = rp[r]; len = rp[r + 1] - st; }
  const bool staged = (seg1 - seg0) <= cap;
  if (staged) {
    for (int i = threadIdx.x; i < seg1 - seg0; i += blockDim.x) {
      s_col[i] = col[seg0 + i];
      s_val[i] = val[seg0 + i];
    }
  }
  __syncthreads();
  if (r >= P) return;
  const int lst = st - seg0;
  for (int j = 0; j < K; j++) {
    int c = -1;
    T v = T(0);
    if (j < len) {
      if (staged) { c = s_col[lst + j]; v = s_val[lst + j]; }
      else { c = col[st + j]; v = val[st + j]; }
    }
    ecol[(long long)j * P + r] = c;
    eval[(long long)j * P + r] = v;
  }
  dep_trigger();
}

// COO part of HYB: entries j >= K of row r go to ovf[r] + (j - K).
template <typename T>
__global__ void __launch_bounds__(kTileThreads) k_hyb_coo_part(const int* __restrict__ rp, const int* __restrict__ col,
                                                               const T* __restrict__ val, long long m, long long z, int K,
                                                               const int* __restrict__ ovf, int* __restrict__ crow,
                                                               int* __restrict__ ccol, T* __restrict__ cval) {
  dep_wait();
  __shared__ int s_rp[kTile + 2];
  __shared__ int s_coord[4];
  long long d0, d1;
  tile_begin(rp, m, z, s_rp, s_coord, d0, d1);
  const int r0 = s_coord[0], k0 = s_coord[1], r1 = s_coord[2], k1 = s_coord[3];
  const int ld = threadIdx.x * kTileIPT, items_all = (int)(d1 - d0);
  if (ld >= items_all) return;
  int r, k;
  merge_local_search(s_rp, r1 - r0, k0, k1, ld, r0, r, k);
  const int items = items_all - ld < kTileIPT ? items_all - ld : kTileIPT;
  for (int it = 0; it < items; it++) {
    if (r < m && s_rp[r - r0 + 1] <= k) { r++; continue; }
    if (k >= k1) break;
    const int j = k - s_rp[r - r0];
    if (j >= K) {
      const int p = ovf[r] + (j - K);
      crow[p] = r;
      ccol[p] = col[k];
      cval[p] = val[k];
    }
    k++;
  }
  dep_trigger();
}

__global__ void k_dia_offsets(const unsigned* __restrict__ bitmap, long long nw, const int* __restrict__ wprefix,
                              long long m, int* __restrict__ offs) {
  dep_wait();
  for (long long w = (long long)blockIdx.x * blockDim.x + threadIdx.x; w < nw; w += (long long)gridDim.x * blockDim.x) {
    unsigned b = bitmap[w];
    int o = wprefix[w];
    while (b) {
      int bit = __ffs(b) - 1;
      offs[o++] = (int)(w * 32 + bit - (m - 1));
      b &= b - 1;
    }
  }
  dep_trigger();
}

// DIA scatter: thread per row; the j-th entry of consecutive rows usually sits on the same diagonal,
// so the stores val[d*P + r] of a warp are coalesced for banded / stencil matrices.
template <typename T>
__global__ void k_csr2dia(const int* __restrict__ rp, const int* __restrict__ col, const T* __restrict__ val,
                          long long m, long long P, const unsigned* __restrict__ bitmap,
                          const int* __restrict__ wprefix, T* __restrict__ dval) {
  dep_wait();
  for (long long r = (long long)blockIdx.x * blockDim.x + threadIdx.x; r < m; r += (long long)gridDim.x * blockDim.x) {
    const int b = rp[r], e = rp[r + 1];
    for (int k = b; k < e; k++) {
      const long long g = (long long)col[k] - r + m - 1;
      const long long w = g >> 5;
      const unsigned below = bitmap[w] & ((1u << (g & 31)) - 1u);
      const long long d = wprefix[w] + __popc(below);
      dval[d * P + r] = val[k];
    }
  }
  dep_trigger();
}

int grid_cap(long long items, int threads, int per_sm) {
  long long g = ceil_div(items, threads), cap = (long long)kSMs * per_sm;
  return (int)(g > cap ? cap : (g < 1 ? 1 : g));
}

}  // namespace

cudaError_t launch_csr2coo(int dtype, const int* rp, const int* col, const void* val, long long m, long long z,
                           int* orow, int* ocol, void* oval, cudaStream_t s) {
  long long tiles = ceil_div(m + z, kTile);
  if (z == 0) return cudaSuccess;
  if (dtype == SFS_F64)
    (void)launch_dep(k_csr2coo<double>, dim3((unsigned)tiles), dim3(kTileThreads), 0, s, rp, col, (const double*)val, m, z, orow, ocol, (double*)oval);
  else
    (void)launch_dep(k_csr2coo<float>, dim3((unsigned)tiles), dim3(kTileThreads), 0, s, rp, col, (const float*)val, m, z, orow, ocol, (float*)oval);
  count_launch();
  return cudaGetLastError();
}

cudaError_t launch_csr2ell(int dtype, const int* rp, const int* col, const void* val, long long m, long long P, int K,
                           int* ecol, void* eval, cudaStream_t s) {
  if (K == 0 || P == 0) return cudaSuccess;
  unsigned g = (unsigned)ceil_div(P, kEllRows);
  long long cap = (long long)kEllRows * K;
  cap = cap < kSegCapMin ? kSegCapMin : (cap > kSegCapMax ? kSegCapMax : cap);
  // opt in to > 48 KB of dynamic shared memory: a function attribute is per device, so once per device
  static std::once_flag attr_once[kMaxDevices];
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= kMaxDevices) return cudaErrorInvalidDevice;
  std::call_once(attr_once[dev], [] {
    cudaFuncSetAttribute(k_csr2ell<double>, cudaFuncAttributeMaxDynamicSharedMemorySize, kSegCapMax * 12);
    cudaFuncSetAttribute(k_csr2ell<float>, cudaFuncAttributeMaxDynamicSharedMemorySize, kSegCapMax * 8);
  });
  if (dtype == SFS_F64)
    (void)launch_dep(k_csr2ell<double>, dim3(g), dim3(kEllRows), cap * 12, s, rp, col, (const double*)val, m, P, K, (int)cap, ecol,
                                                    (double*)eval);
  else
    (void)launch_dep(k_csr2ell<float>, dim3(g), dim3(kEllRows), cap * 8, s, rp, col, (const float*)val, m, P, K, (int)cap, ecol,
                                                  (float*)eval);
  count_launch();
  return cudaGetLastError();
}

cudaError_t launch_hyb_coo_part(int dtype, const int* rp, const int* col, const void* val, long long m, long long z,
                                int K, const int* ovf, int* crow, int* ccol, void* cval, cudaStream_t s) {
  if (z == 0) return cudaSuccess;
  long long tiles = ceil_div(m + z, kTile);
  if (dtype == SFS_F64)
    (void)launch_dep(k_hyb_coo_part<double>, dim3((unsigned)tiles), dim3(kTileThreads), 0, s, rp, col, (const double*)val, m, z, K, ovf, crow,
                                                                     ccol, (double*)cval);
  else
    (void)launch_dep(k_hyb_coo_part<float>, dim3((unsigned)tiles), dim3(kTileThreads), 0, s, rp, col, (const float*)val, m, z, K, ovf, crow,
                                                                    ccol, (float*)cval);
  count_launch();
  return cudaGetLastError();
}

cudaError_t launch_dia_offsets(const unsigned* bitmap, long long nw, const int* wprefix, long long m, int* offs,
                               cudaStream_t s) {
  (void)launch_dep(k_dia_offsets, dim3(grid_cap(nw, 256, 8)), dim3(256), 0, s, bitmap, nw, wprefix, m, offs);
  count_launch();
  return cudaGetLastError();
}

cudaError_t launch_csr2dia(int dtype, const int* rp, const int* col, const void* val, long long m, long long P,
                           const unsigned* bitmap, const int* wprefix, void* dval, cudaStream_t s) {
  if (dtype == SFS_F64)
    (void)launch_dep(k_csr2dia<double>, dim3(grid_cap(m, 256, 8)), dim3(256), 0, s, rp, col, (const double*)val, m, P, bitmap, wprefix, (double*)dval);
  else
    (void)launch_dep(k_csr2dia<float>, dim3(grid_cap(m, 256, 8)), dim3(256), 0, s, rp, col, (const float*)val, m, P, bitmap, wprefix, (float*)dval);
  count_launch();
  return cudaGetLastError();
}

}  // namespace sfs
