// common.cuh — device helpers shared by the libsfs kernels (sm_100a).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "shape.h"

namespace sfs {


// ---------------------------------------------------------------- cache-hinted loads
// A's arrays are streamed once per SpMV: no L1 allocation (they would only evict x).
__device__ __forceinline__ int ld_stream(const int* p) {
  int v;
  asm("ld.global.nc.L1::no_allocate.b32 %0, [%1];" : "=r"(v) : "l"(p));
  return v;
}
__device__ __forceinline__ float ld_stream(const float* p) {
  float v;
  asm("ld.global.nc.L1::no_allocate.f32 %0, [%1];" : "=f"(v) : "l"(p));
  return v;
}
__device__ __forceinline__ double ld_stream(const double* p) {
  double v;
  asm("ld.global.nc.L1::no_allocate.f64 %0, [%1];" : "=d"(v) : "l"(p));
  return v;
}
__device__ __forceinline__ int4 ld_stream4(const int* p) {
  int4 v;
  asm("ld.global.nc.L1::no_allocate.v4.s32 {%0,%1,%2,%3}, [%4];"
               : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p));
  return v;
}
__device__ __forceinline__ float4 ld_stream4(const float* p) {
  float4 v;
  asm("ld.global.nc.L1::no_allocate.v4.f32 {%0,%1,%2,%3}, [%4];"
               : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p));
  return v;
}
__device__ __forceinline__ double2 ld_stream2(const double* p) {
  double2 v;
  asm("ld.global.nc.L1::no_allocate.v2.f64 {%0,%1}, [%2];" : "=d"(v.x), "=d"(v.y) : "l"(p));
  return v;
}
// x is gathered: keep it in L1 / L2 (read-only path).
template <typename T>
__device__ __forceinline__ T ld_x(const T* p) { return __ldg(p); }

// ---------------------------------------------------------------- vectors of 4 values
template <typename T> struct Vec4;
template <> struct Vec4<float> {
  float v[4];
  __device__ __forceinline__ void load_stream(const float* p) {
    float4 a = ld_stream4(p);
    v[0] = a.x; v[1] = a.y; v[2] = a.z; v[3] = a.w;
  }
  __device__ __forceinline__ void load_x(const float* p) {  // 16 B aligned, cached
    float4 a = __ldg((const float4*)p);
    v[0] = a.x; v[1] = a.y; v[2] = a.z; v[3] = a.w;
  }
};
template <> struct Vec4<double> {
  double v[4];
  __device__ __forceinline__ void load_stream(const double* p) {
    double2 a = ld_stream2(p), b = ld_stream2(p + 2);
    v[0] = a.x; v[1] = a.y; v[2] = b.x; v[3] = b.y;
  }
  __device__ __forceinline__ void load_x(const double* p) {  // 16 B aligned, cached
    double2 a = __ldg((const double2*)p), b = __ldg((const double2*)p + 1);
    v[0] = a.x; v[1] = a.y; v[2] = b.x; v[3] = b.y;
  }
};

// ---------------------------------------------------------------- warp helpers
template <typename T>
__device__ __forceinline__ T warp_sum(T v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}

// ---------------------------------------------------------------- merge-path partition
// Merge of A = row ends (row_ptr[1..m]) with B = nnz indices 0..z-1.  At diagonal d returns the
// number of row ends consumed (x) and nnz consumed (y = d - x).  Row end r is consumed before
// nnz k iff row_ptr[r+1] <= k, i.e. nnz k belongs to the first row whose end exceeds k.
__device__ __forceinline__ void merge_path_search(long long d, const int* __restrict__ row_end, int m, int z,
                                                  int& x, int& y) {
  long long lo = d - z > 0 ? d - z : 0;
  long long hi = d < m ? d : m;
  while (lo < hi) {
    long long mid = (lo + hi) >> 1;
    if (row_end[mid] <= d - mid - 1) lo = mid + 1;
    else hi = mid;
  }
  x = (int)lo;
  y = (int)(d - lo);
}

// Inside a tile whose row ends are staged as s_rp[i] = row_ptr[r0 + i] (i = 0..nrow+1) and whose
// nnz range is [k0, k1): coordinates (row, nnz) after `ld` items of the tile.
__device__ __forceinline__ void merge_local_search(const int* s_rp, int nrow, int k0, int k1, int ld, int r0,
                                                   int& r, int& k) {
  int lo = ld - (k1 - k0) > 0 ? ld - (k1 - k0) : 0, hi = ld < nrow ? ld : nrow;
  while (lo < hi) {
    int mid = (lo + hi) >> 1;
    if (s_rp[mid + 1] <= k0 + (ld - mid) - 1) lo = mid + 1;
    else hi = mid;
  }
  r = r0 + lo;
  k = k0 + (ld - lo);
}


}  // namespace sfs
