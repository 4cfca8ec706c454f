// common.cuh — device helpers shared by the libsfs kernels (sm_100a).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdlib.h>

#include "shape.h"

namespace sfs {

// ---------------------------------------------------------------- programmatic dependent launch
// The feature, conversion and preparation chains run as PDL chains like the SpMV kernels: every kernel
// waits (griddepcontrol.wait: a no-op without a programmatic predecessor) before touching memory and
// releases its successor when its work is done; launch_dep sets the launch attribute (SFS_PDL=0: off).
__device__ __forceinline__ void dep_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__device__ __forceinline__ void dep_trigger() { asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }
inline bool dep_enabled() {
  static const bool v = [] {
    const char* e = getenv("SFS_PDL");
    return !(e && e[0] == '0');
  }();
  return v;
}
template <typename... Params, typename... Args>
cudaError_t launch_dep(void (*kern)(Params...), dim3 grid, dim3 block, size_t smem, cudaStream_t s, Args... args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = at;
  cfg.numAttrs = dep_enabled() ? 1 : 0;
  return cudaLaunchKernelEx(&cfg, kern, static_cast<Params>(args)...);
}


// ---------------------------------------------------------------- cache-hinted loads
// A's arrays are streamed once per SpMV: no L1 allocation (they would only evict x).  With
// SFS_STREAM_EVICT_FIRST the streams also carry an L2 evict-first cache policy (createpolicy +
// .L2::cache_hint), so that a matrix larger than L2 does not push x out of it.
#ifdef SFS_STREAM_EVICT_FIRST
#define SFS_LDS(TY, ...)                                                                              \
  asm("{\n .reg .b64 pol;\n createpolicy.fractional.L2::evict_first.b64 pol, 1.0;\n"                    \
      " ld.global.nc.L1::no_allocate.L2::cache_hint" TY ";\n}" : __VA_ARGS__)
#else
#define SFS_LDS(TY, ...) asm("ld.global.nc.L1::no_allocate" TY ";" : __VA_ARGS__)
#endif
__device__ __forceinline__ int ld_stream(const int* p) {
  int v;
#ifdef SFS_STREAM_EVICT_FIRST
  SFS_LDS(".b32 %0, [%1], pol", "=r"(v) : "l"(p));
#else
  SFS_LDS(".b32 %0, [%1]", "=r"(v) : "l"(p));
#endif
  return v;
}
__device__ __forceinline__ float ld_stream(const float* p) {
  float v;
#ifdef SFS_STREAM_EVICT_FIRST
  SFS_LDS(".f32 %0, [%1], pol", "=f"(v) : "l"(p));
#else
  SFS_LDS(".f32 %0, [%1]", "=f"(v) : "l"(p));
#endif
  return v;
}
__device__ __forceinline__ double ld_stream(const double* p) {
  double v;
#ifdef SFS_STREAM_EVICT_FIRST
  SFS_LDS(".f64 %0, [%1], pol", "=d"(v) : "l"(p));
#else
  SFS_LDS(".f64 %0, [%1]", "=d"(v) : "l"(p));
#endif
  return v;
}
__device__ __forceinline__ int4 ld_stream4(const int* p) {
  int4 v;
#ifdef SFS_STREAM_EVICT_FIRST
  SFS_LDS(".v4.s32 {%0,%1,%2,%3}, [%4], pol", "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p));
#else
  SFS_LDS(".v4.s32 {%0,%1,%2,%3}, [%4]", "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p));
#endif
  return v;
}
__device__ __forceinline__ float4 ld_stream4(const float* p) {
  float4 v;
#ifdef SFS_STREAM_EVICT_FIRST
  SFS_LDS(".v4.f32 {%0,%1,%2,%3}, [%4], pol", "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p));
#else
  SFS_LDS(".v4.f32 {%0,%1,%2,%3}, [%4]", "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p));
#endif
  return v;
}
__device__ __forceinline__ double2 ld_stream2(const double* p) {
  double2 v;
#ifdef SFS_STREAM_EVICT_FIRST
  SFS_LDS(".v2.f64 {%0,%1}, [%2], pol", "=d"(v.x), "=d"(v.y) : "l"(p));
#else
  SFS_LDS(".v2.f64 {%0,%1}, [%2]", "=d"(v.x), "=d"(v.y) : "l"(p));
#endif
  return v;
}
// 256-bit streaming loads (sm_100: LDG.E.NA.ENL2.256), 32-byte aligned addresses.
__device__ __forceinline__ void ld_stream8(const int* p, int (&v)[8]) {
  asm("ld.global.nc.L1::no_allocate.v8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
      : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7])
      : "l"(p));
}
__device__ __forceinline__ void ld_stream8(const float* p, float (&v)[8]) {
  asm("ld.global.nc.L1::no_allocate.v8.f32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
      : "=f"(v[0]), "=f"(v[1]), "=f"(v[2]), "=f"(v[3]), "=f"(v[4]), "=f"(v[5]), "=f"(v[6]), "=f"(v[7])
      : "l"(p));
}
__device__ __forceinline__ void ld_stream4d(const double* p, double* v) {
  asm("ld.global.nc.L1::no_allocate.v4.f64 {%0,%1,%2,%3}, [%4];"
      : "=d"(v[0]), "=d"(v[1]), "=d"(v[2]), "=d"(v[3])
      : "l"(p));
}
__device__ __forceinline__ void ld_stream8(const double* p, double (&v)[8]) {
  ld_stream4d(p, v);
  ld_stream4d(p + 4, v + 4);
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
  __device__ __forceinline__ void load_stream(const double* p) { ld_stream4d(p, v); }  // one 256-bit load
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

// The same search by a whole warp (all 32 lanes call it with the same d): 32 probes per step, so the
// dependent global loads drop from log2(m) to ~log32(m) rounds (the tile setups of the feature and
// conversion kernels are latency chains on small matrices).
__device__ __forceinline__ void merge_path_search_warp(long long d, const int* __restrict__ row_end, int m, int z,
                                                       int& x, int& y) {
  const int lane = threadIdx.x & 31;
  long long lo = d - z > 0 ? d - z : 0;
  long long hi = d < m ? d : m;
  // invariant: the answer (first mid with row_end[mid] > d - mid - 1, or hi) lies in [lo, hi]
  while (lo < hi) {
    const long long step = (hi - lo + 31) / 32;
    const long long probe = lo + (long long)(lane + 1) * step - 1;
    const bool right = probe < hi && row_end[probe] <= d - probe - 1;  // the answer lies past the probe
    const int cnt = __popc(__ballot_sync(0xffffffffu, right));
    const long long nlo = lo + (long long)cnt * step;
    const long long nhi = cnt < 32 ? lo + (long long)(cnt + 1) * step - 1 : hi;
    lo = nlo;
    hi = nhi < hi ? nhi : hi;
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
