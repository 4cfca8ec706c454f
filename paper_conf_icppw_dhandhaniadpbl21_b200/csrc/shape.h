// shape.h — host/device shape helpers shared by the kernels and the host API.
#pragma once
#ifdef __CUDACC__
#define SFS_HD __host__ __device__ __forceinline__
#else
#define SFS_HD inline
#endif

namespace sfs {
constexpr int kSMs = 148;                      // B200: 2 dies x 74 SMs
constexpr int kWarpsPerSM = 64;                // 2048 resident threads / SM
constexpr int kCsrWarps = kSMs * kWarpsPerSM;  // grid of the CSR vector kernel (feature csr_max, Q4)
SFS_HD long long ceil_div(long long a, long long b) { return (a + b - 1) / b; }
SFS_HD long long pitch_of(long long m) { return ceil_div(m, 32) * 32; }  // ELL / DIA slab pitch
}  // namespace sfs
