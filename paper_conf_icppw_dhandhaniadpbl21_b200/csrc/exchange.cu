// exchange.cu — the send side of the row-partitioned SpMV's halo exchange.
//
// A rank that holds rows [r_k, r_{k+1}) of A and the same slice of x sends each neighbour only the x
// entries its row block references (its ghost columns), instead of every rank all-gathering all of x.
// The plan (which local entries go to which rank) is built once on the host; per SpMV this kernel packs
// the entries into one contiguous send buffer, ordered by destination, for the point-to-point sends.
#include "common.cuh"
#include "internal.h"

namespace sfs {
namespace {

template <typename T>
__global__ void k_gather(const T* __restrict__ src, const int* __restrict__ idx, long long n, T* __restrict__ dst) {
  for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x)
    dst[i] = __ldg(src + __ldg(idx + i));
}

}  // namespace

cudaError_t launch_gather(int dtype, const void* src, const int* idx, long long n, void* dst, cudaStream_t s) {
  if (n <= 0) return cudaSuccess;
  const long long g = ceil_div(n, 256) < (long long)kSMs * 8 ? ceil_div(n, 256) : (long long)kSMs * 8;
  if (dtype == SFS_F64) k_gather<double><<<(unsigned)g, 256, 0, s>>>((const double*)src, idx, n, (double*)dst);
  else k_gather<float><<<(unsigned)g, 256, 0, s>>>((const float*)src, idx, n, (float*)dst);
  count_launch();
  return cudaGetLastError();
}

}  // namespace sfs
