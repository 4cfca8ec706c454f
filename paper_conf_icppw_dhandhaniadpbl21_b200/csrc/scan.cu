// scan.cu — device-wide exclusive scans used by the conversions:
//   * HYB: ovf[r] = sum_{r' < r} max(0, len_r' - K)   (placement of the COO part, §2.1)
//   * DIA: wprefix[w] = sum_{w' < w} popc(bitmap[w'])  (rank of a diagonal offset)
// Three phases (tile reduce -> scan of tile sums -> tile scan + offset); out has n+1 entries.
#include "common.cuh"
#include "internal.h"

namespace sfs {
namespace {

constexpr int kThreads = 256;
constexpr int kIPT = 8;
constexpr int kTile = kThreads * kIPT;

struct OverflowOp {
  const int* rp;
  int K;
  __device__ __forceinline__ int operator()(long long i) const {
    int len = rp[i + 1] - rp[i];
    return len > K ? len - K : 0;
  }
};
struct NonEmptyOp {
  const int* rp;
  __device__ __forceinline__ int operator()(long long i) const { return rp[i + 1] > rp[i] ? 1 : 0; }
};
struct PopcOp {
  const unsigned* w;
  __device__ __forceinline__ int operator()(long long i) const { return __popc(w[i]); }
};

__device__ __forceinline__ int block_exclusive(int v, int* s_warp, int& total) {
  const int l = threadIdx.x & 31, w = threadIdx.x >> 5;
  int incl = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    int u = __shfl_up_sync(0xffffffffu, incl, o);
    if (l >= o) incl += u;
  }
  if (l == 31) s_warp[w] = incl;
  __syncthreads();
  if (w == 0) {
    int t = l < (int)(blockDim.x >> 5) ? s_warp[l] : 0;
    int ti = t;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      int u = __shfl_up_sync(0xffffffffu, ti, o);
      if (l >= o) ti += u;
    }
    s_warp[l] = ti - t;  // exclusive warp offsets
    if (l == 31) s_warp[32] = ti;
  }
  __syncthreads();
  total = s_warp[32];
  int r = s_warp[w] + incl - v;
  __syncthreads();
  return r;
}

template <typename Op>
__global__ void __launch_bounds__(kThreads) k_tile_reduce(Op op, long long n, int* __restrict__ partial) {
  dep_wait();
  __shared__ int s_warp[33];
  const long long base = (long long)blockIdx.x * kTile + (long long)threadIdx.x * kIPT;
  int s = 0;
#pragma unroll
  for (int i = 0; i < kIPT; i++)
    if (base + i < n) s += op(base + i);
  int total;
  block_exclusive(s, s_warp, total);
  if (threadIdx.x == 0) partial[blockIdx.x] = total;
  dep_trigger();
}

// single block: exclusive scan of nb tile sums in place; total -> *total_out
__global__ void __launch_bounds__(1024) k_scan_partials(int* __restrict__ partial, long long nb, int* total_out) {
  dep_wait();
  __shared__ int s_warp[33];
  int carry = 0;
  for (long long base = 0; base < nb; base += blockDim.x) {
    long long i = base + threadIdx.x;
    int v = i < nb ? partial[i] : 0;
    int total;
    int ex = block_exclusive(v, s_warp, total);
    if (i < nb) partial[i] = carry + ex;
    carry += total;
  }
  if (threadIdx.x == 0) *total_out = carry;
  dep_trigger();
}

template <typename Op>
__global__ void __launch_bounds__(kThreads) k_tile_scan(Op op, long long n, const int* __restrict__ partial,
                                                        int* __restrict__ out) {
  dep_wait();
  __shared__ int s_warp[33];
  const long long base = (long long)blockIdx.x * kTile + (long long)threadIdx.x * kIPT;
  int v[kIPT];
  int s = 0;
#pragma unroll
  for (int i = 0; i < kIPT; i++) {
    v[i] = base + i < n ? op(base + i) : 0;
    s += v[i];
  }
  int total;
  int ex = block_exclusive(s, s_warp, total) + partial[blockIdx.x];
#pragma unroll
  for (int i = 0; i < kIPT; i++) {
    if (base + i < n) out[base + i] = ex;
    ex += v[i];
  }
  dep_trigger();
}

template <typename Op>
cudaError_t run_scan(Op op, long long n, int* out, void* work, cudaStream_t s) {
  long long nb = ceil_div(n, kTile);
  int* partial = (int*)work;
  if (nb == 0) return cudaMemsetAsync(out, 0, sizeof(int), s);
  (void)launch_dep(k_tile_reduce<Op>, dim3((unsigned)nb), dim3(kThreads), 0, s, op, n, partial);
  (void)launch_dep(k_scan_partials, dim3(1), dim3(1024), 0, s, partial, nb, out + n);
  (void)launch_dep(k_tile_scan<Op>, dim3((unsigned)nb), dim3(kThreads), 0, s, op, n, partial, out);
  count_launch(3);
  return cudaGetLastError();
}

}  // namespace

size_t scan_work_bytes(long long n) { return sizeof(int) * (size_t)(ceil_div(n, kTile) + 1); }

cudaError_t launch_overflow_scan(const int* rp, long long m, int K, int* out, void* work, cudaStream_t s) {
  return run_scan(OverflowOp{rp, K}, m, out, work, s);
}

cudaError_t launch_nonempty_scan(const int* rp, long long m, int* out, void* work, cudaStream_t s) {
  return run_scan(NonEmptyOp{rp}, m, out, work, s);
}

cudaError_t launch_popc_scan(const unsigned* words, long long nw, int* out, void* work, cudaStream_t s) {
  return run_scan(PopcOp{words}, nw, out, work, s);
}

}  // namespace sfs
