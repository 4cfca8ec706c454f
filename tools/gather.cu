// Random-gather ceiling probe (B200): how many independent random 8-byte loads per second the SMs can
// pull from an L2-resident array (the x gathers of uniform-random SpMV), by in-flight depth and array size.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/gather_bin tools/gather.cu && ./tools/gather_bin
#include <cstdio>
#include <cuda_runtime.h>

__device__ __forceinline__ unsigned hash32(unsigned v) {
  v ^= v >> 16; v *= 0x7feb352du; v ^= v >> 15; v *= 0x846ca68bu; v ^= v >> 16;
  return v;
}

template <int D, typename T>
__global__ void __launch_bounds__(256) k_gather(const T* __restrict__ x, unsigned nmask, int iters, double* out) {
  const unsigned t = blockIdx.x * blockDim.x + threadIdx.x;
  double acc = 0;
  unsigned s = hash32(t * 2654435761u + 1);
  for (int it = 0; it < iters; it++) {
    T v[D];
#pragma unroll
    for (int d = 0; d < D; d++) {
      s = s * 1664525u + 1013904223u;
      v[d] = __ldg(x + ((s >> 3) & nmask));
    }
#pragma unroll
    for (int d = 0; d < D; d++) acc += (double)v[d];
  }
  if (acc == 123.456) out[0] = acc;
}

template <int D, typename T>
void run(const T* x, unsigned nmask, int ctas_per_sm, double* out) {
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  const int grid = 148 * ctas_per_sm, iters = 64;
  k_gather<D, T><<<grid, 256>>>(x, nmask, iters, out);
  cudaEventRecord(a);
  for (int r = 0; r < 5; r++) k_gather<D, T><<<grid, 256>>>(x, nmask, iters, out);
  cudaEventRecord(b);
  cudaEventSynchronize(b);
  float ms;
  cudaEventElapsedTime(&ms, a, b);
  const double g = 5.0 * grid * 256.0 * iters * D / (ms * 1e-3) / 1e9;
  printf("elem=%zuB array=%6.1f MB depth=%2d ctas/SM=%d : %6.1f G gathers/s (%.2f per SM-clk @1.965GHz)\n", sizeof(T),
         (nmask + 1.0) * sizeof(T) / 1e6, D, ctas_per_sm, g, g / 148 / 1.965);
}

int main() {
  double* out;
  cudaMalloc(&out, 8);
  double* x;
  cudaMalloc(&x, (size_t)1 << 30);
  cudaMemset(x, 0, (size_t)1 << 30);
  for (unsigned n : {1u << 17, 1u << 20, 1u << 23}) {
    const unsigned mask = n - 1;
    run<4, double>(x, mask, 4, out);
    run<8, double>(x, mask, 4, out);
    run<16, double>(x, mask, 4, out);
    run<8, double>(x, mask, 8, out);
    run<16, double>(x, mask, 8, out);
    run<8, float>((const float*)x, mask, 8, out);
  }
  printf("err: %s\n", cudaGetErrorString(cudaGetLastError()));
  return 0;
}
