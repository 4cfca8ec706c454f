// Random-gather probe by load flavour and array size (B200): is the ~1 random sector per SM clock of
// tools/gather.cu an L1 (t-stage / wavefront) limit or an L2 limit?  Arrays from 32 KB (L1-resident) to
// 64 MB (L2-resident); loads: ld.global.nc (__ldg, L1-allocating), ld.global.cg (L2 only), ld.global.ca,
// and shared memory (a CTA's own copy) for the L1-sized arrays.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/gather_flavors_bin tools/gather_flavors.cu
#include <cstdio>
#include <cuda_runtime.h>

template <int F>
__device__ __forceinline__ double ld(const double* p) {
  double v;
  if (F == 0) v = __ldg(p);
  else if (F == 1) asm volatile("ld.global.cg.f64 %0, [%1];" : "=d"(v) : "l"(p));
  else asm volatile("ld.global.ca.f64 %0, [%1];" : "=d"(v) : "l"(p));
  return v;
}

template <int F, int D>
__global__ void __launch_bounds__(256) k_gather(const double* __restrict__ x, unsigned nmask, int iters, double* out) {
  extern __shared__ double sx[];
  const unsigned t = blockIdx.x * blockDim.x + threadIdx.x;
  if (F == 3) {  // smem: the CTA copies the array first
    for (unsigned i = threadIdx.x; i <= nmask; i += blockDim.x) sx[i] = x[i];
    __syncthreads();
  }
  double acc = 0;
  unsigned s = t * 2654435761u + 1;
  for (int it = 0; it < iters; it++) {
    double v[D];
#pragma unroll
    for (int d = 0; d < D; d++) {
      s = s * 1664525u + 1013904223u;
      const unsigned i = (s >> 3) & nmask;
      v[d] = F == 3 ? sx[i] : ld<F>(x + i);
    }
#pragma unroll
    for (int d = 0; d < D; d++) acc += v[d];
  }
  if (acc == 123.456) out[0] = acc;
}

template <int F>
void run(const double* x, unsigned n, double* out) {
  constexpr int D = 16;
  const int ctas = 4, grid = 148 * ctas, iters = 64;
  const size_t smem = F == 3 ? n * sizeof(double) : 0;
  if (F == 3) cudaFuncSetAttribute(k_gather<F, D>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  k_gather<F, D><<<grid, 256, smem>>>(x, n - 1, iters, out);
  cudaEventRecord(a);
  for (int r = 0; r < 5; r++) k_gather<F, D><<<grid, 256, smem>>>(x, n - 1, iters, out);
  cudaEventRecord(b);
  cudaEventSynchronize(b);
  float ms;
  cudaEventElapsedTime(&ms, a, b);
  const char* names[] = {"ld.global.nc", "ld.global.cg", "ld.global.ca", "ld.shared"};
  const double g = 5.0 * grid * 256.0 * iters * D / (ms * 1e-3) / 1e9;
  printf("%-13s array=%8.3f MB : %7.1f G gathers/s (%.2f per SM-clk @1.965GHz)%s\n", names[F], n * 8.0 / 1e6, g,
         g / 148 / 1.965, cudaGetLastError() == cudaSuccess ? "" : " (launch error)");
}

int main() {
  double* out;
  cudaMalloc(&out, 8);
  double* x;
  cudaMalloc(&x, (size_t)64 << 20);
  cudaMemset(x, 0, (size_t)64 << 20);
  for (unsigned n : {1u << 12, 1u << 14, 1u << 17, 1u << 20, 1u << 23}) {
    run<0>(x, n, out);
    run<1>(x, n, out);
    run<2>(x, n, out);
    if (n * 8 <= 48 * 1024) run<3>(x, n, out);
  }
  return 0;
}
