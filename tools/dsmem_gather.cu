// DSMEM random-gather probe (B200): random 8-byte loads from the shared memory of the CTAs of a thread-block
// cluster (ld.shared::cluster after mapa), against the ~290 G/s L2 random-sector ceiling of tools/gather.cu.
// Question: can a cluster hold x (cluster_size x ~200 KB) and serve the x gathers of a uniform-random SpMV
// faster than L2?
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/dsmem_gather_bin tools/dsmem_gather.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ unsigned cluster_rank() {
  unsigned r;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
  return r;
}
__device__ __forceinline__ void cluster_sync() {
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
__device__ __forceinline__ double ld_dsmem(unsigned local_addr, unsigned rank) {
  unsigned ra;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(ra) : "r"(local_addr), "r"(rank));
  double v;
  asm volatile("ld.shared::cluster.f64 %0, [%1];" : "=d"(v) : "r"(ra));
  return v;
}

template <int D>
__global__ void k_dsmem(int words, int csize, int iters, double* out) {
  extern __shared__ double sm[];
  for (int i = threadIdx.x; i < words; i += blockDim.x) sm[i] = 1.0 + i;
  cluster_sync();
  const unsigned base = (unsigned)__cvta_generic_to_shared(sm);
  unsigned s = (blockIdx.x * blockDim.x + threadIdx.x) * 2654435761u + 12345u;
  double acc = 0;
  for (int it = 0; it < iters; it++) {
    double v[D];
#pragma unroll
    for (int d = 0; d < D; d++) {
      s = s * 1664525u + 1013904223u;
      const unsigned r = (s >> 24) % (unsigned)csize;
      const unsigned o = (s >> 3) % (unsigned)words;
      v[d] = ld_dsmem(base + 8 * o, r);
    }
#pragma unroll
    for (int d = 0; d < D; d++) acc += v[d];
  }
  cluster_sync();  // keep every CTA's smem alive until the cluster is done
  if (acc == 1.2345) out[0] = acc;
}

template <int D>
void run(int csize, int threads, int smem_kb) {
  double* out;
  cudaMalloc(&out, 8);
  const int smem = smem_kb * 1024, words = smem / 8;
  cudaFuncSetAttribute(k_dsmem<D>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  cudaFuncSetAttribute(k_dsmem<D>, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
  int maxc = 0;
  const int grid = 148 / csize * csize;
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(threads);
  cfg.dynamicSmemBytes = smem;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeClusterDimension;
  at[0].val.clusterDim.x = csize;
  at[0].val.clusterDim.y = 1;
  at[0].val.clusterDim.z = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  cudaOccupancyMaxActiveClusters(&maxc, k_dsmem<D>, &cfg);
  const int iters = 64;
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  cudaLaunchKernelEx(&cfg, k_dsmem<D>, words, csize, iters, out);
  cudaEventRecord(a);
  for (int r = 0; r < 5; r++) cudaLaunchKernelEx(&cfg, k_dsmem<D>, words, csize, iters, out);
  cudaEventRecord(b);
  cudaError_t e = cudaEventSynchronize(b);
  float ms = 0;
  cudaEventElapsedTime(&ms, a, b);
  const double g = 5.0 * grid * threads * (double)iters * D / (ms * 1e-3) / 1e9;
  printf("cluster=%2d ctas=%3d (max active clusters %3d) threads=%4d smem=%3d KB depth=%2d : %7.1f G gathers/s  "
         "(%.2f per SM-clk)  %s\n", csize, grid, maxc, threads, smem_kb, D, g, g / grid / 1.965,
         cudaGetErrorString(e));
  cudaFree(out);
}

int main() {
  for (int cs : {1, 2, 4, 8, 16}) {
    run<8>(cs, 512, 192);
    run<16>(cs, 1024, 192);
  }
  printf("err: %s\n", cudaGetErrorString(cudaGetLastError()));
  return 0;
}
