// Gather + stream probe (B200): the inner loop of a uniform-random SpMV (stream col/val, gather x[col]) with
// the streamed operands loaded (a) by LDG through L1TEX or (b) by TMA bulk copies into shared memory,
// to see whether the L1TEX miss path (~1 sector/clk/SM) is shared between the streams and the gathers.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/gather_stream_bin tools/gather_stream.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ int4 ldnc_i4(const int* p) {
  int4 v;
  asm volatile("ld.global.nc.L1::no_allocate.v4.s32 {%0,%1,%2,%3}, [%4];"
               : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p));
  return v;
}
__device__ __forceinline__ double2 ldnc_d2(const double* p) {
  double2 v;
  asm volatile("ld.global.nc.L1::no_allocate.v2.f64 {%0,%1}, [%2];" : "=d"(v.x), "=d"(v.y) : "l"(p));
  return v;
}

// (0) gather only: col from a hash, no streamed operand
__global__ void __launch_bounds__(256) k_gather_only(const double* __restrict__ x, unsigned nmask, long long N,
                                                     double* out) {
  double acc = 0;
  const long long T = (long long)gridDim.x * blockDim.x;
  for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i * 8 < N; i += T) {
    double v[8];
#pragma unroll
    for (int u = 0; u < 8; u++) {
      unsigned h = (unsigned)(i * 8 + u) * 2654435761u;
      h ^= h >> 15;
      v[u] = __ldg(x + (h & nmask));
    }
#pragma unroll
    for (int u = 0; u < 8; u++) acc += v[u];
  }
  if (acc == 1.2345) out[0] = acc;
}

// (1) LDG stream: a warp owns 256-entry chunks, lane reads 8 consecutive entries (2 x int4 col, 4 x double2 val)
__global__ void __launch_bounds__(256) k_ldg(const int* __restrict__ col, const double* __restrict__ val,
                                             const double* __restrict__ x, long long N, double* out) {
  double acc = 0;
  const long long T = (long long)gridDim.x * blockDim.x;
  for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i * 8 < N; i += T) {
    const int4 c0 = ldnc_i4(col + i * 8), c1 = ldnc_i4(col + i * 8 + 4);
    const double2 v0 = ldnc_d2(val + i * 8), v1 = ldnc_d2(val + i * 8 + 2), v2 = ldnc_d2(val + i * 8 + 4),
                  v3 = ldnc_d2(val + i * 8 + 6);
    const int c[8] = {c0.x, c0.y, c0.z, c0.w, c1.x, c1.y, c1.z, c1.w};
    const double v[8] = {v0.x, v0.y, v1.x, v1.y, v2.x, v2.y, v3.x, v3.y};
    double xv[8];
#pragma unroll
    for (int u = 0; u < 8; u++) xv[u] = __ldg(x + c[u]);
#pragma unroll
    for (int u = 0; u < 8; u++) acc += v[u] * xv[u];
  }
  if (acc == 1.2345) out[0] = acc;
}

// (2) TMA stream: CTA-wide chunks of 2048 entries (8 KB col + 16 KB val) moved by cp.async.bulk into a
// kStages-deep smem ring (mbarrier complete_tx), consumed by all 256 threads (entry t + 256u).
constexpr int kChunk = 2048;
constexpr int kStages = 4;
__device__ __forceinline__ unsigned smem_u32(const void* p) { return (unsigned)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t* b, unsigned n) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(b)), "r"(n));
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* b, unsigned bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(b)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, unsigned bytes, uint64_t* b) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
               ::"r"(smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(b)) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* b, unsigned parity) {
  asm volatile(
      "{\n .reg .pred p;\n W: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n @!p bra W;\n}\n"
      ::"r"(smem_u32(b)), "r"(parity) : "memory");
}

__global__ void __launch_bounds__(256) k_tma(const int* __restrict__ col, const double* __restrict__ val,
                                             const double* __restrict__ x, long long N, double* out) {
  extern __shared__ __align__(128) unsigned char smem[];
  int* s_col = (int*)smem;                                        // [kStages][kChunk]
  double* s_val = (double*)(smem + kStages * kChunk * 4);        // [kStages][kChunk]
  __shared__ uint64_t full[kStages];
  const long long nch = N / kChunk;
  if (threadIdx.x == 0) {
    for (int s = 0; s < kStages; s++) mbar_init(&full[s], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  auto issue = [&](long long ch, int s) {
    mbar_expect_tx(&full[s], kChunk * 12);
    bulk_g2s(s_col + s * kChunk, col + ch * kChunk, kChunk * 4, &full[s]);
    bulk_g2s(s_val + s * kChunk, val + ch * kChunk, kChunk * 8, &full[s]);
  };
  if (threadIdx.x == 0)
    for (int s = 0; s < kStages; s++) {
      const long long ch = blockIdx.x + (long long)s * gridDim.x;
      if (ch < nch) issue(ch, s);
    }
  double acc = 0;
  int it = 0;
  for (long long ch = blockIdx.x; ch < nch; ch += gridDim.x, it++) {
    const int s = it % kStages;
    mbar_wait(&full[s], (it / kStages) & 1);
    int c[8];
    double v[8], xv[8];
#pragma unroll
    for (int u = 0; u < 8; u++) {
      c[u] = s_col[s * kChunk + threadIdx.x + 256 * u];
      v[u] = s_val[s * kChunk + threadIdx.x + 256 * u];
    }
#pragma unroll
    for (int u = 0; u < 8; u++) xv[u] = __ldg(x + c[u]);
#pragma unroll
    for (int u = 0; u < 8; u++) acc += v[u] * xv[u];
    __syncthreads();  // everyone is done with stage s
    if (threadIdx.x == 0) {
      const long long nx = ch + (long long)kStages * gridDim.x;
      if (nx < nch) issue(nx, s);
    }
  }
  if (acc == 1.2345) out[0] = acc;
}

__global__ void k_init(int* col, double* val, long long N, unsigned nmask) {
  for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < N; i += (long long)gridDim.x * blockDim.x) {
    unsigned h = (unsigned)i * 2654435761u;
    h ^= h >> 13;
    h *= 0x5bd1e995u;
    h ^= h >> 15;
    col[i] = h & nmask;
    val[i] = 1.0;
  }
}

int main() {
  const long long N = 1LL << 25;  // 32M entries: 128 MB col + 256 MB val (> L2)
  int* col;
  double *val, *x, *out;
  cudaMalloc(&col, N * 4);
  cudaMalloc(&val, N * 8);
  cudaMalloc(&x, (1 << 23) * 8);
  cudaMalloc(&out, 8);
  cudaMemset(x, 0, (1 << 23) * 8);
  const int smem = kStages * kChunk * 12;
  cudaFuncSetAttribute(k_tma, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  for (unsigned n : {1u << 17, 1u << 20, 1u << 23}) {
    const unsigned nmask = n - 1;
    k_init<<<148 * 8, 256>>>(col, val, N, nmask);
    for (int mode = 0; mode < 4; mode++) {
      auto go = [&] {
        if (mode == 0) k_gather_only<<<148 * 8, 256>>>(x, nmask, N, out);
        if (mode == 1) k_ldg<<<148 * 8, 256>>>(col, val, x, N, out);
        if (mode == 2) k_tma<<<148 * 2, 256, smem>>>(col, val, x, N, out);
        if (mode == 3) k_tma<<<148 * 1, 256, smem>>>(col, val, x, N, out);
      };
      go();
      cudaEventRecord(a);
      for (int r = 0; r < 5; r++) go();
      cudaEventRecord(b);
      cudaEventSynchronize(b);
      float ms;
      cudaEventElapsedTime(&ms, a, b);
      const double t = ms / 5 * 1e-3;
      const char* nm[] = {"gather only", "LDG stream + gather", "TMA stream + gather (2 CTA/SM)",
                          "TMA stream + gather (1 CTA/SM)"};
      printf("x=%5.1f MB %-32s %7.1f us  %6.1f G entries/s  stream %5.0f GB/s\n", n * 8 / 1e6, nm[mode], t * 1e6,
             N / t / 1e9, mode ? N * 12 / t / 1e9 : 0.0);
    }
  }
  printf("err: %s\n", cudaGetErrorString(cudaGetLastError()));
  return 0;
}
