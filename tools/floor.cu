// Launch-floor probe (B200): per-launch device time of back-to-back dependent launches on one stream.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o floor tools/floor.cu && ./floor
#include <chrono>
#include <cstdio>
#include <cuda_runtime.h>

__global__ void k_empty(int* p) {
  if (p && threadIdx.x == 1023) p[0] = 1;
}
__global__ void k_pdl_empty(int* p) {
  asm volatile("griddepcontrol.wait;" ::: "memory");
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  if (p && threadIdx.x == 1023) p[0] = 1;
}
// three dependent global round trips (row_ptr -> col -> x) and a store, like a tiny SpMV
__global__ void k_pdl_chain(const int* rp, const int* col, const double* x, double* y, int m) {
  asm volatile("griddepcontrol.wait;" ::: "memory");
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  int r = blockIdx.x * blockDim.x + threadIdx.x;
  if (r < m) {
    int b = rp[r], e = rp[r + 1];
    double s = 0;
    for (int k = b; k < e; k++) s += x[col[k]];
    y[r] = s;
  }
}
__global__ void k_chain(const int* rp, const int* col, const double* x, double* y, int m) {
  int r = blockIdx.x * blockDim.x + threadIdx.x;
  if (r < m) {
    int b = rp[r], e = rp[r + 1];
    double s = 0;
    for (int k = b; k < e; k++) s += x[col[k]];
    y[r] = s;
  }
}

template <typename K, typename... A>
void launch(K k, int grid, int block, bool pdl, cudaStream_t s, A... a) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(block);
  cfg.stream = s;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = at;
  cfg.numAttrs = pdl ? 1 : 0;
  cudaLaunchKernelEx(&cfg, k, a...);
}

int main() {
  cudaStream_t s;
  cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
  const int m = 4096;
  int *rp, *col;
  double *x, *y;
  cudaMalloc(&rp, (m + 1) * 4);
  cudaMalloc(&col, m * 5 * 4);
  cudaMalloc(&x, m * 8);
  cudaMalloc(&y, m * 8);
  int* h = new int[m * 5 + 1];
  for (int i = 0; i <= m; i++) h[i] = 5 * i;
  cudaMemcpy(rp, h, (m + 1) * 4, cudaMemcpyHostToDevice);
  for (int i = 0; i < m * 5; i++) h[i] = (i * 7) % m;
  cudaMemcpy(col, h, m * 5 * 4, cudaMemcpyHostToDevice);
  cudaMemset(x, 0, m * 8);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  const int N = 2000;
  auto run = [&](const char* name, auto body) {
    for (int i = 0; i < 200; i++) body();
    cudaEventRecord(a, s);
    auto h0 = std::chrono::steady_clock::now();
    for (int i = 0; i < N; i++) body();
    auto h1 = std::chrono::steady_clock::now();
    cudaEventRecord(b, s);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    printf("%-44s %7.3f us/launch (host enqueue %.3f us/launch)\n", name, 1e3 * ms / N,
           1e6 * std::chrono::duration<double>(h1 - h0).count() / N);
  };
  for (int grid : {1, 16, 148, 592, 1184}) {
    char nm[96];
    snprintf(nm, sizeof nm, "empty plain grid=%d x256", grid);
    run(nm, [&] { launch(k_empty, grid, 256, false, s, (int*)nullptr); });
    snprintf(nm, sizeof nm, "empty PDL(wait+trigger) grid=%d x256", grid);
    run(nm, [&] { launch(k_pdl_empty, grid, 256, true, s, (int*)nullptr); });
  }
  run("chain plain m=4096 grid=16x256", [&] { launch(k_chain, 16, 256, false, s, rp, col, x, y, m); });
  run("chain PDL m=4096 grid=16x256", [&] { launch(k_pdl_chain, 16, 256, true, s, rp, col, x, y, m); });
  run("chain PDL m=4096 grid=4x1024", [&] { launch(k_pdl_chain, 4, 1024, true, s, rp, col, x, y, m); });
  // graph of 100 PDL launches
  cudaStream_t cap;
  cudaStreamCreateWithFlags(&cap, cudaStreamNonBlocking);
  for (int pdl = 0; pdl < 2; pdl++) {
    cudaGraph_t g;
    cudaGraphExec_t ge;
    cudaStreamBeginCapture(cap, cudaStreamCaptureModeThreadLocal);
    for (int i = 0; i < 100; i++) launch(pdl ? k_pdl_chain : k_chain, 16, 256, pdl, cap, rp, col, x, y, m);
    cudaStreamEndCapture(cap, &g);
    cudaGraphInstantiate(&ge, g, 0);
    for (int i = 0; i < 5; i++) cudaGraphLaunch(ge, s);
    cudaEventRecord(a, s);
    for (int i = 0; i < 20; i++) cudaGraphLaunch(ge, s);
    cudaEventRecord(b, s);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    printf("graph of 100 chain launches, pdl=%d            %7.3f us/launch\n", pdl, 1e3 * ms / 2000);
  }
  printf("err: %s\n", cudaGetErrorString(cudaGetLastError()));
  return 0;
}
