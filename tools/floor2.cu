// Launch-floor probe, part 2 (B200): host enqueue cost of the runtime's cudaLaunchKernelEx against the
// driver's cuLaunchKernelEx on a pre-resolved CUfunction, and the DEVICE floor of back-to-back PDL
// launches (inside a graph, so the host is not the limit).
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o floor2 tools/floor2.cu -lcuda && ./floor2
#include <chrono>
#include <cstdio>
#include <cuda.h>
#include <cuda_runtime.h>

__global__ void k_pdl_empty(int* p) {
  asm volatile("griddepcontrol.wait;" ::: "memory");
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  if (p && threadIdx.x == 1023) p[0] = 1;
}
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

int main() {
  cudaFree(0);
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
  const int N = 4000;
  auto run = [&](const char* name, auto body) {
    for (int i = 0; i < 400; i++) body();
    cudaStreamSynchronize(s);
    cudaEventRecord(a, s);
    auto h0 = std::chrono::steady_clock::now();
    for (int i = 0; i < N; i++) body();
    auto h1 = std::chrono::steady_clock::now();
    cudaEventRecord(b, s);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    printf("%-52s %7.3f us/launch (host enqueue %.3f us/launch)\n", name, 1e3 * ms / N,
           1e6 * std::chrono::duration<double>(h1 - h0).count() / N);
  };
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = 1;
  cudaLaunchConfig_t cfg = {};
  cfg.blockDim = dim3(256);
  cfg.stream = s;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  CUfunction f_empty, f_chain;
  cudaGetFuncBySymbol(&f_empty, (const void*)k_pdl_empty);
  cudaGetFuncBySymbol(&f_chain, (const void*)k_pdl_chain);
  CUlaunchAttribute dat[1];
  dat[0].id = CU_LAUNCH_ATTRIBUTE_PROGRAMMATIC_STREAM_SERIALIZATION;
  dat[0].value.programmaticStreamSerializationAllowed = 1;
  CUlaunchConfig dcfg = {};
  dcfg.blockDimX = 256;
  dcfg.blockDimY = dcfg.blockDimZ = 1;
  dcfg.gridDimY = dcfg.gridDimZ = 1;
  dcfg.hStream = (CUstream)s;
  dcfg.attrs = dat;
  dcfg.numAttrs = 1;
  int* np = nullptr;
  for (int grid : {1, 16, 148, 296}) {
    char nm[96];
    cfg.gridDim = dim3(grid);
    dcfg.gridDimX = grid;
    snprintf(nm, sizeof nm, "empty PDL runtime grid=%d", grid);
    run(nm, [&] { cudaLaunchKernelEx(&cfg, k_pdl_empty, np); });
    snprintf(nm, sizeof nm, "empty PDL driver grid=%d", grid);
    run(nm, [&] {
      void* args[] = {&np};
      cuLaunchKernelEx(&dcfg, f_empty, args, nullptr);
    });
  }
  cfg.gridDim = dim3(16);
  dcfg.gridDimX = 16;
  run("chain PDL runtime grid=16", [&] { cudaLaunchKernelEx(&cfg, k_pdl_chain, (const int*)rp, (const int*)col, (const double*)x, y, m); });
  run("chain PDL driver grid=16", [&] {
    void* args[] = {&rp, &col, &x, &y, (void*)&m};
    cuLaunchKernelEx(&dcfg, f_chain, args, nullptr);
  });
  // device floor: graphs of 100 PDL launches (host not the limit)
  cudaStream_t cap;
  cudaStreamCreateWithFlags(&cap, cudaStreamNonBlocking);
  for (int kind = 0; kind < 2; kind++)
    for (int grid : {1, 16, 148}) {
      cudaGraph_t g;
      cudaGraphExec_t ge;
      cudaLaunchConfig_t c2 = cfg;
      c2.stream = cap;
      c2.gridDim = dim3(grid);
      cudaStreamBeginCapture(cap, cudaStreamCaptureModeThreadLocal);
      for (int i = 0; i < 100; i++) {
        if (kind == 0) cudaLaunchKernelEx(&c2, k_pdl_empty, np);
        else cudaLaunchKernelEx(&c2, k_pdl_chain, (const int*)rp, (const int*)col, (const double*)x, y, m);
      }
      cudaStreamEndCapture(cap, &g);
      cudaGraphInstantiate(&ge, g, 0);
      for (int i = 0; i < 5; i++) cudaGraphLaunch(ge, s);
      cudaStreamSynchronize(s);
      cudaEventRecord(a, s);
      for (int i = 0; i < 40; i++) cudaGraphLaunch(ge, s);
      cudaEventRecord(b, s);
      cudaEventSynchronize(b);
      float ms;
      cudaEventElapsedTime(&ms, a, b);
      printf("graph of 100 %s PDL launches grid=%-4d              %7.3f us/launch\n", kind ? "chain" : "empty", grid,
             1e3 * ms / 4000);
    }
  printf("err: %s\n", cudaGetErrorString(cudaGetLastError()));
  return 0;
}
