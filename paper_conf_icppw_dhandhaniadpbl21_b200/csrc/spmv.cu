// spmv.cu — per-format y = A·x (§1; formats L73 §2.1; step (iii) of L331 §5.4).
//
// SpMV is HBM-bound (0.10–0.46 flop/B): every kernel streams the format's arrays once with
// L1-bypassing loads (ld.global.nc.L1::no_allocate) and gathers x through L1/L2 (__ldg).  No tensor
// cores: the path is not a dense contraction.  Sums run in fp64 for both value types; fp64 values form
// fp64 products, fp32 values form each product (or a chain of <= 8 products of one row) in fp32 and
// widen it once (mulp below), so fp32 rows of any length stay far inside the 1e-5 per-row tolerance;
// y is rounded once to its dtype.
//
// Two regimes shape every launch: matrices far larger than the GPU's in-flight capacity are
// bandwidth-bound (one wave, each thread streaming a long slice); L2-resident / mid-size matrices
// are latency-bound, so the work of a row group is split S ways (ELL slots, DIA diagonals, CSR
// windows) and the partial sums are combined in shared memory, keeping each thread to one or two
// dependent memory round trips.  Back-to-back SpMVs (the race's 100 reps) use programmatic
// dependent launch: each kernel waits (griddepcontrol.wait) before touching memory, and releases
// its successor (griddepcontrol.launch_dependents) when its work is issued, hiding launch latency
// without overlapping two SpMVs' memory traffic.
//   CSR vector : TPV lanes per row (TPV from floor(z/m)), grid of 148*64 warps (the csr_max
//                feature, Q4), shuffle reduction.  Kept as the CUSP-mapping variant.
//   CSR stream : warp-groups of 32 consecutive rows; windows of their contiguous nnz streamed with
//                coalesced loads, products staged in smem, lane j sums row j.  S warps per group.
//   CSR merge  : merge-path tiles over (row ends + nnz), products staged in smem, block-wide
//                segmented scan of thread carries, one carry per tile added by a fix-up kernel.
//   COO        : each warp owns a contiguous range of 256-item chunks (8 items per lane, 128-bit
//                loads), warp segmented reduction by row; rows are stored directly except the
//                range's first row and its final carry (atomicAdd).
//   ELL / HYB  : 4 rows per thread, column-major slab read with 128-bit loads (coalesced per slot),
//                S slot-parts per row group; HYB = ELL part (writes y) then COO part (accumulates).
//   DIA        : 4 (fp64) / 8 (fp32) rows per thread 256 apart (coalesced slab and x), S diagonal
//                parts per row block.
#include <stdio.h>
#include <stdlib.h>

#include <algorithm>
#include <mutex>
#include <type_traits>

#include "common.cuh"
#include "internal.h"

namespace sfs {
namespace {

typedef double acc_t;

// Products.  fp64 values: fp64 products.  fp32 values: the product is formed in fp32 (one rounding,
// relative error <= 2^-24) and widened once, and the sums run in fp64 -- per row the error stays below
// (2^-24 + K 2^-53) |A||x|, far inside the 1e-5 fp32 tolerance for any row length K, at one conversion
// per entry instead of two.  The row-owning fp32 kernels (DIA, ELL) go further: a batch of <= 8
// entries of a row is chained in fp32 FMAs and widened once (error <= 8 * 2^-24 |A||x| per batch).
// -DSFS_FP64_PRODUCTS restores fp64 products everywhere (A/B).
#ifdef SFS_FP64_PRODUCTS
constexpr bool kFp32Arith = false;
#else
constexpr bool kFp32Arith = true;
#endif
__device__ __forceinline__ acc_t mulp(double a, double b) { return a * b; }
__device__ __forceinline__ acc_t mulp(float a, float b) {
  if constexpr (kFp32Arith) return (acc_t)__fmul_rn(a, b);
  return (acc_t)a * (acc_t)b;
}

constexpr long long kResidentThreads = (long long)kSMs * 2048;

__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__device__ __forceinline__ void pdl_trigger() { asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }
// SFS_PDL_EARLY: release the successor right after our own wait (it is scheduled once all our CTAs
// are resident, then blocks in griddepcontrol.wait until this grid has completed and flushed).
#ifdef SFS_PDL_EARLY
__device__ __forceinline__ void pdl_early() { pdl_trigger(); }
#else
__device__ __forceinline__ void pdl_early() {}
#endif

// Environment A/B switches are read once per process (thread-safe function-local statics; SFS_PDL: common.cuh).

// cudaLaunchKernelEx with the programmatic-stream-serialization attribute (PDL; common.cuh launch_dep),
// counted as one of the library's launches.
template <typename... Params, typename... Args>
cudaError_t launch_k_smem(void (*kern)(Params...), dim3 grid, dim3 block, size_t smem, cudaStream_t s, Args... args) {
  count_launch();
  return launch_dep(kern, grid, block, smem, s, args...);
}
template <typename... Params, typename... Args>
cudaError_t launch_k(void (*kern)(Params...), dim3 grid, dim3 block, cudaStream_t s, Args... args) {
  return launch_k_smem(kern, grid, block, 0, s, args...);
}

int grid_cap(long long items, int threads, int per_sm) {
  long long g = ceil_div(items, threads), cap = (long long)kSMs * per_sm;
  return (int)(g > cap ? cap : (g < 1 ? 1 : g));
}

[[maybe_unused]] int pow2_ceil(long long v) {
  int p = 1;
  while (p < v && p < (1 << 20)) p <<= 1;
  return p;
}

// Split factor for a latency-bound launch: enough parts that each thread does <= `per_thread` units
// of `units` (slots, diagonals, windows), but stop once `items * S` threads would exceed `fill` x the
// GPU's resident threads (bandwidth-bound sizes keep S = 1).
int split_factor(long long items, long long units, long long per_thread, int smax, long long fill = 2) {
  int S = 1;
  while (S < smax && ceil_div(units, S) > per_thread && items * S * 2 <= fill * kResidentThreads) S <<= 1;
  return S;
}

template <typename T>
__global__ void k_zero(T* __restrict__ y, long long m) {
  pdl_wait();
  pdl_trigger();  // successor (COO) overlaps its loads with this kernel and waits before storing
  for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < m; i += (long long)gridDim.x * blockDim.x)
    y[i] = T(0);
}

// ======================================================================== fused halo push
// sfs_spmv_push (include/sfs.h): the row-owning kernels (DIA, ELL, CSR stream) store each y[r] that a
// neighbour needs as a ghost also into the neighbour's x_ext (peer memory), in the same instruction
// stream that computes it.  PushParam<false> is empty, so the plain kernels are unchanged.
template <bool PUSH> struct PushParam {};
template <> struct PushParam<true> {
  int nseg;
  long long b[SFS_MAX_PUSH], e[SFS_MAX_PUSH];
  void* dst[SFS_MAX_PUSH];
  int nwait;
  const unsigned* wait[SFS_MAX_PEERS];
  unsigned wait_value;
  int nsig;
  unsigned* sig[SFS_MAX_PEERS];
  unsigned sig_value;
  unsigned* counter;
};

PushParam<true> push_param(const sfs_push_t& h) {
  PushParam<true> p;
  p.nseg = h.nseg;
  for (int i = 0; i < SFS_MAX_PUSH; i++) {
    p.b[i] = h.seg_begin[i];
    p.e[i] = h.seg_end[i];
    p.dst[i] = h.seg_dst[i];
  }
  p.nwait = h.nwait;
  p.nsig = h.nsig;
  for (int i = 0; i < SFS_MAX_PEERS; i++) {
    p.wait[i] = h.wait_flag[i];
    p.sig[i] = h.sig_flag[i];
  }
  p.wait_value = h.wait_value;
  p.sig_value = h.sig_value;
  p.counter = h.counter;
  return p;
}

__device__ __forceinline__ unsigned ld_acquire_sys(const unsigned* p) {
  unsigned v;
  asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release_sys(unsigned* p, unsigned v) {
  asm volatile("st.release.sys.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

constexpr unsigned long long kHaloTimeoutNs = 20ull * 1000 * 1000 * 1000;  // 20 s

// Before reading x: the neighbours have pushed this epoch's ghosts and finished reading the buffer
// this grid pushes into.
template <bool PUSH>
__device__ __forceinline__ void halo_wait(const PushParam<PUSH>& p) {
  if constexpr (PUSH) {
    if ((int)threadIdx.x < p.nwait) {
      const unsigned* f = p.wait[threadIdx.x];
      unsigned long long t0 = 0;
      for (int spin = 0; (int)(ld_acquire_sys(f) - p.wait_value) < 0; spin++) {
        __nanosleep(100);
        if ((spin & 1023) == 0) {  // a neighbour that never signals: fail the launch, do not hang the GPU
          unsigned long long t;
          asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
          if (t0 == 0) t0 = t;
          else if (t - t0 > kHaloTimeoutNs) __trap();
        }
      }
    }
    __syncthreads();
  }
}

// y[r] = v, and into every run that contains r.
template <bool PUSH, typename T>
__device__ __forceinline__ void store_row(T* __restrict__ y, long long r, T v, const PushParam<PUSH>& p,
                                          bool& pushed) {
  y[r] = v;
  if constexpr (PUSH) {
    for (int i = 0; i < p.nseg; i++)
      if (r >= p.b[i] && r < p.e[i]) {
        ((T*)p.dst[i])[r - p.b[i]] = v;
        pushed = true;
      }
  }
}

// After this CTA's stores: a thread that pushed publishes its peer stores (system-scope fence); the
// CTA's arrival is counted with an acq_rel atomic (its reads of x and stores of y are done), and the
// last CTA of the grid resets the counter and releases every neighbour's flag (system scope).  With no
// neighbour (nsig == 0, uniform over the grid) nothing waits on this grid: no counting.
template <bool PUSH>
__device__ __forceinline__ void halo_signal(const PushParam<PUSH>& p, bool pushed) {
  if constexpr (PUSH) {
    if (pushed) __threadfence_system();
    if (p.nsig == 0) return;
    __syncthreads();
    if (threadIdx.x == 0) {
      unsigned prev;
      asm volatile("atom.acq_rel.gpu.global.add.u32 %0, [%1], 1;" : "=r"(prev) : "l"(p.counter) : "memory");
      if (prev == gridDim.x - 1) {
        asm volatile("fence.acq_rel.sys;" ::: "memory");
        *p.counter = 0u;
        for (int i = 0; i < p.nsig; i++) st_release_sys(p.sig[i], p.sig_value);
      }
    }
  }
}

__global__ void k_halo_wait(PushParam<true> p) {
  pdl_wait();
  halo_wait<true>(p);
  pdl_trigger();
}

// The push alone: dst runs <- src[r] (initial ghost exchange; the unfused formats' push after their SpMV).
template <typename T>
__global__ void k_halo_push(const T* __restrict__ src, PushParam<true> p) {
  pdl_wait();
  halo_wait<true>(p);
  bool pushed = false;
  for (int i = 0; i < p.nseg; i++) {
    const long long n = p.e[i] - p.b[i];
    T* d = (T*)p.dst[i];
    for (long long t = (long long)blockIdx.x * blockDim.x + threadIdx.x; t < n; t += (long long)gridDim.x * blockDim.x) {
      d[t] = src[p.b[i] + t];
      pushed = true;
    }
  }
  halo_signal<true>(p, pushed);
  pdl_trigger();
}

// ======================================================================== CSR vector
// Vector v (TPV lanes) owns rows v, v+V, v+2V, ... (V = vectors in the grid): the CUSP-style mapping
// the csr_max feature describes (Q4).  It works on two of its rows at once (r and r+V) and
// prefetches the row bounds of the next pair, so each lane has >= 2 independent loads in flight.
template <typename T, int TPV>
__device__ __forceinline__ acc_t csr_row_partial(const int* __restrict__ col, const T* __restrict__ val,
                                                 const T* __restrict__ x, int b, int e, int lane) {
  acc_t s = 0;
  int k = b + lane;
  for (; k + TPV < e; k += 2 * TPV) {
    const int c0 = ld_stream(col + k), c1 = ld_stream(col + k + TPV);
    const T v0 = ld_stream(val + k), v1 = ld_stream(val + k + TPV);
    s += mulp(v0, ld_x(x + c0));
    s += mulp(v1, ld_x(x + c1));
  }
  if (k < e) s += mulp(ld_stream(val + k), ld_x(x + ld_stream(col + k)));
  return s;
}

template <typename T, int TPV>
__global__ void __launch_bounds__(256) k_spmv_csr_vector(const int* __restrict__ rp, const int* __restrict__ col,
                                                         const T* __restrict__ val, const T* __restrict__ x,
                                                         T* __restrict__ y, long long m) {
  pdl_wait();
  pdl_early();
  const long long gt = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  const int lane = threadIdx.x & (TPV - 1);
  const long long V = ((long long)gridDim.x * blockDim.x) / TPV;
  const unsigned mask = TPV == 32 ? 0xffffffffu : (((1u << TPV) - 1u) << ((threadIdx.x & 31) & ~(TPV - 1)));
  long long r = gt / TPV;
  int b0 = 0, e0 = 0, b1 = 0, e1 = 0;
  if (r < m) { b0 = __ldg(rp + r); e0 = __ldg(rp + r + 1); }
  if (r + V < m) { b1 = __ldg(rp + r + V); e1 = __ldg(rp + r + V + 1); }
  for (; r < m; r += 2 * V) {
    const long long rn = r + 2 * V;
    int nb0 = 0, ne0 = 0, nb1 = 0, ne1 = 0;  // prefetch the next pair's bounds
    if (rn < m) { nb0 = __ldg(rp + rn); ne0 = __ldg(rp + rn + 1); }
    if (rn + V < m) { nb1 = __ldg(rp + rn + V); ne1 = __ldg(rp + rn + V + 1); }
    acc_t s0 = csr_row_partial<T, TPV>(col, val, x, b0, e0, lane);
    acc_t s1 = csr_row_partial<T, TPV>(col, val, x, b1, e1, lane);
#pragma unroll
    for (int o = TPV / 2; o > 0; o >>= 1) {
      s0 += __shfl_xor_sync(mask, s0, o);
      s1 += __shfl_xor_sync(mask, s1, o);
    }
    if (lane == 0) {
      y[r] = (T)s0;
      if (r + V < m) y[r + V] = (T)s1;
    }
    b0 = nb0; e0 = ne0; b1 = nb1; e1 = ne1;
  }
  pdl_trigger();
}

// ======================================================================== CSR stream (regular rows)
// A group of 32 consecutive rows has contiguous nnz [rp[r0], rp[r0+32]).  S warps share a group:
// warp part p streams windows p, p+S, ... of kSW items (lane i loads items i, i+32, ...: every load
// instruction is one contiguous 128/256 B request), stages the products in its own smem window, and
// lane j adds row r0+j's part of the window.  The S partial sums meet in shared memory.
constexpr int kSThreads = 256;
constexpr int kSWarps = kSThreads / 32;
template <typename T> constexpr int stream_u() { return sizeof(T) == 4 ? 16 : 8; }  // items per lane per window
template <typename T> constexpr int stream_ctas() { return sizeof(T) == 4 ? 3 : 4; }  // register cap
constexpr int kSWMax = 32 * 16;

template <typename T, bool PUSH = false>
__global__ void __launch_bounds__(kSThreads, stream_ctas<T>()) k_spmv_csr_stream(const int* __restrict__ rp,
                                                               const int* __restrict__ col,
                                                               const T* __restrict__ val, const T* __restrict__ x,
                                                               T* __restrict__ y, long long m, int S,
                                                               PushParam<PUSH> push) {
  constexpr int kSU = stream_u<T>();  // all of a lane's loads of a window are in flight together
  constexpr int kSW = 32 * kSU;
  __shared__ acc_t sbuf[kSWarps][kSW];
  __shared__ acc_t s_part[kSWarps][32];
  pdl_wait();
  pdl_early();
  halo_wait<PUSH>(push);
  bool pushed = false;
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  const int NG = kSWarps / S;  // groups per CTA iteration
  const int p = w / NG, gl = w % NG;
  acc_t* buf = sbuf[w];
  const long long ngroups = ceil_div(m, 32);
  const long long niter = ceil_div(ngroups, NG);
  // row bounds of the group are prefetched one iteration ahead (off the col -> x critical path)
  auto bounds = [&](long long it, int& b, int& e) {
    const long long g = it * NG + gl;
    const long long r = g * 32 + lane;
    const long long rb = g < ngroups ? (r < m ? r : m) : m;
    b = __ldg(rp + rb);
    e = __ldg(rp + (g < ngroups && r < m ? r + 1 : rb));
  };
  int nb = 0, ne = 0;
  if ((long long)blockIdx.x < niter) bounds(blockIdx.x, nb, ne);
  for (long long it = blockIdx.x; it < niter; it += gridDim.x) {
    const long long g = it * NG + gl;
    const long long r = g * 32 + lane;
    const int b = nb, e = ne;
    if (it + gridDim.x < niter) bounds(it + gridDim.x, nb, ne);
    const int s0 = __shfl_sync(0xffffffffu, b, 0), s1 = __shfl_sync(0xffffffffu, e, 31);
    acc_t acc = 0;
    for (int w0 = s0 + p * kSW; w0 < s1; w0 += S * kSW) {
      const int n = s1 - w0 < kSW ? s1 - w0 : kSW;
      int c[kSU];
      T v[kSU], xv[kSU];
      // Loads are unconditional (indices clamped into the window) so that all 2*kSU of them, then
      // all kSU x gathers, issue back to back; only the smem stores are predicated.
      const int last = n - 1;
#pragma unroll
      for (int u = 0; u < kSU; u++) {
        const int i = u * 32 + lane < n ? u * 32 + lane : last;
        c[u] = ld_stream(col + w0 + i);
        v[u] = ld_stream(val + w0 + i);
      }
#pragma unroll
      for (int u = 0; u < kSU; u++) xv[u] = ld_x(x + c[u]);
#pragma unroll
      for (int u = 0; u < kSU; u++) {
        const int i = u * 32 + lane;
        if (i < n) buf[i] = mulp(v[u], xv[u]);
      }
      __syncwarp();
      const int lo = (b > w0 ? b : w0) - w0, hi = (e < w0 + n ? e : w0 + n) - w0;
      acc_t a0 = 0, a1 = 0;
      int i = lo;
      for (; i + 1 < hi; i += 2) {
        a0 += buf[i];
        a1 += buf[i + 1];
      }
      if (i < hi) a0 += buf[i];
      acc += a0 + a1;
      __syncwarp();
    }
    if (S == 1) {
      if (g < ngroups && r < m) store_row<PUSH>(y, r, (T)acc, push, pushed);
    } else {
      s_part[w][lane] = acc;
      __syncthreads();
      if (p == 0) {
        acc_t t = acc;
        for (int q = 1; q < S; q++) t += s_part[q * NG + gl][lane];
        if (g < ngroups && r < m) store_row<PUSH>(y, r, (T)t, push, pushed);
      }
      __syncthreads();
    }
  }
  halo_signal<PUSH>(push, pushed);
  pdl_trigger();
}

// ======================================================================== CSR merge path
constexpr int kMT = 256;  // threads
constexpr int kMI = 7;    // items per thread (odd: conflict-free smem walk)
constexpr int kMTile = kMT * kMI;

// Inclusive segmented scan over the block: S_t = f_t ? v_t : S_{t-1} + v_t.  Returns S_{t-1}
// (0 for thread 0); `total` receives S of the last thread.
__device__ __forceinline__ acc_t block_seg_exclusive(int f, acc_t v, acc_t* s_ws, int* s_wf, acc_t& total) {
  const int l = threadIdx.x & 31, w = threadIdx.x >> 5;
  int cf = f;
  acc_t cs = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    acc_t us = __shfl_up_sync(0xffffffffu, cs, o);
    int uf = __shfl_up_sync(0xffffffffu, cf, o);
    if (l >= o) {
      if (!cf) cs += us;
      cf |= uf;
    }
  }
  if (l == 31) { s_ws[w] = cs; s_wf[w] = cf; }
  __syncthreads();
  if (w == 0) {
    const int nw = blockDim.x >> 5;
    acc_t is = l < nw ? s_ws[l] : 0;
    int iff = l < nw ? s_wf[l] : 0;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      acc_t us = __shfl_up_sync(0xffffffffu, is, o);
      int uf = __shfl_up_sync(0xffffffffu, iff, o);
      if (l >= o) {
        if (!iff) is += us;
        iff |= uf;
      }
    }
    acc_t ex = __shfl_up_sync(0xffffffffu, is, 1);
    if (l == 0) ex = 0;
    s_ws[l] = ex;  // segmented prefix of the warps before l
    if (l == nw - 1) s_ws[32] = is;
  }
  __syncthreads();
  const acc_t wprefix = s_ws[w];
  const acc_t incl = cf ? cs : cs + wprefix;
  total = s_ws[32];
  acc_t prev = __shfl_up_sync(0xffffffffu, incl, 1);
  if (l == 0) prev = wprefix;
  __syncthreads();
  return prev;
}

// Merge-path coordinates of every tile boundary, computed once per matrix (at CSR handle creation),
// so no SpMV tile pays the ~log2(m+z) dependent global loads of the search.
__global__ void k_merge_partition(const int* __restrict__ rp, long long m, long long z, int tile,
                                  int2* __restrict__ coords, long long ntiles) {
  dep_wait();
  for (long long t = (long long)blockIdx.x * blockDim.x + threadIdx.x; t <= ntiles; t += (long long)gridDim.x * blockDim.x) {
    long long d = t * tile;
    if (d > m + z) d = m + z;
    int xx, yy;
    merge_path_search(d, rp + 1, (int)m, (int)z, xx, yy);
    coords[t] = make_int2(xx, yy);
  }
  dep_trigger();
}

template <typename T>
__global__ void __launch_bounds__(kMT) k_spmv_csr_merge(const int* __restrict__ rp, const int* __restrict__ col,
                                                        const T* __restrict__ val, const T* __restrict__ x,
                                                        T* __restrict__ y, long long m, long long z,
                                                        const int2* __restrict__ coords,
                                                        int* __restrict__ carry_row, acc_t* __restrict__ carry_val) {
  __shared__ int s_rp[kMTile + 2];
  __shared__ acc_t s_prod[kMTile];
  __shared__ acc_t s_ws[33];
  __shared__ int s_wf[32];
  pdl_wait();
  pdl_early();
  const long long total = m + z;
  const long long d0 = (long long)blockIdx.x * kMTile;
  const long long d1 = d0 + kMTile < total ? d0 + kMTile : total;
  const int2 c0 = __ldg(coords + blockIdx.x), c1 = __ldg(coords + blockIdx.x + 1);
  const int r0 = c0.x, k0 = c0.y, r1 = c1.x, k1 = c1.y;
  // Load phase, fully unrolled so every thread has all of its loads in flight at once: row ends of
  // the tile, then col/val of its nnz (coalesced: item u*kMT + tid), then the x gathers.
  {
    const int nr = (r1 - r0 + 2 < (int)(m - r0 + 1)) ? r1 - r0 + 2 : (int)(m - r0 + 1);
    const int nk = k1 - k0;
    // Loads unconditional with clamped (always valid) indices so they all issue back to back; only
    // the shared-memory stores are predicated.
    int rv[kMI + 1], cv[kMI];
    T vv[kMI], xv[kMI];
#pragma unroll
    for (int u = 0; u <= kMI; u++) {
      const int i = threadIdx.x + u * kMT;
      rv[u] = __ldg(rp + r0 + (i < nr ? i : nr - 1));
    }
    if (nk > 0) {
#pragma unroll
      for (int u = 0; u < kMI; u++) {
        const int i = threadIdx.x + u * kMT < nk ? threadIdx.x + u * kMT : nk - 1;
        cv[u] = ld_stream(col + k0 + i);
        vv[u] = ld_stream(val + k0 + i);
      }
#pragma unroll
      for (int u = 0; u < kMI; u++) xv[u] = ld_x(x + cv[u]);
    }
#pragma unroll
    for (int u = 0; u <= kMI; u++) {
      const int i = threadIdx.x + u * kMT;
      if (i < nr) s_rp[i] = rv[u];
    }
#pragma unroll
    for (int u = 0; u < kMI; u++) {
      const int i = threadIdx.x + u * kMT;
      if (i < nk) s_prod[i] = mulp(vv[u], xv[u]);
    }
  }
  __syncthreads();
  const int ld = threadIdx.x * kMI;
  const int items_all = (int)(d1 - d0);
  int has_end = 0;
  acc_t acc = 0;
  int first_row = -1;
  acc_t first_val = 0;
  if (ld < items_all) {
    int r, k;
    merge_local_search(s_rp, r1 - r0, k0, k1, ld, r0, r, k);
    const int items = items_all - ld < kMI ? items_all - ld : kMI;
#pragma unroll
    for (int it = 0; it < kMI; it++) {
      if (it >= items) break;
      if (r < m && s_rp[r - r0 + 1] <= k) {  // row r ends
        if (!has_end) { has_end = 1; first_row = r; first_val = acc; }
        else y[r] = (T)acc;
        acc = 0;
        r++;
      } else {
        acc += s_prod[k - k0];
        k++;
      }
    }
  }
  acc_t tile_total;
  const acc_t incoming = block_seg_exclusive(has_end, acc, s_ws, s_wf, tile_total);
  if (has_end) y[first_row] = (T)(first_val + incoming);
  if (threadIdx.x == 0) {
    carry_row[blockIdx.x] = r1;  // row open at the tile end (r1 == m: none)
    carry_val[blockIdx.x] = tile_total;
  }
  pdl_trigger();
}

template <typename T>
__global__ void k_spmv_csr_merge_fixup(const int* __restrict__ carry_row, const acc_t* __restrict__ carry_val,
                                       long long tiles, long long m, T* __restrict__ y) {
  pdl_wait();
  pdl_early();
  for (long long t = (long long)blockIdx.x * blockDim.x + threadIdx.x; t < tiles; t += (long long)gridDim.x * blockDim.x) {
    const int r = carry_row[t];
    if (r < m) {  // carry_val is only written for a carried row
      const acc_t v = carry_val[t];
      if (v != 0) atomicAdd(y + r, (T)v);
    }
  }
  pdl_trigger();
}

// ======================================================================== CSR tile (nnz-balanced)
// The COO kernel's shape on the CSR arrays.  Warp w streams the contiguous chunks [cb, ce) of 256
// entries (8 per lane, 256-bit col/val loads whose addresses do not depend on row_ptr), and the row of
// every entry is rebuilt in shared memory from the chunk's slice of row_ptr, off the col -> x chain:
// the rows that START in chunk c are [a_c, a_{c+1}), a_c = lower_bound(rp[0..m), 256 c) (computed
// once per matrix); each non-empty one marks its start position, a max-scan carries the marks to
// every entry, seeded with a_c - 1 (the row open at the chunk start).  Empty rows are zeroed by the
// chunk that owns them.  Rows lying inside one warp's range are finished with plain stores; a row
// split across ranges (one per range boundary, listed per matrix) is zeroed by k_zero_rows ahead of
// this grid and gets every piece by atomicAdd.  k_zero_rows releases this kernel at once (PDL), so
// the first chunk's loads and x gathers overlap it; the kernel waits before touching y.  No full zero
// pass, no row array: CSR's own bytes only.
constexpr int kTThreads = 256;
#ifndef SFS_TILE_PFD
#define SFS_TILE_PFD 1  // chunks ahead of the L2 prefetch of col / val (A/B builds)
#endif
#ifndef SFS_TILE_CTAS
#define SFS_TILE_CTAS 4  // CTAs per SM of the tile kernel (register cap; A/B builds set 5)
#endif
constexpr int kTV = 8;
constexpr int kTChunk = 32 * kTV;

struct TileGeom {
  long long nchunks, cpw, nwarps;
};
TileGeom tile_geom(long long z) {
  TileGeom g;
  g.nchunks = ceil_div(z, kTChunk);
  const long long max_warps = (long long)kSMs * SFS_TILE_CTAS * (kTThreads / 32);  // one resident wave
  g.cpw = ceil_div(g.nchunks, max_warps) < 1 ? 1 : ceil_div(g.nchunks, max_warps);
  g.nwarps = ceil_div(g.nchunks, g.cpw);
  return g;
}

// a[c] = lower_bound(rp, 256 c) (c < nchunks), a[nchunks] = m: one pass over the rows instead of a binary search
// per chunk (a row r owns the chunk starts in (rp[r-1], rp[r]], row 0 the start 0)
__global__ void k_csr_tile_partition(const int* __restrict__ rp, long long m, long long nchunks, int* __restrict__ a) {
  dep_wait();
  for (long long r = (long long)blockIdx.x * blockDim.x + threadIdx.x; r <= m; r += (long long)gridDim.x * blockDim.x) {
    const long long hi = __ldg(rp + r);
    long long c = r == 0 ? 0 : __ldg(rp + r - 1) / kTChunk + 1;
    const long long ce = hi / kTChunk < nchunks - 1 ? hi / kTChunk : nchunks - 1;
    for (; c <= ce; c++) a[c] = (int)r;
    if (r == m) a[nchunks] = (int)m;
  }
  dep_trigger();
}

// BM (variant 4, matrices without empty rows): the row of every entry comes from a row-start bitmap
// built with the handle (bit k set iff entry k starts a row, z/8 bytes): lane l's 8 entries are byte l
// of the chunk's 32-byte bitmap, row = a - 1 + (row starts up to the entry), a warp scan of the bytes'
// popcounts -- no row_ptr loads and no shared-memory marks on the chunk's critical path.
//
// MAP (variant 5, matrices with empty rows): the bitmap marks the starts of the NON-EMPTY rows only, row
// ids are ranks among the non-empty rows (ca / srow converted to that numbering at handle creation) and
// ne[j] maps rank j to its row; y was zeroed whole ahead of this grid (the empty rows stay 0), so no
// per-chunk row_ptr walk is needed (variant 3's walk over runs of empty rows made it 3x slower than the
// merge path on R-MAT).
template <typename T, bool VEC, bool BM = false, bool MAP = false>
__device__ __forceinline__ void csr_tile_warp(const int* __restrict__ rp, const int* __restrict__ col,
                                              const T* __restrict__ val, const T* __restrict__ x, T* __restrict__ y,
                                              long long m, long long z, long long cpw, long long warp,
                                              const int* __restrict__ ca, const int* __restrict__ srow,
                                              long long nwarps, int* head, const unsigned* __restrict__ bm,
                                              const unsigned short* __restrict__ pb, int pf,
                                              const int* __restrict__ ne) {
  const int l = threadIdx.x & 31;
  const long long nchunks = ceil_div(z, kTChunk);
  const long long cb = warp * cpw;
  const long long ce = cb + cpw < nchunks ? cb + cpw : nchunks;
  const int own_lo = __ldg(ca + cb);  // rows >= own_lo start inside this range
  // the row split at the boundary with the next range (m: none); srow[w] rows were zeroed by
  // k_zero_rows before this grid touched y, and every piece of them is added atomically
  const int next_split = warp + 1 < nwarps ? __ldg(srow + warp + 1) : (MAP ? 0x7fffffff : (int)m);
  int open_row = -1;                  // row left open at the previous chunk's end (all lanes agree)
  int open_y = -1;                    // MAP: its y index
  acc_t open = 0;
  bool waited = false;                // PDL: loads of the first chunk overlap k_zero_rows
  // emit(row, y index, value); MAP: the y index of a lane's first / last row is loaded as soon as the
  // ranks are known (off the store path), rows strictly inside a lane's 8 entries (rare) load it there
  auto emit = [&](int row, int yr, acc_t v) {
    if (row < own_lo) atomicAdd(y + yr, (T)v);  // the piece of the row carried into this range
    else y[yr] = (T)v;
  };
  int a_run = own_lo;  // BM: first row starting at or after the chunk start
  for (long long ch = cb; ch < ce; ch++) {
    const long long k0 = ch * kTChunk;
    const long long k = k0 + l * kTV;
    // footprints >> L2 (pf): the next chunk's col (1 KB) and val (1 / 2 KB) into L2, one 128-byte line
    // per lane (L2-resident matrices skip it: there the prefetches only cost issue slots)
    if (pf && ch + SFS_TILE_PFD < ce) {
      constexpr int kColLines = kTChunk * 4 / 128;
      const long long kn = k0 + (long long)SFS_TILE_PFD * kTChunk;
      const long long e = l < kColLines ? kn + l * 32 : kn + (long long)(l - kColLines) * (128 / (long long)sizeof(T));
      if (l < kColLines + kTChunk * (int)sizeof(T) / 128 && e < z) {
        const void* a = l < kColLines ? (const void*)(col + e) : (const void*)(val + e);
        asm volatile("prefetch.global.L2 [%0];" ::"l"(a));
      }
    }
    const int a_lo = BM ? 0 : __ldg(ca + ch), a_hi = BM ? 0 : __ldg(ca + ch + 1);
    // variant 4 reads its lane's bitmap byte with the row starts of the chunk's earlier bytes (k_tile_pack);
    // variant 5 scans the bitmap bytes (corpus CSR race -1.3 % with the packed form, R-MAT 2^22 +5 %)
#ifndef SFS_TILE_PACK
#define SFS_TILE_PACK 1  // A/B builds: 0 = the warp scan for variant 4 too
#endif
    constexpr bool kPack = BM && !MAP && SFS_TILE_PACK;
    unsigned sb = 0;
    int spre = 0;  // row starts in the chunk before this lane's entries
    if (kPack) {
      const unsigned pv = __ldg(pb + ch * 32 + l);
      sb = pv & 0xFFu;
      spre = (int)(pv >> 8);
    } else if (BM) {
      sb = (__ldg(bm + ch * (kTChunk / 32) + (l >> 2)) >> ((l & 3) * 8)) & 0xFFu;
    }
    acc_t p[kTV];
    {
      int c[kTV];
      T v[kTV];
      if (VEC && k + kTV <= z) {
        ld_stream8(col + k, c);  // 32 B aligned: k is a multiple of 8, the bases were checked on the host
        ld_stream8(val + k, v);
      } else {
#pragma unroll
        for (int i = 0; i < kTV; i++) {
          const long long kk = k + i < z ? k + i : z - 1;  // padding: a valid column, value 0
          c[i] = ld_stream(col + kk);
          v[i] = k + i < z ? ld_stream(val + kk) : T(0);
        }
      }
      T xv[kTV];  // every gather issued before the first product (memory-level parallelism)
#pragma unroll
      for (int i = 0; i < kTV; i++) xv[i] = ld_x(x + c[i]);
#pragma unroll
      for (int i = 0; i < kTV; i++) p[i] = mulp(v[i], xv[i]);
    }
    if (!waited) {
      pdl_wait();
      pdl_trigger();
      waited = true;
    }
    int r[kTV];
    if (BM) {
      if (!kPack) {  // exclusive warp scan of the bytes' popcounts
        const int cnt = __popc(sb);
        int inc = cnt;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
          const int u = __shfl_up_sync(0xffffffffu, inc, o);
          if (l >= o) inc += u;
        }
        spre = inc - cnt;
      }
      const int base = a_run - 1 + spre;
#pragma unroll
      for (int i = 0; i < kTV; i++) r[i] = base + __popc(sb & ((2u << i) - 1u));
      a_run += __shfl_sync(0xffffffffu, spre + __popc(sb), 31);
    } else {
    // start marks of the rows beginning in this chunk (non-empty rows start at distinct positions)
    reinterpret_cast<int4*>(head)[2 * l] = make_int4(-1, -1, -1, -1);
    reinterpret_cast<int4*>(head)[2 * l + 1] = make_int4(-1, -1, -1, -1);
    __syncwarp();
    for (int r = a_lo + l; r < a_hi; r += 32) {
      const int b = __ldg(rp + r), e = __ldg(rp + r + 1);
      if (e > b) head[b - k0] = r;
      else y[r] = T(0);
    }
    __syncwarp();
    {
      const int4 h0 = reinterpret_cast<const int4*>(head)[2 * l], h1 = reinterpret_cast<const int4*>(head)[2 * l + 1];
      const int hv[kTV] = {h0.x, h0.y, h0.z, h0.w, h1.x, h1.y, h1.z, h1.w};
      int run = -1;
#pragma unroll
      for (int i = 0; i < kTV; i++) {
        run = hv[i] > run ? hv[i] : run;
        r[i] = run;
      }
      int inc = run;  // warp inclusive max-scan of the lane maxima
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const int u = __shfl_up_sync(0xffffffffu, inc, o);
        if (l >= o) inc = u > inc ? u : inc;
      }
      int ex = __shfl_up_sync(0xffffffffu, inc, 1);
      if (l == 0 || ex < a_lo - 1) ex = a_lo - 1;
#pragma unroll
      for (int i = 0; i < kTV; i++) r[i] = r[i] > ex ? r[i] : ex;
    }
    __syncwarp();  // head is rewritten by the next chunk
    }
    // segmented reduction of (r[i], p[i]) exactly as in the COO kernel; padding items (past z) have
    // p = 0 and the last row
    const int rf = r[0], rl = r[kTV - 1];
    const int yf = MAP ? __ldg(ne + (rf > 0 ? rf : 0)) : rf, yl = MAP ? __ldg(ne + (rl > 0 ? rl : 0)) : rl;
    const int chunk_first = __shfl_sync(0xffffffffu, rf, 0);
    if (open_row >= 0 && open_row != chunk_first) {
      if (l == 0) emit(open_row, MAP ? open_y : open_row, open);
      open_row = -1;
      open = 0;
    }
    acc_t hsum = p[0], cur = p[0];
    int cr = rf;
    bool in_head = true;
#pragma unroll
    for (int i = 1; i < kTV; i++) {
      if (r[i] != cr) {
        if (in_head) { hsum = cur; in_head = false; }
        else emit(cr, MAP ? __ldg(ne + cr) : cr, cur);
        cr = r[i];
        cur = p[i];
      } else {
        cur += p[i];
      }
    }
    if (in_head) hsum = cur;
    const bool single = (rf == rl);
    const acc_t in0 = (open_row == rf) ? open : acc_t(0);
    const int prev_rl = __shfl_up_sync(0xffffffffu, rl, 1);
    int f = (l == 0) || !single || (prev_rl != rf);
    acc_t S = cur + ((l == 0 && single) ? in0 : acc_t(0));
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const acc_t us = __shfl_up_sync(0xffffffffu, S, o);
      const int uf = __shfl_up_sync(0xffffffffu, f, o);
      if (l >= o) {
        if (!f) S += us;
        f |= uf;
      }
    }
    const acc_t S_prev = __shfl_up_sync(0xffffffffu, S, 1);
    const int next_rf = __shfl_down_sync(0xffffffffu, rf, 1);
    if (!single) emit(rf, yf, hsum + (l == 0 ? in0 : (prev_rl == rf ? S_prev : acc_t(0))));
    if (l < 31 && next_rf != rl) emit(rl, yl, S);
    open_row = __shfl_sync(0xffffffffu, rl, 31);
    if (MAP) open_y = __shfl_sync(0xffffffffu, yl, 31);
    open = __shfl_sync(0xffffffffu, S, 31);
  }
  if (l == 0 && open_row >= 0) {  // a piece of a split row if it continues past the range
    const int oy = MAP ? open_y : open_row;
    if (open_row == next_split) atomicAdd(y + oy, (T)open);
    else emit(open_row, oy, open);
  }
}

// blockDim is 64, 128 or 256 (smaller CTAs spread a small matrix's few warps over more SMs)
template <typename T, bool VEC, bool BM, bool MAP = false>
__global__ void __launch_bounds__(kTThreads, SFS_TILE_CTAS) k_spmv_csr_tile(const int* __restrict__ rp, const int* __restrict__ col,
                                                               const T* __restrict__ val, const T* __restrict__ x,
                                                               T* __restrict__ y, long long m, long long z,
                                                               long long cpw, long long nwarps,
                                                               const int* __restrict__ ca, const int* __restrict__ srow,
                                                               const unsigned* __restrict__ bm,
                                                               const unsigned short* __restrict__ pb, int pf,
                                                               const int* __restrict__ ne) {
  __shared__ __align__(16) int s_head[BM ? 1 : kTThreads / 32][kTChunk];
  const long long warp = ((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  if (warp < nwarps)
    csr_tile_warp<T, VEC, BM, MAP>(rp, col, val, x, y, m, z, cpw, warp, ca, srow, nwarps,
                                   s_head[BM ? 0 : threadIdx.x >> 5], bm, pb, pf, ne);
  else
    pdl_wait();
  pdl_trigger();
}

// Rows split across two warp ranges of the tile kernel (one per range boundary, precomputed): zeroed
// ahead of the tile grid, which adds their pieces atomically.  Releases the tile kernel at once so
// that its first loads overlap this kernel (the tile kernel waits before touching y).
template <typename T>
__global__ void k_zero_rows(T* __restrict__ y, const int* __restrict__ srow, long long n, long long m) {
  pdl_wait();
  pdl_trigger();
  for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
    const int r = srow[i];
    if (r < m) y[r] = T(0);
  }
}

// srow[w] = the row holding the first entry of warp w's range if it started before it, else m; from the
// chunk partition: with r0 = a[w cpw] (the first row with rp[r0] >= kb), the entry kb starts row r0 iff
// rp[r0] == kb, else it lies inside row r0 - 1
__global__ void k_tile_split_rows(const int* __restrict__ rp, const int* __restrict__ a, long long m, long long cpw,
                                  long long nwarps, int* __restrict__ srow) {
  dep_wait();
  for (long long w = (long long)blockIdx.x * blockDim.x + threadIdx.x; w < nwarps; w += (long long)gridDim.x * blockDim.x) {
    const long long kb = w * cpw * kTChunk;
    const int r0 = __ldg(a + w * cpw);
    srow[w] = (w > 0 && (long long)__ldg(rp + r0) != kb) ? r0 - 1 : (int)m;
  }
  dep_trigger();
}

// row-start bitmap: bit k set iff entry k is the first of its row (non-empty rows only: an empty row
// has no entry; variant 4 has none, variant 5 maps ranks back with ne[]).  MAP: ne[pos[r]] = r.
__global__ void k_row_starts(const int* __restrict__ rp, long long m, unsigned* __restrict__ bm,
                             const int* __restrict__ pos, int* __restrict__ ne) {
  dep_wait();
  for (long long r = (long long)blockIdx.x * blockDim.x + threadIdx.x; r < m; r += (long long)gridDim.x * blockDim.x) {
    const int k = __ldg(rp + r);
    if (__ldg(rp + r + 1) > k) {
      atomicOr(bm + (k >> 5), 1u << (k & 31));
      if (ne) ne[pos[r]] = (int)r;
    }
  }
  dep_trigger();
}

// per chunk and lane: (row starts in the chunk's bytes before the lane's) << 8 | the lane's bitmap byte (<= 248
// starts precede lane 31), so the tile kernel reads its row offsets instead of scanning the bitmap bytes
__global__ void k_tile_pack(const unsigned* __restrict__ bm, long long nchunks, unsigned short* __restrict__ pb) {
  dep_wait();
  for (long long c = (long long)blockIdx.x * blockDim.x + threadIdx.x; c < nchunks; c += (long long)gridDim.x * blockDim.x) {
    unsigned run = 0;
    for (int w = 0; w < kTChunk / 32; w++) {
      const unsigned word = bm[c * (kTChunk / 32) + w];
      for (int b = 0; b < 4; b++) {
        const unsigned byte = (word >> (8 * b)) & 0xFFu;
        pb[c * 32 + w * 4 + b] = (unsigned short)((run << 8) | byte);
        run += __popc(byte);
      }
    }
  }
  dep_trigger();
}

// variant 5: chunk starts and split rows renumbered to ranks among the non-empty rows
__global__ void k_tile_rank(const int* __restrict__ pos, long long m, int* __restrict__ a, long long nchunks,
                            int* __restrict__ srow, long long nwarps) {
  dep_wait();
  for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i <= nchunks || i < nwarps;
       i += (long long)gridDim.x * blockDim.x) {
    if (i <= nchunks) a[i] = pos[a[i]];  // a[i] <= m; pos[m] = number of non-empty rows
    if (i < nwarps) srow[i] = srow[i] < m ? pos[srow[i]] : 0x7fffffff;
  }
  dep_trigger();
}

// ======================================================================== COO (also the COO part of HYB)
constexpr int kCooThreads = 256;
constexpr int kCooV = 8;                // items per lane per step (two 128-bit loads per array)
constexpr int kChunk = 32 * kCooV;      // items per warp step

template <typename T, bool ACCUM>
__device__ __forceinline__ void coo_emit(T* y, int row, acc_t v, bool atomic) {
  if (atomic) atomicAdd(y + row, (T)v);
  else if (ACCUM) y[row] = (T)((acc_t)y[row] + v);
  else y[row] = (T)v;
}

// ATOM (the COO part of an overlapped HYB): y was zeroed before the ELL part, which runs concurrently and
// adds atomically -- every row sum is added atomically too, nothing waits before touching y, and the grid
// waits for its predecessor (the ELL part) only at its end, so the SpMV is complete when this grid is.
template <typename T, bool ACCUM, bool ATOM = false>
__global__ void __launch_bounds__(kCooThreads) k_spmv_coo(const int* __restrict__ row, const int* __restrict__ col,
                                                          const T* __restrict__ val, const T* __restrict__ x,
                                                          T* __restrict__ y, long long z, long long chunks_per_warp) {
  // PDL: the predecessor (zero kernel / ELL part of HYB) released us at its start; everything up to
  // the first write (or ACCUM read) of y overlaps it.
  bool waited = false;
  const int l = threadIdx.x & 31;
  const long long nchunks = ceil_div(z, kChunk);
  const long long warp = ((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const long long cb = warp * chunks_per_warp;
  const long long ce = cb + chunks_per_warp < nchunks ? cb + chunks_per_warp : nchunks;
  if (cb < ce) {
    const int last_row = __ldg(row + z - 1);
    const int range_first = __ldg(row + cb * kChunk);
    int carry_row = -1;
    acc_t carry = 0;
    for (long long ch = cb; ch < ce; ch++) {
      const long long k = ch * kChunk + l * kCooV;
      int r[kCooV];
      acc_t p[kCooV];
      if (k + kCooV <= z) {
        int c[kCooV];
        T v[kCooV];
        static_assert(kCooV == 8, "one 256-bit load per array per lane");
        ld_stream8(row + k, r);  // 32 B aligned: k is a multiple of 8 and the arrays are ours
        ld_stream8(col + k, c);
        ld_stream8(val + k, v);
        // fp64 products here even for fp32 values: the fp32-product build of this kernel measured slower on
        // R-MAT 2^22 (286 vs 243 us: ptxas drops to 48 registers and the chunk loop loses its overlap;
        // profiles/r02/micro_ab.txt)
#pragma unroll
        for (int i = 0; i < kCooV; i++) p[i] = (acc_t)v[i] * (acc_t)ld_x(x + c[i]);
      } else {
#pragma unroll
        for (int i = 0; i < kCooV; i++) {
          if (k + i < z) {
            r[i] = ld_stream(row + k + i);
            p[i] = (acc_t)ld_stream(val + k + i) * (acc_t)ld_x(x + ld_stream(col + k + i));
          } else {
            r[i] = last_row;  // padding joins the last segment with value 0
            p[i] = 0;
          }
        }
      }
      if (!ATOM && !waited) {
        pdl_wait();
        pdl_early();
        waited = true;
      }
      const int rf = r[0], rl = r[kCooV - 1];
      // the previous chunk's carry ends exactly at this chunk boundary: emit it
      const int chunk_first = __shfl_sync(0xffffffffu, rf, 0);
      if (carry_row >= 0 && carry_row != chunk_first) {
        if (l == 0) coo_emit<T, ACCUM>(y, carry_row, carry, ATOM || carry_row == range_first);
        carry_row = -1;
        carry = 0;
      }
      // lane-local segments: head (row rf), middles (complete), tail (row rl)
      acc_t head = p[0], cur = p[0];
      int cr = rf;
      bool in_head = true;
#pragma unroll
      for (int i = 1; i < kCooV; i++) {
        if (r[i] != cr) {
          if (in_head) { head = cur; in_head = false; }
          else coo_emit<T, ACCUM>(y, cr, cur, ATOM || cr == range_first);
          cr = r[i];
          cur = p[i];
        } else {
          cur += p[i];
        }
      }
      if (in_head) head = cur;
      const bool single = (rf == rl);
      const acc_t in0 = (carry_row == rf) ? carry : acc_t(0);  // carry into lane 0 (same row)
      // segmented scan of tails across lanes: S_l = f_l ? tail_l : S_{l-1} + tail_l
      const int prev_rl = __shfl_up_sync(0xffffffffu, rl, 1);
      int f = (l == 0) || !single || (prev_rl != rf);
      acc_t S = cur + ((l == 0 && single) ? in0 : acc_t(0));
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        acc_t us = __shfl_up_sync(0xffffffffu, S, o);
        int uf = __shfl_up_sync(0xffffffffu, f, o);
        if (l >= o) {
          if (!f) S += us;
          f |= uf;
        }
      }
      const acc_t S_prev = __shfl_up_sync(0xffffffffu, S, 1);
      const int next_rf = __shfl_down_sync(0xffffffffu, rf, 1);
      if (!single) {
        const acc_t h = head + (l == 0 ? in0 : (prev_rl == rf ? S_prev : acc_t(0)));
        coo_emit<T, ACCUM>(y, rf, h, ATOM || rf == range_first);
      }
      if (l < 31 && next_rf != rl) coo_emit<T, ACCUM>(y, rl, S, ATOM || rl == range_first);
      carry_row = __shfl_sync(0xffffffffu, rl, 31);  // the chunk's last row stays open
      carry = __shfl_sync(0xffffffffu, S, 31);
    }
    if (l == 0 && carry_row >= 0) atomicAdd(y + carry_row, (T)carry);  // may continue in the next range
  }
  // ATOM: complete only after the ELL part (its predecessor) has completed, so the SpMV is done with this
  // grid and the next SpMV's zero kernel cannot overtake the ELL part's atomics
  if (ATOM || !waited) pdl_wait();
  pdl_trigger();
}

// ======================================================================== ELL (and the ELL part of HYB)
// Thread = 4 consecutive rows x one of S slot-parts; slots are read in batches (four / eight 16 B col
// vectors and as many 16/32 B val vectors issued before any x gather).  CTA = S parts x G row
// groups (a warp = 32 consecutive groups of one part); parts meet in shared memory.
constexpr int kEllThreads = 256;
template <typename T> constexpr int ell_batch() { return sizeof(T) == 4 ? 8 : 4; }   // bytes in flight per thread
template <typename T> constexpr int ell_ctas() { return sizeof(T) == 4 ? 3 : 4; }    // CTAs / SM (register cap)

// OVF (HYB whose rows overflow the ELL part by at most kHybRowwiseLarge / kHybRowwiseSmall entries):
// the parts of each row group also add its rows' COO-part entries, located by the per-row overflow
// offsets ovf[0..m] kept from the conversion -- HYB in one launch, y written once.
constexpr long long kHybRowwiseSmall = 64;  // z < 2^20 (latency-bound sizes)
constexpr long long kHybRowwiseLarge = 32;

// ATOM (HYB with long overflow rows, overlapped): y was zeroed ahead and the COO part runs concurrently,
// so the ELL part adds its row sums atomically instead of storing them.
#ifndef SFS_OVF_BATCH
#define SFS_OVF_BATCH 2  // HYB overflow entries per walk step (corpus HYB race: 1: 2683, 2: 2668, 3: 2677, 4: 2687, 8: 2757 us/rep)
#endif
template <typename T, bool OVF, bool PUSH = false, bool ATOM = false>
__global__ void __launch_bounds__(kEllThreads, ell_ctas<T>()) k_spmv_ell(const int* __restrict__ ecol,
                                                                         const T* __restrict__ eval,
                                                                         const T* __restrict__ x, T* __restrict__ y,
                                                                         long long m, long long P, int K, int S,
                                                                         int early_trigger,
                                                                         const int* __restrict__ ovf,
                                                                         const int* __restrict__ ocol,
                                                                         const T* __restrict__ oval,
                                                                         PushParam<PUSH> push) {
  constexpr int kB = ell_batch<T>();
  __shared__ acc_t s_part[kEllThreads][4];
  pdl_wait();
  pdl_early();
  if (early_trigger) pdl_trigger();  // HYB: let the COO part start its loads now
  halo_wait<PUSH>(push);
  bool pushed = false;
  const int G = kEllThreads / S;
  const int p = threadIdx.x / G, g = threadIdx.x % G;
  const int Kp = (K + S - 1) / S;
  const int j0 = p * Kp, j1 = j0 + Kp < K ? j0 + Kp : K;
  const long long groups = P / 4;
  const long long niter = ceil_div(groups, G);
  for (long long it = blockIdx.x; it < niter; it += gridDim.x) {
    const long long grp = it * G + g;
    const long long r = grp * 4;
    acc_t acc[4] = {0, 0, 0, 0};
    if (grp < groups) {
      int ob[5];
      if (OVF) {
#pragma unroll
        for (int q = 0; q <= 4; q++) ob[q] = __ldg(ovf + (r + q < m ? r + q : m));
      }
      const int* cp = ecol + r;
      const T* vp = eval + r;
      int j = j0;
      for (; j + kB <= j1; j += kB) {
        int4 c[kB];
        Vec4<T> v[kB];
#pragma unroll
        for (int u = 0; u < kB; u++) {
          c[u] = ld_stream4(cp + (long long)(j + u) * P);
          v[u].load_stream(vp + (long long)(j + u) * P);
        }
        if constexpr (sizeof(T) == 4 && kFp32Arith) {  // the batch's products per row chained in fp32
          float t[4] = {0.f, 0.f, 0.f, 0.f};
#pragma unroll
          for (int u = 0; u < kB; u++) {
            if (c[u].x >= 0) t[0] = __fmaf_rn(v[u].v[0], ld_x(x + c[u].x), t[0]);
            if (c[u].y >= 0) t[1] = __fmaf_rn(v[u].v[1], ld_x(x + c[u].y), t[1]);
            if (c[u].z >= 0) t[2] = __fmaf_rn(v[u].v[2], ld_x(x + c[u].z), t[2]);
            if (c[u].w >= 0) t[3] = __fmaf_rn(v[u].v[3], ld_x(x + c[u].w), t[3]);
          }
#pragma unroll
          for (int q = 0; q < 4; q++) acc[q] += (acc_t)t[q];
        } else {
#pragma unroll
          for (int u = 0; u < kB; u++) {
            if (c[u].x >= 0) acc[0] += mulp(v[u].v[0], ld_x(x + c[u].x));
            if (c[u].y >= 0) acc[1] += mulp(v[u].v[1], ld_x(x + c[u].y));
            if (c[u].z >= 0) acc[2] += mulp(v[u].v[2], ld_x(x + c[u].z));
            if (c[u].w >= 0) acc[3] += mulp(v[u].v[3], ld_x(x + c[u].w));
          }
        }
      }
      for (; j < j1; j++) {
        const int4 c = ld_stream4(cp + (long long)j * P);
        Vec4<T> v;
        v.load_stream(vp + (long long)j * P);
        if (c.x >= 0) acc[0] += mulp(v.v[0], ld_x(x + c.x));
        if (c.y >= 0) acc[1] += mulp(v.v[1], ld_x(x + c.y));
        if (c.z >= 0) acc[2] += mulp(v.v[2], ld_x(x + c.z));
        if (c.w >= 0) acc[3] += mulp(v.v[3], ld_x(x + c.w));
      }
      if (OVF) {
        // the 4 rows' overflow entries are contiguous: [ob[0], ob[4]); batches of kOB (clamped loads),
        // batch b taken by slot-part b mod S, so the parts share the walk
        constexpr int kOB = SFS_OVF_BATCH;
        for (int k = ob[0] + kOB * p; k < ob[4]; k += kOB * S) {
          int c[kOB];
          T v[kOB];
#pragma unroll
          for (int u = 0; u < kOB; u++) {
            const int kk = k + u < ob[4] ? k + u : ob[4] - 1;
#ifdef SFS_OVF_STREAM
            c[u] = ld_stream(ocol + kk);
            v[u] = ld_stream(oval + kk);
#else
            // L1-allocating: a thread's 4 consecutive entries share a sector, so the 2nd-4th loads hit
            // L1 instead of each requesting the sector from L2 again (L2 sectors bound these SpMVs)
            c[u] = __ldg(ocol + kk);
            v[u] = __ldg(oval + kk);
#endif
          }
#pragma unroll
          for (int u = 0; u < kOB; u++) {
            const acc_t t = mulp(v[u], ld_x(x + c[u]));
            const int kk = k + u;
            if (kk < ob[4]) {
              if (kk < ob[1]) acc[0] += t;
              else if (kk < ob[2]) acc[1] += t;
              else if (kk < ob[3]) acc[2] += t;
              else acc[3] += t;
            }
          }
        }
      }
    }
    if (S > 1) {
#pragma unroll
      for (int q = 0; q < 4; q++) s_part[threadIdx.x][q] = acc[q];
      __syncthreads();
      if (p == 0) {
        for (int pp = 1; pp < S; pp++)
#pragma unroll
          for (int q = 0; q < 4; q++) acc[q] += s_part[pp * G + g][q];
      }
      __syncthreads();
    }
    if (p == 0 && grp < groups) {
#pragma unroll
      for (int q = 0; q < 4; q++) {
        if (r + q < m) {
          if constexpr (ATOM) atomicAdd(y + r + q, (T)acc[q]);
          else store_row<PUSH>(y, r + q, (T)acc[q], push, pushed);
        }
      }
    }
  }
  halo_signal<PUSH>(push, pushed);
  pdl_trigger();
}

// ======================================================================== DIA
// Thread t of a part owns rows R0 + t + Gq (q < 4 for fp64, 8 for fp32, G = 256/S threads per part):
// for every diagonal a warp reads 32 consecutive slab entries and 32 consecutive x entries (coalesced
// whatever the offset's alignment), 4 diagonals per batch, so each thread keeps 16 / 32 independent
// loads in flight.  The S diagonal-parts of a row block meet in shared memory.
constexpr int kDiaThreads = 256;
constexpr int kDiaSmemOffs = 1024;
template <typename T> constexpr int dia_rows() { return 4; }
template <typename T> constexpr int dia_ctas() { return 4; }  // register cap
template <typename T> constexpr int dia_batch() { return 4; }  // diagonals per batch

template <typename T, int S, bool PUSH = false>
__global__ void __launch_bounds__(kDiaThreads, dia_ctas<T>()) k_spmv_dia(const int* __restrict__ offs,
                                                                         const T* __restrict__ dval,
                                                                         const T* __restrict__ x, T* __restrict__ y,
                                                                         long long m, long long n, long long P,
                                                                         int nd, PushParam<PUSH> push) {
  constexpr int kR = dia_rows<T>();
  constexpr int G = kDiaThreads / S;  // threads per part (compile-time: row strides are immediates)
  constexpr int kB = dia_batch<T>();
  __shared__ int s_off[kDiaSmemOffs];
  __shared__ acc_t s_part[S > 1 ? kDiaThreads * kR : 1];
  pdl_wait();
  pdl_early();
  const int nsm = nd < kDiaSmemOffs ? nd : kDiaSmemOffs;
  for (int i = threadIdx.x; i < nsm; i += blockDim.x) s_off[i] = offs[i];
  __syncthreads();
  halo_wait<PUSH>(push);
  bool pushed = false;
  const int p = threadIdx.x / G, g = threadIdx.x % G;
  const int Dp = (nd + S - 1) / S;
  const int d0 = p * Dp, d1 = d0 + Dp < nd ? d0 + Dp : nd;
  constexpr long long rows_per_blk = (long long)G * kR;
  const long long nblk = ceil_div(m, rows_per_blk);
  for (long long blk = blockIdx.x; blk < nblk; blk += gridDim.x) {
    const long long rbase = blk * rows_per_blk;
    const long long r0 = rbase + g;
    const bool full = rbase + rows_per_blk <= m;
    acc_t acc[kR];
#pragma unroll
    for (int q = 0; q < kR; q++) acc[q] = 0;
    for (int d = d0; d < d1; d += kB) {
      const int nb = d1 - d < kB ? d1 - d : kB;
      int off[kB];
#pragma unroll
      for (int u = 0; u < kB; u++) off[u] = u < nb ? (d + u < kDiaSmemOffs ? s_off[d + u] : __ldg(offs + d + u)) : 0;
      bool all_in = full && nb == kB;
#pragma unroll
      for (int u = 0; u < kB; u++) {
        const long long c0 = r0 + off[u];
        all_in = all_in && c0 >= 0 && c0 + (kR - 1) * G < n;
      }
      if (all_in) {
        // fast path (interior blocks): every load unconditional with a per-diagonal base pointer and
        // immediate row offsets, slab values first, then the x gathers, then the FMAs
        T v[kB][kR], xv[kB][kR];
#pragma unroll
        for (int u = 0; u < kB; u++) {
          const T* vp = dval + (long long)(d + u) * P + r0;
#pragma unroll
          for (int q = 0; q < kR; q++) v[u][q] = ld_stream(vp + q * G);
        }
#pragma unroll
        for (int u = 0; u < kB; u++) {
          const T* xp = x + r0 + off[u];
#pragma unroll
          for (int q = 0; q < kR; q++) xv[u][q] = ld_x(xp + q * G);
        }
#pragma unroll
        for (int u = 0; u < kB; u++)
#pragma unroll
          for (int q = 0; q < kR; q++) acc[q] += mulp(v[u][q], xv[u][q]);
      } else {
        for (int u = 0; u < nb; u++) {
          const T* vp = dval + (long long)(d + u) * P + r0;
          const long long c0 = r0 + off[u];
#pragma unroll
          for (int q = 0; q < kR; q++) {
            const long long rr = r0 + q * G, c = c0 + q * G;
            if (rr < m && c >= 0 && c < n) acc[q] += mulp(ld_stream(vp + q * G), ld_x(x + c));
          }
        }
      }
    }
    if (S > 1) {
#pragma unroll
      for (int q = 0; q < kR; q++) s_part[threadIdx.x * kR + q] = acc[q];
      __syncthreads();
      if (p == 0) {
#pragma unroll
        for (int pp = 1; pp < S; pp++)
#pragma unroll
          for (int q = 0; q < kR; q++) acc[q] += s_part[(pp * G + g) * kR + q];
      }
      __syncthreads();
    }
    if (p == 0) {
#pragma unroll
      for (int q = 0; q < kR; q++) {
        const long long rr = r0 + (long long)q * G;
        if (rr < m) store_row<PUSH>(y, rr, (T)acc[q], push, pushed);
      }
    }
  }
  halo_signal<PUSH>(push, pushed);
  pdl_trigger();
}

// Consecutive-row DIA (fp32): thread = 4 CONSECUTIVE rows, so a diagonal's slab values are one 16-byte vector per thread
// (the ELL mapping; warp = 128 consecutive rows, 512 contiguous bytes per slab load) and its 4 x values
// are 4 scalar loads hitting the same lines (L1).  fp32's scalar strided mapping above moves 4 bytes
// per load instruction; this one moves 16.  S diagonal-parts per row block meet in shared memory.
#ifndef SFS_DIA_V4_CTAS
#define SFS_DIA_V4_CTAS 4  // CTAs per SM (register cap); A/B builds set 5 / 6 together with SFS_DIA_V4_KB
#endif
#ifndef SFS_DIA_V4_KB
#define SFS_DIA_V4_KB 4    // fp32 diagonals per batch
#endif
template <typename T, int S, bool PUSH, bool XA = false>
__global__ void __launch_bounds__(kDiaThreads, SFS_DIA_V4_CTAS) k_spmv_dia_v4(const int* __restrict__ offs,
                                                                const T* __restrict__ dval,
                                                                const T* __restrict__ x, T* __restrict__ y,
                                                                long long m, long long n, long long P, int nd,
                                                                PushParam<PUSH> push, int pfd) {
  static_assert(!XA || sizeof(T) == 4, "XA: fp32 x");
  constexpr int G = kDiaThreads / S;
  constexpr int kB = sizeof(T) == 4 ? SFS_DIA_V4_KB : 2;  // diagonals per batch (register cap)
  __shared__ int s_off[kDiaSmemOffs];
  __shared__ acc_t s_part[S > 1 ? kDiaThreads * 4 : 1];
  pdl_wait();
  pdl_early();
  const int nsm = nd < kDiaSmemOffs ? nd : kDiaSmemOffs;
  for (int i = threadIdx.x; i < nsm; i += blockDim.x) s_off[i] = offs[i];
  __syncthreads();
  halo_wait<PUSH>(push);
  bool pushed = false;
  const int p = threadIdx.x / G, g = threadIdx.x % G;
  const int Dp = (nd + S - 1) / S;
  const int d0 = p * Dp, d1 = d0 + Dp < nd ? d0 + Dp : nd;
  constexpr long long rows_per_blk = (long long)G * 4;
  const long long nblk = ceil_div(m, rows_per_blk);
  for (long long blk = blockIdx.x; blk < nblk; blk += gridDim.x) {
    const long long r0 = blk * rows_per_blk + 4 * g;  // < P whenever < m (P is a multiple of 32)
    const bool live = r0 < m;
    acc_t acc[4] = {0, 0, 0, 0};
    if (live) {
      const bool full = r0 + 4 <= m;
      for (int d = d0; d < d1; d += kB) {
        const int nb = d1 - d < kB ? d1 - d : kB;
        int off[kB];
#pragma unroll
        for (int u = 0; u < kB; u++) off[u] = u < nb ? (d + u < kDiaSmemOffs ? s_off[d + u] : __ldg(offs + d + u)) : 0;
        bool all_in = full && nb == kB;
#pragma unroll
        for (int u = 0; u < kB; u++) all_in = all_in && r0 + off[u] >= 0 && r0 + off[u] + 3 < n;
        if (all_in) {
          Vec4<T> v[kB];
          T xv[kB][4];
#pragma unroll
          for (int u = 0; u < kB; u++) v[u].load_stream(dval + (long long)(d + u) * P + r0);
          // slab of the batch pfd batches ahead into L2 (no registers held): more HBM bytes in flight
          if (pfd > 0) {
            const int dp = d + pfd * kB;
#pragma unroll
            for (int u = 0; u < kB; u++)
              if (dp + u < d1)
                asm volatile("prefetch.global.L2 [%0];" ::"l"(dval + (long long)(dp + u) * P + r0));
          }
#pragma unroll
          for (int u = 0; u < kB; u++) {
            const T* xp = x + r0 + off[u];
            if constexpr (XA) {
              // the 4 x values in the widest aligned pieces (x 16 B aligned, r0 a multiple of 4, so the
              // alignment s = off mod 4 is warp-uniform): s = 0 one 16-byte load, s = 2 two 8-byte loads,
              // s odd 4 + 8 + 4 bytes -- a lane-strided warp load costs ~4 L1 wavefronts whatever its width
              const int sft = off[u] & 3;
              if (sft == 0) {
                const float4 a = __ldg(reinterpret_cast<const float4*>(xp));
                xv[u][0] = a.x; xv[u][1] = a.y; xv[u][2] = a.z; xv[u][3] = a.w;
              } else if (sft == 2) {
                const float2 a = __ldg(reinterpret_cast<const float2*>(xp));
                const float2 b = __ldg(reinterpret_cast<const float2*>(xp + 2));
                xv[u][0] = a.x; xv[u][1] = a.y; xv[u][2] = b.x; xv[u][3] = b.y;
              } else {
                const float2 a = __ldg(reinterpret_cast<const float2*>(xp + 1));
                xv[u][0] = ld_x(xp); xv[u][1] = a.x; xv[u][2] = a.y; xv[u][3] = ld_x(xp + 3);
              }
            } else {
#pragma unroll
              for (int q = 0; q < 4; q++) xv[u][q] = ld_x(xp + q);
            }
          }
          if constexpr (sizeof(T) == 4 && kFp32Arith) {  // the batch's products per row chained in fp32
#pragma unroll
            for (int q = 0; q < 4; q++) {
              float t = __fmul_rn(v[0].v[q], xv[0][q]);
#pragma unroll
              for (int u = 1; u < kB; u++) t = __fmaf_rn(v[u].v[q], xv[u][q], t);
              acc[q] += (acc_t)t;
            }
          } else {
#pragma unroll
            for (int u = 0; u < kB; u++)
#pragma unroll
              for (int q = 0; q < 4; q++) acc[q] += mulp(v[u].v[q], xv[u][q]);
          }
        } else {
          for (int u = 0; u < nb; u++) {
            Vec4<T> v;
            v.load_stream(dval + (long long)(d + u) * P + r0);
#pragma unroll
            for (int q = 0; q < 4; q++) {
              const long long c = r0 + q + off[u];
              if (r0 + q < m && c >= 0 && c < n) acc[q] += mulp(v.v[q], ld_x(x + c));
            }
          }
        }
      }
    }
    if (S > 1) {
#pragma unroll
      for (int q = 0; q < 4; q++) s_part[threadIdx.x * 4 + q] = acc[q];
      __syncthreads();
      if (p == 0) {
#pragma unroll
        for (int pp = 1; pp < S; pp++)
#pragma unroll
          for (int q = 0; q < 4; q++) acc[q] += s_part[(pp * G + g) * 4 + q];
      }
      __syncthreads();
    }
    if (p == 0 && live) {
#pragma unroll
      for (int q = 0; q < 4; q++)
        if (r0 + q < m) store_row<PUSH>(y, r0 + q, (T)acc[q], push, pushed);
    }
  }
  halo_signal<PUSH>(push, pushed);
  pdl_trigger();
}

// Shared by the TMA DIA kernel below: rows per block, staged-x window rules, cp.async helpers.
constexpr int kSxRows = 4 * kDiaThreads;  // rows per block: thread t owns rows t + 256 q, q = 0..3
constexpr int kSxBuf = 16384;             // bytes per fp32 x staging buffer (two per CTA)
constexpr int kSxGap = 256;               // offsets closer than this share an x window
constexpr int kSxWin = 32;                // windows tracked (later ones read x from global memory)
__device__ __forceinline__ void cp_async16(void* dst, const void* src, int src_bytes) {
  const unsigned d = (unsigned)__cvta_generic_to_shared(dst);
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(d), "l"(src), "r"(src_bytes) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() { asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory"); }

// Window setup of the staged-x DIA kernel (warp 0; the caller synchronises): offsets closer than kSxGap
// share a window; window w (w < kSxWin) holds (whi - floor4(wlo)) + kSxRows values rounded up to 4 at
// s_wsb[w]; staged windows are the prefix that fits kCap values.  s_xb[d] = window of d (-1: none).
__device__ __forceinline__ void sx_windows(int nd, int kCap, const int* s_off, int* s_xb, int* s_wlo, int* s_whi,
                                           int* s_wlen, int* s_wsb, int* s_nw, int* s_tot, int* s_all) {
  const int lane = threadIdx.x & 31;
  {
    int nw = 0;
    for (int d0 = 0; d0 < nd; d0 += 32) {
      const int d = d0 + lane;
      const bool ok = d < nd;
      const int o = ok ? s_off[d] : 0;
      const bool start = ok && (d == 0 || o - s_off[d - 1] > kSxGap);
      const bool end = ok && (d == nd - 1 || s_off[d + 1] - o > kSxGap);
      const unsigned sb = __ballot_sync(0xffffffffu, start);
      const int w = nw + __popc(sb & ((2u << lane) - 1u)) - 1;  // window of d
      if (ok) s_xb[d] = w < kSxWin ? w : -1;
      if (start && w < kSxWin) s_wlo[w] = o;
      if (end && w < kSxWin) s_whi[w] = o;
      nw += __popc(sb);
    }
    const bool fits = nw <= kSxWin;
    nw = nw < kSxWin ? nw : kSxWin;
    __syncwarp();
    // budget: window w holds (whi - floor4(wlo)) + kSxRows values rounded up to 4; staged windows are a
    // prefix (the running total is monotone)
    int len = 0;
    if (lane < nw) len = ((s_whi[lane] - (s_wlo[lane] & ~3) + kSxRows) + 3) & ~3;
    int inc = len;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const int u = __shfl_up_sync(0xffffffffu, inc, o);
      if (lane >= o) inc += u;
    }
    const bool staged = lane < nw && inc <= kCap;
    if (lane < nw) {
      s_wlen[lane] = staged ? len : 0;
      s_wsb[lane] = inc - len;
    }
    const int ns = __popc(__ballot_sync(0xffffffffu, staged));
    const int tot = __shfl_sync(0xffffffffu, inc, ns > 0 ? ns - 1 : 0);  // values staged per block
    if (lane == 0) {
      *s_nw = ns;
      *s_tot = ns > 0 ? tot : 0;
      *s_all = fits && ns == nw;  // every diagonal's x is staged
    }
  }
}

// DIA with the slab streamed by TMA bulk copies (cp.async.bulk) through a ring of shared-memory stages and
// x staged as in k_spmv_dia_sx (large matrices).  A producer warp issues, per (row block, batch of kTB
// diagonals), one bulk copy of each diagonal's kSxRows-row slab segment (contiguous: the slab is
// diagonal-major) into a free stage and arms that stage's mbarrier with the byte count; the 8 consumer
// warps wait on the stage's mbarrier, read slab and x from shared memory (thread t: rows t + 256 q, both
// reads conflict-free), and release the stage to the producer through a second mbarrier.  The bytes in
// flight per SM are the ring (kTStages x kTB x 4 KB per CTA), held by no register -- the limit of the
// register-staged fp32 kernels (latency-bound at ~0.73-0.79 of HBM).  x windows: cp.async by the
// consumers, double-buffered per block, synchronised by a consumer-only named barrier.
// ring depth (measured, cold, tools/micro.py: fp32 4 stages at 2 CTAs / SM -- 128^3 stencil 0.86 of HBM, 6 or
// 8 stages at 1 CTA / SM 0.66-0.70; fp64 8 stages at 1 CTA / SM -- stencil 0.93, 1M-row band 0.92)
#ifndef SFS_DIA_TMA_STAGES32
#define SFS_DIA_TMA_STAGES32 4
#endif
#ifndef SFS_DIA_TMA_STAGES64
#define SFS_DIA_TMA_STAGES64 8
#endif
template <typename T> constexpr int dia_tma_stages() { return sizeof(T) == 4 ? SFS_DIA_TMA_STAGES32 : SFS_DIA_TMA_STAGES64; }
constexpr int kTConsumers = kDiaThreads;            // 8 consumer warps
constexpr int kTThreadsAll = kDiaThreads + 32;      // + 1 producer warp
template <typename T> constexpr int dia_tma_batch() { return 16384 / (kSxRows * (int)sizeof(T)); }  // 16 KB stages
#ifndef SFS_DIA_TMA_XBUF64
#define SFS_DIA_TMA_XBUF64 32768  // fp64 x buffer bytes (the 128^3 stencil's 3 windows need 30.9 KB)
#endif
template <typename T> constexpr int dia_tma_xbuf() { return sizeof(T) == 8 ? SFS_DIA_TMA_XBUF64 : kSxBuf; }
template <typename T>
constexpr size_t dia_tma_smem() {
  return (size_t)dia_tma_stages<T>() * dia_tma_batch<T>() * kSxRows * sizeof(T) + 2 * (size_t)dia_tma_xbuf<T>();
}
__device__ __forceinline__ unsigned smem_u32(const void* p) { return (unsigned)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(unsigned a, unsigned count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(a), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_wait(unsigned a, unsigned parity) {
  asm volatile(
      "{\n .reg .pred p;\n"
      "WAIT_%=:\n mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n @!p bra WAIT_%=;\n}\n" ::"r"(a),
      "r"(parity)
      : "memory");
}
__device__ __forceinline__ void mbar_arrive(unsigned a) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(a) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(unsigned a, unsigned bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(a), "r"(bytes) : "memory");
}
__device__ __forceinline__ void tma_bulk_g2s(unsigned dst, const void* src, unsigned bytes, unsigned mbar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(dst),
               "l"(src), "r"(bytes), "r"(mbar)
               : "memory");
}
__device__ __forceinline__ void consumers_sync() { asm volatile("bar.sync 1, %0;" ::"n"(kTConsumers) : "memory"); }

template <typename T>
__global__ void __launch_bounds__(kTThreadsAll, 1) k_spmv_dia_tma(const int* __restrict__ offs, const T* __restrict__ dval,
                                                                  const T* __restrict__ x, T* __restrict__ y,
                                                                  long long m, long long n, long long P, int nd) {
  constexpr int kB = dia_tma_batch<T>();
  constexpr int kTStages = dia_tma_stages<T>();
  static_assert(kTStages >= 1 && kTStages <= 16, "the mbarrier arrays hold 16 stages");
  constexpr int kCap = dia_tma_xbuf<T>() / (int)sizeof(T);
  constexpr int kE = 16 / (int)sizeof(T);
  extern __shared__ __align__(128) unsigned char s_dyn[];
  T* s_slab = reinterpret_cast<T*>(s_dyn);                                       // [stage][u][row]
  T* s_xbuf = reinterpret_cast<T*>(s_dyn + (size_t)kTStages * kB * kSxRows * sizeof(T));  // [2][kCap]
  __shared__ __align__(8) unsigned long long s_full[16], s_empty[16];
  __shared__ int s_off[kDiaSmemOffs];
  __shared__ int s_xb[kDiaSmemOffs];
  __shared__ int s_wlo[kSxWin], s_whi[kSxWin], s_wlen[kSxWin], s_wsb[kSxWin];
  __shared__ int s_nw, s_tot, s_all;
  const int t = threadIdx.x, lane = t & 31, warp = t >> 5;
  if (t == 0) {
    for (int i = 0; i < kTStages; i++) {
      mbar_init(smem_u32(&s_full[i]), 1);
      mbar_init(smem_u32(&s_empty[i]), kTConsumers / 32);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  pdl_wait();
  for (int i = t; i < nd; i += blockDim.x) s_off[i] = offs[i];
  __syncthreads();
  if (t < 32) sx_windows(nd, kCap, s_off, s_xb, s_wlo, s_whi, s_wlen, s_wsb, &s_nw, &s_tot, &s_all);
  __syncthreads();
  for (int d = t; d < nd; d += blockDim.x) {
    const int w = s_xb[d];
    s_xb[d] = (w >= 0 && s_wlen[w] > 0) ? s_wsb[w] + (s_off[d] - (s_wlo[w] & ~3)) : -1;
  }
  __syncthreads();
  const long long nblk = ceil_div(m, (long long)kSxRows);
  const int nbatch = (nd + kB - 1) / kB;
  if (warp == kTConsumers / 32) {  // producer warp: one lane issues every bulk copy
    if (lane == 0) {
      long long i = 0;
      for (long long blk = blockIdx.x; blk < nblk; blk += gridDim.x) {
        const long long rbase = blk * kSxRows;
        const long long rows = P - rbase < kSxRows ? P - rbase : kSxRows;  // P: multiple of 32, >= m
        const unsigned seg = (unsigned)(rows * (long long)sizeof(T));
        for (int b = 0; b < nbatch; b++, i++) {
          const int st = (int)(i % kTStages);
          const long long round = i / kTStages;
          if (round > 0) mbar_wait(smem_u32(&s_empty[st]), (unsigned)((round - 1) & 1));
          const int d0 = b * kB, nb = nd - d0 < kB ? nd - d0 : kB;
          const unsigned full = smem_u32(&s_full[st]);
          mbar_expect_tx(full, seg * nb);
          for (int u = 0; u < nb; u++)
            tma_bulk_g2s(smem_u32(s_slab + ((size_t)st * kB + u) * kSxRows), dval + (long long)(d0 + u) * P + rbase,
                         seg, full);
        }
      }
    }
    return;
  }
  // consumers
  const int nws = s_nw, tot = s_tot;
  const bool all_staged = s_all;
  auto stage_x = [&](long long b, int buf) {
    const long long rb = b * kSxRows;
    int w = 0;
    for (int e = t * kE; e < tot; e += kTConsumers * kE) {
      while (w + 1 < nws && e >= s_wsb[w + 1]) w++;
      const long long g = rb + (s_wlo[w] & ~3) + (e - s_wsb[w]);
      const long long avail = g < 0 ? 0 : (n - g) * (long long)sizeof(T);
      const int bytes = avail <= 0 ? 0 : (avail >= 16 ? 16 : (int)avail);
      cp_async16(s_xbuf + (size_t)buf * kCap + e, bytes ? (const void*)(x + g) : (const void*)x, bytes);
    }
    cp_async_commit();
  };
  if ((long long)blockIdx.x < nblk) stage_x(blockIdx.x, 0);
  long long i = 0;
  int it = 0;
  for (long long blk = blockIdx.x; blk < nblk; blk += gridDim.x, it ^= 1) {
    const long long rbase = blk * kSxRows;
    if (blk + gridDim.x < nblk) stage_x(blk + gridDim.x, it ^ 1);
    else cp_async_commit();
    cp_async_wait<1>();
    consumers_sync();  // this block's x windows have landed (every consumer's copies)
    const T* sx = s_xbuf + (size_t)it * kCap;
    acc_t acc[4] = {0, 0, 0, 0};
    for (int b = 0; b < nbatch; b++, i++) {
      const int st = (int)(i % kTStages);
      mbar_wait(smem_u32(&s_full[st]), (unsigned)((i / kTStages) & 1));
      const int d0 = b * kB, nb = nd - d0 < kB ? nd - d0 : kB;
      const T* sl = s_slab + (size_t)st * kB * kSxRows + t;
      if (nb == kB && all_staged) {  // fast path: unrolled, every x read from shared memory
        if constexpr (sizeof(T) == 4 && kFp32Arith) {
          float sq[4];
#pragma unroll
          for (int u = 0; u < kB; u++) {
            const T* xs = sx + s_xb[d0 + u] + t;
#pragma unroll
            for (int q = 0; q < 4; q++)
              sq[q] = u == 0 ? __fmul_rn(sl[q * kDiaThreads], xs[q * kDiaThreads])
                             : __fmaf_rn(sl[u * kSxRows + q * kDiaThreads], xs[q * kDiaThreads], sq[q]);
          }
#pragma unroll
          for (int q = 0; q < 4; q++) acc[q] += (acc_t)sq[q];
        } else {
#pragma unroll
          for (int u = 0; u < kB; u++) {
            const T* xs = sx + s_xb[d0 + u] + t;
#pragma unroll
            for (int q = 0; q < 4; q++) acc[q] += mulp(sl[u * kSxRows + q * kDiaThreads], xs[q * kDiaThreads]);
          }
        }
      } else {
        for (int u = 0; u < nb; u++) {
          const int xb = s_xb[d0 + u], o = s_off[d0 + u];
#pragma unroll
          for (int q = 0; q < 4; q++) {
            const long long c = rbase + t + q * kDiaThreads + o;
            const T xv = xb >= 0 ? sx[xb + t + q * kDiaThreads] : (c >= 0 && c < n ? ld_x(x + c) : T(0));
            acc[q] += mulp(sl[u * kSxRows + q * kDiaThreads], xv);
          }
        }
      }
      __syncwarp();
      if (lane == 0) mbar_arrive(smem_u32(&s_empty[st]));
    }
#pragma unroll
    for (int q = 0; q < 4; q++) {
      const long long r = rbase + t + q * kDiaThreads;
      if (r < m) y[r] = (T)acc[q];
    }
    consumers_sync();  // x buffer `it` is restaged in the next iteration
  }
  cp_async_wait<0>();
  pdl_trigger();
}

// ELL (and HYB without a COO part) for large banded matrices: the slot slabs (ecol, eval: slot-major,
// contiguous per slot) streamed by TMA bulk copies through an mbarrier ring, as k_spmv_dia_tma; the
// consumers read the column indices and values of their rows (t + 256 q) from shared memory
// (conflict-free) and gather x through L1.  Measured (profiles/r02/micro_ab.txt): banded / block-diagonal /
// stencil ELL 0.80-0.94 -> 0.90-0.96 of HBM cold; gather-bound (uniform) patterns and the HYB launch
// shapes with an overflow walk got slower, so they keep k_spmv_ell.
#ifndef SFS_ELL_TMA_KB
#define SFS_ELL_TMA_KB 4  // slots per stage
#endif
#ifndef SFS_ELL_TMA_STAGES
#define SFS_ELL_TMA_STAGES 3
#endif
template <typename T> constexpr size_t ell_tma_stage_bytes() { return (size_t)SFS_ELL_TMA_KB * kSxRows * (4 + sizeof(T)); }
template <typename T> constexpr size_t ell_tma_smem() { return (size_t)SFS_ELL_TMA_STAGES * ell_tma_stage_bytes<T>(); }

template <typename T>
__global__ void __launch_bounds__(kTThreadsAll, 1) k_spmv_ell_tma(const int* __restrict__ ecol, const T* __restrict__ eval,
                                                                  const T* __restrict__ x, T* __restrict__ y,
                                                                  long long m, long long P, int K) {
  constexpr int kB = SFS_ELL_TMA_KB;
  constexpr int kStages = SFS_ELL_TMA_STAGES;
  extern __shared__ __align__(128) unsigned char s_dyn[];
  __shared__ __align__(8) unsigned long long s_full[kStages], s_empty[kStages];
  const int t = threadIdx.x, lane = t & 31, warp = t >> 5;
  if (t == 0) {
    for (int i = 0; i < kStages; i++) {
      mbar_init(smem_u32(&s_full[i]), 1);
      mbar_init(smem_u32(&s_empty[i]), kTConsumers / 32);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  pdl_wait();
  __syncthreads();
  const long long nblk = ceil_div(m, (long long)kSxRows);
  const int nbatch = (K + kB - 1) / kB;
  // stage st: [kB][kSxRows] column indices, then [kB][kSxRows] values
  auto scol = [&](int st) { return reinterpret_cast<int*>(s_dyn + (size_t)st * ell_tma_stage_bytes<T>()); };
  auto sval = [&](int st) {
    return reinterpret_cast<T*>(s_dyn + (size_t)st * ell_tma_stage_bytes<T>() + (size_t)kB * kSxRows * 4);
  };
  if (warp == kTConsumers / 32) {  // producer warp
    if (lane == 0) {
      long long i = 0;
      for (long long blk = blockIdx.x; blk < nblk; blk += gridDim.x) {
        const long long rbase = blk * kSxRows;
        const long long rows = P - rbase < kSxRows ? P - rbase : kSxRows;  // P: multiple of 32, >= m
        for (int b = 0; b < nbatch; b++, i++) {
          const int st = (int)(i % kStages);
          const long long round = i / kStages;
          if (round > 0) mbar_wait(smem_u32(&s_empty[st]), (unsigned)((round - 1) & 1));
          const int j0 = b * kB, nb = K - j0 < kB ? K - j0 : kB;
          const unsigned full = smem_u32(&s_full[st]);
          mbar_expect_tx(full, (unsigned)(rows * (4 + (long long)sizeof(T)) * nb));
          for (int u = 0; u < nb; u++) {
            tma_bulk_g2s(smem_u32(scol(st) + (size_t)u * kSxRows), ecol + (long long)(j0 + u) * P + rbase,
                         (unsigned)(rows * 4), full);
            tma_bulk_g2s(smem_u32(sval(st) + (size_t)u * kSxRows), eval + (long long)(j0 + u) * P + rbase,
                         (unsigned)(rows * (long long)sizeof(T)), full);
          }
        }
      }
    }
    return;
  }
  long long i = 0;
  for (long long blk = blockIdx.x; blk < nblk; blk += gridDim.x) {
    const long long rbase = blk * kSxRows;
    const bool full = rbase + kSxRows <= m;
    acc_t acc[4] = {0, 0, 0, 0};
    for (int b = 0; b < nbatch; b++, i++) {
      const int st = (int)(i % kStages);
      mbar_wait(smem_u32(&s_full[st]), (unsigned)((i / kStages) & 1));
      const int j0 = b * kB, nb = K - j0 < kB ? K - j0 : kB;
      const int* sc = scol(st) + t;
      const T* sv = sval(st) + t;
      if (nb == kB && full) {
        int c[kB][4];
        T v[kB][4], xv[kB][4];
#pragma unroll
        for (int u = 0; u < kB; u++)
#pragma unroll
          for (int q = 0; q < 4; q++) {
            c[u][q] = sc[u * kSxRows + q * kDiaThreads];
            v[u][q] = sv[u * kSxRows + q * kDiaThreads];
          }
#pragma unroll
        for (int u = 0; u < kB; u++)
#pragma unroll
          for (int q = 0; q < 4; q++) xv[u][q] = c[u][q] >= 0 ? ld_x(x + c[u][q]) : T(0);  // padding: (-1, +0)
        if constexpr (sizeof(T) == 4 && kFp32Arith) {
          float sq[4];
#pragma unroll
          for (int q = 0; q < 4; q++) {
            sq[q] = __fmul_rn(v[0][q], xv[0][q]);
#pragma unroll
            for (int u = 1; u < kB; u++) sq[q] = __fmaf_rn(v[u][q], xv[u][q], sq[q]);
            acc[q] += (acc_t)sq[q];
          }
        } else {
#pragma unroll
          for (int u = 0; u < kB; u++)
#pragma unroll
            for (int q = 0; q < 4; q++) acc[q] += mulp(v[u][q], xv[u][q]);
        }
      } else {
        // rows past the copied segment (the last block's rows >= P) hold stale shared memory: rows >= m
        // are skipped
        for (int u = 0; u < nb; u++)
#pragma unroll
          for (int q = 0; q < 4; q++) {
            const int c = rbase + t + q * kDiaThreads < m ? sc[u * kSxRows + q * kDiaThreads] : -1;
            if (c >= 0) acc[q] += mulp(sv[u * kSxRows + q * kDiaThreads], ld_x(x + c));
          }
      }
      __syncwarp();
      if (lane == 0) mbar_arrive(smem_u32(&s_empty[st]));
    }
#pragma unroll
    for (int q = 0; q < 4; q++) {
      const long long r = rbase + t + q * kDiaThreads;
      if (r < m) y[r] = (T)acc[q];
    }
  }
  pdl_trigger();
}

struct MergeWork {
  int2* coords;
  int* crow;
  acc_t* cval;
};
inline size_t al256(size_t b) { return (b + 255) / 256 * 256; }
MergeWork merge_work(void* base, long long tiles) {
  MergeWork w;
  char* p = (char*)base;
  w.coords = (int2*)p;
  p += al256(sizeof(int2) * (tiles + 1));
  w.crow = (int*)p;
  p += al256(sizeof(int) * tiles);
  w.cval = (acc_t*)p;
  return w;
}

struct TileWork {
  int* a;        // a_c = lower_bound(rp, 256 c), c = 0..nchunks
  int* srow;     // row split at the start of each warp range (m: none)
  unsigned* bm;  // variants 4, 5: row-start bitmap, nchunks * 8 words
  unsigned short* pb;  // variants 4, 5: per chunk and lane, (row starts in the chunk's earlier bytes << 8) | byte
  int* ne;       // variant 5: row of each non-empty-row rank (m entries reserved)
};
TileWork tile_work(void* base, const TileGeom& g) {
  TileWork w;
  char* p = (char*)base;
  w.a = (int*)p;
  p += al256(sizeof(int) * (g.nchunks + 1));
  w.srow = (int*)p;
  p += al256(sizeof(int) * g.nwarps);
  w.bm = (unsigned*)p;
  p += al256(sizeof(unsigned) * g.nchunks * (kTChunk / 32));
  w.pb = (unsigned short*)p;
  p += al256(sizeof(unsigned short) * g.nchunks * 32);
  w.ne = (int*)p;
  return w;
}

// COO launch geometry: contiguous chunk ranges, one resident wave of warps at most.
template <typename T, bool ACCUM, bool ATOM = false>
cudaError_t launch_coo(const int* row, const int* col, const T* val, const T* x, T* y, long long z, cudaStream_t s) {
  const long long nchunks = ceil_div(z, kChunk);
  const long long max_warps = (long long)kSMs * 4 * (kCooThreads / 32);  // <= 64 regs: 4 CTAs / SM
  const long long cpw = ceil_div(nchunks, max_warps) < 1 ? 1 : ceil_div(nchunks, max_warps);
  const long long warps = ceil_div(nchunks, cpw);
  const unsigned blocks = (unsigned)ceil_div(warps, kCooThreads / 32);
  return launch_k(k_spmv_coo<T, ACCUM, ATOM>, dim3(blocks), dim3(kCooThreads), s, row, col, val, x, y, z, cpw);
}

template <typename T>
cudaError_t launch_zero(T* y, long long m, cudaStream_t s) {
  return launch_k(k_zero<T>, dim3(grid_cap(m, 256, 8)), dim3(256), s, y, m);
}

template <typename T, bool PUSH = false, bool ATOM = false>
cudaError_t launch_ell(const Matrix* A, const T* x, T* y, int K, cudaStream_t s, int early_trigger,
                       PushParam<PUSH> push = {}) {
  if constexpr (!PUSH) {
    // the TMA kernel for slabs of >= SFS_ELL_TMA_MB megabytes (default 256 = 2 x L2; < 0: never).  In the
    // race's back-to-back reps an L2-resident ELL keeps k_spmv_ell: gating on >= 64 row blocks instead made
    // the corpus-200 ELL race 5 % slower (mid-size bands with few slots: 1.2-3.6x per matrix)
    static const long long tma_mb = [] {
      const char* e = getenv("SFS_ELL_TMA_MB");
      return e ? atoll(e) : 256LL;
    }();
    // ... and >= SFS_ELL_TMA_K slots (corpus-2000: 5- and 7-slot stencils 1.24-1.31x slower, 27 slots faster)
    static const int tma_k = [] {
      const char* e = getenv("SFS_ELL_TMA_K");
      return e ? atoi(e) : 16;
    }();
    const long long nb = ceil_div(A->m, (long long)kSxRows);
    const long long slab = (long long)K * A->pitch * (4 + (long long)sizeof(T));
    if (!ATOM && tma_mb >= 0 && slab >= tma_mb * (1ll << 20) && K >= tma_k && K >= 1 && A->banded &&
        (A->fmt == SFS_ELL || A->coo_nnz == 0)) {
      static std::once_flag attr_once[kMaxDevices];
      int dev = 0;
      if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= kMaxDevices) return cudaErrorInvalidDevice;
      std::call_once(attr_once[dev], [] {
        cudaFuncSetAttribute(k_spmv_ell_tma<T>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)ell_tma_smem<T>());
      });
      constexpr int per_sm = (int)((228 * 1024) / (ell_tma_smem<T>() + 2 * 1024)) < 1
                                 ? 1 : (int)((228 * 1024) / (ell_tma_smem<T>() + 2 * 1024));
      const int gt = (int)(nb < (long long)kSMs * per_sm ? nb : (long long)kSMs * per_sm);
      return launch_k_smem(k_spmv_ell_tma<T>, dim3(gt), dim3(kTThreadsAll), ell_tma_smem<T>(), s,
                           (const int*)A->ptr[0], (const T*)A->ptr[1], x, y, A->m, A->pitch, K);
    }
  }
  const long long groups = A->pitch / 4;
  const int S = split_factor(groups, K, 2 * ell_batch<T>(), 16);
  const long long niter = ceil_div(groups, kEllThreads / S);
  const int grid = (int)(niter < (long long)kSMs * ell_ctas<T>() ? niter : (long long)kSMs * ell_ctas<T>());
  if (!PUSH && A->fmt == SFS_HYB && A->variant == 1)
    return launch_k(k_spmv_ell<T, true, false>, dim3(grid), dim3(kEllThreads), s, (const int*)A->ptr[0],
                    (const T*)A->ptr[1], x, y, A->m, A->pitch, K, S, 0, (const int*)A->ptr[5], (const int*)A->ptr[3],
                    (const T*)A->ptr[4], PushParam<false>{});
  return launch_k(k_spmv_ell<T, false, PUSH, ATOM>, dim3(grid), dim3(kEllThreads), s, (const int*)A->ptr[0],
                  (const T*)A->ptr[1], x, y, A->m, A->pitch, K, S, early_trigger, (const int*)nullptr,
                  (const int*)nullptr, (const T*)nullptr, push);
}

template <typename T, bool PUSH>
cudaError_t launch_csr_stream(const int* rp, const int* col, const T* val, const T* x, T* y, long long m, long long z,
                              cudaStream_t s, PushParam<PUSH> push) {
  const long long groups = ceil_div(m, 32);
  const long long windows = ceil_div(z, 32 * stream_u<T>());  // ~ windows over all groups
  const int S = split_factor(groups * 32, ceil_div(windows, groups), 1, kSWarps);
  const long long niter = ceil_div(groups, kSWarps / S);
  const int grid = (int)(niter < (long long)kSMs * stream_ctas<T>() ? niter : (long long)kSMs * stream_ctas<T>());
  return launch_k(k_spmv_csr_stream<T, PUSH>, dim3(grid < 1 ? 1 : grid), dim3(kSThreads), s, rp, col, val, x, y, m, S,
                  push);
}

// consecutive-row DIA (k_spmv_dia_v4): fp32 by default (SFS_DIA_F4=0 disables), fp64 on request
// (SFS_DIA_V4_F64=1) -- A/B switches
bool dia_v4_enabled(size_t elem) {
  static const bool f32 = [] {
    const char* e = getenv("SFS_DIA_F4");
    return !(e && e[0] == '0');
  }();
  static const bool f64 = [] {
    const char* d = getenv("SFS_DIA_V4_F64");
    return d && d[0] == '1';
  }();
  return elem == 4 ? f32 : f64;
}

template <typename T, bool PUSH>
cudaError_t launch_dia(const Matrix* A, const T* x, T* y, cudaStream_t s, PushParam<PUSH> push) {
  const long long m = A->m;
  const long long blocks_rows = ceil_div(m, dia_rows<T>());  // threads needed at S = 1
  int S = split_factor(blocks_rows, A->ndiag, 2 * dia_batch<T>(), 16);
  // bandwidth-bound fp64: parts of ~12+ diagonals stream faster than one long walk (measured, cold,
  // tools/micro.py: 128^3 27-point S 1 -> 2: 0.91 -> 0.93 of peak; 1M-row band of 49 diagonals S 2 -> 4:
  // 0.73 -> 0.80); fp32 keeps the latency rule (its S = 1 is fastest)
  if (sizeof(T) == 8)
    while (S < 16 && A->ndiag / (2 * S) >= 12) S <<= 1;
  static const int force_s = [] {  // SFS_DIA_S: A/B override of the diagonal split (1, 2, 4, 8, 16)
    const char* e = getenv("SFS_DIA_S");
    return e ? atoi(e) : -1;
  }();
  if (force_s == 1 || force_s == 2 || force_s == 4 || force_s == 8 || force_s == 16) S = force_s;
  const long long nblk = ceil_div(m, (long long)(kDiaThreads / S) * dia_rows<T>());
  const int grid = (int)(nblk < (long long)kSMs * dia_ctas<T>() ? nblk : (long long)kSMs * dia_ctas<T>());
  const dim3 gd(grid < 1 ? 1 : grid), bd(kDiaThreads);
  const int* offs = (const int*)A->ptr[0];
  const T* dv = (const T*)A->ptr[1];
  const int nd = (int)A->ndiag;
  if constexpr (!PUSH) {
    // the TMA kernel for matrices of >= SFS_DIA_SX_MIN blocks of kSxRows rows (< 0: never).  Corpus-200
    // DIA race (race_probe, us/rep): never 874, >= 296 blocks 816, 148: 802, 64: 800, 16: 820
    static const long long sx_min = [] {
      const char* e = getenv("SFS_DIA_SX_MIN");
      return e ? atoll(e) : 64LL;
    }();
    // ... with >= SFS_DIA_TMA_ND (12) diagonals: with few diagonals per row block the ring never fills and the x
    // windows cost as much as the slab (corpus-2000: 2D 5-point 1.6-2.3x, 3D 7-point 1.2-1.6x, 3-diagonal
    // bands 1.2-1.7x slower than the register kernels; 27-point stencils and bands of >= 17 diagonals faster)
    static const int tma_nd = [] {  // corpus-200 / corpus-2000 DIA race: >= 12 best (12: 802 / 1945, 16: 811 / 1945, 24: 822 / 1951 us/rep)
      const char* e = getenv("SFS_DIA_TMA_ND");
      return e ? atoi(e) : 12;
    }();
    const long long nsx = ceil_div(m, (long long)kSxRows);
    if (sx_min >= 0 && nsx >= sx_min && nd >= tma_nd && nd >= 1 && nd <= kDiaSmemOffs && ((uintptr_t)x % 16) == 0) {
      // TMA-streamed slab: 8 consumer warps + 1 producer warp per CTA
      static std::once_flag attr_once[kMaxDevices];
      int dev = 0;
      if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= kMaxDevices) return cudaErrorInvalidDevice;
      std::call_once(attr_once[dev], [] {
        cudaFuncSetAttribute(k_spmv_dia_tma<T>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)dia_tma_smem<T>());
      });
      constexpr int per_sm = (int)((228 * 1024) / (dia_tma_smem<T>() + 10 * 1024)) < 1
                                 ? 1 : (int)((228 * 1024) / (dia_tma_smem<T>() + 10 * 1024));  // smem-bound
      const int gt = (int)(nsx < (long long)kSMs * per_sm ? nsx : (long long)kSMs * per_sm);
      return launch_k_smem(k_spmv_dia_tma<T>, dim3(gt), dim3(kTThreadsAll), dia_tma_smem<T>(), s, offs, dv, x, y, m,
                           A->n, A->pitch, nd);
    }
  }
  if (dia_v4_enabled(sizeof(T))) {
    // L2 prefetch of the next batch's slab (SFS_DIA_PF: distance in batches, 0 = off; A/B switch).
    // 128^3 fp32 stencil cold (tools/ab_dia_pf.sh): off 54.3 us (0.69), 1: 52.2 us (0.71), 2: 53.2, 3: 55.3
    static const int pfd = [] {
      const char* e = getenv("SFS_DIA_PF");
      return e ? atoi(e) : 1;
    }();
    // same split rule; 4 consecutive rows per thread (G * 4 rows per block, as the strided mapping)
    const int g4 = (int)(nblk < (long long)kSMs * SFS_DIA_V4_CTAS ? nblk : (long long)kSMs * SFS_DIA_V4_CTAS);
    const dim3 gd(g4 < 1 ? 1 : g4);
    if constexpr (sizeof(T) == 4) {
      static const bool xa = [] {  // SFS_DIA_XA=0: 4 scalar x loads per diagonal (A/B)
        const char* e = getenv("SFS_DIA_XA");
        return !(e && e[0] == '0');
      }();
      if (xa && ((uintptr_t)x % 16) == 0) {
        switch (S) {
          case 1: return launch_k(k_spmv_dia_v4<T, 1, PUSH, true>, gd, bd, s, offs, dv, x, y, m, A->n, A->pitch, nd, push, pfd);
          case 2: return launch_k(k_spmv_dia_v4<T, 2, PUSH, true>, gd, bd, s, offs, dv, x, y, m, A->n, A->pitch, nd, push, pfd);
          case 4: return launch_k(k_spmv_dia_v4<T, 4, PUSH, true>, gd, bd, s, offs, dv, x, y, m, A->n, A->pitch, nd, push, pfd);
          case 8: return launch_k(k_spmv_dia_v4<T, 8, PUSH, true>, gd, bd, s, offs, dv, x, y, m, A->n, A->pitch, nd, push, pfd);
          default: return launch_k(k_spmv_dia_v4<T, 16, PUSH, true>, gd, bd, s, offs, dv, x, y, m, A->n, A->pitch, nd, push, pfd);
        }
      }
    }
    switch (S) {
      case 1: return launch_k(k_spmv_dia_v4<T, 1, PUSH>, gd, bd, s, offs, dv, x, y, m, A->n, A->pitch, nd, push, pfd);
      case 2: return launch_k(k_spmv_dia_v4<T, 2, PUSH>, gd, bd, s, offs, dv, x, y, m, A->n, A->pitch, nd, push, pfd);
      case 4: return launch_k(k_spmv_dia_v4<T, 4, PUSH>, gd, bd, s, offs, dv, x, y, m, A->n, A->pitch, nd, push, pfd);
      case 8: return launch_k(k_spmv_dia_v4<T, 8, PUSH>, gd, bd, s, offs, dv, x, y, m, A->n, A->pitch, nd, push, pfd);
      default: return launch_k(k_spmv_dia_v4<T, 16, PUSH>, gd, bd, s, offs, dv, x, y, m, A->n, A->pitch, nd, push, pfd);
    }
  }
  switch (S) {
    case 1: return launch_k(k_spmv_dia<T, 1, PUSH>, gd, bd, s, offs, dv, x, y, m, A->n, A->pitch, nd, push);
    case 2: return launch_k(k_spmv_dia<T, 2, PUSH>, gd, bd, s, offs, dv, x, y, m, A->n, A->pitch, nd, push);
    case 4: return launch_k(k_spmv_dia<T, 4, PUSH>, gd, bd, s, offs, dv, x, y, m, A->n, A->pitch, nd, push);
    case 8: return launch_k(k_spmv_dia<T, 8, PUSH>, gd, bd, s, offs, dv, x, y, m, A->n, A->pitch, nd, push);
    default: return launch_k(k_spmv_dia<T, 16, PUSH>, gd, bd, s, offs, dv, x, y, m, A->n, A->pitch, nd, push);
  }
}

// HYB with long overflow rows: overlapped parts (SFS_HYB_OVERLAP=0: the ELL part -> COO<ACCUM> pair)
bool hyb_overlap() {
  static const bool v = [] {
    const char* e = getenv("SFS_HYB_OVERLAP");
    return !(e && e[0] == '0');
  }();
  return v;
}

template <typename T>
cudaError_t spmv_t(const Matrix* A, const T* x, T* y, cudaStream_t s) {
  const long long m = A->m, z = A->nnz;
  cudaError_t e = cudaSuccess;
  switch (A->fmt) {
    case SFS_CSR: {
      const int* rp = (const int*)A->ptr[0];
      const int* col = (const int*)A->ptr[1];
      const T* val = (const T*)A->ptr[2];
      if (A->variant == 3 || A->variant == 4 || A->variant == 5) {
        if (z == 0) {
          e = launch_zero<T>(y, m, s);
          break;
        }
        const TileGeom g = tile_geom(z);
        TileWork w = tile_work(A->work, g);
        // small matrices: fewer warps per CTA so that the CTAs cover >= 2 x 148 SMs where possible
        int tpb = kTThreads;
        while (tpb > 64 && ceil_div(g.nwarps, tpb / 32) < 2 * kSMs) tpb >>= 1;
        const dim3 grid((unsigned)ceil_div(g.nwarps, tpb / 32));
        // borrowed arrays (e.g. a row block of a larger CSR) may not be 32 B aligned: scalar loads
        const bool vec = ((((uintptr_t)col) | ((uintptr_t)val)) % 32) == 0;
        // next-chunk L2 prefetch above SFS_TILE_PF_MB of footprint (default 256 = 2 x L2; < 0: never).
        // Cold, tools/ab_tile_pf.sh: 1M-row band fp64 0.81 -> 0.85 of peak; applied to every matrix the
        // corpus CSR race got 2.5 % slower (L2-resident matrices), hence the gate.
        static const long long pf_mb = [] {
          const char* ev = getenv("SFS_TILE_PF_MB");
          return ev ? atoll(ev) : 256LL;
        }();
        const long long foot = 4 * (m + 1) + (4 + (long long)sizeof(T)) * z + (long long)sizeof(T) * (A->n + m);
        const int pf = pf_mb >= 0 && foot > pf_mb * (1ll << 20);
        auto go = [&](auto kern) {
          return launch_k(kern, grid, dim3(tpb), s, rp, col, val, x, y, m, z, g.cpw, g.nwarps, (const int*)w.a,
                          (const int*)w.srow, (const unsigned*)w.bm, (const unsigned short*)w.pb, pf, (const int*)w.ne);
        };
        if (A->variant == 5) {  // empty rows: all of y zeroed ahead (PDL-overlapped), ranks mapped to rows
          e = launch_zero<T>(y, m, s);
          if (e == cudaSuccess)
            e = vec ? go(k_spmv_csr_tile<T, true, true, true>) : go(k_spmv_csr_tile<T, false, true, true>);
          break;
        }
        e = launch_k(k_zero_rows<T>, dim3(grid_cap(g.nwarps, 256, 4)), dim3(256), s, y, (const int*)w.srow, g.nwarps, m);
        if (e == cudaSuccess) {
          if (A->variant == 4) e = vec ? go(k_spmv_csr_tile<T, true, true>) : go(k_spmv_csr_tile<T, false, true>);
          else e = vec ? go(k_spmv_csr_tile<T, true, false>) : go(k_spmv_csr_tile<T, false, false>);
        }
      } else if (A->variant == 2) {
        const long long groups = ceil_div(m, 32);
        const long long windows = ceil_div(z, 32 * stream_u<T>());  // ~ windows over all groups
        const int S = split_factor(groups * 32, ceil_div(windows, groups), 1, kSWarps);
        const long long niter = ceil_div(groups, kSWarps / S);
        const int grid = (int)(niter < (long long)kSMs * stream_ctas<T>() ? niter : (long long)kSMs * stream_ctas<T>());
        e = launch_csr_stream<T, false>(rp, col, val, x, y, m, z, s, PushParam<false>{});
      } else if (A->variant == 0) {
        // kCsrWarps warps grid-stride over rows (the mapping the csr_max feature describes, Q4); a
        // matrix covered in one pass gets only the warps that own rows (same row -> warp mapping).
        const int tpv = csr_vector_tpv(m, z);
        const long long warps_needed = ceil_div(m, 32 / tpv);
        const int blocks = (int)ceil_div(warps_needed < kCsrWarps ? warps_needed : kCsrWarps, 256 / 32);
        switch (tpv) {
          case 2: e = launch_k(k_spmv_csr_vector<T, 2>, dim3(blocks), dim3(256), s, rp, col, val, x, y, m); break;
          case 4: e = launch_k(k_spmv_csr_vector<T, 4>, dim3(blocks), dim3(256), s, rp, col, val, x, y, m); break;
          case 8: e = launch_k(k_spmv_csr_vector<T, 8>, dim3(blocks), dim3(256), s, rp, col, val, x, y, m); break;
          case 16: e = launch_k(k_spmv_csr_vector<T, 16>, dim3(blocks), dim3(256), s, rp, col, val, x, y, m); break;
          default: e = launch_k(k_spmv_csr_vector<T, 32>, dim3(blocks), dim3(256), s, rp, col, val, x, y, m); break;
        }
      } else {
        const long long tiles = ceil_div(m + z, kMTile);
        MergeWork w = merge_work(A->work, tiles);
        e = launch_k(k_spmv_csr_merge<T>, dim3((unsigned)tiles), dim3(kMT), s, rp, col, val, x, y, m, z, w.coords,
                     w.crow, w.cval);
        if (e == cudaSuccess)
          e = launch_k(k_spmv_csr_merge_fixup<T>, dim3(grid_cap(tiles, 256, 4)), dim3(256), s, (const int*)w.crow,
                       (const acc_t*)w.cval, tiles, m, y);
      }
      break;
    }
    case SFS_COO: {
      e = launch_zero<T>(y, m, s);
      if (e == cudaSuccess && z > 0)
        e = launch_coo<T, false>((const int*)A->ptr[0], (const int*)A->ptr[1], (const T*)A->ptr[2], x, y, z, s);
      break;
    }
    case SFS_ELL:
    case SFS_HYB: {
      const int K = (int)A->width;
      const bool two = A->fmt == SFS_HYB && A->coo_nnz > 0 && A->variant == 0;  // ELL part -> COO part
      if (two && K > 0 && hyb_overlap()) {
        // zero -> ELL part (atomic adds, releases the COO part at its start) -> COO part (atomic adds,
        // waits for the ELL part only before it exits): the two parts run concurrently
        e = launch_zero<T>(y, m, s);
        if (e == cudaSuccess) e = launch_ell<T, false, true>(A, x, y, K, s, 1);
        if (e == cudaSuccess)
          e = launch_coo<T, true, true>((const int*)A->ptr[2], (const int*)A->ptr[3], (const T*)A->ptr[4], x, y,
                                        A->coo_nnz, s);
        break;
      }
      e = K == 0 ? launch_zero<T>(y, m, s) : launch_ell<T>(A, x, y, K, s, two);
      if (e == cudaSuccess && two)
        e = launch_coo<T, true>((const int*)A->ptr[2], (const int*)A->ptr[3], (const T*)A->ptr[4], x, y, A->coo_nnz, s);
      break;
    }
    case SFS_DIA:
      e = launch_dia<T, false>(A, x, y, s, PushParam<false>{});
      break;
    default:
      return cudaErrorInvalidValue;
  }
  return e;
}

// Cold-cache mode: stream a 2x-L2 buffer through L2 with plain reads (clean lines, so the next SpMV
// does not pay dirty write-backs); the sink store is never taken unless the buffer holds NaN bits.
__global__ void k_l2_flush(const uint4* __restrict__ buf, long long n16, unsigned* __restrict__ sink) {
  unsigned acc = 0;
  for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < n16; i += (long long)gridDim.x * blockDim.x) {
    const uint4 v = __ldcg(buf + i);
    acc ^= v.x ^ v.y ^ v.z ^ v.w;
  }
  if (acc == 0x7fc00001u) sink[0] = acc;
}

template <typename T>
__global__ void k_fill(T* __restrict__ p, long long n, T v) {
  for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) p[i] = v;
}

}  // namespace

int csr_vector_tpv(long long m, long long z) {
  const long long avg = z / m;
  return avg <= 2 ? 2 : avg <= 4 ? 4 : avg <= 8 ? 8 : avg <= 16 ? 16 : 32;
}

size_t csr_merge_work_bytes(long long m, long long z, int dtype) {
  (void)dtype;
  const long long tiles = ceil_div(m + z, kMTile);
  return al256(sizeof(int2) * (tiles + 1)) + al256(sizeof(int) * tiles) + al256(sizeof(acc_t) * tiles);
}

cudaError_t launch_csr_merge_prepare(const int* rp, long long m, long long z, void* work, cudaStream_t s) {
  const long long tiles = ceil_div(m + z, kMTile);
  MergeWork w = merge_work(work, tiles);
  (void)launch_dep(k_merge_partition, dim3(grid_cap(tiles + 1, 256, 8)), dim3(256), 0, s, rp, m, z, kMTile, w.coords, tiles);
  count_launch();
  return cudaGetLastError();
}

// bitmap: 0 = variant 3, 1 = variant 4 (row-start bitmap), 2 = variant 5 (bitmap over the non-empty rows
// + rank -> row map)
size_t csr_tile_work_bytes(long long m, long long z, int bitmap) {
  const TileGeom g = tile_geom(z);
  return al256(sizeof(int) * (g.nchunks + 1)) + al256(sizeof(int) * g.nwarps) +
         (bitmap ? al256(sizeof(unsigned) * g.nchunks * (kTChunk / 32)) + al256(sizeof(unsigned short) * g.nchunks * 32) : 0) +
         (bitmap == 2 ? al256(sizeof(int) * m) : 0);
}

cudaError_t launch_csr_tile_prepare(const int* rp, long long m, long long z, void* work, int bitmap, cudaStream_t s) {
  const TileGeom g = tile_geom(z);
  TileWork w = tile_work(work, g);
  (void)launch_dep(k_csr_tile_partition, dim3(grid_cap(m + 1, 256, 8)), dim3(256), 0, s, rp, m, g.nchunks, w.a);
  count_launch();
  (void)launch_dep(k_tile_split_rows, dim3(grid_cap(g.nwarps, 256, 8)), dim3(256), 0, s, rp, w.a, m, g.cpw, g.nwarps, w.srow);
  count_launch();
  if (bitmap) {
    cudaError_t e = cudaMemsetAsync(w.bm, 0, sizeof(unsigned) * g.nchunks * (kTChunk / 32), s);
    count_launch();
    if (e != cudaSuccess) return e;
    int* pos = nullptr;
    void* sw = nullptr;
    if (bitmap == 2) {  // ranks of the non-empty rows
      pos = (int*)dalloc(sizeof(int) * (m + 1), s);
      sw = dalloc(scan_work_bytes(m), s);
      if (!pos || !sw) {
        dfree(pos, s);
        dfree(sw, s);
        return cudaErrorMemoryAllocation;
      }
      e = launch_nonempty_scan(rp, m, pos, sw, s);
      if (e != cudaSuccess) return e;
    }
    (void)launch_dep(k_row_starts, dim3(grid_cap(m, 256, 8)), dim3(256), 0, s, rp, m, w.bm, pos, bitmap == 2 ? w.ne : nullptr);
    count_launch();
    (void)launch_dep(k_tile_pack, dim3(grid_cap(g.nchunks, 256, 8)), dim3(256), 0, s, w.bm, g.nchunks, w.pb);
    count_launch();
    if (bitmap == 2) {
      const long long items = std::max(g.nchunks + 1, g.nwarps);
      (void)launch_dep(k_tile_rank, dim3(grid_cap(items, 256, 8)), dim3(256), 0, s, pos, m, w.a, g.nchunks, w.srow, g.nwarps);
      count_launch();
      dfree(pos, s);
      dfree(sw, s);
    }
  }
  return cudaGetLastError();
}

// One-launch HYB when the overflow per row is short: <= 32 entries (<= 64 below 2^20 nnz), the walk
// shared by the slot-parts.  Measured on 50 corpus-200 matrices with a COO part (tools/hyb_ab.sh,
// profiles/r01/csr_variants.txt): HYB race time -4.8 % against the previous rule (<= 4, or <= 32
// below 2^20) and -10 % against always two kernels; rows overflowing by thousands (power-law) keep
// the ELL-part -> COO-part pair.
int hyb_rowwise(long long nnz_max, long long K, long long coo_nnz, long long z) {
  const long long o = nnz_max - K;
  struct Lim { long long small, large; };
  static const Lim lim = [] {  // SFS_HYB_ROWWISE="small,large": A/B overrides of the limits
    Lim l{kHybRowwiseSmall, kHybRowwiseLarge};
    const char* e = getenv("SFS_HYB_ROWWISE");
    if (e) sscanf(e, "%lld,%lld", &l.small, &l.large);
    return l;
  }();
  const long long small = lim.small, large = lim.large;
  return coo_nnz > 0 && (o <= large || (z < (1LL << 20) && o <= small));
}

int spmv_kernels_per_call(const Matrix* A) {
  switch (A->fmt) {
    case SFS_CSR: return (A->variant == 1 || ((A->variant >= 3 && A->variant <= 5) && A->nnz > 0)) ? 2 : 1;
    case SFS_COO: return A->nnz > 0 ? 2 : 1;
    case SFS_HYB: return (A->coo_nnz > 0 && A->variant == 0) ? (A->width > 0 && hyb_overlap() ? 3 : 2) : 1;
    default: return 1;
  }
}

cudaError_t launch_spmv(const Matrix* A, const void* x, void* y, cudaStream_t s) {
  if (A->dtype == SFS_F64) return spmv_t<double>(A, (const double*)x, (double*)y, s);
  return spmv_t<float>(A, (const float*)x, (float*)y, s);
}

cudaError_t launch_l2_flush(const void* buf, size_t bytes, cudaStream_t s) {
  k_l2_flush<<<kSMs * 8, 256, 0, s>>>((const uint4*)buf, (long long)(bytes / 16), (unsigned*)buf);
  count_launch();
  return cudaGetLastError();
}

template <typename T>
cudaError_t spmv_push_t(const Matrix* A, const T* x, T* y, const sfs_push_t& h, cudaStream_t s) {
  const PushParam<true> p = push_param(h);
  if (A->fmt == SFS_DIA && A->ndiag > 0) return launch_dia<T, true>(A, x, y, s, p);
  if (A->fmt == SFS_ELL && A->width > 0) return launch_ell<T, true>(A, x, y, (int)A->width, s, 0, p);
  if (A->fmt == SFS_CSR && A->variant == 2 && A->m > 0)
    return launch_csr_stream<T, true>((const int*)A->ptr[0], (const int*)A->ptr[1], (const T*)A->ptr[2], x, y, A->m,
                                      A->nnz, s, p);
  // kernels that do not own their rows (atomics, carries): wait kernel -> SpMV -> push kernel
  cudaError_t e = cudaSuccess;
  if (p.nwait > 0) e = launch_k(k_halo_wait, dim3(1), dim3(32), s, p);
  if (e == cudaSuccess) e = spmv_t<T>(A, x, y, s);
  if (e == cudaSuccess) {
    PushParam<true> q = p;
    q.nwait = 0;
    long long most = 0;
    for (int i = 0; i < h.nseg; i++) most = std::max(most, (long long)(h.seg_end[i] - h.seg_begin[i]));
    e = launch_k(k_halo_push<T>, dim3(grid_cap(most, 256, 2)), dim3(256), s, (const T*)y, q);
  }
  return e;
}

cudaError_t launch_spmv_push(const Matrix* A, const void* x, void* y, const sfs_push_t& p, cudaStream_t s) {
  if (A->dtype == SFS_F64) return spmv_push_t<double>(A, (const double*)x, (double*)y, p, s);
  return spmv_push_t<float>(A, (const float*)x, (float*)y, p, s);
}

cudaError_t launch_halo_push(int dtype, const void* src, long long nrows, const sfs_push_t& h, cudaStream_t s) {
  const PushParam<true> p = push_param(h);
  long long most = 0;
  for (int i = 0; i < h.nseg; i++) most = std::max(most, (long long)(h.seg_end[i] - h.seg_begin[i]));
  (void)nrows;
  const dim3 g(grid_cap(most, 256, 2));
  if (dtype == SFS_F64) return launch_k(k_halo_push<double>, g, dim3(256), s, (const double*)src, p);
  return launch_k(k_halo_push<float>, g, dim3(256), s, (const float*)src, p);
}

cudaError_t launch_fill(int dtype, void* p, long long n, double v, cudaStream_t s) {
  if (n <= 0) return cudaSuccess;
  const int g = (int)(ceil_div(n, 256) < kSMs * 8 ? ceil_div(n, 256) : kSMs * 8);
  if (dtype == SFS_F64) k_fill<double><<<g, 256, 0, s>>>((double*)p, n, v);
  else k_fill<float><<<g, 256, 0, s>>>((float*)p, n, (float)v);
  count_launch();
  return cudaGetLastError();
}

}  // namespace sfs
