// spmv.cu — per-format y = A·x (§1; formats L73 §2.1; step (iii) of L331 §5.4).
//
// SpMV is HBM-bound (0.10–0.46 flop/B): every kernel streams the format's arrays once with
// L1-bypassing loads (ld.global.nc.L1::no_allocate) and gathers x through L1/L2 (__ldg).  No tensor
// cores: the path is not a dense contraction.  Products and sums are formed in fp64 for both value
// types (an fp32 product is exact in fp64), so fp32 rows of ~10^5 entries stay within the 1e-5
// per-row tolerance; y is rounded once to its dtype.
//   CSR vector : TPV lanes per row (TPV from floor(z/m)), grid of 148*64 warps (the csr_max
//                feature, Q4), shuffle reduction.
//   CSR merge  : merge-path tiles over (row ends + nnz), products staged in smem, block-wide
//                segmented scan of thread carries, one carry per tile added by a fix-up kernel.
//   COO        : each warp owns a contiguous range of 128-item chunks (4 items per lane, 128-bit
//                loads), warp segmented reduction by row; rows are stored directly except the
//                range's first row and its final carry (atomicAdd).
//   ELL / HYB  : 4 rows per thread, column-major slab read with 128-bit loads (coalesced per slot);
//                HYB = ELL part (writes y) then COO part (accumulates).
//   DIA        : 4 rows per thread, slab read with 128-bit loads, x through L1.
#include "common.cuh"
#include "internal.h"

namespace sfs {
namespace {

typedef double acc_t;

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
    s += (acc_t)v0 * (acc_t)ld_x(x + c0);
    s += (acc_t)v1 * (acc_t)ld_x(x + c1);
  }
  if (k < e) s += (acc_t)ld_stream(val + k) * (acc_t)ld_x(x + ld_stream(col + k));
  return s;
}

template <typename T, int TPV>
__global__ void __launch_bounds__(256) k_spmv_csr_vector(const int* __restrict__ rp, const int* __restrict__ col,
                                                         const T* __restrict__ val, const T* __restrict__ x,
                                                         T* __restrict__ y, long long m) {
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
  for (long long t = (long long)blockIdx.x * blockDim.x + threadIdx.x; t <= ntiles; t += (long long)gridDim.x * blockDim.x) {
    long long d = t * tile;
    if (d > m + z) d = m + z;
    int xx, yy;
    merge_path_search(d, rp + 1, (int)m, (int)z, xx, yy);
    coords[t] = make_int2(xx, yy);
  }
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
  const long long total = m + z;
  const long long d0 = (long long)blockIdx.x * kMTile;
  const long long d1 = d0 + kMTile < total ? d0 + kMTile : total;
  const int2 c0 = __ldg(coords + blockIdx.x), c1 = __ldg(coords + blockIdx.x + 1);
  const int r0 = c0.x, k0 = c0.y, r1 = c1.x, k1 = c1.y;
  for (int i = threadIdx.x; i <= r1 - r0 + 1 && r0 + i <= m; i += kMT) s_rp[i] = __ldg(rp + r0 + i);
  for (int i = threadIdx.x; i < k1 - k0; i += kMT)
    s_prod[i] = (acc_t)ld_stream(val + k0 + i) * (acc_t)ld_x(x + ld_stream(col + k0 + i));
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
}

template <typename T>
__global__ void k_spmv_csr_merge_fixup(const int* __restrict__ carry_row, const acc_t* __restrict__ carry_val,
                                       long long tiles, long long m, T* __restrict__ y) {
  for (long long t = (long long)blockIdx.x * blockDim.x + threadIdx.x; t < tiles; t += (long long)gridDim.x * blockDim.x) {
    const int r = carry_row[t];
    const acc_t v = carry_val[t];
    if (r < m && v != 0) atomicAdd(y + r, (T)v);
  }
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

template <typename T, bool ACCUM>
__global__ void __launch_bounds__(kCooThreads) k_spmv_coo(const int* __restrict__ row, const int* __restrict__ col,
                                                          const T* __restrict__ val, const T* __restrict__ x,
                                                          T* __restrict__ y, long long z, long long chunks_per_warp) {
  const int l = threadIdx.x & 31;
  const long long nchunks = ceil_div(z, kChunk);
  const long long warp = ((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const long long cb = warp * chunks_per_warp;
  const long long ce = cb + chunks_per_warp < nchunks ? cb + chunks_per_warp : nchunks;
  if (cb >= ce) return;
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
#pragma unroll
      for (int q = 0; q < kCooV / 4; q++) {
        const int4 rr = ld_stream4(row + k + 4 * q), cc = ld_stream4(col + k + 4 * q);
        Vec4<T> vv;
        vv.load_stream(val + k + 4 * q);
        r[4 * q] = rr.x; r[4 * q + 1] = rr.y; r[4 * q + 2] = rr.z; r[4 * q + 3] = rr.w;
        c[4 * q] = cc.x; c[4 * q + 1] = cc.y; c[4 * q + 2] = cc.z; c[4 * q + 3] = cc.w;
#pragma unroll
        for (int i = 0; i < 4; i++) v[4 * q + i] = vv.v[i];
      }
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
    const int rf = r[0], rl = r[kCooV - 1];
    // the previous chunk's carry ends exactly at this chunk boundary: emit it
    const int chunk_first = __shfl_sync(0xffffffffu, rf, 0);
    if (carry_row >= 0 && carry_row != chunk_first) {
      if (l == 0) coo_emit<T, ACCUM>(y, carry_row, carry, carry_row == range_first);
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
        else coo_emit<T, ACCUM>(y, cr, cur, cr == range_first);
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
      coo_emit<T, ACCUM>(y, rf, h, rf == range_first);
    }
    if (l < 31 && next_rf != rl) coo_emit<T, ACCUM>(y, rl, S, rl == range_first);
    carry_row = __shfl_sync(0xffffffffu, rl, 31);  // the chunk's last row stays open
    carry = __shfl_sync(0xffffffffu, S, 31);
  }
  if (l == 0 && carry_row >= 0) atomicAdd(y + carry_row, (T)carry);  // may continue in the next range
}

// ======================================================================== ELL (and the ELL part of HYB)
// Thread = 4 consecutive rows; slots are read in batches of 4 (four 16 B col vectors and four 16/32 B
// val vectors issued before any x gather), grid of one wave striding over row groups.
constexpr int kEllThreads = 256;
constexpr int kEllBatch = 4;

template <typename T>
__global__ void __launch_bounds__(kEllThreads, 4) k_spmv_ell(const int* __restrict__ ecol, const T* __restrict__ eval,
                                                             const T* __restrict__ x, T* __restrict__ y, long long m,
                                                             long long P, int K) {
  const long long groups = P / 4;
  for (long long g = (long long)blockIdx.x * blockDim.x + threadIdx.x; g < groups; g += (long long)gridDim.x * blockDim.x) {
    const long long r = g * 4;
    acc_t acc[4] = {0, 0, 0, 0};
    const int* cp = ecol + r;
    const T* vp = eval + r;
    int j = 0;
    for (; j + kEllBatch <= K; j += kEllBatch) {
      int4 c[kEllBatch];
      Vec4<T> v[kEllBatch];
#pragma unroll
      for (int u = 0; u < kEllBatch; u++) {
        c[u] = ld_stream4(cp + (long long)(j + u) * P);
        v[u].load_stream(vp + (long long)(j + u) * P);
      }
#pragma unroll
      for (int u = 0; u < kEllBatch; u++) {
        if (c[u].x >= 0) acc[0] += (acc_t)v[u].v[0] * (acc_t)ld_x(x + c[u].x);
        if (c[u].y >= 0) acc[1] += (acc_t)v[u].v[1] * (acc_t)ld_x(x + c[u].y);
        if (c[u].z >= 0) acc[2] += (acc_t)v[u].v[2] * (acc_t)ld_x(x + c[u].z);
        if (c[u].w >= 0) acc[3] += (acc_t)v[u].v[3] * (acc_t)ld_x(x + c[u].w);
      }
    }
    for (; j < K; j++) {
      const int4 c = ld_stream4(cp + (long long)j * P);
      Vec4<T> v;
      v.load_stream(vp + (long long)j * P);
      if (c.x >= 0) acc[0] += (acc_t)v.v[0] * (acc_t)ld_x(x + c.x);
      if (c.y >= 0) acc[1] += (acc_t)v.v[1] * (acc_t)ld_x(x + c.y);
      if (c.z >= 0) acc[2] += (acc_t)v.v[2] * (acc_t)ld_x(x + c.z);
      if (c.w >= 0) acc[3] += (acc_t)v.v[3] * (acc_t)ld_x(x + c.w);
    }
#pragma unroll
    for (int q = 0; q < 4; q++)
      if (r + q < m) y[r + q] = (T)acc[q];
  }
}

// ======================================================================== DIA
constexpr int kDiaThreads = 256;
constexpr int kDiaSmemOffs = 1024;
constexpr int kDiaBatch = 4;

template <typename T>
__device__ __forceinline__ void dia_accum(acc_t* acc, const Vec4<T>& v, const T* __restrict__ x, long long c0,
                                          long long n) {
  if (c0 >= 0 && c0 + 3 < n) {
    acc[0] += (acc_t)v.v[0] * (acc_t)ld_x(x + c0);
    acc[1] += (acc_t)v.v[1] * (acc_t)ld_x(x + c0 + 1);
    acc[2] += (acc_t)v.v[2] * (acc_t)ld_x(x + c0 + 2);
    acc[3] += (acc_t)v.v[3] * (acc_t)ld_x(x + c0 + 3);
  } else {
#pragma unroll
    for (int q = 0; q < 4; q++)
      if (c0 + q >= 0 && c0 + q < n) acc[q] += (acc_t)v.v[q] * (acc_t)ld_x(x + c0 + q);
  }
}

template <typename T>
__global__ void __launch_bounds__(kDiaThreads, 4) k_spmv_dia(const int* __restrict__ offs, const T* __restrict__ dval,
                                                             const T* __restrict__ x, T* __restrict__ y, long long m,
                                                             long long n, long long P, int nd) {
  __shared__ int s_off[kDiaSmemOffs];
  const int nsm = nd < kDiaSmemOffs ? nd : kDiaSmemOffs;
  for (int i = threadIdx.x; i < nsm; i += blockDim.x) s_off[i] = offs[i];
  __syncthreads();
  const long long groups = P / 4;
  for (long long g = (long long)blockIdx.x * blockDim.x + threadIdx.x; g < groups; g += (long long)gridDim.x * blockDim.x) {
    const long long r = g * 4;
    acc_t acc[4] = {0, 0, 0, 0};
    const T* vp = dval + r;
    int d = 0;
    for (; d + kDiaBatch <= nd; d += kDiaBatch) {
      Vec4<T> v[kDiaBatch];
#pragma unroll
      for (int u = 0; u < kDiaBatch; u++) v[u].load_stream(vp + (long long)(d + u) * P);
#pragma unroll
      for (int u = 0; u < kDiaBatch; u++) {
        const long long off = d + u < kDiaSmemOffs ? s_off[d + u] : __ldg(offs + d + u);
        dia_accum<T>(acc, v[u], x, r + off, n);
      }
    }
    for (; d < nd; d++) {
      Vec4<T> v;
      v.load_stream(vp + (long long)d * P);
      const long long off = d < kDiaSmemOffs ? s_off[d] : __ldg(offs + d);
      dia_accum<T>(acc, v, x, r + off, n);
    }
#pragma unroll
    for (int q = 0; q < 4; q++)
      if (r + q < m) y[r + q] = (T)acc[q];
  }
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

int grid_cap(long long items, int threads, int per_sm) {
  long long g = ceil_div(items, threads), cap = (long long)kSMs * per_sm;
  return (int)(g > cap ? cap : (g < 1 ? 1 : g));
}

// COO launch geometry: contiguous chunk ranges, at most 148*16 CTAs of 8 warps.
template <typename T, bool ACCUM>
void launch_coo(const int* row, const int* col, const T* val, const T* x, T* y, long long z, cudaStream_t s) {
  const long long nchunks = ceil_div(z, kChunk);
  const long long max_warps = (long long)kSMs * 4 * (kCooThreads / 32);  // one resident wave (<= 64 regs)
  const long long cpw = ceil_div(nchunks, max_warps) < 1 ? 1 : ceil_div(nchunks, max_warps);
  const long long warps = ceil_div(nchunks, cpw);
  const unsigned blocks = (unsigned)ceil_div(warps, kCooThreads / 32);
  k_spmv_coo<T, ACCUM><<<blocks, kCooThreads, 0, s>>>(row, col, val, x, y, z, cpw);
}

template <typename T>
cudaError_t spmv_t(const Matrix* A, const T* x, T* y, cudaStream_t s) {
  const long long m = A->m, z = A->nnz;
  switch (A->fmt) {
    case SFS_CSR: {
      const int* rp = (const int*)A->ptr[0];
      const int* col = (const int*)A->ptr[1];
      const T* val = (const T*)A->ptr[2];
      if (A->variant == 0) {
        // kCsrWarps warps grid-stride over rows (the mapping the csr_max feature describes, Q4); a
        // matrix covered in one pass gets only the warps that own rows (same row -> warp mapping).
        const int tpv = csr_vector_tpv(m, z);
        const long long warps_needed = ceil_div(m, 32 / tpv);
        const int blocks = (int)ceil_div(warps_needed < kCsrWarps ? warps_needed : kCsrWarps, 256 / 32);
        switch (tpv) {
          case 2: k_spmv_csr_vector<T, 2><<<blocks, 256, 0, s>>>(rp, col, val, x, y, m); break;
          case 4: k_spmv_csr_vector<T, 4><<<blocks, 256, 0, s>>>(rp, col, val, x, y, m); break;
          case 8: k_spmv_csr_vector<T, 8><<<blocks, 256, 0, s>>>(rp, col, val, x, y, m); break;
          case 16: k_spmv_csr_vector<T, 16><<<blocks, 256, 0, s>>>(rp, col, val, x, y, m); break;
          default: k_spmv_csr_vector<T, 32><<<blocks, 256, 0, s>>>(rp, col, val, x, y, m); break;
        }
        count_launch();
      } else {
        const long long tiles = ceil_div(m + z, kMTile);
        MergeWork w = merge_work(A->work, tiles);
        k_spmv_csr_merge<T><<<(unsigned)tiles, kMT, 0, s>>>(rp, col, val, x, y, m, z, w.coords, w.crow, w.cval);
        k_spmv_csr_merge_fixup<T><<<grid_cap(tiles, 256, 4), 256, 0, s>>>(w.crow, w.cval, tiles, m, y);
        count_launch(2);
      }
      break;
    }
    case SFS_COO: {
      cudaError_t e = cudaMemsetAsync(y, 0, sizeof(T) * m, s);
      if (e != cudaSuccess) return e;
      count_launch();
      if (z > 0) {
        launch_coo<T, false>((const int*)A->ptr[0], (const int*)A->ptr[1], (const T*)A->ptr[2], x, y, z, s);
        count_launch();
      }
      break;
    }
    case SFS_ELL:
    case SFS_HYB: {
      const int K = (int)A->width;
      if (K == 0) {
        cudaError_t e = cudaMemsetAsync(y, 0, sizeof(T) * m, s);
        if (e != cudaSuccess) return e;
      } else {
        k_spmv_ell<T><<<grid_cap(A->pitch / 4, kEllThreads, 4), kEllThreads, 0, s>>>(
            (const int*)A->ptr[0], (const T*)A->ptr[1], x, y, m, A->pitch, K);
      }
      count_launch();
      if (A->fmt == SFS_HYB && A->coo_nnz > 0) {
        launch_coo<T, true>((const int*)A->ptr[2], (const int*)A->ptr[3], (const T*)A->ptr[4], x, y, A->coo_nnz, s);
        count_launch();
      }
      break;
    }
    case SFS_DIA: {
      k_spmv_dia<T><<<grid_cap(A->pitch / 4, kDiaThreads, 4), kDiaThreads, 0, s>>>(
          (const int*)A->ptr[0], (const T*)A->ptr[1], x, y, m, A->n, A->pitch, (int)A->ndiag);
      count_launch();
      break;
    }
    default:
      return cudaErrorInvalidValue;
  }
  return cudaGetLastError();
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
  k_merge_partition<<<grid_cap(tiles + 1, 256, 8), 256, 0, s>>>(rp, m, z, kMTile, w.coords, tiles);
  count_launch();
  return cudaGetLastError();
}

int spmv_kernels_per_call(const Matrix* A) {
  switch (A->fmt) {
    case SFS_CSR: return A->variant == 0 ? 1 : 2;
    case SFS_COO: return A->nnz > 0 ? 2 : 1;
    case SFS_HYB: return A->coo_nnz > 0 ? 2 : 1;
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

cudaError_t launch_fill(int dtype, void* p, long long n, double v, cudaStream_t s) {
  if (n <= 0) return cudaSuccess;
  const int g = (int)(ceil_div(n, 256) < kSMs * 8 ? ceil_div(n, 256) : kSMs * 8);
  if (dtype == SFS_F64) k_fill<double><<<g, 256, 0, s>>>((double*)p, n, v);
  else k_fill<float><<<g, 256, 0, s>>>((float*)p, n, (float)v);
  count_launch();
  return cudaGetLastError();
}

}  // namespace sfs
