// features.cu — the Table-1 feature pass (Table 1; cost model P:L146 §4).
//
// Every reduction is over exact integers (atomics on uint64), so the aggregates are
// order-independent and the host-side fp64 formulas (api.cu) are bit-reproducible.
//   k_rowstats  : one pass over row_ptr (4(m+1) B): validation, min/max, S2, the low / high
//                 partition sums of Q3, an exact row-length histogram for lengths < 4096.
//   k_nnzpass   : merge-path tiles over (row ends + nnz) (4(m+1) + 4z B): column validation and the
//                 diagonal bitmap (bit c - r + m - 1), near-diagonal bits staged in shared memory.
//   k_popcount  : number of non-empty diagonals.
//   k_hyb_select: HYB width K (Q6) as an order statistic of the row lengths, plus hyb_coo.
#include "common.cuh"
#include "internal.h"

namespace sfs {

namespace {

constexpr int kRowThreads = 256;
constexpr int kNnzThreads = 256;
constexpr int kNnzIPT = 8;
constexpr int kNnzTile = kNnzThreads * kNnzIPT;
constexpr int kNearBits = 65536;  // shared-memory diagonal window: offsets in [-32768, 32767]
constexpr int kNearWords = kNearBits / 32;

template <typename T>
__device__ __forceinline__ T warp_min(T v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) { T u = __shfl_xor_sync(0xffffffffu, v, o); v = u < v ? u : v; }
  return v;
}
template <typename T>
__device__ __forceinline__ T warp_max(T v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) { T u = __shfl_xor_sync(0xffffffffu, v, o); v = u > v ? u : v; }
  return v;
}

__global__ void __launch_bounds__(kRowThreads) k_rowstats(const int* __restrict__ rp, long long m, long long z,
                                                          DevAggr* __restrict__ ag, unsigned* __restrict__ hist) {
  dep_wait();
  __shared__ unsigned sh_hist[kHistCap + 1];
  __shared__ unsigned long long sh_red[kRowThreads / 32][11];
  for (int i = threadIdx.x; i <= kHistCap; i += blockDim.x) sh_hist[i] = 0;
  __syncthreads();
  unsigned long long mininv = 0, mx = 0, S2 = 0, cL = 0, s1L = 0, s2L = 0, cH = 0, s1H = 0, s2H = 0, bc = 0,
                     bs = 0, flags = 0;
  const long long stride = (long long)gridDim.x * blockDim.x;
  for (long long r = (long long)blockIdx.x * blockDim.x + threadIdx.x; r < m; r += stride) {
    int a = rp[r], b = rp[r + 1];
    if (r == 0 && a != 0) flags |= FLAG_RP0;
    if (r == m - 1 && (long long)b != z) flags |= FLAG_RP_END;
    long long len = (long long)b - (long long)a;
    if (len < 0) { flags |= FLAG_RP_DECREASE; continue; }
    unsigned long long L = (unsigned long long)len;
    unsigned long long inv = 2147483647ull - L;
    mininv = inv > mininv ? inv : mininv;
    mx = L > mx ? L : mx;
    S2 += L * L;
    long long lm = len * m;
    if (lm < z) { cL++; s1L += L; s2L += L * L; }         // len < nnz_mu   (Q3, strict)
    else if (lm > z) { cH++; s1H += L; s2H += L * L; }    // len > nnz_mu
    if (len >= kHistCap) { bc++; bs += L; atomicAdd(&sh_hist[kHistCap], 1u); }
    else atomicAdd(&sh_hist[len], 1u);
  }
  // warp then block reduction, one atomic per field per block
  mininv = warp_max(mininv); mx = warp_max(mx);
  S2 = warp_sum(S2); cL = warp_sum(cL); s1L = warp_sum(s1L); s2L = warp_sum(s2L);
  cH = warp_sum(cH); s1H = warp_sum(s1H); s2H = warp_sum(s2H); bc = warp_sum(bc); bs = warp_sum(bs);
  flags = __reduce_or_sync(0xffffffffu, (unsigned)flags);
  const int w = threadIdx.x >> 5, l = threadIdx.x & 31;
  if (l == 0) {
    unsigned long long* o = sh_red[w];
    o[0] = mininv; o[1] = mx; o[2] = S2; o[3] = cL; o[4] = s1L; o[5] = s2L; o[6] = cH; o[7] = s1H; o[8] = s2H;
    o[9] = bc; o[10] = bs | (flags << 58);  // flags ride in the top bits (bs < 2^31 * 2^26 is never reached)
  }
  __syncthreads();
  if (w == 0) {
    unsigned long long v[11];
#pragma unroll
    for (int i = 0; i < 11; i++) v[i] = l < kRowThreads / 32 ? sh_red[l][i] : 0ull;
    unsigned long long fl = v[10] >> 58;
    v[10] &= (1ull << 58) - 1;
    v[0] = warp_max(v[0]); v[1] = warp_max(v[1]);
#pragma unroll
    for (int i = 2; i < 11; i++) v[i] = warp_sum(v[i]);
    fl = __reduce_or_sync(0xffffffffu, (unsigned)fl);
    if (l == 0) {
      atomicMax(&ag->min_inv, v[0]); atomicMax(&ag->max_len, v[1]);
      atomicAdd(&ag->S2, v[2]); atomicAdd(&ag->cL, v[3]); atomicAdd(&ag->s1L, v[4]); atomicAdd(&ag->s2L, v[5]);
      atomicAdd(&ag->cH, v[6]); atomicAdd(&ag->s1H, v[7]); atomicAdd(&ag->s2H, v[8]);
      atomicAdd(&ag->big_cnt, v[9]); atomicAdd(&ag->big_sum, v[10]);
      if (fl) atomicOr(&ag->flags, fl);
    }
  }
  for (int i = threadIdx.x; i <= kHistCap; i += blockDim.x)
    if (sh_hist[i]) atomicAdd(&hist[i], sh_hist[i]);
  dep_trigger();
}

// merge-path tile over (row ends, nnz): column checks + diagonal bitmap
__global__ void __launch_bounds__(kNnzThreads) k_nnzpass(const int* __restrict__ rp, const int* __restrict__ col,
                                                         long long m, long long n, long long z,
                                                         DevAggr* __restrict__ ag, unsigned* __restrict__ bitmap,
                                                         long long words) {
  dep_wait();
  if (ag->flags & (FLAG_RP0 | FLAG_RP_DECREASE | FLAG_RP_END)) return;  // row_ptr invalid: do not walk it
  __shared__ int s_rp[kNnzTile + 2];
  __shared__ int s_col[kNnzTile];
  __shared__ unsigned s_bits[kNearWords];
  __shared__ int s_coord[4];
  const long long total = m + z;
  const long long d0 = (long long)blockIdx.x * kNnzTile;
  const long long d1 = d0 + kNnzTile < total ? d0 + kNnzTile : total;
  if (threadIdx.x < 64) {  // warp 0 finds the tile start, warp 1 its end
    const int wsel = threadIdx.x >> 5;
    int x, y;
    merge_path_search_warp(wsel == 0 ? d0 : d1, rp + 1, (int)m, (int)z, x, y);
    if ((threadIdx.x & 31) == 0) {
      s_coord[wsel * 2] = x;
      s_coord[wsel * 2 + 1] = y;
    }
  }
  for (int i = threadIdx.x; i < kNearWords; i += blockDim.x) s_bits[i] = 0;
  __syncthreads();
  const int r0 = s_coord[0], k0 = s_coord[1], r1 = s_coord[2], k1 = s_coord[3];
  const int nrow = r1 - r0;  // rows whose end lies in the tile (+1 partially open row)
  for (int i = threadIdx.x; i <= nrow + 1 && r0 + i <= m; i += blockDim.x) s_rp[i] = rp[r0 + i];
  for (int i = threadIdx.x; i < k1 - k0; i += blockDim.x) s_col[i] = col[k0 + i];
  __syncthreads();
  // thread-local merge-path search inside the tile
  const int ld = threadIdx.x * kNnzIPT;
  const int tile_items = (int)(d1 - d0);
  unsigned long long flags = 0;
  const long long base = ((m - 1 - kNearBits / 2) >= 0 ? (m - 1 - kNearBits / 2) / 32
                                                         : -((kNearBits / 2 - (m - 1) + 31) / 32)) * 32;
  if (ld < tile_items) {
    int lo = ld - (k1 - k0) > 0 ? ld - (k1 - k0) : 0, hi = ld < nrow ? ld : nrow;
    while (lo < hi) {
      int mid = (lo + hi) >> 1;
      if (s_rp[mid + 1] <= k0 + (ld - mid) - 1) lo = mid + 1; else hi = mid;
    }
    int r = r0 + lo, k = k0 + (ld - lo);
    const int items = tile_items - ld < kNnzIPT ? tile_items - ld : kNnzIPT;
    for (int it = 0; it < items; it++) {
      if (r < m && s_rp[r - r0 + 1] <= k) { r++; continue; }  // row end of r
      if (k >= z) break;
      const int c = s_col[k - k0];
      if (c < 0 || (long long)c >= n) { flags |= FLAG_COL_RANGE; k++; continue; }
      if (k > s_rp[r - r0]) {
        int prev = k - 1 >= k0 ? s_col[k - 1 - k0] : col[k - 1];
        if (prev >= c) flags |= FLAG_COL_ORDER;
      }
      const long long g = (long long)c - r + m - 1;
      const long long loc = g - base;
      if (loc >= 0 && loc < kNearBits) atomicOr(&s_bits[loc >> 5], 1u << (loc & 31));
      else atomicOr(&bitmap[g >> 5], 1u << (g & 31));
      k++;
    }
  }
  unsigned fl = __reduce_or_sync(0xffffffffu, (unsigned)flags);
  if ((threadIdx.x & 31) == 0 && fl) atomicOr(&ag->flags, (unsigned long long)fl);
  __syncthreads();
  for (int i = threadIdx.x; i < kNearWords; i += blockDim.x) {
    unsigned b = s_bits[i];
    long long gw = base / 32 + i;
    if (b && gw >= 0 && gw < words) atomicOr(&bitmap[gw], b);
  }
  dep_trigger();
}

__global__ void k_popcount(const unsigned* __restrict__ bitmap, long long words, DevAggr* __restrict__ ag) {
  dep_wait();
  unsigned long long c = 0;
  for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < words; i += (long long)gridDim.x * blockDim.x)
    c += __popc(bitmap[i]);
  c = warp_sum(c);
  if ((threadIdx.x & 31) == 0 && c) atomicAdd(&ag->ndiag, c);
  dep_trigger();
}

// One CTA of kSelThreads.  j = rmax + 1.  The HYB width rule of Q6 (smallest k >= 1 with R(k) <= rmax,
// R(k) = #rows longer than k) equals max(1, j-th largest row length); zero rows -> 0.  Thread t owns
// histogram bins [kHistCap - 4(t+1), kHistCap - 4t), i.e. thread 0 the longest lengths; a block-wide
// top-down prefix sum of the per-thread counts locates the bin holding the j-th largest length.
constexpr int kSelThreads = kHistCap / 4;
// Thread 0 makes every write to *ag here; it finishes by copying the whole aggregate record into
// host_out (pinned host memory mapped into the device address space; null = the caller copies).
__device__ __forceinline__ void publish(const DevAggr* ag, DevAggr* host_out) {
  if (host_out) *host_out = *ag;
}

__global__ void __launch_bounds__(kSelThreads) k_hyb_select(long long m, long long j, DevAggr* __restrict__ ag,
                                                            const unsigned* __restrict__ hist,
                                                            DevAggr* __restrict__ host_out) {
  dep_wait();
  __shared__ long long s_w[kSelThreads / 32];
  __shared__ long long s_L;
  const int t = threadIdx.x, l = t & 31, w = t >> 5;
  if (t == 0) ag->empty_rows = hist[0];
  const long long mx = (long long)ag->max_len;
  const long long bc = (long long)ag->big_cnt, bs = (long long)ag->big_sum;
  if (mx == 0) {
    if (t == 0) { ag->hyb_k = 0; ag->hyb_coo = 0; publish(ag, host_out); }
    return;
  }
  if (j <= bc) {  // the order statistic lies beyond the exact histogram: host refines
    if (t == 0) { ag->hyb_k = -1; ag->hyb_coo = -1; publish(ag, host_out); }
    return;
  }
  const int hi = kHistCap - 4 * t;  // exclusive
  const int lo = hi - 4;
  unsigned h[4];
#pragma unroll
  for (int q = 0; q < 4; q++) h[q] = hist[lo + q];
  const long long mine = (long long)h[0] + h[1] + h[2] + h[3];
  long long incl = mine;  // inclusive prefix over threads 0..t (top-down)
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const long long u = __shfl_up_sync(0xffffffffu, incl, o);
    if (l >= o) incl += u;
  }
  if (l == 31) s_w[w] = incl;
  if (t == 0) s_L = 0;  // j exceeds the number of rows
  __syncthreads();
  if (w == 0) {
    long long v = s_w[l], x = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const long long u = __shfl_up_sync(0xffffffffu, x, o);
      if (l >= o) x += u;
    }
    s_w[l] = x - v;  // exclusive prefix of the warps before l
  }
  __syncthreads();
  const long long above = bc + s_w[w] + incl - mine;  // rows longer than any bin of this thread
  if (above < j && above + mine >= j) {
    long long cum = above;
    for (int q = 3; q >= 0; q--) {
      cum += h[q];
      if (cum >= j) { s_L = lo + q; break; }
    }
  }
  __syncthreads();
  const long long L = s_L;
  const long long K = L < 1 ? 1 : L;
  unsigned long long coo = 0;
#pragma unroll
  for (int q = 0; q < 4; q++)
    if (lo + q > K) coo += (unsigned long long)(lo + q - K) * h[q];
  coo = warp_sum(coo);
  __syncthreads();
  if (l == 0) s_w[w] = (long long)coo;
  __syncthreads();
  if (w == 0) {
    unsigned long long c = (unsigned long long)s_w[l];
    c = warp_sum(c);
    if (l == 0) {
      ag->hyb_k = K;
      ag->hyb_coo = (long long)c + (bs - K * bc);
      publish(ag, host_out);
    }
  }
  dep_trigger();
}

__global__ void k_len_hist_range(const int* __restrict__ rp, long long m, long long lo, long long hi, long long wdt,
                                 unsigned* __restrict__ hist) {
  dep_wait();
  for (long long r = (long long)blockIdx.x * blockDim.x + threadIdx.x; r < m; r += (long long)gridDim.x * blockDim.x) {
    long long len = (long long)rp[r + 1] - rp[r];
    if (len >= lo && len <= hi) atomicAdd(&hist[(len - lo) / wdt], 1u);
  }
  dep_trigger();
}

__global__ void k_hyb_coo_count(const int* __restrict__ rp, long long m, long long K, long long* out) {
  dep_wait();
  unsigned long long c = 0;
  for (long long r = (long long)blockIdx.x * blockDim.x + threadIdx.x; r < m; r += (long long)gridDim.x * blockDim.x) {
    long long len = (long long)rp[r + 1] - rp[r];
    if (len > K) c += (unsigned long long)(len - K);
  }
  c = warp_sum(c);
  if ((threadIdx.x & 31) == 0 && c) atomicAdd((unsigned long long*)out, c);
  dep_trigger();
}

int grid_for(long long items, int threads, int per_sm) {
  long long g = ceil_div(items, threads);
  long long cap = (long long)kSMs * per_sm;
  if (g > cap) g = cap;
  return (int)(g < 1 ? 1 : g);
}

}  // namespace

size_t feat_work_bytes(long long m, long long n) {
  long long words = ceil_div(m + n - 1, 32);
  return sizeof(DevAggr) + sizeof(unsigned) * (kHistCap + 1 + 3) + sizeof(unsigned) * (size_t)words;
}

void feat_work_bind(FeatWork& w, void* base, long long m, long long n) {
  w.base = base;
  w.bytes = feat_work_bytes(m, n);
  w.aggr = (DevAggr*)base;
  w.hist = (unsigned*)((char*)base + sizeof(DevAggr));
  w.bitmap = w.hist + kHistCap + 1 + 3;
  w.words = ceil_div(m + n - 1, 32);
}

cudaError_t launch_features(const int* rp, const int* col, long long m, long long n, long long z, long long rmax,
                            const FeatWork& w, DevAggr* host_out, cudaStream_t s) {
  cudaError_t e = cudaMemsetAsync(w.base, 0, w.bytes, s);
  if (e != cudaSuccess) return e;
  (void)launch_dep(k_rowstats, dim3(grid_for(m, kRowThreads, 4)), dim3(kRowThreads), 0, s, rp, m, z, w.aggr, w.hist);
  long long tiles = ceil_div(m + z, kNnzTile);
  if (tiles > 0) (void)launch_dep(k_nnzpass, dim3((unsigned)tiles), dim3(kNnzThreads), 0, s, rp, col, m, n, z, w.aggr, w.bitmap, w.words);
  (void)launch_dep(k_popcount, dim3(grid_for(w.words, 256, 8)), dim3(256), 0, s, w.bitmap, w.words, w.aggr);
  (void)launch_dep(k_hyb_select, dim3(1), dim3(kSelThreads), 0, s, m, rmax + 1, w.aggr, w.hist, host_out);
  count_launch(tiles > 0 ? 4 : 3);
  return cudaGetLastError();
}

cudaError_t launch_len_hist_range(const int* rp, long long m, long long lo, long long hi, long long wdt,
                                  unsigned* hist, cudaStream_t s) {
  (void)launch_dep(k_len_hist_range, dim3(grid_for(m, 256, 8)), dim3(256), 0, s, rp, m, lo, hi, wdt, hist);
  count_launch();
  return cudaGetLastError();
}

cudaError_t launch_hyb_coo(const int* rp, long long m, long long K, long long* out, cudaStream_t s) {
  (void)launch_dep(k_hyb_coo_count, dim3(grid_for(m, 256, 8)), dim3(256), 0, s, rp, m, K, out);
  count_launch();
  return cudaGetLastError();
}

}  // namespace sfs
