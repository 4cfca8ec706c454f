// gen_device.cu — the sfsgen generators on the GPU (TEST / BENCH INPUT ONLY; see sfsgen.h).
//
// "host and device must emit bit-identical CSR"; §8(d) C5: the configs[4] corpus is
// "Generated on device per rank" (the host generator needs ~139 s for corpus-2000 on one process, which
// would dominate an 8-rank run sharing the host's cores).  Every entry is the same pure function of
// (seed, row, col) as gen.c: splitmix64 on uint64, U(h) = (h >> 11) * 2^-53, explicitly rounded fp64
// operations (__dadd_rn / __dmul_rn / __ddiv_rn: no FMA contraction) in gen.c's order, the power-law
// threshold table built on the host with the same libm pow and passed in as data, fp32 values as
// round-to-nearest of the fp64 value.  Rows are built count -> scan -> fill; the sampled classes sort
// and deduplicate each row's draws (CUB segmented sort), R-MAT sorts and deduplicates the edge keys
// (CUB radix sort + unique).  Nothing here computes a feature, a conversion or a product.
#include <cuda_runtime.h>
#include <math.h>
#include <stdint.h>
#include <string.h>

#include <cub/cub.cuh>
#include <vector>

#include "sfsgen.h"

namespace {

struct DSpec {
  int cls, dtype;
  uint64_t seed;
  long long m, n, ia, ib;
  double pa;
  const double* T;  // power-law thresholds (device), T[L] for L = 0..cap
  long long cap;
};

__device__ __forceinline__ uint64_t sm64(uint64_t x) {
  x += 0x9E3779B97F4A7C15ULL;
  uint64_t z = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ULL;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
  return z ^ (z >> 31);
}
__device__ __forceinline__ uint64_t H(uint64_t seed, uint64_t a, uint64_t b) {
  return sm64(seed ^ sm64(a ^ sm64(b ^ 0x243F6A8885A308D3ULL)));
}
__device__ __forceinline__ double U(uint64_t h) { return __dmul_rn((double)(h >> 11), 1.0 / 9007199254740992.0); }
__device__ __forceinline__ double value_of(uint64_t seed, long long r, long long c) {
  const double mag = __dadd_rn(0.5, __dmul_rn(0.5, U(H(seed ^ 0xA5ULL, (uint64_t)r, (uint64_t)c))));
  return (H(seed, (uint64_t)r, (uint64_t)c) & 1ULL) ? -mag : mag;
}
__device__ __forceinline__ double entry_value(const DSpec& s, long long r, long long c) {
  switch (s.cls) {
    case SFSGEN_ST2D5: return r == c ? 4.0 : -1.0;
    case SFSGEN_ST3D7: return r == c ? 6.0 : -1.0;
    case SFSGEN_ST3D27: return r == c ? 26.0 : -1.0;
    default: return value_of(s.seed, r, c);
  }
}
__device__ __forceinline__ void store_val(void* val, long long o, int dtype, double v) {
  if (dtype) ((double*)val)[o] = v;
  else ((float*)val)[o] = __double2float_rn(v);
}

// ---------------------------------------------------------------- classes without draws to sort
// band / block-diagonal / stencils: columns come out increasing; cols == nullptr counts only.
__device__ long long row_direct(const DSpec& s, long long r, int* col, void* val) {
  const long long n = s.n;
  long long len = 0;
  auto emit = [&](long long c) {
    if (col) {
      col[len] = (int)c;
      store_val(val, len, s.dtype, entry_value(s, r, c));
    }
    len++;
  };
  switch (s.cls) {
    case SFSGEN_BAND: {
      const long long b = s.ia, lo = r - b < 0 ? 0 : r - b, hi = r + b > n - 1 ? n - 1 : r + b;
      for (long long c = lo; c <= hi; c++)
        if (c == r || U(H(s.seed, (uint64_t)r, (uint64_t)c)) < s.pa) emit(c);
      break;
    }
    case SFSGEN_BLOCKDIAG: {
      const long long B = s.ia, q = r / B, lo = q * B, hi = (q + 1) * B < n ? (q + 1) * B : n;
      for (long long c = lo; c < hi; c++)
        if (c == r || U(H(s.seed, (uint64_t)r, (uint64_t)c)) < s.pa) emit(c);
      break;
    }
    case SFSGEN_ST2D5: {
      const long long N = s.ia, i = r / N, j = r % N;
      const int d[5][2] = {{-1, 0}, {0, -1}, {0, 0}, {0, 1}, {1, 0}};
      for (int t = 0; t < 5; t++) {
        const long long ii = i + d[t][0], jj = j + d[t][1];
        if (ii >= 0 && ii < N && jj >= 0 && jj < N) emit(ii * N + jj);
      }
      break;
    }
    default: {  // ST3D7, ST3D27
      const long long N = s.ia, i = r / (N * N), j = (r / N) % N, k = r % N;
      for (int di = -1; di <= 1; di++)
        for (int dj = -1; dj <= 1; dj++)
          for (int dk = -1; dk <= 1; dk++) {
            if (s.cls == SFSGEN_ST3D7 && (di != 0) + (dj != 0) + (dk != 0) > 1) continue;
            const long long ii = i + di, jj = j + dj, kk = k + dk;
            if (ii >= 0 && ii < N && jj >= 0 && jj < N && kk >= 0 && kk < N) emit((ii * N + jj) * N + kk);
          }
      break;
    }
  }
  return len;
}

__global__ void k_direct_count(DSpec s, int* len) {
  for (long long r = (long long)blockIdx.x * blockDim.x + threadIdx.x; r < s.m; r += (long long)gridDim.x * blockDim.x)
    len[r] = (int)row_direct(s, r, nullptr, nullptr);
}
__global__ void k_direct_fill(DSpec s, const int* rp, int* col, void* val) {
  for (long long r = (long long)blockIdx.x * blockDim.x + threadIdx.x; r < s.m; r += (long long)gridDim.x * blockDim.x) {
    const long long o = rp[r];
    row_direct(s, r, col + o, s.dtype ? (void*)((double*)val + o) : (void*)((float*)val + o));
  }
}

// ---------------------------------------------------------------- uniform / power-law draws
// len0 (draws before dedup); power-law rows with len0 > n/8 take the Bernoulli mode (len0 = 0 here,
// their columns are counted / filled by one CTA each).
__device__ long long draws_of(const DSpec& s, long long r) {
  if (s.cls == SFSGEN_UNIFORM) {
    const double f = __dmul_rn(s.pa, __dadd_rn(0.5, U(H(s.seed, (uint64_t)r, 1ULL << 40))));
    long long len0 = (long long)floor(f);
    return len0 < 1 ? 1 : len0;
  }
  const double u = __dsub_rn(1.0, U(H(s.seed, (uint64_t)r, 1ULL << 40)));  // U1
  long long lo = 2, hi = s.cap < 2 ? 2 : s.cap;
  while (lo < hi) {
    const long long mid = lo + (hi - lo + 1) / 2;
    if (u <= s.T[mid]) lo = mid;
    else hi = mid - 1;
  }
  return lo < s.n ? lo : s.n;
}

__global__ void k_draw_count(DSpec s, long long* len0, int* bern_rows, int* nbern) {
  for (long long r = (long long)blockIdx.x * blockDim.x + threadIdx.x; r < s.m; r += (long long)gridDim.x * blockDim.x) {
    const long long l = draws_of(s, r);
    if (s.cls == SFSGEN_POWERLAW && l > s.n / 8) {
      len0[r] = 0;
      bern_rows[atomicAdd(nbern, 1)] = (int)r;
    } else {
      len0[r] = l;
    }
  }
}
__global__ void k_draw_fill(DSpec s, const long long* off0, int* keys) {
  for (long long r = (long long)blockIdx.x * blockDim.x + threadIdx.x; r < s.m; r += (long long)gridDim.x * blockDim.x) {
    const long long b = off0[r], e = off0[r + 1];
    for (long long k = 0; k < e - b; k++) keys[b + k] = (int)(H(s.seed, (uint64_t)r, (uint64_t)k) % (uint64_t)s.n);
  }
}
__global__ void k_unique_count(DSpec s, const long long* off0, const int* sorted, int* len) {
  for (long long r = (long long)blockIdx.x * blockDim.x + threadIdx.x; r < s.m; r += (long long)gridDim.x * blockDim.x) {
    const long long b = off0[r], e = off0[r + 1];
    int u = 0;
    for (long long k = b; k < e; k++) u += (k == b || sorted[k] != sorted[k - 1]);
    len[r] = u;
  }
}
__global__ void k_unique_fill(DSpec s, const long long* off0, const int* sorted, const int* rp, int* col, void* val) {
  for (long long r = (long long)blockIdx.x * blockDim.x + threadIdx.x; r < s.m; r += (long long)gridDim.x * blockDim.x) {
    const long long b = off0[r], e = off0[r + 1];
    long long o = rp[r];
    for (long long k = b; k < e; k++)
      if (k == b || sorted[k] != sorted[k - 1]) {
        col[o] = sorted[k];
        store_val(val, o, s.dtype, value_of(s.seed, r, sorted[k]));
        o++;
      }
  }
}
// Bernoulli rows: keep c iff U(H(seed, r, c)) < len0 / n (threshold in fp64, IEEE division)
__global__ void k_bern_count(DSpec s, const int* rows, int* len) {
  const long long r = rows[blockIdx.x];
  const double thr = __ddiv_rn((double)draws_of(s, r), (double)s.n);
  int cnt = 0;
  for (long long c = threadIdx.x; c < s.n; c += blockDim.x) cnt += U(H(s.seed, (uint64_t)r, (uint64_t)c)) < thr;
  __shared__ int acc;
  if (threadIdx.x == 0) acc = 0;
  __syncthreads();
  atomicAdd(&acc, cnt);
  __syncthreads();
  if (threadIdx.x == 0) len[r] = acc;
}
__global__ void k_bern_fill(DSpec s, const int* rows, const int* rp, int* col, void* val) {
  const long long r = rows[blockIdx.x];
  const double thr = __ddiv_rn((double)draws_of(s, r), (double)s.n);
  __shared__ int s_w[32];
  __shared__ int s_base;
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, nw = blockDim.x >> 5;
  if (threadIdx.x == 0) s_base = rp[r];
  __syncthreads();
  for (long long c0 = 0; c0 < s.n; c0 += blockDim.x) {  // ordered compaction, one block-chunk at a time
    const long long c = c0 + threadIdx.x;
    const bool keep = c < s.n && U(H(s.seed, (uint64_t)r, (uint64_t)c)) < thr;
    const unsigned bal = __ballot_sync(0xffffffffu, keep);
    if (lane == 0) s_w[w] = __popc(bal);
    __syncthreads();
    int before = 0, total = 0;
    for (int i = 0; i < nw; i++) {
      if (i < w) before += s_w[i];
      total += s_w[i];
    }
    if (keep) {
      const long long o = s_base + before + __popc(bal & ((1u << lane) - 1u));
      col[o] = (int)c;
      store_val(val, o, s.dtype, value_of(s.seed, r, c));
    }
    __syncthreads();
    if (threadIdx.x == 0) s_base += total;
    __syncthreads();
  }
}

// ---------------------------------------------------------------- R-MAT
__global__ void k_rmat_edges(uint64_t seed, int scale, long long ne, double ta, double tb, unsigned long long* keys) {
  for (long long e = (long long)blockIdx.x * blockDim.x + threadIdx.x; e < ne; e += (long long)gridDim.x * blockDim.x) {
    long long r = 0, c = 0;
    for (int l = 0; l < scale; l++) {
      const uint64_t l0 = sm64((uint64_t)(2 * l) ^ 0x243F6A8885A308D3ULL), l1 = sm64((uint64_t)(2 * l + 1) ^ 0x243F6A8885A308D3ULL);
      const double u1 = U(sm64(seed ^ sm64((uint64_t)e ^ l0)));
      const double u2 = U(sm64(seed ^ sm64((uint64_t)e ^ l1)));
      const int rb = u1 >= 0.76;
      const int cb = rb ? (u2 >= tb) : (u2 >= ta);
      r |= (long long)rb << l;
      c |= (long long)cb << l;
    }
    keys[e] = ((unsigned long long)r << 32) | (unsigned long long)c;
  }
}
__global__ void k_rmat_csr(uint64_t seed, long long m, const unsigned long long* keys, const long long* nnz_p, int* rp,
                           int* col, void* val, int dtype) {
  const long long nnz = *nnz_p;
  for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < nnz; i += (long long)gridDim.x * blockDim.x) {
    const long long row = (long long)(keys[i] >> 32), c = (long long)(keys[i] & 0xffffffffULL);
    const long long prev = i ? (long long)(keys[i - 1] >> 32) : -1;
    for (long long rr = prev + 1; rr <= row; rr++) rp[rr] = (int)i;
    if (i == nnz - 1)
      for (long long rr = row + 1; rr <= m; rr++) rp[rr] = (int)nnz;
    col[i] = (int)c;
    store_val(val, i, dtype, value_of(seed, row, c));
  }
}
__global__ void k_fill_int(int* p, long long n, int v) {
  for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) p[i] = v;
}

__global__ void k_vector(uint64_t seed, long long n, int dtype, void* out) {
  for (long long j = (long long)blockIdx.x * blockDim.x + threadIdx.x; j < n; j += (long long)gridDim.x * blockDim.x) {
    const double x = __dsub_rn(__dmul_rn(2.0, U(H(seed ^ 0x78ULL, (uint64_t)j, 0))), 1.0);
    store_val(out, j, dtype, x);
  }
}

// m, n of a spec (the rule of gen.c's sfsgen_dims)
int dims_of(const sfsgen_spec* s, int64_t* m, int64_t* n) {
  switch (s->cls) {
    case SFSGEN_RMAT: *m = *n = (int64_t)1 << s->ia; return 0;
    case SFSGEN_ST2D5: *m = *n = s->ia * s->ia; return 0;
    case SFSGEN_ST3D7:
    case SFSGEN_ST3D27: *m = *n = s->ia * s->ia * s->ia; return 0;
    case SFSGEN_BAND:
    case SFSGEN_BLOCKDIAG:
    case SFSGEN_UNIFORM:
    case SFSGEN_POWERLAW: *m = s->m; *n = s->n; return (s->m >= 1 && s->n >= 1) ? 0 : -1;
    default: return -1;
  }
}

inline unsigned grid_for(long long n) {
  long long g = (n + 255) / 256;
  return (unsigned)(g < 1 ? 1 : (g > 148 * 16 ? 148 * 16 : g));
}

// RAII list of device allocations
struct Bufs {
  std::vector<void*> v;
  void* get(size_t b) {
    void* p = nullptr;
    if (cudaMalloc(&p, b ? b : 16) != cudaSuccess) return nullptr;
    v.push_back(p);
    return p;
  }
  void release(void* p) {  // keep: hand ownership to the caller
    for (auto& q : v)
      if (q == p) q = nullptr;
  }
  ~Bufs() {
    for (void* p : v)
      if (p) cudaFree(p);
  }
};

int scan_lengths(const int* len, int* rp, long long m, cudaStream_t st, Bufs& B) {
  // rp[0] = 0, rp[r+1] = rp[r] + len[r] (int32: the generator refuses nnz >= 2^31 like gen.c)
  size_t tb = 0;
  if (cudaMemsetAsync(rp, 0, sizeof(int), st) != cudaSuccess) return -1;
  cub::DeviceScan::InclusiveSum(nullptr, tb, len, rp + 1, (int)m, st);
  void* t = B.get(tb);
  if (!t) return -1;
  return cub::DeviceScan::InclusiveSum(t, tb, len, rp + 1, (int)m, st) == cudaSuccess ? 0 : -1;
}

}  // namespace

extern "C" {

int sfsgen_generate_device(const sfsgen_spec* sp, sfsgen_csr* out, void* stream) {
  memset(out, 0, sizeof(*out));
  cudaStream_t st = (cudaStream_t)stream;
  int64_t m = 0, n = 0;
  if (dims_of(sp, &m, &n)) return -1;
  Bufs B;
  const size_t vb = sp->dtype ? 8 : 4;
  out->m = m;
  out->n = n;
  out->dtype = sp->dtype;
  DSpec s{sp->cls, sp->dtype, sp->seed, m, n, sp->ia, sp->ib, sp->pa, nullptr, 0};
  int* rp = (int*)B.get(sizeof(int) * (size_t)(m + 1));
  if (!rp) return -1;
  long long nnz = 0;
  int* col = nullptr;
  void* val = nullptr;
  if (sp->cls == SFSGEN_RMAT) {
    if (sp->ia < 1 || sp->ia > 30) return -1;
    const int scale = (int)sp->ia;
    const long long ef = sp->ib > 0 ? sp->ib : 16, ne = (long long)m * ef;
    unsigned long long *k0 = (unsigned long long*)B.get(8 * (size_t)ne), *k1 = (unsigned long long*)B.get(8 * (size_t)ne),
                       *ku = (unsigned long long*)B.get(8 * (size_t)ne);
    long long* dn = (long long*)B.get(sizeof(long long));
    if (!k0 || !k1 || !ku || !dn) return -1;
    k_rmat_edges<<<grid_for(ne), 256, 0, st>>>(sp->seed, scale, ne, 0.57 / 0.76, 0.19 / 0.24, k0);
    cub::DoubleBuffer<unsigned long long> db(k0, k1);
    size_t tb = 0;
    cub::DeviceRadixSort::SortKeys(nullptr, tb, db, (int)ne, 0, 32 + scale, st);
    void* t = B.get(tb);
    if (!t || cub::DeviceRadixSort::SortKeys(t, tb, db, (int)ne, 0, 32 + scale, st) != cudaSuccess) return -1;
    size_t tu = 0;
    cub::DeviceSelect::Unique(nullptr, tu, db.Current(), ku, dn, (int)ne, st);
    void* t2 = B.get(tu);
    if (!t2 || cub::DeviceSelect::Unique(t2, tu, db.Current(), ku, dn, (int)ne, st) != cudaSuccess) return -1;
    if (cudaMemcpyAsync(&nnz, dn, sizeof(long long), cudaMemcpyDeviceToHost, st) != cudaSuccess ||
        cudaStreamSynchronize(st) != cudaSuccess)
      return -1;
    col = (int*)B.get(sizeof(int) * (size_t)(nnz ? nnz : 1));
    val = B.get(vb * (size_t)(nnz ? nnz : 1));
    if (!col || !val) return -1;
    if (nnz == 0) k_fill_int<<<grid_for(m + 1), 256, 0, st>>>(rp, m + 1, 0);
    else k_rmat_csr<<<grid_for(nnz), 256, 0, st>>>(sp->seed, m, ku, dn, rp, col, val, sp->dtype);
  } else if (sp->cls == SFSGEN_UNIFORM || sp->cls == SFSGEN_POWERLAW) {
    std::vector<double> T;
    double* dT = nullptr;
    if (sp->cls == SFSGEN_POWERLAW) {  // the same table as gen.c, built by the same libm pow
      long long cap = n < (1LL << 17) ? n : (1LL << 17);
      if (cap < 2) cap = 2;
      T.resize((size_t)cap + 1);
      T[0] = T[1] = 1.0;
      for (long long L = 2; L <= cap; L++) T[(size_t)L] = pow(2.0 / (double)L, sp->pa - 1.0);
      dT = (double*)B.get(sizeof(double) * T.size());
      if (!dT || cudaMemcpyAsync(dT, T.data(), sizeof(double) * T.size(), cudaMemcpyHostToDevice, st) != cudaSuccess)
        return -1;
      s.T = dT;
      s.cap = cap;
    }
    long long* len0 = (long long*)B.get(sizeof(long long) * (size_t)m);
    long long* off0 = (long long*)B.get(sizeof(long long) * (size_t)(m + 1));
    int* brows = (int*)B.get(sizeof(int) * (size_t)m);
    int* nb = (int*)B.get(sizeof(int));
    int* len = (int*)B.get(sizeof(int) * (size_t)m);
    if (!len0 || !off0 || !brows || !nb || !len) return -1;
    cudaMemsetAsync(nb, 0, sizeof(int), st);
    cudaMemsetAsync(off0, 0, sizeof(long long), st);
    k_draw_count<<<grid_for(m), 256, 0, st>>>(s, len0, brows, nb);
    size_t tb = 0;
    cub::DeviceScan::InclusiveSum(nullptr, tb, len0, off0 + 1, (int)m, st);
    void* t = B.get(tb);
    if (!t || cub::DeviceScan::InclusiveSum(t, tb, len0, off0 + 1, (int)m, st) != cudaSuccess) return -1;
    long long total = 0;
    int nbern = 0;
    cudaMemcpyAsync(&total, off0 + m, sizeof(long long), cudaMemcpyDeviceToHost, st);
    cudaMemcpyAsync(&nbern, nb, sizeof(int), cudaMemcpyDeviceToHost, st);
    if (cudaStreamSynchronize(st) != cudaSuccess) return -1;
    int* keys = (int*)B.get(sizeof(int) * (size_t)(total ? total : 1));
    int* sorted = (int*)B.get(sizeof(int) * (size_t)(total ? total : 1));
    if (!keys || !sorted) return -1;
    k_draw_fill<<<grid_for(m), 256, 0, st>>>(s, off0, keys);
    if (total > 0) {
      size_t ts = 0;
      cub::DeviceSegmentedSort::SortKeys(nullptr, ts, keys, sorted, (int)total, (int)m, off0, off0 + 1, st);
      void* t3 = B.get(ts);
      if (!t3 || cub::DeviceSegmentedSort::SortKeys(t3, ts, keys, sorted, (int)total, (int)m, off0, off0 + 1, st) !=
                     cudaSuccess)
        return -1;
    }
    k_unique_count<<<grid_for(m), 256, 0, st>>>(s, off0, sorted, len);
    if (nbern) k_bern_count<<<nbern, 256, 0, st>>>(s, brows, len);
    if (scan_lengths(len, rp, m, st, B)) return -1;
    int nz32 = 0;
    cudaMemcpyAsync(&nz32, rp + m, sizeof(int), cudaMemcpyDeviceToHost, st);
    if (cudaStreamSynchronize(st) != cudaSuccess) return -1;
    nnz = nz32;
    col = (int*)B.get(sizeof(int) * (size_t)(nnz ? nnz : 1));
    val = B.get(vb * (size_t)(nnz ? nnz : 1));
    if (!col || !val) return -1;
    k_unique_fill<<<grid_for(m), 256, 0, st>>>(s, off0, sorted, rp, col, val);
    if (nbern) k_bern_fill<<<nbern, 256, 0, st>>>(s, brows, rp, col, val);
  } else {
    int* len = (int*)B.get(sizeof(int) * (size_t)m);
    if (!len) return -1;
    k_direct_count<<<grid_for(m), 256, 0, st>>>(s, len);
    if (scan_lengths(len, rp, m, st, B)) return -1;
    int nz32 = 0;
    cudaMemcpyAsync(&nz32, rp + m, sizeof(int), cudaMemcpyDeviceToHost, st);
    if (cudaStreamSynchronize(st) != cudaSuccess) return -1;
    nnz = nz32;
    col = (int*)B.get(sizeof(int) * (size_t)(nnz ? nnz : 1));
    val = B.get(vb * (size_t)(nnz ? nnz : 1));
    if (!col || !val) return -1;
    k_direct_fill<<<grid_for(m), 256, 0, st>>>(s, rp, col, val);
  }
  if (cudaStreamSynchronize(st) != cudaSuccess || cudaGetLastError() != cudaSuccess) return -1;
  B.release(rp);
  B.release(col);
  B.release(val);
  out->nnz = nnz;
  out->rp = rp;
  out->col = col;
  out->val = val;
  return 0;
}

void sfsgen_free_device(sfsgen_csr* c) {
  if (!c) return;
  cudaFree(c->rp);
  cudaFree(c->col);
  cudaFree(c->val);
  c->rp = nullptr;
  c->col = nullptr;
  c->val = nullptr;
}

int sfsgen_vector_device(uint64_t seed, int64_t n, int32_t dtype, void* out, void* stream) {
  if (n <= 0) return 0;
  k_vector<<<grid_for(n), 256, 0, (cudaStream_t)stream>>>(seed, n, dtype, out);
  return cudaGetLastError() == cudaSuccess ? 0 : -1;
}

}  // extern "C"
