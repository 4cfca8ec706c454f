// api.cpp — the C ABI of include/sfs.h: handles, allocator, feature finalisation, conversions and
// the device-timed format race (§5.1 "average over 100 trials"; L331 §5.4 steps
// (ii)–(iii); label = fastest format, L56 §1).
#include <cuda_runtime.h>
#include <stdint.h>
#include <string.h>

#include <algorithm>
#include <atomic>
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <cmath>
#include <mutex>
#include <string>
#include <vector>

#include "internal.h"
#include "sfs.h"

namespace sfs {

std::atomic<int64_t> g_launches{0};

// ---------------------------------------------------------------- errors
static thread_local std::string t_err;
void set_error(const std::string& msg) { t_err = msg; }

static sfs_status fail(sfs_status s, const std::string& msg) {
  set_error(msg);
  return s;
}
static sfs_status cuda_fail(cudaError_t e, const char* what) {
  set_error(std::string(what) + ": " + cudaGetErrorString(e));
  return e == cudaErrorMemoryAllocation ? SFS_ERR_OOM : SFS_ERR_CUDA;
}
#define TRY_CUDA(expr)                                    \
  do {                                                    \
    cudaError_t _e = (expr);                              \
    if (_e != cudaSuccess) return cuda_fail(_e, #expr);   \
  } while (0)

// ---------------------------------------------------------------- allocator
static void* (*g_user_alloc)(size_t, void*) = nullptr;
static void (*g_user_free)(void*, void*) = nullptr;
static std::mutex g_pool_mu;
static cudaMemPool_t g_pools[kMaxDevices] = {};

static cudaMemPool_t pool_for_current_device() {
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= kMaxDevices) return nullptr;
  std::lock_guard<std::mutex> lk(g_pool_mu);
  if (!g_pools[dev]) {
    cudaMemPoolProps props;
    memset(&props, 0, sizeof(props));
    props.allocType = cudaMemAllocationTypePinned;
    props.handleTypes = cudaMemHandleTypeNone;
    props.location.type = cudaMemLocationTypeDevice;
    props.location.id = dev;
    cudaMemPool_t p = nullptr;
    if (cudaMemPoolCreate(&p, &props) != cudaSuccess) return nullptr;
    uint64_t thr = UINT64_MAX;  // keep freed blocks cached: steady-state races never hit cudaMalloc
    cudaMemPoolSetAttribute(p, cudaMemPoolAttrReleaseThreshold, &thr);
    g_pools[dev] = p;
  }
  return g_pools[dev];
}

void* dalloc(size_t bytes, cudaStream_t s) {
  if (bytes == 0) bytes = 256;
  bytes = (bytes + 255) & ~(size_t)255;
  if (g_user_alloc) return g_user_alloc(bytes, (void*)s);
  cudaMemPool_t p = pool_for_current_device();
  if (!p) return nullptr;
  void* ptr = nullptr;
  if (cudaMallocFromPoolAsync(&ptr, bytes, p, s) != cudaSuccess) {
    cudaGetLastError();
    return nullptr;
  }
  return ptr;
}

void dfree(void* p, cudaStream_t s) {
  if (!p) return;
  if (g_user_free) { g_user_free(p, (void*)s); return; }
  cudaFreeAsync(p, s);
}

// A handle outlives the call that built it: its buffers go back to the allocator that provided them,
// even if sfs_set_allocator changed in between.
static void dfree_from(void* p, cudaStream_t s, void (*user_free)(void*, void*)) {
  if (!p) return;
  if (user_free) user_free(p, (void*)s);
  else cudaFreeAsync(p, s);
}

// RAII list of stream-ordered temporaries
struct Temps {
  cudaStream_t s;
  std::vector<void*> v;
  explicit Temps(cudaStream_t st) : s(st) {}
  void* get(size_t b) {
    void* p = dalloc(b, s);
    if (p) v.push_back(p);
    return p;
  }
  ~Temps() {
    for (void* p : v) dfree(p, s);
  }
};

// ---------------------------------------------------------------- options / rules
static void defaults(sfs_race_opts* o) {
  o->reps = 100;
  o->warmup = 5;
  o->formats_mask = 0x1F;
  o->cold = 0;
  o->max_fill = 3.0;
  o->fill_slack = (int64_t)1 << 20;
  o->hyb_rel_speed = 3.0;
  o->hyb_breakeven = 4096;
  o->csr_variant = -1;
  o->use_graphs = 0;  // direct PDL launches: measured faster than per-(matrix, format) graphs
  o->race_mask = nullptr;
}

// Q6: largest R with  rel * R < m  or  R < breakeven  (the condition is monotone in R).
static long long hyb_rmax(long long m, const sfs_race_opts& o) {
  long long r1 = -1;
  if (o.hyb_rel_speed <= 0) return m;  // condition always true -> K = 1
  long long R = (long long)std::floor((double)m / o.hyb_rel_speed);
  while (R >= 0 && !(o.hyb_rel_speed * (double)R < (double)m)) R--;
  while (o.hyb_rel_speed * (double)(R + 1) < (double)m) R++;
  r1 = R;
  long long r2 = o.hyb_breakeven - 1;
  long long r = std::max(r1, r2);
  return std::min(r, m);
}

typedef __int128 i128;
static inline double i2d(i128 v) { return (double)v; }

// Q4: csr_max = sum over the first warp's vectors of ceil((m - v) / V).
static long long csr_max_closed_form(long long m, long long z) {
  const long long tpv = csr_vector_tpv(m, z), vpw = 32 / tpv, V = (long long)kCsrWarps * vpw;
  long long s = 0;
  for (long long v = 0; v < std::min(vpw, m); v++) s += (m - v + V - 1) / V;
  return s;
}

// Finalise Table-1 features from the exact device aggregates (fixed fp64 formulas).
static void finalize(long long m, long long n, long long z, const DevAggr& a, long long K, long long hcoo,
                     const sfs_race_opts& o, sfs_features_t* f) {
  memset(f, 0, sizeof(*f));
  const long long mn = 2147483647LL - (long long)a.min_inv, mx = (long long)a.max_len, nd = (long long)a.ndiag;
  const i128 M = m, Z = z;
  f->nrows = m;
  f->ncols = n;
  f->nnz = z;
  f->nnz_min = mn;
  f->nnz_max = mx;
  f->csr_max = csr_max_closed_form(m, z);
  f->ell_size = m * mx;
  f->hyb_k = K;
  f->hyb_ell_size = m * K;
  f->hyb_coo = hcoo;
  f->hyb_ell_nnz = z - hcoo;
  f->diagonals = nd;
  f->dia_size = nd * m;
  f->nnz_frac = i2d(Z) / i2d(M * (i128)n);
  f->nnz_mu = i2d(Z) / i2d(M);
  f->nnz_sig = std::sqrt(i2d(M * (i128)a.S2 - Z * Z) / i2d(M * M));
  f->max_mu = i2d((i128)mx * M - Z) / i2d(M);
  f->mu_min = i2d(Z - (i128)mn * M) / i2d(M);
  f->sig_lower = a.cL == 0 ? 0.0
                           : std::sqrt(i2d(M * M * (i128)a.s2L - 2 * M * Z * (i128)a.s1L + (i128)a.cL * Z * Z) /
                                       i2d((i128)a.cL * M * M));
  f->sig_higher = a.cH == 0 ? 0.0
                            : std::sqrt(i2d(M * M * (i128)a.s2H - 2 * M * Z * (i128)a.s1H + (i128)a.cH * Z * Z) /
                                        i2d((i128)a.cH * M * M));
  f->hyb_ell_frac = z == 0 ? 0.0 : i2d(Z - hcoo) / i2d(Z);
  f->dia_frac = f->dia_size == 0 ? 0.0 : i2d(Z) / i2d((i128)f->dia_size);
  f->ell_frac = f->ell_size == 0 ? 0.0 : i2d(Z) / i2d((i128)f->ell_size);
  long long lim = (long long)(o.max_fill * (double)z);
  if (lim < o.fill_slack) lim = o.fill_slack;
  uint32_t mask = (1u << SFS_CSR) | (1u << SFS_COO) | (1u << SFS_HYB);
  if (f->ell_size <= lim) mask |= 1u << SFS_ELL;
  if (f->dia_size <= lim) mask |= 1u << SFS_DIA;
  f->admissible_mask = mask;
  // Q17 (measured; profiles/r02/csr_variants.txt): matrices with empty rows take the tile
  // kernel over the non-empty rows (variant 5: R-MAT 2^22 290 us against 336 for the merge path and
  // 1020 for the row_ptr tile kernel); otherwise the tile kernel (nnz-balanced chunks, row ids from a
  // row-start bitmap, variant 4) for skewed rows or nnz >= 2^20, else the stream kernel (warp per 32
  // rows), whose single launch is fastest on small regular matrices.
  const long long avg = std::max(1LL, z / m);
  if (a.empty_rows * 256 > (long long)z) f->csr_variant = 5;
  else if (mx > 4 * avg + 32 || z >= (1LL << 20)) f->csr_variant = a.empty_rows == 0 ? 4 : 5;
  else f->csr_variant = 2;
  if (o.csr_variant >= 0 && o.csr_variant <= 5) f->csr_variant = o.csr_variant;
}

static sfs_status check_csr(const sfs_csr* A) {
  if (!A) return fail(SFS_ERR_INVALID_ARG, "null matrix");
  if (A->nrows < 1 || A->ncols < 1 || A->nnz < 0) return fail(SFS_ERR_INVALID_ARG, "bad sizes");
  if (A->nrows >= (1LL << 31) - 1 || A->ncols >= (1LL << 31) - 1 || A->nnz >= (1LL << 31) - 1)
    return fail(SFS_ERR_UNSUPPORTED, "int32 index overflow");
  if (A->dtype != SFS_F32 && A->dtype != SFS_F64) return fail(SFS_ERR_INVALID_ARG, "bad dtype");
  if (A->mem != SFS_MEM_DEVICE && A->mem != SFS_MEM_HOST) return fail(SFS_ERR_INVALID_ARG, "bad mem");
  if (!A->row_ptr || (A->nnz > 0 && (!A->col_idx || !A->values))) return fail(SFS_ERR_INVALID_ARG, "null array");
  return SFS_OK;
}

static inline size_t vbytes(int dtype) { return dtype == SFS_F64 ? 8 : 4; }

// Device view of an input CSR (staged to the device if it lives in host memory).
struct DevCSR {
  long long m = 0, n = 0, z = 0;
  int dtype = 0;
  const int* rp = nullptr;
  const int* col = nullptr;
  const void* val = nullptr;
  const void* x = nullptr;
  void* staged[4] = {nullptr, nullptr, nullptr, nullptr};
  bool host = false;
};

static sfs_status stage(const sfs_csr* A, DevCSR& d, cudaStream_t s, bool with_x) {
  d.m = A->nrows;
  d.n = A->ncols;
  d.z = A->nnz;
  d.dtype = A->dtype;
  d.host = A->mem == SFS_MEM_HOST;
  if (!d.host) {
    d.rp = A->row_ptr;
    d.col = A->col_idx;
    d.val = A->values;
    d.x = A->x;
    return SFS_OK;
  }
  const size_t b[4] = {sizeof(int) * (size_t)(d.m + 1), sizeof(int) * (size_t)d.z, vbytes(d.dtype) * (size_t)d.z,
                       vbytes(d.dtype) * (size_t)d.n};
  const void* src[4] = {A->row_ptr, A->col_idx, A->values, A->x};
  for (int i = 0; i < 4; i++) {
    if (i == 3 && (!with_x || !A->x)) break;
    d.staged[i] = dalloc(b[i], s);
    if (!d.staged[i]) return fail(SFS_ERR_OOM, "staging host CSR");
    if (b[i]) TRY_CUDA(cudaMemcpyAsync(d.staged[i], src[i], b[i], cudaMemcpyHostToDevice, s));
  }
  d.rp = (const int*)d.staged[0];
  d.col = (const int*)d.staged[1];
  d.val = d.staged[2];
  d.x = d.staged[3];
  return SFS_OK;
}

static void unstage(DevCSR& d, cudaStream_t s) {
  for (int i = 0; i < 4; i++) {
    dfree(d.staged[i], s);
    d.staged[i] = nullptr;
  }
}

// Host-side refinement of the HYB order statistic when it lies beyond the exact histogram (rare).
static sfs_status refine_hyb(const DevCSR& d, const DevAggr& a, long long rmax, long long* K, long long* hcoo,
                             cudaStream_t s) {
  const long long j = rmax + 1;
  long long lo = kHistCap, hi = (long long)a.max_len, above = 0;
  const int nb = 4096;
  Temps tmp(s);  // freed on every return path
  unsigned* dh = (unsigned*)tmp.get(sizeof(unsigned) * nb + sizeof(long long));
  if (!dh) return fail(SFS_ERR_OOM, "refine");
  std::vector<unsigned> hh(nb);
  while (true) {
    const long long w = (hi - lo + 1 + nb - 1) / nb;
    TRY_CUDA(cudaMemsetAsync(dh, 0, sizeof(unsigned) * nb, s));
    TRY_CUDA(launch_len_hist_range(d.rp, d.m, lo, hi, w, dh, s));
    TRY_CUDA(cudaMemcpyAsync(hh.data(), dh, sizeof(unsigned) * nb, cudaMemcpyDeviceToHost, s));
    TRY_CUDA(cudaStreamSynchronize(s));
    const long long nbins = (hi - lo + 1 + w - 1) / w;
    long long cum = above;
    long long b = nbins - 1;
    for (; b >= 0; b--) {
      if (cum + hh[b] >= j) break;
      cum += hh[b];
    }
    if (b < 0) { lo = 0; break; }  // cannot happen when j <= big_cnt
    const long long nlo = lo + b * w, nhi = std::min(hi, lo + (b + 1) * w - 1);
    above = cum;
    lo = nlo;
    hi = nhi;
    if (w == 1) break;
  }
  *K = std::max(1LL, lo);
  long long* dc = (long long*)(dh);
  TRY_CUDA(cudaMemsetAsync(dc, 0, sizeof(long long), s));
  TRY_CUDA(launch_hyb_coo(d.rp, d.m, *K, dc, s));
  TRY_CUDA(cudaMemcpyAsync(hcoo, dc, sizeof(long long), cudaMemcpyDeviceToHost, s));
  TRY_CUDA(cudaStreamSynchronize(s));
  return SFS_OK;
}

// Host memory the device can store to with the same address (cudaMallocHost under unified addressing).
static bool host_mapped(const void* p) {
  cudaPointerAttributes at;
  if (cudaPointerGetAttributes(&at, p) != cudaSuccess) {
    cudaGetLastError();
    return false;
  }
  return at.type == cudaMemoryTypeHost && at.devicePointer == p;
}

// Feature pass for one device CSR; leaves the bitmap in `w` (caller frees) and copies aggregates to `ha`.
static sfs_status features_device(const DevCSR& d, const sfs_race_opts& o, FeatWork& w, DevAggr* ha_pinned,
                                  cudaStream_t s) {
  void* base = dalloc(feat_work_bytes(d.m, d.n), s);
  if (!base) return fail(SFS_ERR_OOM, "feature workspace");
  feat_work_bind(w, base, d.m, d.n);
  // the last feature kernel writes the aggregates straight into the mapped pinned record (no D2H copy
  // operation in the stream); unmapped host memory gets a copy
  const bool mapped = host_mapped(ha_pinned);
  TRY_CUDA(launch_features(d.rp, d.col, d.m, d.n, d.z, hyb_rmax(d.m, o), w, mapped ? ha_pinned : nullptr, s));
  if (!mapped) TRY_CUDA(cudaMemcpyAsync(ha_pinned, w.aggr, sizeof(DevAggr), cudaMemcpyDeviceToHost, s));
  return SFS_OK;
}

// After the aggregates are on the host: validation, refinement, finalisation.
static sfs_status features_finish(const DevCSR& d, const sfs_race_opts& o, const DevAggr& a, sfs_features_t* f,
                                  cudaStream_t s) {
  if (a.flags) {
    return fail(SFS_ERR_INVALID_CSR, "invalid CSR (flags " + std::to_string(a.flags) + ")");
  }
  long long K = a.hyb_k, hcoo = a.hyb_coo;
  if (K < 0) {
    sfs_status st = refine_hyb(d, a, hyb_rmax(d.m, o), &K, &hcoo, s);
    if (st != SFS_OK) return st;
  }
  finalize(d.m, d.n, d.z, a, K, hcoo, o, f);
  return SFS_OK;
}

// ---------------------------------------------------------------- conversion
static sfs_status convert_impl(const DevCSR& d, sfs_format fmt, const sfs_features_t& f, const FeatWork& fw,
                               Matrix** out, cudaStream_t s) {
  Matrix* A = new Matrix();
  A->fmt = fmt;
  A->dtype = d.dtype;
  A->m = d.m;
  A->n = d.n;
  A->nnz = d.z;
  A->pitch = pitch_of(d.m);
  A->stream = s;
  A->variant = f.csr_variant;
  A->banded = (f.admissible_mask >> SFS_DIA) & 1u;
  A->user_free = g_user_free;  // the allocator this handle's buffers come from
  const size_t sv = vbytes(d.dtype);
  auto own = [&](size_t b) -> void* {
    void* p = dalloc(b, s);
    if (p) {
      A->owned[A->n_owned++] = p;
      A->bytes += (long long)b;
    }
    return p;
  };
  auto bail = [&](sfs_status st, const std::string& what) {
    for (int i = 0; i < A->n_owned; i++) dfree(A->owned[i], s);
    delete A;
    return fail(st, what);
  };
  // every CUDA failure releases the partly built handle (no leak of its pool blocks)
#define BAIL_CUDA(expr)                                                                             \
  do {                                                                                              \
    cudaError_t _e = (expr);                                                                        \
    if (_e != cudaSuccess)                                                                          \
      return bail(_e == cudaErrorMemoryAllocation ? SFS_ERR_OOM : SFS_ERR_CUDA,                     \
                  std::string(#expr) + ": " + cudaGetErrorString(_e));                              \
  } while (0)
  const long long m = d.m, z = d.z, P = A->pitch;
  switch (fmt) {
    case SFS_CSR: {
      if (d.host) {  // own device copies
        int* rp = (int*)own(sizeof(int) * (m + 1));
        int* col = (int*)own(sizeof(int) * std::max(z, 1LL));
        void* val = own(sv * std::max(z, 1LL));
        if (!rp || !col || !val) return bail(SFS_ERR_OOM, "csr copy");
        BAIL_CUDA(cudaMemcpyAsync(rp, d.rp, sizeof(int) * (m + 1), cudaMemcpyDeviceToDevice, s));
        if (z) {
          BAIL_CUDA(cudaMemcpyAsync(col, d.col, sizeof(int) * z, cudaMemcpyDeviceToDevice, s));
          BAIL_CUDA(cudaMemcpyAsync(val, d.val, sv * z, cudaMemcpyDeviceToDevice, s));
        }
        A->ptr[0] = rp; A->ptr[1] = col; A->ptr[2] = val;
      } else {
        A->ptr[0] = d.rp; A->ptr[1] = d.col; A->ptr[2] = d.val;
      }
      A->width = 0;
      if (A->variant == 1) {
        A->work = own(csr_merge_work_bytes(m, z, d.dtype));
        if (!A->work) return bail(SFS_ERR_OOM, "csr merge carries");
        BAIL_CUDA(launch_csr_merge_prepare((const int*)A->ptr[0], m, z, A->work, s));
      } else if ((A->variant == 3 || A->variant == 4 || A->variant == 5) && z > 0) {
        if (A->variant == 4 && f.nnz_min < 1) A->variant = 5;  // empty rows: bitmap over the non-empty rows + map
        const int bitmap = A->variant == 4 ? 1 : (A->variant == 5 ? 2 : 0);
        A->work = own(csr_tile_work_bytes(m, z, bitmap));
        if (!A->work) return bail(SFS_ERR_OOM, "csr tile partition");
        BAIL_CUDA(launch_csr_tile_prepare((const int*)A->ptr[0], m, z, A->work, bitmap, s));
      }
      break;
    }
    case SFS_COO: {
      int* r = (int*)own(sizeof(int) * std::max(z, 1LL));
      int* c = (int*)own(sizeof(int) * std::max(z, 1LL));
      void* v = own(sv * std::max(z, 1LL));
      if (!r || !c || !v) return bail(SFS_ERR_OOM, "coo");
      BAIL_CUDA(launch_csr2coo(d.dtype, d.rp, d.col, d.val, m, z, r, c, v, s));
      A->ptr[0] = r; A->ptr[1] = c; A->ptr[2] = v;
      break;
    }
    case SFS_ELL: {
      if (!(f.admissible_mask & (1u << SFS_ELL))) return bail(SFS_ERR_INADMISSIBLE, "ELL inadmissible (Q11)");
      const long long K = f.nnz_max;
      int* ec = (int*)own(sizeof(int) * std::max(K * P, 1LL));
      void* ev = own(sv * std::max(K * P, 1LL));
      if (!ec || !ev) return bail(SFS_ERR_OOM, "ell");
      BAIL_CUDA(launch_csr2ell(d.dtype, d.rp, d.col, d.val, m, P, (int)K, ec, ev, s));
      A->ptr[0] = ec; A->ptr[1] = ev;
      A->width = K;
      break;
    }
    case SFS_HYB: {
      const long long K = f.hyb_k, nc = f.hyb_coo;
      int* ec = (int*)own(sizeof(int) * std::max(K * P, 1LL));
      void* ev = own(sv * std::max(K * P, 1LL));
      int* cr = (int*)own(sizeof(int) * std::max(nc, 1LL));
      int* cc = (int*)own(sizeof(int) * std::max(nc, 1LL));
      void* cv = own(sv * std::max(nc, 1LL));
      if (!ec || !ev || !cr || !cc || !cv) return bail(SFS_ERR_OOM, "hyb");
      BAIL_CUDA(launch_csr2ell(d.dtype, d.rp, d.col, d.val, m, P, (int)K, ec, ev, s));
      // rows overflowing by <= 32 (64 below 2^20 nnz): keep the per-row overflow offsets for the one-launch SpMV
      A->variant = hyb_rowwise(f.nnz_max, K, nc, z);
      if (nc > 0) {
        Temps t(s);
        int* ovf = A->variant ? (int*)own(sizeof(int) * (m + 1)) : (int*)t.get(sizeof(int) * (m + 1));
        void* work = t.get(scan_work_bytes(m));
        if (!ovf || !work) return bail(SFS_ERR_OOM, "hyb scan");
        BAIL_CUDA(launch_overflow_scan(d.rp, m, (int)K, ovf, work, s));
        BAIL_CUDA(launch_hyb_coo_part(d.dtype, d.rp, d.col, d.val, m, z, (int)K, ovf, cr, cc, cv, s));
        if (A->variant) A->ptr[5] = ovf;
      }
      A->ptr[0] = ec; A->ptr[1] = ev; A->ptr[2] = cr; A->ptr[3] = cc; A->ptr[4] = cv;
      A->width = K;
      A->coo_nnz = nc;
      break;
    }
    case SFS_DIA: {
      if (!(f.admissible_mask & (1u << SFS_DIA))) return bail(SFS_ERR_INADMISSIBLE, "DIA inadmissible (Q11)");
      const long long nd = f.diagonals;
      int* offs = (int*)own(sizeof(int) * std::max(nd, 1LL));
      void* dv = own(sv * std::max(nd * P, 1LL));
      if (!offs || !dv) return bail(SFS_ERR_OOM, "dia");
      {
        Temps t(s);
        int* wp = (int*)t.get(sizeof(int) * (fw.words + 1));
        void* work = t.get(scan_work_bytes(fw.words));
        if (!wp || !work) return bail(SFS_ERR_OOM, "dia scan");
        BAIL_CUDA(launch_popc_scan(fw.bitmap, fw.words, wp, work, s));
        BAIL_CUDA(launch_dia_offsets(fw.bitmap, fw.words, wp, m, offs, s));
        if (nd > 0) {
          BAIL_CUDA(cudaMemsetAsync(dv, 0, sv * nd * P, s));
          count_launch();
          BAIL_CUDA(launch_csr2dia(d.dtype, d.rp, d.col, d.val, m, P, fw.bitmap, wp, dv, s));
        }
      }
      A->ptr[0] = offs; A->ptr[1] = dv;
      A->ndiag = nd;
      break;
    }
    default:
      return bail(SFS_ERR_INVALID_ARG, "bad format");
  }
#undef BAIL_CUDA
  *out = A;
  return SFS_OK;
}

static void matrix_free(Matrix* A) {
  if (!A) return;
  for (int i = 0; i < A->n_owned; i++) dfree_from(A->owned[i], A->stream, A->user_free);
  delete A;
}

// ---------------------------------------------------------------- events
struct EventPool {
  std::vector<cudaEvent_t> all;
  size_t used = 0;
  cudaEvent_t get() {
    if (used == all.size()) {
      cudaEvent_t e;
      if (cudaEventCreate(&e) != cudaSuccess) return nullptr;
      all.push_back(e);
    }
    return all[used++];
  }
  ~EventPool() {
    for (auto e : all) cudaEventDestroy(e);
  }
};

static float elapsed_us(cudaEvent_t a, cudaEvent_t b) {
  float ms = 0.f;
  if (cudaEventElapsedTime(&ms, a, b) != cudaSuccess) return -1.f;
  return ms * 1000.f;
}

}  // namespace sfs

using namespace sfs;

// ======================================================================== C ABI
extern "C" {

void sfs_default_opts(sfs_race_opts* opt) {
  if (opt) defaults(opt);
}

const char* sfs_version(void) { return "sfs 0.1 (sm_100a)"; }

const char* sfs_status_string(sfs_status s) {
  switch (s) {
    case SFS_OK: return "SFS_OK";
    case SFS_ERR_INVALID_ARG: return "SFS_ERR_INVALID_ARG";
    case SFS_ERR_INVALID_CSR: return "SFS_ERR_INVALID_CSR";
    case SFS_ERR_INADMISSIBLE: return "SFS_ERR_INADMISSIBLE";
    case SFS_ERR_OOM: return "SFS_ERR_OOM";
    case SFS_ERR_CUDA: return "SFS_ERR_CUDA";
    case SFS_ERR_UNSUPPORTED: return "SFS_ERR_UNSUPPORTED";
    case SFS_ERR_NOT_RUN: return "SFS_ERR_NOT_RUN";
  }
  return "SFS_ERR_UNKNOWN";
}

const char* sfs_last_error(void) { return t_err.c_str(); }

void sfs_set_allocator(void* (*alloc)(size_t, void*), void (*dealloc)(void*, void*)) {
  g_user_alloc = (alloc && dealloc) ? alloc : nullptr;
  g_user_free = (alloc && dealloc) ? dealloc : nullptr;
}

int64_t sfs_launch_count(void) { return g_launches.load(); }

int64_t sfs_spmv_bytes(const sfs_features_t* F, sfs_format f, sfs_dtype dtype) {
  if (!F) return -1;
  const long long s = dtype == SFS_F64 ? 8 : 4, m = F->nrows, n = F->ncols, z = F->nnz;
  const long long xy = s * n + s * m;
  switch (f) {
    case SFS_CSR: return 4 * (m + 1) + (4 + s) * z + xy;
    case SFS_COO: return (8 + s) * z + xy;
    case SFS_ELL: return (4 + s) * F->ell_size + xy;
    case SFS_HYB: return (4 + s) * F->hyb_ell_size + (8 + s) * F->hyb_coo + xy;
    case SFS_DIA: return s * F->dia_size + 4 * F->diagonals + xy;
    default: return -1;
  }
}

sfs_status sfs_features(const sfs_csr* A, const sfs_race_opts* opt, sfs_features_t* out, void* stream) {
  sfs_status st = check_csr(A);
  if (st != SFS_OK) return st;
  if (!out) return fail(SFS_ERR_INVALID_ARG, "null out");
  sfs_race_opts o;
  defaults(&o);
  if (opt) o = *opt;
  cudaStream_t s = (cudaStream_t)stream;
  DevCSR d;
  if ((st = stage(A, d, s, false)) != SFS_OK) { unstage(d, s); return st; }
  DevAggr* ha = nullptr;
  if (cudaError_t e = cudaMallocHost(&ha, sizeof(DevAggr)); e != cudaSuccess) {
    unstage(d, s);
    return cuda_fail(e, "pinned aggregate record");
  }
  FeatWork w;
  st = features_device(d, o, w, ha, s);
  if (st == SFS_OK) {
    cudaError_t e = cudaStreamSynchronize(s);
    st = e == cudaSuccess ? features_finish(d, o, *ha, out, s) : cuda_fail(e, "features sync");
  }
  dfree(w.base, s);
  unstage(d, s);
  cudaFreeHost(ha);
  return st;
}

sfs_status sfs_convert(const sfs_csr* A, sfs_format f, const sfs_race_opts* opt, sfs_matrix* out, void* stream) {
  sfs_status st = check_csr(A);
  if (st != SFS_OK) return st;
  if (!out || f < 0 || f >= SFS_NFMT) return fail(SFS_ERR_INVALID_ARG, "bad format / out");
  *out = nullptr;
  sfs_race_opts o;
  defaults(&o);
  if (opt) o = *opt;
  cudaStream_t s = (cudaStream_t)stream;
  DevCSR d;
  if ((st = stage(A, d, s, false)) != SFS_OK) { unstage(d, s); return st; }
  DevAggr* ha = nullptr;
  if (cudaError_t e = cudaMallocHost(&ha, sizeof(DevAggr)); e != cudaSuccess) {
    unstage(d, s);
    return cuda_fail(e, "pinned aggregate record");
  }
  FeatWork w;
  sfs_features_t F;
  st = features_device(d, o, w, ha, s);
  if (st == SFS_OK) {
    cudaError_t e = cudaStreamSynchronize(s);
    st = e == cudaSuccess ? features_finish(d, o, *ha, &F, s) : cuda_fail(e, "features sync");
  }
  Matrix* M = nullptr;
  if (st == SFS_OK) st = convert_impl(d, f, F, w, &M, s);
  dfree(w.base, s);
  unstage(d, s);
  cudaFreeHost(ha);
  if (st == SFS_OK) *out = (sfs_matrix)M;
  return st;
}

sfs_status sfs_spmv(sfs_format f, sfs_matrix Ah, const void* x, void* y, void* stream) {
  Matrix* A = (Matrix*)Ah;
  if (!A || !x || !y) return fail(SFS_ERR_INVALID_ARG, "null argument");
  if ((int)f != A->fmt) return fail(SFS_ERR_INVALID_ARG, "format does not match the handle");
  cudaError_t e = launch_spmv(A, x, y, (cudaStream_t)stream);
  if (e != cudaSuccess) return cuda_fail(e, "spmv launch");
  return SFS_OK;
}

sfs_status sfs_gather(sfs_dtype dtype, const void* src, const int32_t* idx, int64_t n, void* dst, void* stream) {
  if (n < 0 || (n > 0 && (!src || !idx || !dst)) || (dtype != SFS_F32 && dtype != SFS_F64))
    return fail(SFS_ERR_INVALID_ARG, "sfs_gather: bad argument");
  cudaError_t e = launch_gather((int)dtype, src, idx, n, dst, (cudaStream_t)stream);
  if (e != cudaSuccess) return cuda_fail(e, "gather launch");
  return SFS_OK;
}

// Row-partitioned SpMV with the halo push fused in (include/sfs.h).
static sfs_status check_push(const sfs_push_t* p, long long nrows) {
  if (!p) return fail(SFS_ERR_INVALID_ARG, "null push plan");
  if (p->nseg < 0 || p->nseg > SFS_MAX_PUSH || p->nwait < 0 || p->nwait > SFS_MAX_PEERS || p->nsig < 0 ||
      p->nsig > SFS_MAX_PEERS)
    return fail(SFS_ERR_INVALID_ARG, "push plan counts out of range");
  if (!p->counter) return fail(SFS_ERR_INVALID_ARG, "push plan needs a counter");
  for (int i = 0; i < p->nseg; i++) {
    if (p->seg_begin[i] < 0 || p->seg_end[i] < p->seg_begin[i] || p->seg_end[i] > nrows || !p->seg_dst[i])
      return fail(SFS_ERR_INVALID_ARG, "push run outside the row block or null destination");
    for (int j = 0; j < i; j++)
      if (p->seg_begin[i] < p->seg_end[j] && p->seg_begin[j] < p->seg_end[i])
        return fail(SFS_ERR_INVALID_ARG, "push runs overlap");
  }
  for (int i = 0; i < p->nwait; i++)
    if (!p->wait_flag[i]) return fail(SFS_ERR_INVALID_ARG, "null wait flag");
  for (int i = 0; i < p->nsig; i++)
    if (!p->sig_flag[i]) return fail(SFS_ERR_INVALID_ARG, "null signal flag");
  return SFS_OK;
}

sfs_status sfs_spmv_push(sfs_format f, sfs_matrix Ah, const void* x, void* y, const sfs_push_t* push, void* stream) {
  Matrix* A = (Matrix*)Ah;
  if (!A || ((!x || !y) && A->m > 0)) return fail(SFS_ERR_INVALID_ARG, "null argument");
  if ((int)f != A->fmt) return fail(SFS_ERR_INVALID_ARG, "format argument does not match the handle");
  sfs_status st = check_push(push, A->m);
  if (st != SFS_OK) return st;
  TRY_CUDA(launch_spmv_push(A, x, y, *push, (cudaStream_t)stream));
  return SFS_OK;
}

sfs_status sfs_halo_push(sfs_dtype dtype, const void* src, int64_t nrows, const sfs_push_t* push, void* stream) {
  if ((dtype != SFS_F32 && dtype != SFS_F64) || nrows < 0 || (!src && nrows > 0))
    return fail(SFS_ERR_INVALID_ARG, "bad dtype / source");
  sfs_status st = check_push(push, nrows);
  if (st != SFS_OK) return st;
  TRY_CUDA(launch_halo_push(dtype, src, nrows, *push, (cudaStream_t)stream));
  return SFS_OK;
}

sfs_status sfs_ipc_alloc(size_t bytes, void** ptr, uint8_t handle[64]) {
  if (!ptr || !handle || bytes == 0) return fail(SFS_ERR_INVALID_ARG, "null argument / zero size");
  static_assert(sizeof(cudaIpcMemHandle_t) == 64, "IPC handle size");
  TRY_CUDA(cudaMalloc(ptr, bytes));
  cudaIpcMemHandle_t h;
  cudaError_t e = cudaMemset(*ptr, 0, bytes);
  if (e == cudaSuccess) e = cudaIpcGetMemHandle(&h, *ptr);
  if (e != cudaSuccess) {
    cudaFree(*ptr);
    *ptr = nullptr;
    return cuda_fail(e, "sfs_ipc_alloc");
  }
  memcpy(handle, &h, 64);
  return SFS_OK;
}

sfs_status sfs_ipc_open(const uint8_t handle[64], void** ptr) {
  if (!ptr || !handle) return fail(SFS_ERR_INVALID_ARG, "null argument");
  cudaIpcMemHandle_t h;
  memcpy(&h, handle, 64);
  TRY_CUDA(cudaIpcOpenMemHandle(ptr, h, cudaIpcMemLazyEnablePeerAccess));
  return SFS_OK;
}

sfs_status sfs_ipc_close(void* ptr) {
  TRY_CUDA(cudaIpcCloseMemHandle(ptr));
  return SFS_OK;
}

sfs_status sfs_ipc_free(void* ptr) {
  TRY_CUDA(cudaFree(ptr));
  return SFS_OK;
}

sfs_status sfs_matrix_free(sfs_matrix A) {
  matrix_free((Matrix*)A);
  return SFS_OK;
}

sfs_status sfs_matrix_describe(sfs_matrix Ah, sfs_layout_t* out) {
  Matrix* A = (Matrix*)Ah;
  if (!A || !out) return fail(SFS_ERR_INVALID_ARG, "null argument");
  memset(out, 0, sizeof(*out));
  out->fmt = A->fmt;
  out->dtype = A->dtype;
  out->nrows = A->m;
  out->ncols = A->n;
  out->nnz = A->nnz;
  out->pitch = A->pitch;
  out->width = A->width;
  out->ndiag = A->ndiag;
  out->coo_nnz = A->coo_nnz;
  for (int i = 0; i < 6; i++) out->ptr[i] = A->ptr[i];
  out->bytes = A->bytes;
  out->variant = A->variant;
  return SFS_OK;
}

sfs_status sfs_label_corpus(const sfs_csr* mats, int64_t n, const sfs_race_opts* opt, sfs_features_t* feats,
                            sfs_label_t* labels, void* stream) {
  if (n < 0 || (n > 0 && (!mats || !feats || !labels))) return fail(SFS_ERR_INVALID_ARG, "bad corpus arguments");
  sfs_race_opts o;
  defaults(&o);
  if (opt) o = *opt;
  if (o.reps < 1 || o.warmup < 0) return fail(SFS_ERR_INVALID_ARG, "reps >= 1, warmup >= 0");
  cudaStream_t s = (cudaStream_t)stream;
  EventPool ev;
  std::vector<DevCSR> d(n);
  std::vector<FeatWork> w(n);
  std::vector<sfs_status> mst(n, SFS_OK);
  std::vector<cudaEvent_t> fe0(n, nullptr), fe1(n, nullptr), ce(n, nullptr);
  struct Timed {
    int64_t i;
    int f;
    cudaEvent_t c0, c1, t0, t1;
    std::vector<cudaEvent_t> cold;
  };
  std::vector<Timed> timed;
  std::vector<cudaGraphExec_t> execs;
  std::vector<cudaGraph_t> graphs;
  // Everything the call owns is released by this guard on every return path (streams, the pinned
  // aggregate records, graphs, staged inputs, feature workspaces, the L2 flush buffer).
  struct Owned {
    cudaStream_t s = nullptr, cap = nullptr, up = nullptr, cs = nullptr;
    DevAggr* ha = nullptr;
    void* flush = nullptr;
    std::vector<DevCSR>* d = nullptr;
    std::vector<FeatWork>* w = nullptr;
    std::vector<cudaGraphExec_t>* execs = nullptr;
    std::vector<cudaGraph_t>* graphs = nullptr;
    ~Owned() {
      for (auto ge : *execs) cudaGraphExecDestroy(ge);
      for (auto g : *graphs) cudaGraphDestroy(g);
      for (auto& x : *w) dfree(x.base, s);
      for (auto& x : *d) unstage(x, s);
      dfree(flush, s);
      if (cap) cudaStreamDestroy(cap);
      if (up) cudaStreamDestroy(up);
      if (cs) cudaStreamDestroy(cs);
      if (ha) cudaFreeHost(ha);
    }
  } own;
  own.s = s;
  own.d = &d;
  own.w = &w;
  own.execs = &execs;
  own.graphs = &graphs;
  TRY_CUDA(cudaStreamCreateWithFlags(&own.cap, cudaStreamNonBlocking));  // capture-only (records graphs)
  {
    const char* eu = getenv("SFS_GRAPH_UPLOAD");  // graph uploads on a side stream (0 disables)
    if (!(eu && eu[0] == '0')) TRY_CUDA(cudaStreamCreateWithFlags(&own.up, cudaStreamNonBlocking));
  }
  TRY_CUDA(cudaMallocHost(&own.ha, sizeof(DevAggr) * std::max<int64_t>(n, 1)));
  cudaStream_t cap = own.cap, up = own.up;
  DevAggr* ha = own.ha;
  for (int64_t i = 0; i < n; i++) {
    memset(&labels[i], 0, sizeof(sfs_label_t));
    memset(&feats[i], 0, sizeof(sfs_features_t));
    labels[i].label = -1;
    for (int f = 0; f < SFS_NFMT; f++) labels[i].status[f] = SFS_ERR_NOT_RUN;
  }
  for (int64_t i = 0; i < n; i++)
    if (mats[i].mem == SFS_MEM_HOST) {  // H2D copy stream for host-memory inputs
      TRY_CUDA(cudaStreamCreateWithFlags(&own.cs, cudaStreamNonBlocking));
      break;
    }
  cudaStream_t cs = own.cs;
  // Chunks.  A device-resident corpus is one chunk: every feature pass, one synchronisation (the host
  // needs the features to enqueue the race), then the whole race enqueued.  Host-memory inputs come in
  // chunks of 1, 2, 4, ... matrices: the H2D copies of chunk c+1 (copy stream) run during the race of
  // chunk c, so only the first matrix's copy is exposed.  The copies are ~10x faster than the race
  // consumes the same bytes, so each chunk's inputs are resident before its predecessor's race ends.
  std::vector<int64_t> cb{0};
  if (cs) {
    for (int64_t len = 1; cb.back() < n; len *= 2) cb.push_back(std::min<int64_t>(n, cb.back() + len));
  } else if (n > 0) {
    cb.push_back(n);
  }
  const int nchunks = (int)cb.size() - 1;
  // stage: (host inputs) allocate + H2D on the copy stream, one event per matrix
  auto stage_chunk = [&](int c) {
    for (int64_t i = cb[c]; i < cb[c + 1]; i++) {
      sfs_status st = check_csr(&mats[i]);
      if (st == SFS_OK) st = stage(&mats[i], d[i], cs ? cs : s, true);
      if (st == SFS_OK && d[i].host && cs) {
        ce[i] = ev.get();
        cudaEventRecord(ce[i], cs);
      }
      mst[i] = st;
    }
  };
  // features on the compute stream (after the matrix's copy)
  auto features_chunk = [&](int c) {
    for (int64_t i = cb[c]; i < cb[c + 1]; i++) {
      if (mst[i] != SFS_OK) continue;
      if (ce[i]) cudaStreamWaitEvent(s, ce[i], 0);
      fe0[i] = ev.get();
      fe1[i] = ev.get();
      cudaEventRecord(fe0[i], s);
      mst[i] = features_device(d[i], o, w[i], &ha[i], s);
      cudaEventRecord(fe1[i], s);
    }
  };
  using clk = std::chrono::steady_clock;
  const bool prof = getenv("SFS_PROFILE") != nullptr;
  double t_graph = 0, t_inst = 0, t_conv = 0, t_warm = 0, t_sync = 0;
  size_t flush_bytes = 0;
  if (o.cold && n > 0) {
    int dev = 0, l2 = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&l2, cudaDevAttrL2CacheSize, dev);
    flush_bytes = (size_t)std::max(l2, 1 << 20) * 2;
    own.flush = dalloc(flush_bytes, s);
  }
  void* flush = own.flush;
  // The race of one matrix: every format of its race set converted, warmed up and timed; nothing
  // synchronises.  The race set is formats_mask & race_mask[i] (a matrix with an
  // empty set is featurised only -- no conversion, no SpMV).  A launch error of any SpMV of a format
  // marks that format SFS_ERR_CUDA and keeps it out of the label (no silent near-zero time).
  auto race_one = [&](int64_t i) {
    sfs_label_t& L = labels[i];
    if (mst[i] != SFS_OK) {
      L.matrix_status = mst[i];
      return;
    }
    const sfs_features_t& F = feats[i];
    L.admissible_mask = F.admissible_mask;
    L.csr_variant = F.csr_variant;
    const DevCSR& D = d[i];
    const uint32_t race_set = o.formats_mask & (o.race_mask ? o.race_mask[i] : 0x1Fu);
    for (int f = 0; f < SFS_NFMT; f++) L.bytes[f] = sfs_spmv_bytes(&F, (sfs_format)f, (sfs_dtype)D.dtype);
    if (!(race_set & 0x1Fu)) return;  // features only
    const size_t sv = vbytes(D.dtype);
    void* y = dalloc(sv * D.m, s);
    void* xo = nullptr;
    const void* x = D.x;
    if (!x) {
      xo = dalloc(sv * D.n, s);
      if (xo) launch_fill(D.dtype, xo, D.n, 1.0, s);
      x = xo;
    }
    if (!y || !x) {
      L.matrix_status = SFS_ERR_OOM;
      dfree(y, s);
      dfree(xo, s);
      return;
    }
    for (int f = 0; f < SFS_NFMT; f++) {
      if (!(race_set & (1u << f))) { L.status[f] = SFS_ERR_NOT_RUN; continue; }
      if (!(F.admissible_mask & (1u << f))) { L.status[f] = SFS_ERR_INADMISSIBLE; continue; }
      Timed T;
      T.i = i;
      T.f = f;
      T.c0 = ev.get();
      T.c1 = ev.get();
      cudaEventRecord(T.c0, s);
      Matrix* A = nullptr;
      const auto tc0 = clk::now();
      sfs_status st = convert_impl(D, (sfs_format)f, F, w[i], &A, s);
      cudaEventRecord(T.c1, s);
      const auto tc1 = clk::now();
      t_conv += std::chrono::duration<double>(tc1 - tc0).count();
      if (st != SFS_OK) { L.status[f] = st; continue; }
      cudaError_t le = cudaSuccess;  // first launch error of this (matrix, format)
      auto chk = [&](cudaError_t e) {
        if (le == cudaSuccess && e != cudaSuccess) le = e;
      };
      for (int r = 0; r < o.warmup; r++) chk(launch_spmv(A, x, y, s));
      t_warm += std::chrono::duration<double>(clk::now() - tc1).count();
      const int kpc = spmv_kernels_per_call(A);
      if (o.cold) {
        for (int r = 0; r < o.reps; r++) {
          if (flush) chk(launch_l2_flush(flush, flush_bytes, s));
          cudaEvent_t a = ev.get(), b = ev.get();
          chk(cudaEventRecord(a, s));
          chk(launch_spmv(A, x, y, s));
          chk(cudaEventRecord(b, s));
          T.cold.push_back(a);
          T.cold.push_back(b);
        }
      } else if (o.use_graphs) {
        cudaGraph_t g = nullptr;
        cudaGraphExec_t ge = nullptr;
        const int64_t before = g_launches.load();
        const auto tg0 = clk::now();
        bool ok = cudaStreamBeginCapture(cap, cudaStreamCaptureModeThreadLocal) == cudaSuccess;
        if (ok) {
          for (int r = 0; r < o.reps; r++) ok = launch_spmv(A, x, y, cap) == cudaSuccess && ok;
          ok = cudaStreamEndCapture(cap, &g) == cudaSuccess && ok;
        }
        g_launches.store(before);
        const auto ti0 = clk::now();
        if (ok) ok = cudaGraphInstantiate(&ge, g, 0) == cudaSuccess;
        if (ok && up) {
          // upload the executable graph on a side stream (overlapping the work already queued on s)
          // instead of paying the implicit upload inside the timed launch
          cudaEvent_t eu = ev.get();
          ok = cudaGraphUpload(ge, up) == cudaSuccess && cudaEventRecord(eu, up) == cudaSuccess &&
               cudaStreamWaitEvent(s, eu, 0) == cudaSuccess;
        }
        t_inst += std::chrono::duration<double>(clk::now() - ti0).count();
        t_graph += std::chrono::duration<double>(clk::now() - tg0).count();
        if (ge) execs.push_back(ge);
        if (g) graphs.push_back(g);
        T.t0 = ev.get();
        T.t1 = ev.get();
        chk(cudaEventRecord(T.t0, s));
        if (ok) {
          chk(cudaGraphLaunch(ge, s));
          count_launch((int64_t)o.reps * kpc);
        } else {
          cudaGetLastError();  // a failed capture falls back to direct launches
          for (int r = 0; r < o.reps; r++) chk(launch_spmv(A, x, y, s));
        }
        chk(cudaEventRecord(T.t1, s));
      } else {
        T.t0 = ev.get();
        T.t1 = ev.get();
        chk(cudaEventRecord(T.t0, s));
        for (int r = 0; r < o.reps; r++) chk(launch_spmv(A, x, y, s));
        chk(cudaEventRecord(T.t1, s));
      }
      matrix_free(A);
      if (le != cudaSuccess) {
        cudaGetLastError();
        set_error(std::string("spmv launch (") + std::to_string(i) + ", " + std::to_string(f) +
                  "): " + cudaGetErrorString(le));
        L.status[f] = le == cudaErrorMemoryAllocation ? SFS_ERR_OOM : SFS_ERR_CUDA;
        continue;
      }
      L.status[f] = SFS_OK;
      timed.push_back(std::move(T));
    }
    dfree(y, s);
    dfree(xo, s);
  };
  const auto t_phase2 = clk::now();
  if (nchunks > 0) {
    stage_chunk(0);
    features_chunk(0);
  }
  cudaError_t e = cudaSuccess;
  for (int c = 0; c < nchunks; c++) {
    const auto ts0 = clk::now();
    e = cudaStreamSynchronize(s);  // this chunk's features (and the previous chunk's race) are done
    t_sync += std::chrono::duration<double>(clk::now() - ts0).count();
    if (e != cudaSuccess) return cuda_fail(e, c == 0 ? "feature phase" : "race");
    for (int64_t i = cb[c]; i < cb[c + 1]; i++) {
      if (mst[i] == SFS_OK) mst[i] = features_finish(d[i], o, ha[i], &feats[i], s);
      if (mst[i] == SFS_OK) labels[i].t_features_us = elapsed_us(fe0[i], fe1[i]);
    }
    if (c + 1 < nchunks) stage_chunk(c + 1);  // H2D of the next chunk overlaps this chunk's race
    for (int64_t i = cb[c]; i < cb[c + 1]; i++) race_one(i);
    // release the chunk's feature workspaces and staged inputs (stream-ordered)
    for (int64_t i = cb[c]; i < cb[c + 1]; i++) {
      dfree(w[i].base, s);
      w[i].base = nullptr;
      unstage(d[i], s);
    }
    if (c + 1 < nchunks) features_chunk(c + 1);
  }
  const auto t_enq = clk::now();
  e = cudaStreamSynchronize(s);
  if (prof) {
    const auto t_end = clk::now();
    fprintf(stderr,
            "[sfs] label_corpus n=%lld chunks=%d: enqueue %.1f ms (convert %.1f, warmup %.1f, graph capture %.1f + "
            "instantiate %.1f ms, chunk syncs %.1f ms), sync wait %.1f ms\n",
            (long long)n, nchunks, 1e3 * std::chrono::duration<double>(t_enq - t_phase2).count(), 1e3 * t_conv,
            1e3 * t_warm, 1e3 * (t_graph - t_inst), 1e3 * t_inst, 1e3 * t_sync,
            1e3 * std::chrono::duration<double>(t_end - t_enq).count());
  }
  if (e != cudaSuccess) return cuda_fail(e, "race");
  if (prof && !o.cold && !o.use_graphs && !timed.empty()) {  // where the device time of the race goes
    double conv = 0, warm = 0, reps = 0, gap = 0, conv_csr = 0;
    for (size_t k = 0; k < timed.size(); k++) {
      const Timed& T = timed[k];
      const double c = elapsed_us(T.c0, T.c1);
      (T.f == SFS_CSR ? conv_csr : conv) += c;
      warm += elapsed_us(T.c1, T.t0);
      reps += elapsed_us(T.t0, T.t1);
      if (k + 1 < timed.size()) gap += elapsed_us(T.t1, timed[k + 1].c0);
    }
    fprintf(stderr, "[sfs] race device time: conversions %.1f ms (CSR handles %.1f), warm-ups %.1f, timed reps %.1f, "
            "between formats %.1f ms\n", 1e-3 * conv, 1e-3 * conv_csr, 1e-3 * warm, 1e-3 * reps, 1e-3 * gap);
  }
  for (auto& T : timed) {
    sfs_label_t& L = labels[T.i];
    L.t_convert_us[T.f] = T.f == SFS_CSR ? 0.f : elapsed_us(T.c0, T.c1);
    double t = 0;
    if (o.cold) {
      for (size_t k = 0; k + 1 < T.cold.size(); k += 2) {
        const float u = elapsed_us(T.cold[k], T.cold[k + 1]);
        t = (u < 0 || t < 0) ? -1.0 : t + u;
      }
      if (t >= 0) t /= o.reps;
    } else {
      const float u = elapsed_us(T.t0, T.t1);
      t = u < 0 ? -1.0 : (double)u / o.reps;
    }
    if (!(t >= 0)) {  // an event that cannot be read is a failed format, not a time
      L.status[T.f] = SFS_ERR_CUDA;
      L.t_spmv_us[T.f] = 0.f;
      set_error("race: unreadable timing event");
      continue;
    }
    L.t_spmv_us[T.f] = (float)t;
  }
  // label: argmin over formats that ran, ties to the lowest id (Q14)
  for (int64_t i = 0; i < n; i++) {
    sfs_label_t& L = labels[i];
    if (L.matrix_status != SFS_OK) continue;
    int best = -1;
    for (int f = 0; f < SFS_NFMT; f++) {
      if (L.status[f] != SFS_OK) continue;
      if (best < 0 || L.t_spmv_us[f] < L.t_spmv_us[best]) best = f;
    }
    L.label = best;
  }
  return SFS_OK;
}

// ---------------------------------------------------------------- semi-supervised predictor (f1)
sfs_status sfs_features_table1(const sfs_features_t* f, int64_t n, double* out) {
  if (n < 0 || (n > 0 && (!f || !out))) return fail(SFS_ERR_INVALID_ARG, "null argument");
  for (int64_t i = 0; i < n; i++) {
    const sfs_features_t& F = f[i];
    const double row[SFS_NFEAT] = {(double)F.nrows,     (double)F.ncols,    (double)F.nnz,        F.nnz_frac,
                                   F.nnz_mu,            (double)F.nnz_min,  (double)F.nnz_max,    F.nnz_sig,
                                   F.max_mu,            F.mu_min,           (double)F.csr_max,    F.sig_lower,
                                   F.sig_higher,        (double)F.hyb_ell_size, (double)F.hyb_coo, F.hyb_ell_frac,
                                   (double)F.diagonals, (double)F.dia_size, F.dia_frac,           F.ell_frac,
                                   (double)F.ell_size};
    memcpy(out + i * SFS_NFEAT, row, sizeof(row));
  }
  return SFS_OK;
}

sfs_status sfs_cluster_fit(const double* table1, int64_t n, const int32_t* init_idx, const sfs_cluster_opts* opt,
                           sfs_cluster_model* out, void* stream) {
  if (!table1 || !init_idx || !opt || !out || n < 1) return fail(SFS_ERR_INVALID_ARG, "null argument / empty corpus");
  if (opt->nc < 1 || opt->nc > n || opt->pcs < 1 || opt->pcs > 16 || opt->max_iter < 1)
    return fail(SFS_ERR_INVALID_ARG, "need 1 <= nc <= n, 1 <= pcs <= 16, max_iter >= 1");
  if ((size_t)opt->nc * opt->pcs * sizeof(double) > 200 * 1024) return fail(SFS_ERR_UNSUPPORTED, "nc * pcs too large");
  for (int c = 0; c < opt->nc; c++)
    if (init_idx[c] < 0 || init_idx[c] >= n) return fail(SFS_ERR_INVALID_ARG, "init index out of range");
  ClusterModel* M = cluster_new();
  cudaError_t e = cluster_fit(table1, n, init_idx, opt->nc, opt->pcs, opt->max_iter, M, (cudaStream_t)stream);
  if (e != cudaSuccess) {
    cluster_free(M);
    return cuda_fail(e, "cluster fit");
  }
  *out = (sfs_cluster_model)M;
  return SFS_OK;
}

sfs_status sfs_cluster_vote(sfs_cluster_model Mh, const int32_t* labels, int32_t* cluster_label, void* stream) {
  if (!Mh || !labels || !cluster_label) return fail(SFS_ERR_INVALID_ARG, "null argument");
  cudaError_t e = cluster_vote((const ClusterModel*)Mh, labels, cluster_label, (cudaStream_t)stream);
  return e == cudaSuccess ? SFS_OK : cuda_fail(e, "cluster vote");
}

sfs_status sfs_cluster_predict(sfs_cluster_model Mh, const double* table1, int64_t q, int32_t* cluster, void* stream) {
  if (!Mh || !table1 || !cluster || q < 1) return fail(SFS_ERR_INVALID_ARG, "null argument");
  cudaError_t e = cluster_predict((const ClusterModel*)Mh, table1, q, cluster, (cudaStream_t)stream);
  return e == cudaSuccess ? SFS_OK : cuda_fail(e, "cluster predict");
}

sfs_status sfs_cluster_describe(sfs_cluster_model Mh, sfs_cluster_info* out) {
  if (!Mh || !out) return fail(SFS_ERR_INVALID_ARG, "null argument");
  cluster_info((const ClusterModel*)Mh, out);
  return SFS_OK;
}

sfs_status sfs_cluster_free(sfs_cluster_model Mh) {
  cluster_free((ClusterModel*)Mh);
  return SFS_OK;
}

}  // extern "C"
