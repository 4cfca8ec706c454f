/* sfs.h — C ABI of libsfs: B200-native featurisation, format conversion, per-format SpMV and
 * format-race labelling of sparse matrices.
 *
 * Paper: Dhandhania, Deodhar, Pogorelov, Biswas, Langguth, "Explaining the Performance of Supervised
 * and Semi-Supervised Methods for Automated Sparse Matrix Format Selection", ICPP Workshops '21
 * (/root/reference/PAPER.md; "P:L<n>" = its line n).  The library implements the benchmarking /
 * labelling pass the paper identifies as the cost of supervised training (§1, §5.1,
 * P:L331–333 §5.4): for each matrix, the Table-1 features, conversion of the CSR input
 * into every candidate format (§2.1, P:L331 step ii), timed SpMV y = A·x in each format
 * ("average over 100 trials" P:L217, step iii of P:L331) and the fastest format as label
 * (§1).  Readings where the paper is silent are DESIGN.md §"Readings" (Q1–Q18).
 *
 * Conventions (every function):
 *  - All array pointers are DEVICE pointers unless a field says otherwise (sfs_csr.mem).
 *  - `stream` is a cudaStream_t passed as void* (NULL = legacy default stream).  All work is
 *    stream-ordered on it.  Only functions that return host results synchronize it (marked
 *    "syncs").  sfs_spmv never synchronizes.
 *  - No C++ exception crosses the ABI.  Every call returns an sfs_status; CUDA errors map to
 *    SFS_ERR_CUDA with the detail in sfs_last_error() (thread-local string).
 *  - Indices are int32: nnz >= 2^31 or nrows/ncols >= 2^31 gives SFS_ERR_UNSUPPORTED.  Size
 *    features are int64 (an inadmissible ELL can have > 2^31 slots).
 *  - x, y and the matrix values share one dtype (fp32 or fp64).
 *  - Input CSR must be canonical (Q16): row_ptr[0] = 0, row_ptr non-decreasing,
 *    row_ptr[nrows] = nnz, 0 <= col < ncols, columns strictly increasing within a row.  Empty
 *    rows and explicit zeros are allowed.  Checked on the device; violation -> SFS_ERR_INVALID_CSR.
 *  - Library-owned buffers (sfs_matrix) come from the allocator hook (default: a CUDA
 *    stream-ordered memory pool) and live until sfs_matrix_free.
 *  - GPU only: without a CUDA device every compute call returns SFS_ERR_CUDA.  There is no CPU
 *    fallback.
 */
#ifndef SFS_H
#define SFS_H
#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  SFS_OK = 0,
  SFS_ERR_INVALID_ARG = -1,
  SFS_ERR_INVALID_CSR = -2,
  SFS_ERR_INADMISSIBLE = -3, /* ELL / DIA past the fill guard (Q11; cf. CUSP size failures P:L194) */
  SFS_ERR_OOM = -4,
  SFS_ERR_CUDA = -5,
  SFS_ERR_UNSUPPORTED = -6,
  SFS_ERR_NOT_RUN = -7       /* format excluded by formats_mask */
} sfs_status;

/* Formats of P:L73 (§2.1) raced by the paper plus DIA.  The enum order is the
   tie-break order of the label rule (Q14). */
typedef enum { SFS_CSR = 0, SFS_COO = 1, SFS_ELL = 2, SFS_HYB = 3, SFS_DIA = 4, SFS_NFMT = 5 } sfs_format;
typedef enum { SFS_F32 = 0, SFS_F64 = 1 } sfs_dtype;
typedef enum { SFS_MEM_DEVICE = 0, SFS_MEM_HOST = 1 } sfs_memspace;

/* A borrowed CSR matrix (caller-owned; never freed or written by the library).
   mem = SFS_MEM_HOST: row_ptr/col_idx/values (and x) are host pointers (pinned for speed); the
   library copies them to the device inside the call (this is the end-to-end path). */
typedef struct {
  int64_t nrows, ncols, nnz;
  const int32_t *row_ptr; /* nrows+1 */
  const int32_t *col_idx; /* nnz */
  const void *values;     /* nnz of float (SFS_F32) or double (SFS_F64) */
  int32_t dtype;          /* sfs_dtype */
  int32_t mem;            /* sfs_memspace of the four pointers */
  const void *x;          /* sfs_label_corpus only: race input vector (ncols); NULL = all ones */
} sfs_csr;

/* Table-1 features, host struct.  Integer features are exact; each double is one
   fixed fp64 expression of exact integer aggregates (DESIGN.md §"Readings" Q1–Q9). */
typedef struct {
  int64_t nrows, ncols, nnz, nnz_min, nnz_max, csr_max, ell_size, hyb_k, hyb_ell_size, hyb_coo,
      hyb_ell_nnz, diagonals, dia_size;
  double nnz_frac, nnz_mu, nnz_sig, max_mu, mu_min, sig_lower, sig_higher, hyb_ell_frac, dia_frac,
      ell_frac;
  uint32_t admissible_mask; /* bit f set iff format f is admissible (Q11) */
  int32_t csr_variant;      /* CSR kernel the library picks for this matrix (Q17): 0 vector (CUSP
                               mapping), 1 merge path, 2 stream (warp per 32 rows), 3 tile
                               (nnz-balanced 256-entry chunks, rows rebuilt from row_ptr), 4 tile
                               with rows from a row-start bitmap (no empty rows), 5 tile with a
                               bitmap over the non-empty rows and a rank -> row map (empty rows) */
} sfs_features_t;

typedef struct sfs_matrix_ *sfs_matrix; /* opaque, library-owned */

/* Physical layout of a converted matrix (read-only device pointers, for tests / inspection).
   pitch P = ceil(nrows/32)*32.  ptr[] by format:
     CSR: 0 row_ptr, 1 col, 2 val                       (borrowed from the caller for device input)
     COO: 0 row, 1 col, 2 val                           (nnz each, CSR order)
     ELL: 0 col[width*P], 1 val[width*P]                column-major slab: entry (r, j) at j*P + r;
                                                        padding col = -1, val = +0 (Q10)
     HYB: 0 ell col, 1 ell val (width = hyb_k, as ELL), 2 coo row, 3 coo col, 4 coo val (coo_nnz)
     DIA: 0 offsets[ndiag] (ascending), 1 val[ndiag*P]  entry (d, r) at d*P + r, +0 where absent */
typedef struct {
  int32_t fmt, dtype;
  int64_t nrows, ncols, nnz, pitch, width, ndiag, coo_nnz;
  const void *ptr[6];
  int64_t bytes;     /* device bytes owned by the handle */
  int32_t variant;   /* CSR kernel variant (Q17) */
} sfs_layout_t;

/* Race options (mean of 100 trials).  sfs_default_opts fills the DESIGN.md defaults. */
typedef struct {
  int32_t reps;          /* timed SpMVs per format (100) */
  int32_t warmup;        /* untimed SpMVs before timing (5) (Q13) */
  uint32_t formats_mask; /* formats to race (0x1F = all five; 0x0F = the paper's four) */
  int32_t cold;          /* 0 = back-to-back reps (labels); 1 = flush L2 before every rep */
  double max_fill;       /* Q11 ELL/DIA guard: slots <= max(trunc(max_fill*nnz), fill_slack) (3.0) */
  int64_t fill_slack;    /* (1<<20) */
  double hyb_rel_speed;  /* Q6 HYB width rule (3.0) */
  int64_t hyb_breakeven; /* (4096) */
  int32_t csr_variant;   /* -1 = pick by Q17; 0 = vector; 1 = merge; 2 = stream; 3 = tile; 4 = tile with row ids from a row-start bitmap (becomes 5 when a row is empty); 5 = tile with a bitmap over the non-empty rows + rank -> row map */
  int32_t use_graphs;    /* 1 = capture the `reps` launches in one CUDA graph (0: direct launches with PDL) */
  const uint32_t *race_mask; /* sfs_label_corpus only, nullable (HOST array of n): matrix i races the
                                formats formats_mask & race_mask[i]; 0 = features only (no conversion,
                                no SpMV; label -1, every status SFS_ERR_NOT_RUN) -- the cluster-subset
                                labelling of P:L134 / P:L167-169 ("benchmark only one matrix from each
                                cluster").  NULL = every matrix races formats_mask. */
} sfs_race_opts;

/* Result of racing one matrix. */
typedef struct {
  int32_t label;            /* argmin t_spmv over run formats, ties to the lowest id (Q14); -1 if none */
  uint32_t admissible_mask; /* Q11 */
  int32_t matrix_status;    /* SFS_OK or the error that stopped this matrix (e.g. INVALID_CSR) */
  int32_t csr_variant;
  float t_spmv_us[SFS_NFMT];    /* mean device time of one SpMV (CUDA events around `reps`) */
  float t_convert_us[SFS_NFMT]; /* device time of CSR -> f (0 for CSR) */
  int32_t status[SFS_NFMT];     /* SFS_OK, SFS_ERR_INADMISSIBLE, SFS_ERR_NOT_RUN, SFS_ERR_OOM, ... */
  int64_t bytes[SFS_NFMT];      /* algorithmic bytes of one SpMV in format f */
  float t_features_us;          /* device time of the feature pass (batched: 0 if not measured) */
} sfs_label_t;

void sfs_default_opts(sfs_race_opts *opt);

/* Table-1 features of A.  opt may be NULL (defaults; used for HYB width and
   admissibility).  One fused device pass over row_ptr and col_idx + two small kernels.  Syncs.
   Errors: INVALID_ARG (null/negative sizes), UNSUPPORTED (int32 overflow), INVALID_CSR, CUDA. */
sfs_status sfs_features(const sfs_csr *A, const sfs_race_opts *opt, sfs_features_t *out, void *stream);

/* Convert A into format f (step (ii) of P:L331) into a new library-owned handle *out.
   Runs the feature pass internally (needed for widths / diagonals).  Syncs once (after features).
   INADMISSIBLE for ELL / DIA past the fill guard (Q11).  For f = CSR with device input the handle
   borrows A's arrays (the caller keeps them alive); with host input it owns device copies. */
sfs_status sfs_convert(const sfs_csr *A, sfs_format f, const sfs_race_opts *opt, sfs_matrix *out, void *stream);

/* y = A·x with A in format f (f must equal A's format, else INVALID_ARG).  x has ncols
   entries, y has nrows entries, device pointers of A's dtype; y is fully overwritten.  Asynchronous:
   1–3 kernel launches on `stream` (a zero pass and the kernels of the format; HYB with long overflow
   rows runs its ELL and COO parts concurrently), no synchronization. */
sfs_status sfs_spmv(sfs_format f, sfs_matrix A, const void *x, void *y, void *stream);

/* Label a batch of matrices: features of all n matrices (batched), then for each
   matrix and each admissible format in opt->formats_mask: convert (event-timed), `warmup` untimed
   SpMVs, `reps` timed SpMVs (CUDA events), free; label = argmin (Q14).  feats / labels are host
   arrays of n entries.  A matrix-level error (e.g. INVALID_CSR) is reported in
   labels[i].matrix_status and does not abort the batch; a format-level error (OOM) only marks
   status[f].  A launch error or an unreadable timing event of one format marks status[f] =
   SFS_ERR_CUDA (detail in sfs_last_error) and keeps that format out of the label; the batch goes on.
   opt->race_mask restricts the race per matrix (featurisation always runs).  Host-memory matrices are copied to the device inside the call and stay resident
   until it returns (callers batch large corpora).  Syncs.  Returns SFS_OK unless an argument is
   invalid or CUDA fails. */
sfs_status sfs_label_corpus(const sfs_csr *mats, int64_t n, const sfs_race_opts *opt, sfs_features_t *feats,
                            sfs_label_t *labels, void *stream);

/* Halo send buffer of the row-partitioned SpMV (y = A·x of P:L31 split by
   rows): dst[i] = src[idx[i]] for 0 <= i < n.  src: the rank's slice of x (device, dtype); idx: int32
   device array of local indices, each in [0, len(src)) (not checked); dst: n entries (device, dtype),
   caller-owned.  Asynchronous on `stream`, one kernel launch (none if n == 0).  INVALID_ARG for a bad
   dtype, n < 0 or a null pointer with n > 0. */
sfs_status sfs_gather(sfs_dtype dtype, const void *src, const int32_t *idx, int64_t n, void *dst, void *stream);

/* Row-partitioned SpMV with the halo exchange fused in (SURVEY §8(e) 2, §8(f) f3 "stores of y into
   every peer's x"; y = A·x of P:L31 split by rows).  Rank k holds a row block of A with its columns
   renumbered into x_ext = [ghosts below | own slice | ghosts above] and writes y into the own slice of
   its next x_ext.  Each neighbour j needs some of those y entries as its ghosts; they form contiguous
   runs of local rows (a banded/stencil block: one run per neighbour) and land in contiguous runs of
   j's next x_ext.  sfs_spmv_push computes y = A·x and stores every y[r] with r in a run also into the
   run's destination -- peer memory mapped into this process (NVLink P2P / symmetric memory, or plain
   device memory when P ranks are simulated on one GPU) -- from the same kernel that computes it, so
   the transfer overlaps the SpMV tile by tile.  Completion protocol (flags are uint32 in device
   memory, monotonically increasing epochs):
     start: every CTA waits until *wait_flag[i] >= wait_value for all i < nwait (acquire, system
            scope) before reading x: the neighbours have pushed this epoch's ghosts into x and have
            finished reading the buffer this call pushes into (double-buffered x_ext);
     end:   after all CTAs' stores, the last CTA (counted in *counter, which it resets to 0) stores
            sig_value into every *sig_flag[i] (release, system scope).
   Fused in one kernel for DIA, ELL and the CSR stream kernel; the other kernels run as
   wait kernel -> SpMV -> push kernel (same protocol, three launches).  Runs must not overlap and must
   lie in [0, nrows).  INVALID_ARG for bad counts / null pointers, else as sfs_spmv.  Asynchronous. */
#define SFS_MAX_PUSH 8
#define SFS_MAX_PEERS 16
typedef struct {
  int32_t nseg;                              /* runs, <= SFS_MAX_PUSH */
  int64_t seg_begin[SFS_MAX_PUSH];           /* local rows [seg_begin, seg_end) of y ... */
  int64_t seg_end[SFS_MAX_PUSH];
  void *seg_dst[SFS_MAX_PUSH];               /* ... also stored at seg_dst[r - seg_begin] (dtype) */
  int32_t nwait;                             /* <= SFS_MAX_PEERS */
  const uint32_t *wait_flag[SFS_MAX_PEERS];  /* this rank's flag slots, written by its neighbours */
  uint32_t wait_value;
  int32_t nsig;                              /* <= SFS_MAX_PEERS */
  uint32_t *sig_flag[SFS_MAX_PEERS];         /* this rank's slot in each neighbour's flags */
  uint32_t sig_value;
  uint32_t *counter;                         /* device, zero before the first call; one per rank */
} sfs_push_t;
sfs_status sfs_spmv_push(sfs_format f, sfs_matrix A, const void *x, void *y, const sfs_push_t *push,
                         void *stream);
/* Peer memory for the push (plumbing; CUDA IPC): sfs_ipc_alloc allocates `bytes` of zeroed device memory
   on the current device and writes its 64-byte IPC handle; another process on the node maps it with
   sfs_ipc_open (peer access enabled lazily, so a buffer on another GPU is reached over NVLink) and
   unmaps it with sfs_ipc_close; the owner frees it with sfs_ipc_free.  Synchronous; CUDA errors ->
   SFS_ERR_CUDA. */
sfs_status sfs_ipc_alloc(size_t bytes, void **ptr, uint8_t handle[64]);
sfs_status sfs_ipc_open(const uint8_t handle[64], void **ptr);
sfs_status sfs_ipc_close(void *ptr);
sfs_status sfs_ipc_free(void *ptr);
/* The push alone (no SpMV): stores src[r] (r in the runs) into the runs' destinations with the same
   wait / signal protocol -- the initial ghost exchange before the first sfs_spmv_push.  src: nrows
   entries of dtype (device).  One kernel launch. */
sfs_status sfs_halo_push(sfs_dtype dtype, const void *src, int64_t nrows, const sfs_push_t *push, void *stream);

sfs_status sfs_matrix_free(sfs_matrix A); /* stream-ordered on the stream it was created on */
sfs_status sfs_matrix_describe(sfs_matrix A, sfs_layout_t *out);

/* Algorithmic bytes of one SpMV in format f for a matrix with features F and dtype (§8(a)
   a9–a13: each format array read once, x read once, y written once; padding counted). */
int64_t sfs_spmv_bytes(const sfs_features_t *F, sfs_format f, sfs_dtype dtype);

const char *sfs_status_string(sfs_status s);
const char *sfs_last_error(void);

/* Allocator hook: both NULL restores the default pool.  alloc must return 256-byte aligned device
   memory usable on `stream`; dealloc is called stream-ordered. */
void sfs_set_allocator(void *(*alloc)(size_t bytes, void *stream), void (*dealloc)(void *p, void *stream));

/* Number of kernels this library has launched in this process (graph replays count every node).
   Lets benchmarks state how many of *our* kernels ran inside a timed region. */
int64_t sfs_launch_count(void);

/* ---------------------------------------------------------------------------------------------
 * Semi-supervised format predictor (§4), fitted on the
 * Table-1 features of a labelled corpus: log1p / sqrt transform and min-max scaling, PCA to
 * `pcs` components, K-Means with `nc` clusters, cluster label = majority
 * vote of the benchmarked members, prediction = label of the nearest centroid.
 * Readings F1–F7 (transform per feature, PCA sign, K-Means start / stop, vote ties): DESIGN.md.
 * All arrays are HOST arrays (the data is small); the corpus-sized work runs on the GPU.  Syncs. */
#define SFS_NFEAT 21
typedef struct {
  int32_t nc;       /* clusters */
  int32_t pcs;      /* PCA components (8; <= 16) */
  int32_t max_iter; /* K-Means iteration cap (100); stops early when no assignment changes */
} sfs_cluster_opts;
typedef struct sfs_cluster_model_ *sfs_cluster_model;
typedef struct {
  int64_t n;                 /* training matrices */
  int32_t nc, pcs, iters;
  const int32_t *assign;     /* n: cluster of every training matrix */
  const double *centroids;   /* nc x pcs */
  const double *basis;       /* pcs x 21 (row = component) */
  const double *eigval;      /* pcs */
  const double *mins, *maxs; /* 21: transformed-feature ranges used for scaling */
  const double *mean;        /* 21: mean of the scaled training features */
} sfs_cluster_info;

/* n x 21 Table-1 matrix (P:L79–102 order) from feature records (host in, host out). */
sfs_status sfs_features_table1(const sfs_features_t *f, int64_t n, double *out);
/* Fit on n matrices (table1: n x 21 host).  init_idx: nc distinct indices of the starting points
   (drawn by the caller, e.g. from a seeded generator).  INVALID_ARG on bad sizes / indices. */
sfs_status sfs_cluster_fit(const double *table1, int64_t n, const int32_t *init_idx, const sfs_cluster_opts *opt,
                           sfs_cluster_model *out, void *stream);
/* labels: n formats of the training matrices, -1 = not benchmarked; cluster_label: nc (host). */
sfs_status sfs_cluster_vote(sfs_cluster_model M, const int32_t *labels, int32_t *cluster_label, void *stream);
/* Nearest-centroid cluster of q new matrices (table1: q x 21 host) -> cluster (q, host). */
sfs_status sfs_cluster_predict(sfs_cluster_model M, const double *table1, int64_t q, int32_t *cluster, void *stream);
sfs_status sfs_cluster_describe(sfs_cluster_model M, sfs_cluster_info *out);
sfs_status sfs_cluster_free(sfs_cluster_model M);
/* The PCA eigen-step of sfs_cluster_fit on its own (host arrays, host computation, no GPU needed):
   leading k eigenpairs of the symmetric n x n matrix cov (row-major, 1 <= k <= n <= 64) by Householder
   tridiagonalisation + implicit QL; eigval descending, basis k x n (row = eigenvector) with each row's
   largest-magnitude entry (first on ties) positive (reading F3).  INVALID_ARG on bad sizes,
   UNSUPPORTED if the iteration does not converge. */
sfs_status sfs_pca_basis(int32_t n, const double *cov, int32_t k, double *basis, double *eigval);

/* Library version string. */
const char *sfs_version(void);

#ifdef __cplusplus
}
#endif
#endif
