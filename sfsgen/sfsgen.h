/* sfsgen.h — seeded synthetic sparse-matrix generators (TEST / BENCH INPUT ONLY).
 *
 * This module is shared input infrastructure: it is the ONLY code that both the CPU oracle
 * (oracle/) and the CUDA path (paper_conf_icppw_dhandhaniadpbl21_b200/) are fed from.  It holds
 * none of the method's arithmetic (no features, no conversion, no SpMV): it only draws matrices.
 *
 * The paper's workloads are SuiteSparse matrices (§5.1 "Benchmarks"), which are not
 * available offline.  These generators stand in for the structure classes the paper draws on
 * (banded, uniform random, block-diagonal, power-law / R-MAT graphs, PDE stencils); the recipe is
 * SURVEY.md Appendix B and DESIGN.md §"Input recipe".
 *
 * All arithmetic is uint64 with wrap-around (splitmix64 counter hash), so every entry is a pure
 * function of (seed, row, col) and the output does not depend on the thread count.
 * Output CSR is canonical: rp[0] = 0, columns strictly increasing within a row, no explicit zeros.
 */
#ifndef SFSGEN_H
#define SFSGEN_H
#include <stdint.h>
#ifdef __cplusplus
extern "C" {
#endif

enum {
  SFSGEN_BAND = 0,      /* ia = half-bandwidth b, pa = fill p              */
  SFSGEN_BLOCKDIAG = 1, /* ia = block size B,   pa = fill p                */
  SFSGEN_UNIFORM = 2,   /* pa = lambda (mean row length before dedup)      */
  SFSGEN_POWERLAW = 3,  /* pa = alpha (row-length tail exponent)           */
  SFSGEN_RMAT = 4,      /* ia = scale, ib = edge factor                    */
  SFSGEN_ST2D5 = 5,     /* ia = N (grid N x N)                             */
  SFSGEN_ST3D7 = 6,     /* ia = N (grid N^3)                               */
  SFSGEN_ST3D27 = 7     /* ia = N (grid N^3)                               */
};

typedef struct {
  int32_t cls;
  int32_t dtype; /* 0 = fp32 values, 1 = fp64 values */
  uint64_t seed;
  int64_t m, n;  /* ignored (derived) for RMAT and stencils */
  int64_t ia, ib;
  double pa, pb;
} sfsgen_spec;

typedef struct {
  int64_t m, n, nnz;
  int32_t *rp;  /* m+1 */
  int32_t *col; /* nnz */
  void *val;    /* nnz of float or double (spec.dtype) */
  int32_t dtype;
} sfsgen_csr;

uint64_t sfsgen_splitmix64(uint64_t x);
uint64_t sfsgen_hash(uint64_t seed, uint64_t a, uint64_t b);

/* Fill dimensions for a spec (m, n) without generating. */
int sfsgen_dims(const sfsgen_spec *s, int64_t *m, int64_t *n);
/* Generate into malloc'd buffers (free with sfsgen_free). Returns 0 on success. */
int sfsgen_generate(const sfsgen_spec *s, sfsgen_csr *out);
void sfsgen_free(sfsgen_csr *c);
/* Dense vector x_j = 2*U(H(seed^0x78, j, 0)) - 1, j < n, as fp32 (dtype 0) or fp64 (dtype 1). */
void sfsgen_vector(uint64_t seed, int64_t n, int32_t dtype, void *out);
/* Per-matrix parameters of a named corpus (200 = BASELINE configs[1], 2000 = configs[4]). */
int sfsgen_corpus_spec(int32_t corpus, int64_t i, sfsgen_spec *out);
/* Number of threads the generator uses (OpenMP). */
int sfsgen_threads(void);

/* The same generators on the GPU (gen_device.cu, libsfsgen_dev.so): bit-identical CSR in device memory
   (cudaMalloc'd rp/col/val; free with sfsgen_free_device), stream-ordered on `stream` (a cudaStream_t),
   synchronizes it before returning.  Returns 0 on success. */
int sfsgen_generate_device(const sfsgen_spec *s, sfsgen_csr *out, void *stream);
void sfsgen_free_device(sfsgen_csr *c);
/* x on the device (out: n entries of dtype), asynchronous on `stream`. */
int sfsgen_vector_device(uint64_t seed, int64_t n, int32_t dtype, void *out, void *stream);

#ifdef __cplusplus
}
#endif
#endif
