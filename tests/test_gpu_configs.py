"""GPU parity at BASELINE.json's full sizes (configs[0], [2], [3], a slice of configs[1], every generator class of configs[4] and its largest early matrix),
through the same C-ABI calls the bench times."""
import numpy as np
import pytest

import oracle
import paper_conf_icppw_dhandhaniadpbl21_b200 as sfs
import sfsgen
from gpu_util import assert_features_equal, check_conversion, check_spmv, to_dev

pytestmark = pytest.mark.gpu


def _full_check(A, formats=range(5), conv=True, ctx=""):
    fo = oracle.features(A.m, A.n, A.rp, A.col)
    dA = to_dev(A)
    assert_features_equal(sfs.features(dA), fo, ctx)
    x = sfsgen.vector(2024, A.n, A.dtype)
    for fmt in formats:
        if not (fo["admissible_mask"] >> fmt) & 1:
            continue
        M = sfs.convert(dA, fmt)
        if conv:
            check_conversion(A, fmt, M, fo)
        check_spmv(A, fmt, M, x, A.dtype, ctx=ctx)
        M.free()
    return fo


def test_config0_laplace_64_fp64():
    A = sfsgen.laplace2d(64)
    fo = _full_check(A, ctx="configs[0]")
    assert fo["admissible_mask"] == 31


def test_config2_rmat_22_fp32():
    A = sfsgen.rmat(22, seed=1)
    fo = _full_check(A, formats=(sfs.CSR, sfs.COO, sfs.HYB), conv=True, ctx="configs[2]")
    assert not (fo["admissible_mask"] >> sfs.ELL) & 1 and not (fo["admissible_mask"] >> sfs.DIA) & 1
    assert fo["nnz"] > 60_000_000 and fo["nnz_max"] > 50_000
    # every CSR kernel that handles empty rows, at full size (52 % of R-MAT's rows are empty)
    dA = to_dev(A)
    x = sfsgen.vector(2024, A.n, A.dtype)
    for v in (1, 3, 5):
        M = sfs.convert(dA, sfs.CSR, sfs.default_opts(csr_variant=v))
        assert M.layout().variant == v
        check_spmv(A, sfs.CSR, M, x, A.dtype, ctx=f"configs[2] CSR variant {v}")
        M.free()


def test_config3_stencil3d27_128_fp64():
    A = sfsgen.stencil3d27(128)
    fo = _full_check(A, ctx="configs[3]")
    assert (fo["nnz"], fo["diagonals"], fo["hyb_k"]) == (55742968, 27, 27)


@pytest.mark.parametrize("i", [0, 1, 2, 3, 4, 5, 6, 7])
def test_config1_corpus_slice(i):
    A = sfsgen.generate(sfsgen.corpus_spec(200, i))
    _full_check(A, conv=(A.nnz < 20_000_000), ctx=f"corpus200[{i}]")


# configs[4] (SuiteSparse-shaped corpus-2000): one small matrix of every generator class (band,
# uniform, block-diagonal, power-law, R-MAT, 2D5 / 3D7 / 3D27 stencils) fully, plus the largest of
# the first 200 corpus-2000 matrices (features bit-exact, SpMV per row) at full size.
@pytest.mark.parametrize("i", [1, 2, 5, 8, 12, 20, 24, 61, 75])
def test_config4_corpus2000_classes(i):
    A = sfsgen.generate(sfsgen.corpus_spec(2000, i))
    _full_check(A, ctx=f"corpus2000[{i}]")


def test_config4_corpus2000_largest_sample():
    A = sfsgen.generate(sfsgen.corpus_spec(2000, 164))  # 47.0 M nnz, uniform random, fp64
    assert A.nnz > 40_000_000
    _full_check(A, conv=False, ctx="corpus2000[164]")


# fp32 DIA / ELL at bandwidth-bound sizes (the TMA slab-ring kernels k_spmv_dia_tma / k_spmv_ell_tma at the
# default size and diagonal / slot gates): the configs[3] stencil in fp32, a ragged stencil (343000 rows:
# partial last 1024-row block) and a ragged 1M-row band, all formats, element by element against the
# oracle.
def test_config3_stencil3d27_128_fp32():
    A = sfsgen.stencil3d27(128, dtype=sfsgen.F32)
    fo = _full_check(A, formats=(sfs.ELL, sfs.DIA), conv=True, ctx="configs[3] fp32")
    assert fo["diagonals"] == 27


@pytest.mark.parametrize("mk", ["st70", "band"])
def test_dia_fp32_bandwidth_bound_ragged(mk):
    if mk == "st70":
        A = sfsgen.stencil3d27(70, dtype=sfsgen.F32)
    else:
        A = sfsgen.generate(sfsgen.make_spec(sfsgen.BAND, seed=12, m=1_000_003, ia=24, pa=0.8, dtype=sfsgen.F32))
    assert A.m >= 148 * 2 * 1024 and A.m % 1024 != 0
    fo = _full_check(A, ctx=f"dia fp32 {mk}")
    assert (fo["admissible_mask"] >> sfs.DIA) & 1
