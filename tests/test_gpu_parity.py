"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle on the same seeded inputs.

Bars (BASELINE.json north_star): features and conversions bit-exact; SpMV per row
|y - y_ref| <= tol * (|A||x|)_r with tol 1e-12 (fp64) / 1e-5 (fp32), rows with |A||x| = 0 exactly 0.
"""
import numpy as np
import pytest

import oracle
import paper_conf_icppw_dhandhaniadpbl21_b200 as sfs
import sfsgen
from gpu_util import assert_features_equal, check_conversion, check_spmv, to_dev
from helpers import golden, q11_boundary_cases, random_csr

pytestmark = pytest.mark.gpu


def _cases():
    rng = np.random.default_rng(1234)
    cases = {
        "tiny4x4": sfsgen.from_dense(np.array(golden("tiny4x4.json")["A"], float)),
        "1x1": sfsgen.from_dense(np.array([[2.5]])),
        "empty": sfsgen.CSR(7, 5, np.zeros(8, np.int32), np.zeros(0, np.int32), np.zeros(0)),
        "laplace64": sfsgen.laplace2d(64),
        "rand_ragged": random_csr(rng, 3001, 2777, 0.004, empty_rows=0.3, dense_rows=2),
        "rand_zeros": random_csr(rng, 500, 700, 0.02, explicit_zero=0.2),
        "band": sfsgen.generate(sfsgen.make_spec(sfsgen.BAND, seed=3, m=20011, ia=9, pa=0.7)),
        "blockdiag32": sfsgen.generate(sfsgen.make_spec(sfsgen.BLOCKDIAG, seed=4, m=9001, ia=37, pa=0.8,
                                                         dtype=sfsgen.F32)),
        "uniform": sfsgen.generate(sfsgen.make_spec(sfsgen.UNIFORM, seed=5, m=12000, n=9000, pa=17.0)),
        "powerlaw32": sfsgen.generate(sfsgen.make_spec(sfsgen.POWERLAW, seed=6, m=30000, pa=2.15, dtype=sfsgen.F32)),
        "rmat14": sfsgen.rmat(14, seed=7),
        "st3d27_20": sfsgen.generate(sfsgen.make_spec(sfsgen.ST3D27, ia=20)),
        "st3d7_32f": sfsgen.generate(sfsgen.make_spec(sfsgen.ST3D7, ia=33, dtype=sfsgen.F32)),
    }
    return cases


CASES = None


def cases():
    global CASES
    if CASES is None:
        CASES = _cases()
    return CASES


NAMES = ["tiny4x4", "1x1", "empty", "laplace64", "rand_ragged", "rand_zeros", "band", "blockdiag32", "uniform",
         "powerlaw32", "rmat14", "st3d27_20", "st3d7_32f"]


@pytest.mark.parametrize("name", NAMES)
def test_features_bit_exact(name):
    A = cases()[name]
    fg = sfs.features(to_dev(A))
    fo = oracle.features(A.m, A.n, A.rp, A.col)
    assert_features_equal(fg, fo, name)


@pytest.mark.parametrize("name", NAMES)
def test_conversions_bit_exact(name):
    A = cases()[name]
    fo = oracle.features(A.m, A.n, A.rp, A.col)
    dA = to_dev(A)
    for fmt in range(5):
        if not (fo["admissible_mask"] >> fmt) & 1:
            with pytest.raises(sfs.SfsError) as ei:
                sfs.convert(dA, fmt)
            assert ei.value.status == sfs.ERR_INADMISSIBLE
            continue
        M = sfs.convert(dA, fmt)
        check_conversion(A, fmt, M, fo)
        M.free()


@pytest.mark.parametrize("name", NAMES)
@pytest.mark.parametrize("variant", [0, 1, 2, 3, 4, 5])
def test_spmv_tolerance(name, variant):
    A = cases()[name]
    fo = oracle.features(A.m, A.n, A.rp, A.col)
    x = sfsgen.vector(99, A.n, A.dtype)
    dA = to_dev(A)
    opts = sfs.default_opts(csr_variant=variant)
    for fmt in range(5):
        if not (fo["admissible_mask"] >> fmt) & 1:
            continue
        if fmt != sfs.CSR and variant != 2:
            continue
        M = sfs.convert(dA, fmt, opts)
        check_spmv(A, fmt, M, x, A.dtype, ctx=f"{name}/v{variant}")
        M.free()


@pytest.mark.parametrize("dtype", [sfsgen.F64, sfsgen.F32])
@pytest.mark.parametrize("cls,N,pts", [(sfsgen.ST2D5, 64, 5), (sfsgen.ST3D27, 24, 27)])
def test_spmv_x_ones_bitwise(dtype, cls, N, pts):
    """x = 1 on a stencil: every partial sum is a small integer, so every format in both precisions
    must give y = points - len exactly (SURVEY §8(c) exact special case)."""
    import torch
    A = sfsgen.generate(sfsgen.make_spec(cls, ia=N, dtype=dtype))
    expect = (pts - np.diff(A.rp)).astype(np.float64)
    dA = to_dev(A)
    tdt = torch.float64 if dtype == sfsgen.F64 else torch.float32
    x = torch.ones(A.n, dtype=tdt, device="cuda")
    for variant in (0, 1, 2, 3):
        for fmt in range(5):
            if variant != 2 and fmt != sfs.CSR:
                continue
            M = sfs.convert(dA, fmt, sfs.default_opts(csr_variant=variant))
            y = torch.empty(A.m, dtype=tdt, device="cuda")
            sfs.spmv(fmt, M, x, y)
            assert (y.cpu().numpy().astype(np.float64) == expect).all(), sfs.FORMAT_NAMES[fmt]


def test_spmv_unit_vector_bitwise():
    import torch
    A = cases()["rand_ragged"]
    dense_col = np.zeros(A.m)
    j = 17
    for r in range(A.m):
        for k in range(A.rp[r], A.rp[r + 1]):
            if A.col[k] == j:
                dense_col[r] = A.val[k]
    dA = to_dev(A)
    e = torch.zeros(A.n, dtype=torch.float64, device="cuda")
    e[j] = 1.0
    fo = oracle.features(A.m, A.n, A.rp, A.col)
    for fmt in range(5):
        if (fo["admissible_mask"] >> fmt) & 1:
            M = sfs.convert(dA, fmt)
            y = torch.empty(A.m, dtype=torch.float64, device="cuda")
            sfs.spmv(fmt, M, e, y)
            assert (y.cpu().numpy() == dense_col).all()


def test_hyb_order_statistic_refine_path():
    """HYB width beyond the exact histogram (>= 4096 rows of length >= 4096) -> host refinement."""
    m, n = 4500, 9700
    lens = 4096 + (np.arange(m) * 7919) % 700
    rp = np.concatenate([[0], np.cumsum(lens)]).astype(np.int32)
    col = np.concatenate([np.arange(L) * 2 + (r % 2) for r, L in enumerate(lens)]).astype(np.int32)
    A = sfsgen.CSR(m, n, rp, col, np.ones(len(col)))
    fg = sfs.features(to_dev(A))
    fo = oracle.features(m, n, rp, col)
    assert fo["hyb_k"] >= 4096
    assert_features_equal(fg, fo, "refine")


def test_errors():
    import torch
    A = cases()["laplace64"]
    bad = sfsgen.CSR(A.m, A.n, A.rp.copy(), A.col.copy(), A.val)
    bad.col[10], bad.col[11] = bad.col[11], bad.col[10]  # not increasing
    with pytest.raises(sfs.SfsError) as ei:
        sfs.features(to_dev(bad))
    assert ei.value.status == sfs.ERR_INVALID_CSR
    bad2 = sfsgen.CSR(A.m, A.n, A.rp.copy(), A.col.copy(), A.val)
    bad2.rp[100] = bad2.rp[101] + 1  # decreasing row_ptr
    with pytest.raises(sfs.SfsError) as ei:
        sfs.features(to_dev(bad2))
    assert ei.value.status == sfs.ERR_INVALID_CSR
    bad3 = sfsgen.CSR(A.m, 50, A.rp, A.col, A.val)  # column out of range
    with pytest.raises(sfs.SfsError) as ei:
        sfs.features(to_dev(bad3))
    assert ei.value.status == sfs.ERR_INVALID_CSR
    M = sfs.convert(to_dev(A), sfs.COO)
    x = torch.ones(A.n, dtype=torch.float64, device="cuda")
    y = torch.empty(A.m, dtype=torch.float64, device="cuda")
    with pytest.raises(sfs.SfsError) as ei:
        sfs.spmv(sfs.CSR, M, x, y)
    assert ei.value.status == sfs.ERR_INVALID_ARG
    anti = sfsgen.CSR(3000, 3000, np.arange(3001, dtype=np.int32), (2999 - np.arange(3000)).astype(np.int32),
                      np.ones(3000))
    with pytest.raises(sfs.SfsError) as ei:
        sfs.convert(to_dev(anti), sfs.DIA, sfs.default_opts(fill_slack=0))
    assert ei.value.status == sfs.ERR_INADMISSIBLE


def test_host_memory_input_matches_device():
    """The end-to-end path (host CSR, copies inside the call) computes the same features."""
    import torch
    A = cases()["uniform"]
    host = sfs.Csr(A.m, A.n, torch.from_numpy(A.rp).pin_memory(), torch.from_numpy(A.col).pin_memory(),
                   torch.from_numpy(A.val).pin_memory())
    assert_features_equal(sfs.features(host), oracle.features(A.m, A.n, A.rp, A.col), "host")
    M = sfs.convert(host, sfs.HYB)
    check_conversion(A, sfs.HYB, M, oracle.features(A.m, A.n, A.rp, A.col))


def test_label_corpus_small():
    names = ["laplace64", "band", "blockdiag32", "uniform", "powerlaw32", "rmat14", "empty", "tiny4x4"]
    mats = [to_dev(cases()[k]) for k in names]
    opts = sfs.default_opts(reps=20, warmup=2)
    feats, labs = sfs.label_corpus(mats, opts)
    for k, f, L in zip(names, feats, labs):
        A = cases()[k]
        fo = oracle.features(A.m, A.n, A.rp, A.col)
        assert_features_equal(f, fo, k)
        assert L["matrix_status"] == 0 and L["admissible_mask"] == fo["admissible_mask"]
        ran = [i for i in range(5) if L["status"][i] == 0]
        assert ran == [i for i in range(5) if (fo["admissible_mask"] >> i) & 1]
        t = np.array(L["t_spmv_us"], dtype=np.float64)
        assert all(t[i] > 0 for i in ran)
        # decision rule (Q14) reproduced by the oracle from the measured times
        assert L["label"] == oracle.label(t, sum(1 << i for i in ran))
        for i in range(5):
            assert L["bytes"][i] == sfs.spmv_bytes(f, i, A.dtype)
        assert L["t_convert_us"][0] == 0 and all(L["t_convert_us"][i] > 0 for i in ran if i)
    # masks: the paper's four formats only
    feats2, labs2 = sfs.label_corpus(mats[:2], sfs.default_opts(reps=5, warmup=1, formats_mask=0x0F))
    assert all(L["status"][4] == sfs.ERR_NOT_RUN and L["label"] != 4 for L in labs2)


def test_label_corpus_invalid_matrix_does_not_abort():
    A = cases()["laplace64"]
    bad = sfsgen.CSR(A.m, A.n, A.rp.copy(), A.col.copy(), A.val)
    bad.col[5] = bad.col[4]
    feats, labs = sfs.label_corpus([to_dev(bad), to_dev(A)], sfs.default_opts(reps=3, warmup=1))
    assert labs[0]["matrix_status"] == sfs.ERR_INVALID_CSR and labs[0]["label"] == -1
    assert labs[1]["matrix_status"] == 0 and labs[1]["label"] >= 0


def test_label_corpus_host_inputs_chunked():
    """Host-memory corpus: inputs staged in chunks of 1, 2, 4, ... matrices, each chunk's H2D overlapping the
    previous chunk's race.  Features bit-exact, statuses per matrix (an invalid one in the middle of a chunk),
    the same admissible formats raced as from device memory."""
    import torch
    names = ["laplace64", "band", "blockdiag32", "uniform", "powerlaw32", "rmat14", "empty", "tiny4x4"]
    A = {k: cases()[k] for k in names}
    bad = sfsgen.CSR(A["band"].m, A["band"].n, A["band"].rp.copy(), A["band"].col.copy(), A["band"].val)
    bad.col[5] = bad.col[4]
    order = names[:4] + ["bad"] + names[4:]
    A["bad"] = bad
    pin = lambda a: torch.from_numpy(np.ascontiguousarray(a)).pin_memory()
    mats = [sfs.Csr(A[k].m, A[k].n, pin(A[k].rp), pin(A[k].col), pin(A[k].val),
                    pin(sfsgen.vector(3, A[k].n, A[k].dtype))) for k in order]
    feats, labs = sfs.label_corpus(mats, sfs.default_opts(reps=5, warmup=1))
    for k, f, L in zip(order, feats, labs):
        if k == "bad":
            assert L["matrix_status"] == sfs.ERR_INVALID_CSR and L["label"] == -1
            continue
        fo = oracle.features(A[k].m, A[k].n, A[k].rp, A[k].col)
        assert_features_equal(f, fo, k)
        assert L["matrix_status"] == 0
        ran = [i for i in range(5) if L["status"][i] == 0]
        assert ran == [i for i in range(5) if (fo["admissible_mask"] >> i) & 1], k
        assert L["label"] == oracle.label(np.array(L["t_spmv_us"], np.float64), sum(1 << i for i in ran))


def test_launch_count_increases():
    import torch
    A = cases()["band"]
    M = sfs.convert(to_dev(A), sfs.COO)
    x = torch.ones(A.n, dtype=torch.float64, device="cuda")
    y = torch.empty(A.m, dtype=torch.float64, device="cuda")
    c0 = sfs.launch_count()
    for _ in range(3):
        sfs.spmv(sfs.COO, M, x, y)
    assert sfs.launch_count() - c0 == 6  # zero kernel + COO kernel per COO SpMV


def _tile_edge_csr(dtype, cap=None, no_empty=False):
    """Rows that stress the CSR tile kernel (variant 3): leading / trailing / mid-matrix runs of empty
    rows, rows of exactly 255/256/257/512 entries, one row of 400,000 entries spanning many warp
    ranges, and nnz large enough (> 148*4*8 chunks of 256) that each warp owns several chunks.
    cap: clip row lengths (cap = 256 selects the carry-free mode, every row <= one chunk)."""
    rng = np.random.default_rng(77)
    m, n = 200_000, 500_000
    lens = rng.poisson(6, m).astype(np.int64)
    lens[:1000] = 0
    lens[-5000:] = 0
    lens[90_000:93_000] = 0
    lens[rng.integers(0, m, 20_000)] = 0
    lens[[5000, 5001, 5002, 77_777]] = [255, 256, 257, 512]
    lens[123_456] = 400_000
    if cap is not None:
        lens = np.minimum(lens, cap)
        lens[rng.integers(0, m, 3000)] = cap  # many rows of exactly one chunk
    if no_empty:
        lens = np.maximum(lens, 1)
    rp = np.zeros(m + 1, np.int64)
    np.cumsum(lens, out=rp[1:])
    z = int(rp[-1])
    col = np.empty(z, np.int64)
    starts = rng.integers(0, n - 3 * 1000, m)
    for r in np.nonzero(lens)[0]:
        L = int(lens[r])
        if L >= 1000:
            col[rp[r]:rp[r + 1]] = np.sort(rng.choice(n, L, replace=False))
        else:
            col[rp[r]:rp[r + 1]] = starts[r] + np.cumsum(rng.integers(1, 4, L))
    val = rng.uniform(0.5, 1.0, z) * rng.choice([-1.0, 1.0], z)
    return sfsgen.CSR(m, n, rp.astype(np.int32), col.astype(np.int32),
                      val.astype(np.float64 if dtype == sfsgen.F64 else np.float32))


@pytest.mark.parametrize("cap", [None, 256])
@pytest.mark.parametrize("dtype", [sfsgen.F64, sfsgen.F32])
def test_csr_tile_edges(dtype, cap):
    import torch
    A = _tile_edge_csr(dtype, cap)
    x = sfsgen.vector(5, A.n, A.dtype)
    dA = to_dev(A)
    M = sfs.convert(dA, sfs.CSR, sfs.default_opts(csr_variant=3))
    assert M.layout().variant == 3
    check_spmv(A, sfs.CSR, M, x, A.dtype, ctx="tile-edges")
    M.free()
    # the same rows through the one-launch COO kernel (gaps, split rows, a row over ~1000 warp ranges)
    M = sfs.convert(dA, sfs.COO)
    check_spmv(A, sfs.COO, M, x, A.dtype, ctx="coo-edges")
    M.free()
    # borrowed arrays that are not 32 B aligned (a view at an element offset): scalar-load path
    t = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
    colb = torch.empty(A.nnz + 1, dtype=torch.int32, device="cuda")
    valb = torch.empty(A.nnz + 1, dtype=t(A.val).dtype, device="cuda")
    colb[1:] = t(A.col)
    valb[1:] = t(A.val)
    dB = sfs.Csr(A.m, A.n, t(A.rp), colb[1:], valb[1:])
    M = sfs.convert(dB, sfs.CSR, sfs.default_opts(csr_variant=3))
    check_spmv(A, sfs.CSR, M, x, A.dtype, ctx="tile-edges-misaligned")
    M.free()


@pytest.mark.parametrize("shape", ["one_row", "two_rows", "first_last", "diag_gaps"])
def test_split_rows_and_gaps(shape):
    """Row layouts that exercise the carries of the one-launch COO and CSR tile kernels: one row holding
    every entry (all warps but the first are middle pieces), two long rows meeting mid-range, entries only
    in the first and last rows (one long run of empty rows), and a sparse diagonal (gaps everywhere)."""
    rng = np.random.default_rng(5)
    m, n = 40_000, 3_000_000
    lens = np.zeros(m, np.int64)
    if shape == "one_row":
        lens[m // 2] = 2_000_000
    elif shape == "two_rows":
        lens[7] = 1_234_567
        lens[8] = 1_000_003
    elif shape == "first_last":
        lens[0] = 700_001
        lens[-1] = 900_000
    else:
        lens[::3] = 1
        lens[5] = 1_500_000
    rp = np.zeros(m + 1, np.int64)
    np.cumsum(lens, out=rp[1:])
    z = int(rp[-1])
    col = np.empty(z, np.int64)
    for r in np.nonzero(lens)[0]:
        L = int(lens[r])
        col[rp[r]:rp[r + 1]] = np.sort(rng.choice(n, L, replace=False)) if L > 1 else [r % n]
    val = rng.uniform(0.5, 1.0, z) * rng.choice([-1.0, 1.0], z)
    A = sfsgen.CSR(m, n, rp.astype(np.int32), col.astype(np.int32), val)
    x = sfsgen.vector(3, n, A.dtype)
    dA = to_dev(A)
    for fmt, opts in [(sfs.CSR, sfs.default_opts(csr_variant=3)), (sfs.CSR, sfs.default_opts(csr_variant=1)),
                      (sfs.CSR, sfs.default_opts(csr_variant=5)), (sfs.COO, None)]:
        M = sfs.convert(dA, fmt, opts)
        check_spmv(A, fmt, M, x, A.dtype, ctx=f"{shape}/{sfs.FORMAT_NAMES[fmt]}")
        M.free()


@pytest.mark.parametrize("cap", [None, 256])
@pytest.mark.parametrize("dtype", [sfsgen.F64, sfsgen.F32])
def test_csr_bitmap_tile(dtype, cap):
    """CSR variant 4 (tile kernel with row ids from a row-start bitmap) on rows of 1..400,000 entries,
    rows of exactly 255/256/257/512, a row spanning many warp ranges; with empty rows present the
    handle takes variant 5 (bitmap over the non-empty rows + rank -> row map, y zeroed ahead)."""
    A = _tile_edge_csr(dtype, cap, no_empty=True)
    x = sfsgen.vector(6, A.n, A.dtype)
    M = sfs.convert(to_dev(A), sfs.CSR, sfs.default_opts(csr_variant=4))
    assert M.layout().variant == 4
    check_spmv(A, sfs.CSR, M, x, A.dtype, ctx="bitmap-tile")
    M.free()
    M = sfs.convert(to_dev(A), sfs.COO)
    check_spmv(A, sfs.COO, M, x, A.dtype, ctx="coo-no-empty-rows")
    M.free()
    B = _tile_edge_csr(dtype, cap)
    for v in (4, 5):
        M = sfs.convert(to_dev(B), sfs.CSR, sfs.default_opts(csr_variant=v))
        assert M.layout().variant == 5
        check_spmv(B, sfs.CSR, M, x[:B.n] if len(x) >= B.n else sfsgen.vector(6, B.n, B.dtype), B.dtype,
                   ctx=f"bitmap-map/{v}")
        M.free()


@pytest.mark.parametrize("name", ["slack_at", "slack_past", "fill_at_dia", "fill_past_dia", "fill_at_ell",
                                  "fill_past_ell", "trunc_at", "trunc_past"])
def test_q11_admissibility_boundary_gpu(name):
    """The library's Q11 decision at E = lim and lim + 1 (Q11) equals the hand-derived bits (and
    the oracle's features, bitwise); an inadmissible ELL / DIA conversion returns SFS_ERR_INADMISSIBLE."""
    A, kw, e = q11_boundary_cases()[name]
    opts = sfs.default_opts(**kw)
    fg = sfs.features(to_dev(A), opts)
    assert_features_equal(fg, oracle.features(A.m, A.n, A.rp, A.col, oracle.default_opts(**kw) if kw else None), name)
    assert bool((fg["admissible_mask"] >> sfs.ELL) & 1) == e["ell_ok"]
    assert bool((fg["admissible_mask"] >> sfs.DIA) & 1) == e["dia_ok"]
    for fmt, ok in ((sfs.ELL, e["ell_ok"]), (sfs.DIA, e["dia_ok"])):
        if ok:
            sfs.convert(to_dev(A), fmt, opts).free()
        else:
            with pytest.raises(sfs.SfsError) as ei:
                sfs.convert(to_dev(A), fmt, opts)
            assert ei.value.status == sfs.ERR_INADMISSIBLE


@pytest.mark.parametrize("shape", ["one_row", "two_rows", "first_last", "all_short"])
def test_split_rows_no_empty(shape):
    """COO and the bitmap CSR tile kernel (variant 4, which needs every row non-empty) on rows split across
    warp ranges: one row holding almost every entry (pieces in ~every warp range), two long rows meeting
    mid-range, long first and last rows, and only short rows (every boundary splits a row)."""
    rng = np.random.default_rng(6)
    m, n = 40_000, 3_000_000
    lens = np.ones(m, np.int64)
    if shape == "one_row":
        lens[m // 2] = 2_000_000
    elif shape == "two_rows":
        lens[7] = 1_234_567
        lens[8] = 1_000_003
    elif shape == "first_last":
        lens[0] = 700_001
        lens[-1] = 900_000
    else:
        lens[:] = rng.integers(1, 40, m)
    rp = np.zeros(m + 1, np.int64)
    np.cumsum(lens, out=rp[1:])
    z = int(rp[-1])
    col = np.empty(z, np.int64)
    for r in range(m):
        L = int(lens[r])
        col[rp[r]:rp[r + 1]] = np.sort(rng.choice(n, L, replace=False)) if L > 1 else [(r * 7919) % n]
    val = rng.uniform(0.5, 1.0, z) * rng.choice([-1.0, 1.0], z)
    for dt in (np.float64, np.float32):
        A = sfsgen.CSR(m, n, rp.astype(np.int32), col.astype(np.int32), val.astype(dt))
        x = sfsgen.vector(3, n, A.dtype)
        dA = to_dev(A)
        for fmt, opts in [(sfs.CSR, sfs.default_opts(csr_variant=4)), (sfs.COO, None)]:
            M = sfs.convert(dA, fmt, opts)
            if fmt == sfs.CSR:
                assert M.layout().variant == 4
            check_spmv(A, fmt, M, x, A.dtype, ctx=f"{shape}/{sfs.FORMAT_NAMES[fmt]}/{np.dtype(dt).name}")
            M.free()
