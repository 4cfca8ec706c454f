"""Pins of the CPU oracle against things other than itself (CPU only, -m "not gpu").

Each test names what fixes the expected value: a hand-worked matrix (tests/golden/tiny4x4.json),
closed forms (stencil row-length histograms derived combinatorially), brute force from a dense
pattern, exact rational arithmetic, or an invariant of the definitions (round trips, HYB = ELL part
+ COO part, x = 1 / x = e_j / x -> 2^k x exactness).  Paper passages: Table 1,
formats (§2.1), SpMV, label rule.
"""
import math
from fractions import Fraction

import numpy as np
import pytest

import oracle
import sfsgen
from helpers import (q11_boundary_cases, csr_max_closed_form, dense_of, exact_matvec, features_from_histogram, golden, kth_largest,
                     pattern_of, random_csr, stencil_histogram, ulp_close)

F = Fraction


def _fr(pair):
    return F(pair[0], pair[1])


# ------------------------------------------------------------------ hand-worked 4x4 (golden)
def test_tiny4x4_features_golden():
    g = golden("tiny4x4.json")
    A = sfsgen.from_dense(np.array(g["A"], float))
    f = oracle.features(A.m, A.n, A.rp, A.col)
    e = g["features"]
    for k in ["nrows", "ncols", "nnz", "nnz_min", "nnz_max", "csr_max", "ell_size", "hyb_k", "hyb_ell_size",
              "hyb_coo", "hyb_ell_nnz", "diagonals", "dia_size", "admissible_mask"]:
        assert f[k] == e[k], k
    for k in ["nnz_frac", "nnz_mu", "max_mu", "mu_min", "hyb_ell_frac", "dia_frac", "ell_frac"]:
        assert f[k] == float(_fr(e[k])), k
    assert f["nnz_sig"] == math.sqrt(float(_fr(e["nnz_sig_sq"])))
    assert f["sig_lower"] == math.sqrt(float(_fr(e["sig_lower_sq"])))
    assert f["sig_higher"] == math.sqrt(float(_fr(e["sig_higher_sq"])))


def test_tiny4x4_conversions_and_spmv_golden():
    g = golden("tiny4x4.json")
    A = sfsgen.from_dense(np.array(g["A"], float))
    ell = oracle.convert(oracle.ELL, A.m, A.n, A.rp, A.col, A.val)
    assert ell.arrays["K"] == g["ell"]["K"]
    assert (ell.arrays["ecol"] == np.array(g["ell"]["col"])).all()
    assert (ell.arrays["eval"] == np.array(g["ell"]["val"], float)).all()
    hyb = oracle.convert(oracle.HYB, A.m, A.n, A.rp, A.col, A.val)
    assert hyb.arrays["K"] == g["hyb"]["K"]
    assert (hyb.arrays["ecol"] == np.array(g["hyb"]["ell_col"])).all()
    assert (hyb.arrays["eval"] == np.array(g["hyb"]["ell_val"], float)).all()
    coo = np.stack([hyb.arrays["crow"], hyb.arrays["ccol"], hyb.arrays["cval"]], 1)
    assert (coo == np.array(g["hyb"]["coo"], float)).all()
    dia = oracle.convert(oracle.DIA, A.m, A.n, A.rp, A.col, A.val)
    assert (dia.arrays["offs"] == np.array(g["dia"]["offsets"])).all()
    assert (dia.arrays["dval"] == np.array(g["dia"]["val"], float)).all()
    x = np.array(g["x"], float)
    for fmt in range(5):
        cv = oracle.convert(fmt, A.m, A.n, A.rp, A.col, A.val)
        y, ay = oracle.spmv(cv, x)
        assert (y == np.array(g["y"], float)).all(), oracle.FORMAT_NAMES[fmt]
        assert (ay == np.array(g["y"], float)).all()  # A and x are nonnegative here: |A||x| = y


# ------------------------------------------------------------------ stencil closed forms
@pytest.mark.parametrize("kind,cls,N", [("2d5", sfsgen.ST2D5, 64), ("2d5", sfsgen.ST2D5, 7),
                                        ("3d7", sfsgen.ST3D7, 9), ("3d27", sfsgen.ST3D27, 12),
                                        ("3d27", sfsgen.ST3D27, 3)])
def test_stencil_features_closed_form(kind, cls, N):
    A = sfsgen.generate(sfsgen.make_spec(cls, ia=N))
    d = 2 if kind == "2d5" else 3
    m = N ** d
    hist = stencil_histogram(kind, N)
    cf = features_from_histogram(hist, m, m)
    f = oracle.features(A.m, A.n, A.rp, A.col)
    assert f["nrows"] == m and f["nnz"] == cf["nnz"]
    assert f["nnz_min"] == cf["nnz_min"] and f["nnz_max"] == cf["nnz_max"]
    assert f["diagonals"] == {"2d5": 5, "3d7": 7, "3d27": 27}[kind]
    assert f["dia_size"] == f["diagonals"] * m and f["ell_size"] == m * cf["nnz_max"]
    assert f["csr_max"] == csr_max_closed_form(m, cf["nnz"])
    # exact rationals, rounded once; the sqrt-of-quotient features within 4 ulp of the exact value
    assert f["nnz_mu"] == float(cf["mu"])
    assert f["max_mu"] == float(cf["max_mu"]) and f["mu_min"] == float(cf["mu_min"])
    assert f["nnz_frac"] == float(F(cf["nnz"], m * m))
    assert ulp_close(f["nnz_sig"], math.sqrt(float(cf["var"])))
    assert ulp_close(f["sig_lower"], math.sqrt(float(cf["sig_lower_sq"])))
    assert ulp_close(f["sig_higher"], math.sqrt(float(cf["sig_higher_sq"])))
    assert f["ell_frac"] == float(F(cf["nnz"], m * cf["nnz_max"]))
    # HYB width: order-statistic form of the Q6 rule (independent of the oracle's loop):
    # K = max(1, (Rmax+1)-th largest length), Rmax = largest R with 3R < m or R < 4096
    rmax = max((m - 1) // 3, 4095)
    K = max(1, kth_largest(hist, rmax + 1))
    assert f["hyb_k"] == K
    assert f["hyb_coo"] == sum(max(0, L - K) * c for L, c in hist.items())


def test_appendix_a2_laplacian_values():
    """SURVEY App. A2 values for configs[0] (2D 5-pt 64x64)."""
    A = sfsgen.laplace2d(64)
    f = oracle.features(A.m, A.n, A.rp, A.col)
    assert (f["nnz"], f["nnz_min"], f["nnz_max"], f["csr_max"]) == (20224, 3, 5, 8)
    assert (f["hyb_k"], f["hyb_ell_size"], f["hyb_coo"]) == (3, 12288, 7936)
    assert f["nnz_frac"] == 0.0012054443359375 and f["nnz_mu"] == 4.9375
    assert f["nnz_sig"] ** 2 == pytest.approx(0.060546875, rel=1e-15)
    assert f["dia_frac"] == f["ell_frac"] == 0.9875


@pytest.mark.slow
def test_appendix_a3_3d27_values():
    """SURVEY App. A3 closed forms for configs[3] (3D 27-pt 128^3)."""
    A = sfsgen.stencil3d27(128)
    f = oracle.features(A.m, A.n, A.rp, A.col)
    hist = stencil_histogram("3d27", 128)
    assert hist == {8: 8, 12: 1512, 18: 95256, 27: 2000376}
    assert (f["nrows"], f["nnz"], f["nnz_min"], f["nnz_max"]) == (2097152, 55742968, 8, 27)
    assert (f["csr_max"], f["diagonals"], f["hyb_k"], f["hyb_coo"]) == (222, 27, 27, 0)
    assert f["dia_size"] == f["ell_size"] == 56623104


# ------------------------------------------------------------------ brute force from dense
@pytest.mark.parametrize("seed", range(12))
def test_features_brute_force(seed):
    rng = np.random.default_rng(seed)
    m, n = int(rng.integers(1, 60)), int(rng.integers(1, 60))
    A = random_csr(rng, m, n, float(rng.uniform(0.0, 0.5)), empty_rows=0.2 * (seed % 2),
                   dense_rows=seed % 3)
    P = pattern_of(A)
    lens = P.sum(1)
    f = oracle.features(A.m, A.n, A.rp, A.col)
    z = int(lens.sum())
    assert f["nnz"] == z and f["nnz_min"] == lens.min() and f["nnz_max"] == lens.max()
    r, c = np.nonzero(P)
    assert f["diagonals"] == len(set((c - r).tolist()))
    assert f["csr_max"] == csr_max_closed_form(m, z)
    assert ulp_close(f["nnz_sig"], float(np.std(lens.astype(np.float64))), ulps=8) or abs(f["nnz_sig"]) < 1e-12
    mu = z / m
    lo, hi = lens[lens * m < z], lens[lens * m > z]
    if len(lo):
        assert f["sig_lower"] == pytest.approx(float(np.sqrt(np.mean((lo - mu) ** 2))), rel=1e-13)
    else:
        assert f["sig_lower"] == 0.0
    if len(hi):
        assert f["sig_higher"] == pytest.approx(float(np.sqrt(np.mean((hi - mu) ** 2))), rel=1e-13)
    else:
        assert f["sig_higher"] == 0.0
    # HYB K: the rule holds at K and fails at K-1 (direct count over rows)
    K = f["hyb_k"]
    ok = lambda k: 3.0 * int((lens > k).sum()) < m or int((lens > k).sum()) < 4096
    if lens.max() == 0:
        assert K == 0
    else:
        assert 1 <= K <= lens.max() and ok(K) and (K == 1 or not ok(K - 1))
    assert f["hyb_coo"] == int(np.maximum(lens - K, 0).sum())


def test_hyb_width_large_threshold_branch():
    """A matrix with > 4096 rows where the 3R < m branch decides (not the breakeven)."""
    m = 30000
    lens = np.array([1] * 20000 + [5] * 6000 + [9] * 4000)
    rp = np.concatenate([[0], np.cumsum(lens)]).astype(np.int32)
    col = np.concatenate([np.arange(L) for L in lens]).astype(np.int32)
    f = oracle.features(m, 16, rp, col)
    # R(k): k=1 -> 10000 (3*10000 = m, not < m; 10000 >= 4096) ; k=2..4 -> 10000 ; k=5 -> 4000 < 4096
    assert f["hyb_k"] == 5
    assert f["hyb_coo"] == 4000 * 4


def test_empty_and_degenerate():
    # z = 0: all fractions 0, K = 0, no diagonals, every format admissible
    rp = np.zeros(6, np.int32)
    f = oracle.features(5, 3, rp, np.zeros(0, np.int32))
    assert f["nnz"] == 0 and f["hyb_k"] == 0 and f["diagonals"] == 0 and f["admissible_mask"] == 31
    assert f["nnz_frac"] == 0 and f["nnz_sig"] == 0 and f["dia_frac"] == 0 and f["ell_frac"] == 0
    # 1x1
    f = oracle.features(1, 1, np.array([0, 1], np.int32), np.array([0], np.int32))
    assert (f["nnz"], f["diagonals"], f["hyb_k"], f["csr_max"]) == (1, 1, 1, 1)
    # anti-diagonal: m distinct offsets -> dia_size = m^2 (P:L106 O(n^2) worst case) -> DIA inadmissible
    m = 2000
    rp = np.arange(m + 1, dtype=np.int32)
    col = (m - 1 - np.arange(m)).astype(np.int32)
    f = oracle.features(m, m, rp, col)
    assert f["diagonals"] == m and f["dia_size"] == m * m
    assert not (f["admissible_mask"] >> oracle.DIA) & 1
    # arrowhead: one dense row makes ELL inadmissible
    m = 3000
    lens = np.ones(m, int)
    lens[0] = m
    rp = np.concatenate([[0], np.cumsum(lens)]).astype(np.int32)
    col = np.concatenate([np.arange(m)] + [[r] for r in range(1, m)]).astype(np.int32)
    f = oracle.features(m, m, rp, col)
    assert f["ell_size"] == m * m and not (f["admissible_mask"] >> oracle.ELL) & 1
    assert (f["admissible_mask"] >> oracle.HYB) & 1


@pytest.mark.parametrize("name", ["slack_at", "slack_past", "fill_at_dia", "fill_past_dia", "fill_at_ell",
                                  "fill_past_ell", "trunc_at", "trunc_past"])
def test_q11_admissibility_boundary(name):
    """Q11 (CUSP size restrictions P:L194): ELL / DIA admissible iff padded slots E <=
    max(trunc(max_fill * z), fill_slack).  Each case sits at E = lim or lim + 1, once where fill_slack
    binds, once where trunc(3z) binds (for ELL and for DIA), once where trunc of a non-integer limit
    decides; the expected bits are literal numbers derived by hand (tests/helpers.q11_boundary_cases)."""
    A, kw, e = q11_boundary_cases()[name]
    f = oracle.features(A.m, A.n, A.rp, A.col, oracle.default_opts(**kw) if kw else None)
    assert (f["nnz"], f["ell_size"], f["dia_size"]) == (e["z"], e["ell_size"], e["dia_size"])
    assert bool((f["admissible_mask"] >> oracle.ELL) & 1) == e["ell_ok"]
    assert bool((f["admissible_mask"] >> oracle.DIA) & 1) == e["dia_ok"]
    assert f["admissible_mask"] & 0b1011 == 0b1011  # CSR, COO, HYB always


# ------------------------------------------------------------------ conversions: invariants
def _decode_to_dense(cv, m, n):
    D = np.zeros((m, n))
    a = cv.arrays
    if cv.fmt == oracle.COO:
        D[a["row"], a["col"]] = a["val"]
    elif cv.fmt in (oracle.ELL, oracle.HYB):
        for r in range(m):
            for j in range(a["K"]):
                if a["ecol"][r, j] >= 0:
                    D[r, a["ecol"][r, j]] = a["eval"][r, j]
        if cv.fmt == oracle.HYB:
            D[a["crow"], a["ccol"]] = a["cval"]
    elif cv.fmt == oracle.DIA:
        for d, off in enumerate(a["offs"]):
            for r in range(m):
                if 0 <= r + off < n:
                    D[r, r + off] = a["dval"][d, r]
    return D


@pytest.mark.parametrize("seed", range(8))
def test_conversion_round_trips(seed):
    rng = np.random.default_rng(100 + seed)
    m, n = int(rng.integers(1, 50)), int(rng.integers(1, 50))
    A = random_csr(rng, m, n, float(rng.uniform(0.02, 0.6)), empty_rows=0.3 * (seed % 2), dense_rows=seed % 2)
    D = dense_of(A)
    f = oracle.features(A.m, A.n, A.rp, A.col)
    for fmt in range(1, 5):
        cv = oracle.convert(fmt, A.m, A.n, A.rp, A.col, A.val)
        assert (_decode_to_dense(cv, m, n) == D).all(), oracle.FORMAT_NAMES[fmt]
    coo = oracle.convert(oracle.COO, A.m, A.n, A.rp, A.col, A.val).arrays
    assert (np.diff(coo["row"]) >= 0).all() and (coo["col"] == A.col).all() and (coo["val"] == A.val).all()
    ell = oracle.convert(oracle.ELL, A.m, A.n, A.rp, A.col, A.val).arrays
    assert ell["ecol"].size == f["ell_size"] and int((ell["ecol"] >= 0).sum()) == A.nnz
    assert (ell["eval"][ell["ecol"] < 0] == 0).all()
    hyb = oracle.convert(oracle.HYB, A.m, A.n, A.rp, A.col, A.val).arrays
    assert int((hyb["ecol"] >= 0).sum()) == f["hyb_ell_nnz"] and len(hyb["crow"]) == f["hyb_coo"]
    dia = oracle.convert(oracle.DIA, A.m, A.n, A.rp, A.col, A.val).arrays
    assert dia["dval"].size == f["dia_size"] and int((dia["dval"] != 0).sum()) == A.nnz  # no stored zeros
    assert (np.diff(dia["offs"]) > 0).all()


def test_explicit_zeros_kept_by_csr_coo_ell_hyb():
    rng = np.random.default_rng(7)
    A = random_csr(rng, 30, 30, 0.3, explicit_zero=0.3)
    assert (A.val == 0).any()
    f = oracle.features(A.m, A.n, A.rp, A.col)
    dia = oracle.convert(oracle.DIA, A.m, A.n, A.rp, A.col, A.val).arrays
    assert len(dia["offs"]) == f["diagonals"]  # Q9: explicit zeros count as stored entries
    ell = oracle.convert(oracle.ELL, A.m, A.n, A.rp, A.col, A.val).arrays
    assert int((ell["ecol"] >= 0).sum()) == A.nnz  # sentinel keeps stored zeros distinguishable (Q10)


# ------------------------------------------------------------------ SpMV pins
@pytest.mark.parametrize("seed", range(6))
def test_spmv_exact_rational(seed):
    rng = np.random.default_rng(200 + seed)
    m, n = int(rng.integers(1, 25)), int(rng.integers(1, 25))
    A = random_csr(rng, m, n, 0.4, empty_rows=0.2)
    x = rng.uniform(-1, 1, n)
    yex = exact_matvec(A, x)
    for fmt in range(5):
        y, ay = oracle.spmv(oracle.convert(fmt, A.m, A.n, A.rp, A.col, A.val), x)
        for r in range(m):
            # long-double accumulation of <= 25 fp64 products: within 2^-60 relative of |A||x|
            assert abs(F(float(y[r])) - yex[r]) <= F(1, 2 ** 50) * F(float(ay[r])) + F(1, 2 ** 1074), (fmt, r)


@pytest.mark.parametrize("kind,cls,N", [("2d5", sfsgen.ST2D5, 64), ("3d27", sfsgen.ST3D27, 10)])
def test_spmv_stencil_x_ones_integer_exact(kind, cls, N):
    """x = 1: y_r = coefficient sum = (points - len_r) for interior-diagonal stencils (exact ints)."""
    A = sfsgen.generate(sfsgen.make_spec(cls, ia=N))
    lens = np.diff(A.rp)
    pts = 5 if kind == "2d5" else 27
    x = np.ones(A.n)
    for fmt in range(5):
        y, _ = oracle.spmv(oracle.convert(fmt, A.m, A.n, A.rp, A.col, A.val), x)
        assert (y == (pts - lens)).all(), oracle.FORMAT_NAMES[fmt]
    if kind == "2d5" and N == 64:
        vals, cnt = np.unique(pts - lens, return_counts=True)
        assert dict(zip(vals.tolist(), cnt.tolist())) == {0: 3844, 1: 248, 2: 4}


def test_spmv_unit_vectors_and_scaling():
    rng = np.random.default_rng(9)
    A = random_csr(rng, 40, 33, 0.25, empty_rows=0.1)
    D = dense_of(A)
    cvs = [oracle.convert(f, A.m, A.n, A.rp, A.col, A.val) for f in range(5)]
    for j in [0, 5, 32]:
        e = np.zeros(A.n)
        e[j] = 1.0
        for cv in cvs:
            assert (oracle.spmv(cv, e)[0] == D[:, j]).all()
    x = rng.uniform(-1, 1, A.n)
    for cv in cvs:
        y1 = oracle.spmv(cv, x)[0]
        y2 = oracle.spmv(cv, x * 2.0 ** 7)[0]
        assert (y2 == y1 * 2.0 ** 7).all()


def test_spmv_formats_agree_with_dense_tolerance():
    A = sfsgen.generate(sfsgen.make_spec(sfsgen.POWERLAW, seed=5, m=3000, pa=2.3))
    x = sfsgen.vector(5, A.n)
    D = dense_of(A)
    yd = D @ x
    ad = np.abs(D) @ np.abs(x)
    for fmt in range(5):
        f = oracle.features(A.m, A.n, A.rp, A.col)
        if fmt == oracle.DIA and f["diagonals"] > 1000:
            continue
        y, ay = oracle.spmv(oracle.convert(fmt, A.m, A.n, A.rp, A.col, A.val), x)
        assert np.all(np.abs(y - yd) <= 1e-13 * ad + 1e-300)
        assert np.allclose(ay, ad, rtol=1e-13, atol=0)


# ------------------------------------------------------------------ label rule, validation
def test_label_rule():
    t = [3.0, 2.0, 2.0, 5.0, 1.0]
    assert oracle.label(t, 0x1F) == 4
    assert oracle.label(t, 0x0F) == 1  # tie COO/ELL -> lower id
    assert oracle.label([1, 1, 1, 1, 1], 0x1F) == 0
    assert oracle.label(t, 0x08) == 3
    assert oracle.label(t, 0) == -1


def test_validation_codes():
    rp = np.array([0, 2, 3], np.int32)
    assert oracle.validate(2, 4, rp, np.array([0, 3, 1], np.int32)) == 0
    assert oracle.validate(2, 4, np.array([1, 2, 3], np.int32), np.array([0, 3, 1], np.int32)) != 0
    assert oracle.validate(2, 4, np.array([0, 3, 2], np.int32), np.array([0, 1, 2], np.int32)) != 0
    assert oracle.validate(2, 4, rp, np.array([0, 4, 1], np.int32)) != 0  # col out of range
    assert oracle.validate(2, 4, rp, np.array([3, 0, 1], np.int32)) != 0  # not increasing
    assert oracle.validate(2, 4, rp, np.array([1, 1, 1], np.int32)) != 0  # duplicate


def test_label_matrix_pass_runs():
    A = sfsgen.laplace2d(16)
    x = sfsgen.vector(1, A.n)
    lab, f, ts, tc = oracle.label_matrix(A.m, A.n, A.rp, A.col, A.val, x, reps=2)
    assert 0 <= lab < 5 and f["admissible_mask"] == 31
    assert (ts > 0).all() and lab == int(np.argmin(ts))
