"""Test-side helpers: independent brute-force computations used to PIN the oracle (and, in the
GPU tests, to decode the library's documented layouts).  Nothing here is imported by the product
package or by the oracle."""
from __future__ import annotations

import json
import math
import os
from fractions import Fraction

import numpy as np

import sfsgen

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")


def golden(name):
    with open(os.path.join(GOLDEN, name)) as fh:
        return json.load(fh)


def random_csr(rng: np.random.Generator, m: int, n: int, density: float, dtype=np.float64,
               empty_rows=0.0, dense_rows=0, explicit_zero=0.0) -> sfsgen.CSR:
    """Random canonical CSR from a dense boolean pattern (brute-force-friendly sizes)."""
    pat = rng.random((m, n)) < density
    if empty_rows:
        pat[rng.random(m) < empty_rows, :] = False
    for r in rng.choice(m, size=min(dense_rows, m), replace=False):
        pat[r, :] = True
    vals = rng.uniform(0.5, 1.0, size=(m, n)) * rng.choice([-1.0, 1.0], size=(m, n))
    if explicit_zero:
        vals[rng.random((m, n)) < explicit_zero] = 0.0
    rp = np.zeros(m + 1, np.int64)
    rp[1:] = np.cumsum(pat.sum(1))
    rows, cols = np.nonzero(pat)
    return sfsgen.CSR(m, n, rp.astype(np.int32), cols.astype(np.int32), vals[rows, cols].astype(dtype))


def dense_of(A: sfsgen.CSR) -> np.ndarray:
    D = np.zeros((A.m, A.n), np.float64)
    for r in range(A.m):
        for k in range(A.rp[r], A.rp[r + 1]):
            D[r, A.col[k]] = A.val[k]
    return D


def pattern_of(A: sfsgen.CSR) -> np.ndarray:
    P = np.zeros((A.m, A.n), bool)
    rows = np.repeat(np.arange(A.m), np.diff(A.rp))
    P[rows, A.col] = True
    return P


def exact_matvec(A: sfsgen.CSR, x) -> list:
    """Exact rational y = A x (brute force over the dense pattern) — tiny matrices only."""
    xs = [Fraction(float(v)) for v in x]
    y = []
    for r in range(A.m):
        s = Fraction(0)
        for k in range(A.rp[r], A.rp[r + 1]):
            s += Fraction(float(A.val[k])) * xs[A.col[k]]
        y.append(s)
    return y


# ------------------------------------------------------------------ closed forms for stencils
def axis_counts(N):
    """Per-axis neighbour counts in {-1,0,+1}: 2 at the two boundary cells, 3 inside."""
    return {2: 2, 3: N - 2} if N > 2 else {2: N}


def stencil_histogram(kind: str, N: int) -> dict:
    """Row-length histogram of the 2D5 / 3D7 / 3D27 stencil on N^d, derived combinatorially."""
    ac = axis_counts(N)
    hist = {}
    if kind == "2d5":
        # length = 1 + (a_i - 1) + (a_j - 1)
        for ai, ci in ac.items():
            for aj, cj in ac.items():
                L = 1 + (ai - 1) + (aj - 1)
                hist[L] = hist.get(L, 0) + ci * cj
    elif kind == "3d7":
        for ai, ci in ac.items():
            for aj, cj in ac.items():
                for ak, ck in ac.items():
                    L = 1 + (ai - 1) + (aj - 1) + (ak - 1)
                    hist[L] = hist.get(L, 0) + ci * cj * ck
    elif kind == "3d27":
        for ai, ci in ac.items():
            for aj, cj in ac.items():
                for ak, ck in ac.items():
                    L = ai * aj * ak
                    hist[L] = hist.get(L, 0) + ci * cj * ck
    return hist


def stencil_offsets(kind: str, N: int) -> int:
    return {"2d5": 5, "3d7": 7, "3d27": 27}[kind] if N >= 2 else 1


def features_from_histogram(hist: dict, m: int, n: int) -> dict:
    """Exact rational Table-1 statistics from a row-length histogram (independent derivation)."""
    z = sum(L * c for L, c in hist.items())
    mu = Fraction(z, m)
    var = sum(c * (L - mu) ** 2 for L, c in hist.items()) / m
    low = [(L, c) for L, c in hist.items() if L < mu]
    high = [(L, c) for L, c in hist.items() if L > mu]
    cl, ch = sum(c for _, c in low), sum(c for _, c in high)
    sl2 = sum(c * (L - mu) ** 2 for L, c in low) / cl if cl else Fraction(0)
    sh2 = sum(c * (L - mu) ** 2 for L, c in high) / ch if ch else Fraction(0)
    return {"nnz": z, "nnz_min": min(hist), "nnz_max": max(hist), "mu": mu, "var": var,
            "sig_lower_sq": sl2, "sig_higher_sq": sh2, "max_mu": max(hist) - mu, "mu_min": mu - min(hist)}


def kth_largest(hist: dict, k: int) -> int:
    """k-th largest row length (1-based) from a histogram; 0 if k exceeds the row count."""
    seen = 0
    for L in sorted(hist, reverse=True):
        seen += hist[L]
        if seen >= k:
            return L
    return 0


def csr_max_closed_form(m, z, warps=148 * 64):
    """Q4 closed form: max over warps of rows handled = sum_{v < min(VPW, m)} ceil((m - v) / V)."""
    avg = z // m
    tpv = 2 if avg <= 2 else 4 if avg <= 4 else 8 if avg <= 8 else 16 if avg <= 16 else 32
    vpw = 32 // tpv
    V = warps * vpw
    return sum(-(-(m - v) // V) for v in range(min(vpw, m)))


def ulp_close(a: float, b: float, ulps=4) -> bool:
    if a == b:
        return True
    return abs(a - b) <= ulps * math.ulp(max(abs(a), abs(b)))


# ------------------------------------------------------------------ Q11 admissibility boundary matrices
def csr_from_rows(m: int, n: int, rows) -> sfsgen.CSR:
    """Canonical CSR from {row: sorted column list} (other rows empty); values 1.0 (never 0)."""
    lens = np.zeros(m, np.int64)
    for r, cs in rows.items():
        lens[r] = len(cs)
    rp = np.zeros(m + 1, np.int64)
    rp[1:] = np.cumsum(lens)
    col = np.zeros(int(rp[-1]), np.int32)
    for r, cs in rows.items():
        col[rp[r]:rp[r + 1]] = cs
    return sfsgen.CSR(m, n, rp.astype(np.int32), col, np.ones(len(col)))


def csr_from_arrays(m: int, n: int, row: np.ndarray, col: np.ndarray) -> sfsgen.CSR:
    """Canonical CSR from (row, col) pairs already in row-major, strictly increasing column order."""
    rp = np.zeros(m + 1, np.int64)
    np.add.at(rp, np.asarray(row, np.int64) + 1, 1)
    return sfsgen.CSR(m, n, np.cumsum(rp).astype(np.int32), np.asarray(col, np.int32), np.ones(len(col)))


def q11_boundary_cases():
    """Matrices whose padded slot count E sits exactly at the Q11 limit lim = max(trunc(max_fill*z),
    fill_slack) and one past it (Q11), with the expected admissibility
    written out as literal numbers (derivations in each entry's comment).
    Returns {name: (A, opts_kw, expect)} with expect = {"z", "ell_size", "dia_size", "ell_ok", "dia_ok"}."""
    out = {}
    # (1) fill_slack binds (3z < 2^20): 2^18 rows, diagonal + row 0 = cols 0..3.
    #     z = 262147, 3z = 786441 -> lim = 1048576; ELL E = 2^18 * 4 = 1048576 = lim (admissible);
    #     offsets {0,1,2,3}: DIA E = 4 * 2^18 = lim (admissible)
    m = 1 << 18
    row = np.concatenate([[0, 0, 0, 0], np.arange(1, m)])
    col = np.concatenate([[0, 1, 2, 3], np.arange(1, m)])
    out["slack_at"] = (csr_from_arrays(m, m, row, col), {},
                       dict(z=262147, ell_size=1048576, dia_size=1048576, ell_ok=True, dia_ok=True))
    # (2) fill_slack binds, one past: 61681 rows (61681 * 17 = 1048577 = 2^20 + 1), diagonal + row 0 =
    #     cols 0..16.  z = 61697, 3z = 185091 -> lim = 1048576; ELL E = 1048577, DIA 17 offsets -> 1048577
    m = 61681
    row = np.concatenate([np.zeros(17, np.int64), np.arange(1, m)])
    col = np.concatenate([np.arange(17), np.arange(1, m)])
    out["slack_past"] = (csr_from_arrays(m, m, row, col), {},
                         dict(z=61697, ell_size=1048577, dia_size=1048577, ell_ok=False, dia_ok=False))
    # (3) trunc(3z) binds, exactly at: 600000 rows, row r holds one entry at column r + d(r),
    #     d(r) = ((r + 1) mod 3) - 1 in {0, +1, -1}: z = 600000, 3 offsets -> DIA E = 1800000 = 3z
    #     (admissible); ELL width 1 -> E = 600000 (admissible)
    m = 600000
    rr = np.arange(m)
    col = rr + ((rr + 1) % 3) - 1
    out["fill_at_dia"] = (csr_from_arrays(m, m, rr, col), {},
                          dict(z=600000, ell_size=600000, dia_size=1800000, ell_ok=True, dia_ok=True))
    # (4) trunc(3z) binds, one past (DIA): 600001 rows, every row its diagonal, rows 3j (j < 200000) one
    #     extra entry at offset +1 / +2 / -1 for j mod 3 = 0 / 1 / 2: z = 800001, 3z = 2400003;
    #     4 offsets -> DIA E = 2400004 (inadmissible); ELL width 2 -> 1200002 (admissible)
    m = 600001
    rows, cols = [np.arange(m)], [np.arange(m)]
    j = np.arange(200000)
    off = np.choose(j % 3, [1, 2, -1])
    rows.append(3 * j)
    cols.append(3 * j + off)
    row = np.concatenate(rows)
    col = np.concatenate(cols)
    o = np.lexsort((col, row))
    out["fill_past_dia"] = (csr_from_arrays(m, m, row[o], col[o]), {},
                            dict(z=800001, ell_size=1200002, dia_size=2400004, ell_ok=True, dia_ok=False))
    # (5) trunc(3z) binds, ELL exactly at: 600000 rows, rows 3j hold 3 entries (cols 3j..3j+2), others
    #     empty: z = 600000, K = 3 -> ELL E = 1800000 = 3z (admissible); offsets {0, 1, 2} -> DIA E =
    #     1800000 (admissible)
    m = 600000
    j = np.arange(200000)
    row = np.repeat(3 * j, 3)
    col = (3 * j[:, None] + np.arange(3)[None, :]).ravel()
    out["fill_at_ell"] = (csr_from_arrays(m, m, row, col), {},
                          dict(z=600000, ell_size=1800000, dia_size=1800000, ell_ok=True, dia_ok=True))
    # (6) trunc(3z) binds, ELL one past: 600001 rows, rows 3j (j < 200000) hold 4 entries (cols 3j..3j+3),
    #     row 600000 holds its diagonal: z = 800001, 3z = 2400003, K = 4 -> ELL E = 2400004 (inadmissible);
    #     offsets {0,1,2,3} -> DIA E = 2400004 (inadmissible)
    m = 600001
    row = np.concatenate([np.repeat(3 * j, 4), [600000]])
    col = np.concatenate([(3 * j[:, None] + np.arange(4)[None, :]).ravel(), [600000]])
    out["fill_past_ell"] = (csr_from_arrays(m, m, row, col), {},
                            dict(z=800001, ell_size=2400004, dia_size=2400004, ell_ok=False, dia_ok=False))
    # (7) truncation of a non-integer limit: max_fill = 2.5, fill_slack = 0, z = 7 -> 2.5z = 17.5 ->
    #     lim = 17.  17 rows, rows 0..6 hold their diagonal: ELL E = 17 (admissible; K = 1); offsets {0}
    #     -> DIA E = 17 (admissible).  18 rows: E = 18 = ceil(17.5) (inadmissible, a rounding-up slip
    #     admits it)
    for mm, ok, name in ((17, True, "trunc_at"), (18, False, "trunc_past")):
        A = csr_from_arrays(mm, mm, np.arange(7), np.arange(7))
        out[name] = (A, dict(max_fill=2.5, fill_slack=0),
                     dict(z=7, ell_size=mm, dia_size=mm, ell_ok=ok, dia_ok=ok))
    return out
