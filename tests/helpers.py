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
