"""CPU oracle (TEST INFRASTRUCTURE ONLY).

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` / ``--impl
reference`` leg may import this module.  The product package never imports it; it shares no code
with the CUDA path.  The arithmetic lives in ``oracle/oracle.c`` (plain C, fp64, long-double SpMV
accumulation); this file only marshals numpy arrays through ctypes.

Every function cites the paper passage it follows (``P:L<n>`` = /root/reference/PAPER.md line n)
and the SURVEY.md §8(c) reading (Q1–Q18) it takes where the paper is silent.  Pins:
``tests/test_oracle_pins.py``.  Parity of the *label* (a timing result) is unpinned: only the
decision rule is pinned.
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "liboracle.so")
CSR, COO, ELL, HYB, DIA = range(5)
NFMT = 5
FORMAT_NAMES = ["CSR", "COO", "ELL", "HYB", "DIA"]

_I64 = ctypes.c_int64
_P = ctypes.c_void_p


class Opts(ctypes.Structure):
    _fields_ = [("max_fill", ctypes.c_double), ("fill_slack", _I64), ("hyb_rel_speed", ctypes.c_double),
                ("hyb_breakeven", _I64), ("csr_warps", _I64)]


INT_FIELDS = ["nrows", "ncols", "nnz", "nnz_min", "nnz_max", "csr_max", "ell_size", "hyb_k", "hyb_ell_size",
              "hyb_coo", "hyb_ell_nnz", "diagonals", "dia_size"]
FLOAT_FIELDS = ["nnz_frac", "nnz_mu", "nnz_sig", "max_mu", "mu_min", "sig_lower", "sig_higher", "hyb_ell_frac",
                "dia_frac", "ell_frac"]


class Features(ctypes.Structure):
    _fields_ = ([(f, _I64) for f in INT_FIELDS] + [(f, ctypes.c_double) for f in FLOAT_FIELDS]
                + [("admissible_mask", ctypes.c_uint32)])

    def as_dict(self) -> dict:
        d = {f: int(getattr(self, f)) for f in INT_FIELDS}
        d.update({f: float(getattr(self, f)) for f in FLOAT_FIELDS})
        d["admissible_mask"] = int(self.admissible_mask)
        return d


_lib = None


def lib():
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise RuntimeError(f"{LIB_PATH} missing: run __graft_entry__.build()")
        L = ctypes.CDLL(LIB_PATH)
        L.or_validate.restype = ctypes.c_int
        L.or_validate.argtypes = [_I64, _I64, _I64, _P, _P]
        L.or_default_opts.argtypes = [ctypes.POINTER(Opts)]
        L.or_features_compute.argtypes = [_I64, _I64, _P, _P, ctypes.POINTER(Opts), ctypes.POINTER(Features)]
        L.or_csr_to_coo.argtypes = [_I64, _P, _P, _P, _P, _P, _P]
        L.or_csr_to_ell.argtypes = [_I64, _P, _P, _P, _I64, _P, _P]
        L.or_csr_to_hyb.argtypes = [_I64, _P, _P, _P, _I64, _P, _P, _P, _P, _P]
        L.or_dia_offsets.argtypes = [_I64, _I64, _P, _P, _P]
        L.or_dia_offsets.restype = _I64
        L.or_csr_to_dia.argtypes = [_I64, _P, _P, _P, _I64, _P, _P]
        L.or_spmv_csr.argtypes = [_I64, _P, _P, _P, _P, _P, _P]
        L.or_spmv_coo.argtypes = [_I64, _I64, _P, _P, _P, _P, _P, _P]
        L.or_spmv_ell.argtypes = [_I64, _I64, _P, _P, _P, _P, _P]
        L.or_spmv_hyb.argtypes = [_I64, _I64, _P, _P, _I64, _P, _P, _P, _P, _P, _P]
        L.or_spmv_dia.argtypes = [_I64, _I64, _I64, _P, _P, _P, _P, _P]
        L.or_label.argtypes = [_P, ctypes.c_uint32]
        L.or_label.restype = ctypes.c_int32
        L.or_label_matrix.argtypes = [_I64, _I64, _P, _P, _P, _P, ctypes.POINTER(Opts), ctypes.c_int32,
                                      ctypes.c_uint32, ctypes.POINTER(Features), _P, _P]
        L.or_label_matrix.restype = ctypes.c_int32
        _lib = L
    return _lib


def _p(a: np.ndarray):
    return a.ctypes.data if a is not None else None


def _i32(a):
    return np.ascontiguousarray(a, dtype=np.int32)


def _f64(a):
    return np.ascontiguousarray(a, dtype=np.float64)


def default_opts(**kw) -> Opts:
    o = Opts()
    lib().or_default_opts(ctypes.byref(o))
    for k, v in kw.items():
        setattr(o, k, v)
    return o


def validate(m, n, rp, col) -> int:
    """Q16 canonical-CSR check (0 = valid)."""
    rp, col = _i32(rp), _i32(col)
    return int(lib().or_validate(m, n, int(rp[-1]) if len(rp) else 0, _p(rp), _p(col) if len(col) else None))


def features(m, n, rp, col, opts: Opts | None = None) -> dict:
    """Table-1 features as fixed fp64 formulas of exact integer aggregates (§8(c))."""
    rp, col = _i32(rp), _i32(col)
    f = Features()
    lib().or_features_compute(m, n, _p(rp), _p(col) if len(col) else None,
                              ctypes.byref(opts or default_opts()), ctypes.byref(f))
    return f.as_dict()


@dataclass
class Converted:
    fmt: int
    m: int
    n: int
    # COO: row, col, val ; ELL: K, ecol (m,K), eval ; HYB: K, ecol, eval, crow, ccol, cval ; DIA: offs, dval (nd,m)
    arrays: dict


def convert(fmt, m, n, rp, col, val, feats: dict | None = None) -> Converted:
    """CSR -> fmt (§2.1; step (ii) of P:L331). Oracle row-major layouts (see oracle.h)."""
    rp, col, val = _i32(rp), _i32(col), _f64(val)
    z = int(rp[-1])
    L = lib()
    if fmt == CSR:
        return Converted(fmt, m, n, {"rp": rp.copy(), "col": col.copy(), "val": val.copy()})
    if fmt == COO:
        r, c, v = np.empty(z, np.int32), np.empty(z, np.int32), np.empty(z, np.float64)
        L.or_csr_to_coo(m, _p(rp), _p(col), _p(val), _p(r), _p(c), _p(v))
        return Converted(fmt, m, n, {"row": r, "col": c, "val": v})
    feats = feats or features(m, n, rp, col)
    if fmt == ELL:
        K = feats["nnz_max"]
        ec, ev = np.empty(m * K, np.int32), np.empty(m * K, np.float64)
        L.or_csr_to_ell(m, _p(rp), _p(col), _p(val), K, _p(ec), _p(ev))
        return Converted(fmt, m, n, {"K": K, "ecol": ec.reshape(m, K), "eval": ev.reshape(m, K)})
    if fmt == HYB:
        K, nc = feats["hyb_k"], feats["hyb_coo"]
        ec, ev = np.empty(m * K, np.int32), np.empty(m * K, np.float64)
        cr, cc, cv = np.empty(nc, np.int32), np.empty(nc, np.int32), np.empty(nc, np.float64)
        L.or_csr_to_hyb(m, _p(rp), _p(col), _p(val), K, _p(ec), _p(ev), _p(cr), _p(cc), _p(cv))
        return Converted(fmt, m, n, {"K": K, "ecol": ec.reshape(m, K), "eval": ev.reshape(m, K),
                                     "crow": cr, "ccol": cc, "cval": cv})
    if fmt == DIA:
        nd = int(L.or_dia_offsets(m, n, _p(rp), _p(col), None))
        offs = np.empty(nd, np.int32)
        L.or_dia_offsets(m, n, _p(rp), _p(col), _p(offs))
        dv = np.empty(nd * m, np.float64)
        L.or_csr_to_dia(m, _p(rp), _p(col), _p(val), nd, _p(offs), _p(dv))
        return Converted(fmt, m, n, {"offs": offs, "dval": dv.reshape(nd, m)})
    raise ValueError(fmt)


def spmv(cv: Converted, x, with_abs=True):
    """y = A x over the format's own arrays; long-double accumulation rounded once.
    Returns (y, |A||x|)."""
    x = _f64(x)
    m = cv.m
    y = np.empty(m, np.float64)
    ay = np.empty(m, np.float64) if with_abs else None
    a = cv.arrays
    L = lib()
    if cv.fmt == CSR:
        L.or_spmv_csr(m, _p(a["rp"]), _p(a["col"]), _p(a["val"]), _p(x), _p(y), _p(ay))
    elif cv.fmt == COO:
        L.or_spmv_coo(m, len(a["row"]), _p(a["row"]), _p(a["col"]), _p(a["val"]), _p(x), _p(y), _p(ay))
    elif cv.fmt == ELL:
        L.or_spmv_ell(m, a["K"], _p(np.ascontiguousarray(a["ecol"])), _p(np.ascontiguousarray(a["eval"])),
                      _p(x), _p(y), _p(ay))
    elif cv.fmt == HYB:
        L.or_spmv_hyb(m, a["K"], _p(np.ascontiguousarray(a["ecol"])), _p(np.ascontiguousarray(a["eval"])),
                      len(a["crow"]), _p(a["crow"]), _p(a["ccol"]), _p(a["cval"]), _p(x), _p(y), _p(ay))
    elif cv.fmt == DIA:
        L.or_spmv_dia(m, cv.n, len(a["offs"]), _p(a["offs"]), _p(np.ascontiguousarray(a["dval"])), _p(x),
                      _p(y), _p(ay))
    else:
        raise ValueError(cv.fmt)
    return y, ay


def spmv_csr(m, n, rp, col, val, x):
    return spmv(convert(CSR, m, n, rp, col, val), x)


def label(times, mask) -> int:
    """Decision rule (P:L217 'average over 100 trials'; Q14 ties -> lowest id)."""
    t = _f64(times)
    return int(lib().or_label(_p(t), mask))


def label_matrix(m, n, rp, col, val, x, reps=3, formats_mask=0x1F, opts: Opts | None = None):
    """Whole oracle labelling pass of one matrix (the cpu_baseline): features, admissible
    conversions, `reps` timed SpMVs per format, argmin.  Releases the GIL (ctypes)."""
    rp, col, val, x = _i32(rp), _i32(col), _f64(val), _f64(x)
    f = Features()
    ts, tc = np.zeros(NFMT), np.zeros(NFMT)
    lab = lib().or_label_matrix(m, n, _p(rp), _p(col), _p(val), _p(x), ctypes.byref(opts or default_opts()),
                                reps, formats_mask, ctypes.byref(f), _p(ts), _p(tc))
    return int(lab), f.as_dict(), ts, tc


# ---------------------------------------------------------------------------- semi-supervised (f1)
# Oracle of the paper's semi-supervised predictor (§4): transform + min-max +
# PCA(8) + K-Means + VOTE; see oracle/semisup.c and DESIGN.md readings F1–F7.
NFEAT = 21
TABLE1 = ["nrows", "ncols", "nnz", "nnz_frac", "nnz_mu", "nnz_min", "nnz_max", "nnz_sig", "max_mu", "mu_min",
          "csr_max", "sig_lower", "sig_higher", "hyb_ell_size", "hyb_coo", "hyb_ell_frac", "diagonals", "dia_size",
          "dia_frac", "ell_frac", "ell_size"]
_ss_ready = False


def _ss():
    global _ss_ready
    L = lib()
    if not _ss_ready:
        L.or_ss_preprocess.argtypes = [_I64, _P, _P, _P, _P]
        L.or_ss_pca.argtypes = [_I64, ctypes.c_int, _P, ctypes.c_int, _P, _P, _P]
        L.or_ss_project.argtypes = [_I64, ctypes.c_int, _P, _P, ctypes.c_int, _P, _P]
        L.or_ss_assign.argtypes = [_I64, ctypes.c_int, _P, ctypes.c_int, _P, _P]
        L.or_ss_kmeans.argtypes = [_I64, ctypes.c_int, _P, ctypes.c_int, _P, ctypes.c_int, _P, _P]
        L.or_ss_kmeans.restype = ctypes.c_int
        L.or_ss_vote.argtypes = [_I64, _P, _P, ctypes.c_int, ctypes.c_int, _P]
        L.or_ss_purity.argtypes = [_I64, _P, _P, ctypes.c_int, ctypes.c_int, _P]
        L.or_ss_purity.restype = ctypes.c_double
        L.or_ss_vote_expected_accuracy.argtypes = [_P, ctypes.c_int, ctypes.c_int, _P]
        L.or_ss_vote_expected_accuracy.restype = ctypes.c_double
        L.or_ss_feature_kind.argtypes = [ctypes.c_int]
        L.or_ss_feature_kind.restype = ctypes.c_int
        _ss_ready = True
    return L


def table1_matrix(feature_dicts) -> np.ndarray:
    """n x 21 fp64 matrix of the Table-1 features (P:L79–102 order)."""
    return np.array([[float(f[k]) for k in TABLE1] for f in feature_dicts], dtype=np.float64).reshape(-1, NFEAT)


def ss_preprocess(raw):
    """F1 transform (log1p / sqrt per feature kind) + F2 min-max to [0, 1]."""
    raw = _f64(raw).reshape(-1, NFEAT)
    n = raw.shape[0]
    out = np.empty_like(raw)
    mins, maxs = np.empty(NFEAT), np.empty(NFEAT)
    _ss().or_ss_preprocess(n, _p(raw), _p(out), _p(mins), _p(maxs))
    return out, mins, maxs


def ss_pca(X, k=8):
    """F3: population covariance, cyclic Jacobi, descending eigenvalues, sign-normalised."""
    X = _f64(X)
    n, d = X.shape
    mean, basis, ev = np.empty(d), np.empty((k, d)), np.empty(k)
    _ss().or_ss_pca(n, d, _p(X), k, _p(mean), _p(basis), _p(ev))
    return mean, basis, ev


def ss_project(X, mean, basis):
    X = _f64(X)
    n, d = X.shape
    k = basis.shape[0]
    Y = np.empty((n, k))
    _ss().or_ss_project(n, d, _p(X), _p(_f64(mean)), k, _p(_f64(basis)), _p(Y))
    return Y


def ss_kmeans(Y, init_idx, max_iter=100):
    """F4: Lloyd's K-Means from the given initial points."""
    Y = _f64(Y)
    n, k = Y.shape
    init = _i32(init_idx)
    nc = len(init)
    cent = np.empty((nc, k))
    assign = np.empty(n, np.int32)
    it = _ss().or_ss_kmeans(n, k, _p(Y), nc, _p(init), max_iter, _p(cent), _p(assign))
    return cent, assign, int(it)


def ss_assign(Y, cent):
    """Nearest centroid, ties to the lowest id."""
    Y, cent = _f64(Y), _f64(cent)
    n, k = Y.shape
    assign = np.empty(n, np.int32)
    _ss().or_ss_assign(n, k, _p(Y), cent.shape[0], _p(cent), _p(assign))
    return assign


def ss_vote(assign, labels, nc, nfmt=NFMT):
    """F5/F6: majority of benchmarked members (labels < 0 = not benchmarked)."""
    a, lab = _i32(assign), _i32(labels)
    out = np.empty(nc, np.int32)
    _ss().or_ss_vote(len(a), _p(a), _p(lab), nc, nfmt, _p(out))
    return out


def ss_purity(assign, labels, nc, nfmt=NFMT):
    """P:L140 purity per cluster and the size-weighted mean."""
    a, lab = _i32(assign), _i32(labels)
    pur = np.empty(nc)
    mean = _ss().or_ss_purity(len(a), _p(a), _p(lab), nc, nfmt, _p(pur))
    return pur, float(mean)


def ss_vote_expected_accuracy(counts, draws):
    """P:L169 worked example: expected accuracy of a cluster labelled by `draws` benchmarked members."""
    c = np.ascontiguousarray(counts, dtype=np.int64)
    p = np.empty(len(c))
    acc = _ss().or_ss_vote_expected_accuracy(_p(c), len(c), draws, _p(p))
    return float(acc), p


def ss_scale(raw, mins, maxs):
    """Prediction-path scaling of new matrices with the fitted ranges (F2)."""
    raw = _f64(raw).reshape(-1, NFEAT)
    out = np.empty_like(raw)
    L = _ss()
    L.or_ss_scale.argtypes = [_I64, _P, _P, _P, _P]
    L.or_ss_scale(raw.shape[0], _p(raw), _p(_f64(mins)), _p(_f64(maxs)), _p(out))
    return out


def ss_fit(raw, init_idx, pcs=8, max_iter=100):
    """The whole oracle fit chain: preprocess -> PCA -> project -> K-Means."""
    X, mins, maxs = ss_preprocess(raw)
    mean, basis, ev = ss_pca(X, pcs)
    Y = ss_project(X, mean, basis)
    cent, assign, it = ss_kmeans(Y, init_idx, max_iter)
    return {"mins": mins, "maxs": maxs, "mean": mean, "basis": basis, "eigval": ev, "centroids": cent,
            "assign": assign, "iters": it}


def ss_predict(fit, raw):
    X = ss_scale(raw, fit["mins"], fit["maxs"])
    return ss_assign(ss_project(X, fit["mean"], fit["basis"]), fit["centroids"])
