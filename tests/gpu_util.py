"""GPU-test helpers: run the library through the C ABI and compare with the oracle."""
from __future__ import annotations

import numpy as np

import oracle
import paper_conf_icppw_dhandhaniadpbl21_b200 as sfs

TOL = {sfs.F64: 1e-12, sfs.F32: 1e-5}


def to_dev(A, x=None):
    import torch
    t = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
    return sfs.Csr(A.m, A.n, t(A.rp), t(A.col), t(A.val), t(x) if x is not None else None)


def assert_features_equal(fg: dict, fo: dict, ctx=""):
    for k in oracle.INT_FIELDS + ["admissible_mask"]:
        assert fg[k] == fo[k], f"{ctx} feature {k}: gpu {fg[k]} oracle {fo[k]}"
    for k in oracle.FLOAT_FIELDS:
        a, b = fg[k], fo[k]
        assert np.float64(a).tobytes() == np.float64(b).tobytes(), f"{ctx} feature {k}: gpu {a!r} oracle {b!r}"


def check_conversion(A, fmt, M: sfs.Matrix, feats: dict):
    """Decoded physical layout == oracle logical content, bit for bit (values compared in fp64:
    fp32 -> fp64 is exact)."""
    g = sfs.decode(M)
    ov = A.val.astype(np.float64)
    cv = oracle.convert(fmt, A.m, A.n, A.rp, A.col, ov, feats)
    a = cv.arrays
    m, P = A.m, g["pitch"]
    if fmt == sfs.CSR:
        assert (g["rp"] == A.rp).all() and (g["col"] == A.col).all() and (g["val"] == A.val).all()
    elif fmt == sfs.COO:
        assert (g["row"] == a["row"]).all() and (g["col"] == a["col"]).all()
        assert (g["val"].astype(np.float64) == a["val"]).all()
    elif fmt in (sfs.ELL, sfs.HYB):
        K = a["K"]
        assert g["width"] == K and P == ((m + 31) // 32) * 32
        ec, ev = g["ecol"], g["eval"].astype(np.float64)
        assert ec.shape == (K, P)
        assert (ec[:, :m].T == a["ecol"]).all()
        assert (ev[:, :m].T == a["eval"]).all()
        assert (ec[:, m:] == -1).all() and (ev[:, m:] == 0).all()
        assert not np.signbit(ev[ec < 0]).any()  # padding is +0.0
        if fmt == sfs.HYB:
            assert g["coo_nnz"] == len(a["crow"])
            assert (g["crow"] == a["crow"]).all() and (g["ccol"] == a["ccol"]).all()
            assert (g["cval"].astype(np.float64) == a["cval"]).all()
    elif fmt == sfs.DIA:
        assert (g["offs"] == a["offs"]).all()
        dv = g["dval"].astype(np.float64)
        assert dv.shape == (len(a["offs"]), P)
        assert (dv[:, :m] == a["dval"]).all() and (dv[:, m:] == 0).all()
        assert not np.signbit(dv[dv == 0]).any()


def check_spmv(A, fmt, M: sfs.Matrix, x: np.ndarray, dtype: int, ctx=""):
    """Per-row |y_gpu - y_ref| <= tol * (|A||x|)_r; rows with (|A||x|)_r = 0 must give exactly 0."""
    import torch
    xd = torch.from_numpy(x).cuda()
    yr, ay = oracle.spmv_csr(A.m, A.n, A.rp, A.col, A.val.astype(np.float64), x.astype(np.float64))
    tol = TOL[dtype]
    # twice, y poisoned with NaN before each call: every row must be written, and the kernels' carry
    # flags must be back to their initial state after a call
    for rep in range(2):
        y = torch.full((A.m,), float("nan"), dtype=xd.dtype, device="cuda")
        sfs.spmv(fmt, M, xd, y)
        torch.cuda.synchronize()
        yg = y.cpu().numpy().astype(np.float64)
        err = np.abs(yg - yr)
        bad = ~(err <= tol * ay)
        zero_rows = ay == 0
        bad |= zero_rows & (yg != 0)
        assert not bad.any(), (f"{ctx} {sfs.FORMAT_NAMES[fmt]} call {rep}: {int(bad.sum())} rows out of tolerance; "
                               f"first {np.nonzero(bad)[0][:5]} gpu {yg[bad][:5]} ref {yr[bad][:5]} "
                               f"|A||x| {ay[bad][:5]}")
    return yg
