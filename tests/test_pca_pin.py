"""CPU pin of the LIBRARY's PCA eigen-step (sfs_pca_basis: Householder + implicit QL, csrc/eigen.cpp)
against numpy's LAPACK eigh -- a third, independent solver -- so that the f1 GPU parity with the oracle's
Jacobi (tests/test_gpu_semisup.py) is not parity by construction.  PAPER.md §4 P:L148 ("PCA ... feature
vector of size 8"); reading F3.  Host-only call: runs without a GPU."""
import ctypes

import numpy as np
import pytest

import oracle
import paper_conf_icppw_dhandhaniadpbl21_b200 as sfs
import sfsgen


def pca_basis(C, k):
    L = sfs.lib()
    f = L.sfs_pca_basis
    f.restype = ctypes.c_int32
    f.argtypes = [ctypes.c_int32, ctypes.c_void_p, ctypes.c_int32, ctypes.c_void_p, ctypes.c_void_p]
    C = np.ascontiguousarray(C, dtype=np.float64)
    n = C.shape[0]
    B, ev = np.zeros((k, n)), np.zeros(k)
    st = f(n, C.ctypes.data, k, B.ctypes.data, ev.ctypes.data)
    assert st == 0, sfs.lib().sfs_last_error()
    return B, ev


def _check_against_eigh(C, k, tol=1e-13):
    B, ev = pca_basis(C, k)
    w, V = np.linalg.eigh(C)
    w, V = w[::-1], V[:, ::-1]
    scale = max(1.0, float(np.abs(w).max()))
    assert np.abs(ev - w[:k]).max() <= tol * scale
    assert np.abs(B @ B.T - np.eye(k)).max() <= 1e-13
    assert np.abs(C @ B.T - B.T * ev).max() <= tol * scale  # residual of every returned pair
    for c in range(k):
        gap = min([abs(w[c] - w[j]) for j in range(len(w)) if j != c] or [np.inf])
        big = int(np.argmax(np.abs(B[c])))
        assert B[c][big] > 0 and np.abs(B[c]).max() == abs(B[c][big])  # F3 sign convention
        if gap > 1e-6 * scale:  # an isolated eigenvalue has a unique direction
            v = V[:, c] * np.sign(V[np.argmax(np.abs(V[:, c])), c])
            mags = np.sort(np.abs(v))
            if mags[-1] - mags[-2] < 1e-9:  # two entries of equal magnitude: the sign is a rounding tie
                v = v if np.dot(v, B[c]) > 0 else -v
            assert np.abs(B[c] - v).max() <= 1e-10 * scale / gap
    return B, ev


@pytest.mark.parametrize("seed", range(6))
def test_pca_basis_random_symmetric(seed):
    rng = np.random.default_rng(seed)
    n = 21
    A = rng.normal(size=(n, n))
    C = np.cov((rng.normal(size=(400, n)) @ A).T, bias=True) if seed % 2 else (A + A.T) / 2
    _check_against_eigh(np.ascontiguousarray((C + C.T) / 2), 8)


def test_pca_basis_repeated_and_zero_eigenvalues():
    rng = np.random.default_rng(7)
    Q, _ = np.linalg.qr(rng.normal(size=(21, 21)))
    w = np.array([5, 5, 5, 3, 3, 1] + [0] * 15, float)
    C = (Q * w) @ Q.T
    B, ev = _check_against_eigh((C + C.T) / 2, 8)
    assert np.allclose(ev, [5, 5, 5, 3, 3, 1, 0, 0], atol=1e-13)
    # diagonal and already-tridiagonal inputs; 1x1
    B, ev = pca_basis(np.diag(np.arange(21.0)), 21)
    assert list(ev) == list(np.arange(20.0, -1.0, -1.0)) and np.array_equal(np.abs(B), np.eye(21)[::-1])
    T = np.diag(np.full(21, 2.0)) - np.diag(np.ones(20), 1) - np.diag(np.ones(20), -1)
    _check_against_eigh(T, 21)
    B, ev = pca_basis(np.array([[3.5]]), 1)
    assert ev[0] == 3.5 and B[0, 0] == 1.0


def test_pca_basis_on_feature_covariance():
    """The covariance the predictor actually decomposes: scaled Table-1 features of a seeded corpus of the
    four structure classes (oracle features; the same recipe as tests/test_gpu_semisup.py)."""
    rng = np.random.default_rng(5)
    feats = []
    for i in range(80):
        cls = [sfsgen.BAND, sfsgen.UNIFORM, sfsgen.BLOCKDIAG, sfsgen.POWERLAW][i % 4]
        m = int(rng.integers(800, 4000))
        pa = (float(rng.uniform(0.5, 1.0)) if cls in (sfsgen.BAND, sfsgen.BLOCKDIAG)
              else (float(rng.uniform(4, 40)) if cls == sfsgen.UNIFORM else float(rng.uniform(2.1, 3.0))))
        A = sfsgen.generate(sfsgen.make_spec(cls, seed=5000 + i, m=m, ia=int(rng.integers(2, 20)), pa=pa))
        feats.append(oracle.features(A.m, A.n, A.rp, A.col))
    X, _, _ = oracle.ss_preprocess(oracle.table1_matrix(feats))
    C = np.cov(X.T, bias=True)
    _check_against_eigh(np.ascontiguousarray((C + C.T) / 2), 8)


def test_pca_basis_rejects_bad_sizes():
    L = sfs.lib()
    L.sfs_pca_basis.restype = ctypes.c_int32
    L.sfs_pca_basis.argtypes = [ctypes.c_int32, ctypes.c_void_p, ctypes.c_int32, ctypes.c_void_p, ctypes.c_void_p]
    C = np.eye(3)
    B, ev = np.zeros((3, 3)), np.zeros(3)
    assert L.sfs_pca_basis(3, C.ctypes.data, 4, B.ctypes.data, ev.ctypes.data) == sfs.ERR_INVALID_ARG
    assert L.sfs_pca_basis(0, C.ctypes.data, 1, B.ctypes.data, ev.ctypes.data) == sfs.ERR_INVALID_ARG
