"""Input generators: canonical CSR, determinism, class structure, thread-count invariance."""
import os
import subprocess
import sys

import numpy as np
import pytest

import sfsgen


def _canonical(A):
    assert A.rp[0] == 0 and A.rp[-1] == A.nnz and (np.diff(A.rp) >= 0).all()
    assert (A.col >= 0).all() and (A.col < A.n).all()
    rows = np.repeat(np.arange(A.m), np.diff(A.rp))
    key = rows.astype(np.int64) * A.n + A.col
    assert (np.diff(key) > 0).all()  # strictly increasing within rows, rows in order
    assert (A.val != 0).all()


SPECS = [
    sfsgen.make_spec(sfsgen.BAND, seed=3, m=5000, ia=7, pa=0.7),
    sfsgen.make_spec(sfsgen.BLOCKDIAG, seed=4, m=5000, ia=33, pa=0.6, dtype=sfsgen.F32),
    sfsgen.make_spec(sfsgen.UNIFORM, seed=5, m=4000, n=3000, pa=20.0),
    sfsgen.make_spec(sfsgen.POWERLAW, seed=6, m=8000, pa=2.2),
    sfsgen.make_spec(sfsgen.POWERLAW, seed=7, m=500, pa=2.05),  # forces the Bernoulli branch
    sfsgen.make_spec(sfsgen.RMAT, seed=8, ia=12, ib=16, dtype=sfsgen.F32),
    sfsgen.make_spec(sfsgen.ST2D5, ia=20),
    sfsgen.make_spec(sfsgen.ST3D7, ia=9),
    sfsgen.make_spec(sfsgen.ST3D27, ia=9),
]


@pytest.mark.parametrize("spec", SPECS, ids=lambda s: sfsgen.CLASS_NAMES[s.cls])
def test_canonical_and_deterministic(spec):
    A = sfsgen.generate(spec)
    _canonical(A)
    B = sfsgen.generate(spec)
    assert (A.rp == B.rp).all() and (A.col == B.col).all() and (A.val == B.val).all()
    assert A.val.dtype == (np.float64 if spec.dtype else np.float32)


def test_class_structure():
    A = sfsgen.generate(SPECS[0])
    rows = np.repeat(np.arange(A.m), np.diff(A.rp))
    assert (np.abs(A.col - rows) <= 7).all() and (A.col[np.searchsorted(A.col, 0):] >= 0).all()
    B = sfsgen.generate(SPECS[1])
    rows = np.repeat(np.arange(B.m), np.diff(B.rp))
    assert (A.col.size > 0) and (rows // 33 == B.col // 33).all()
    # every row keeps its diagonal in band / block classes
    for M in (A, B):
        rows = np.repeat(np.arange(M.m), np.diff(M.rp))
        assert len(np.unique(rows[rows == M.col])) == M.m


def test_rmat_shape():
    A = sfsgen.rmat(14, seed=1)
    assert A.m == 2 ** 14
    # ~2.8% duplicates at scale 22; at least some are dropped at scale 14, most edges survive
    assert 0.8 * 16 * 2 ** 14 < A.nnz < 16 * 2 ** 14
    lens = np.diff(A.rp)
    assert (lens == 0).mean() > 0.3 and lens.max() > 50 * lens.mean()  # skewed, many empty rows


def test_thread_count_invariance():
    code = ("import sfsgen,hashlib;A=sfsgen.generate(sfsgen.make_spec(sfsgen.UNIFORM,seed=11,m=20000,pa=9.0));"
            "print(hashlib.sha1(A.rp.tobytes()+A.col.tobytes()+A.val.tobytes()).hexdigest())")
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    outs = set()
    for t in ("1", "3"):
        env = dict(os.environ, OMP_NUM_THREADS=t, PYTHONPATH=root)
        outs.add(subprocess.check_output([sys.executable, "-c", code], env=env, cwd=root).strip())
    assert len(outs) == 1


def test_corpus_specs():
    seen = set()
    for i in range(200):
        s = sfsgen.corpus_spec(200, i)
        assert 10_000 <= s.m < 1_000_000
        seen.add((s.cls, s.dtype))
    assert len(seen) == 8
    for i in range(0, 2000, 97):
        s = sfsgen.corpus_spec(2000, i)
        m, n = sfsgen.dims(s)
        assert m >= 64 and n == m


def test_vector():
    x = sfsgen.vector(3, 1000)
    assert (x >= -1).all() and (x < 1).all() and abs(x.mean()) < 0.1
    assert (sfsgen.vector(3, 1000, sfsgen.F32) == x.astype(np.float32)).all()
