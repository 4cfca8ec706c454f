"""GPU parity of the semi-supervised predictor against the oracle chain: ranges and
means bit-exact (same fixed-order definitions); the PCA step is solved independently on each side
(library: Householder + implicit QL, csrc/eigen.cpp, itself pinned to numpy eigh in tests/test_pca_pin.py;
oracle: cyclic Jacobi), so eigenvalues / basis / centroids agree to a tolerance and the discrete results
(assignments, iterations, votes, predictions) exactly."""
import numpy as np
import pytest

import oracle
import paper_conf_icppw_dhandhaniadpbl21_b200 as sfs
import sfsgen

pytestmark = pytest.mark.gpu


def _table(count, seed):
    rng = np.random.default_rng(seed)
    feats, labels = [], []
    for i in range(count):
        cls = [sfsgen.BAND, sfsgen.UNIFORM, sfsgen.BLOCKDIAG, sfsgen.POWERLAW][i % 4]
        m = int(rng.integers(800, 6000))
        spec = sfsgen.make_spec(cls, seed=seed * 1000 + i, m=m, ia=int(rng.integers(2, 20)),
                                pa=float(rng.uniform(0.5, 1.0)) if cls in (sfsgen.BAND, sfsgen.BLOCKDIAG)
                                else (float(rng.uniform(4, 40)) if cls == sfsgen.UNIFORM else float(rng.uniform(2.1, 3.0))))
        A = sfsgen.generate(spec)
        feats.append(oracle.features(A.m, A.n, A.rp, A.col))
        labels.append(int(rng.integers(0, 5)) if i % 7 else i % 4)
    return oracle.table1_matrix(feats), np.array(labels, np.int32), feats


@pytest.mark.parametrize("nc,pcs", [(6, 8), (20, 8), (9, 4)])
def test_fit_vote_predict_parity(nc, pcs):
    raw, labels, _ = _table(120, 5)
    init = np.random.default_rng(nc).choice(len(raw), size=nc, replace=False).astype(np.int32)
    ref = oracle.ss_fit(raw, init, pcs=pcs)
    M = sfs.ClusterModel(raw, init, pcs=pcs)
    g = M.info
    for k in ("mins", "maxs", "mean"):
        assert np.array_equal(g[k], ref[k]), k
    scale = float(ref["eigval"][0])
    assert np.abs(g["eigval"] - ref["eigval"]).max() <= 1e-12 * scale
    ev_all = ref["eigval"]
    for c in range(pcs):
        gap = min(abs(ev_all[c] - ev_all[j]) for j in range(pcs) if j != c)
        if gap > 1e-6 * scale:
            assert np.abs(g["basis"][c] - ref["basis"][c]).max() <= 1e-9 * scale / gap, c
    assert np.allclose(g["centroids"], ref["centroids"], rtol=0, atol=1e-10)
    assert (g["assign"] == ref["assign"]).all() and g["iters"] == ref["iters"]
    bench = labels.copy()
    bench[::3] = -1  # a third of the corpus not benchmarked
    assert (M.vote(bench) == oracle.ss_vote(ref["assign"], bench, nc)).all()
    new_raw, _, _ = _table(40, 17)
    assert (M.predict(new_raw) == oracle.ss_predict(ref, new_raw)).all()
    M.free()


def test_table1_from_gpu_features_matches_oracle_table():
    import torch
    _, _, feats = _table(8, 3)
    specs = [sfsgen.generate(sfsgen.make_spec(sfsgen.ST2D5, ia=20 + i)) for i in range(4)]
    t = lambda a: torch.from_numpy(a).cuda()
    gf = [sfs.features(sfs.Csr(A.m, A.n, t(A.rp), t(A.col), t(A.val))) for A in specs]
    of = [oracle.features(A.m, A.n, A.rp, A.col) for A in specs]
    assert np.array_equal(sfs.features_table1(gf), oracle.table1_matrix(of))
