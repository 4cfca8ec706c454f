"""Pins of the semi-supervised oracle (§4): the paper's worked
VOTE example (tests/golden/vote_example.json), closed forms, and independent library routines
(numpy eigh, scikit-learn KMeans) the oracle does not call."""
import math

import numpy as np
import pytest

import oracle
from helpers import golden


@pytest.mark.parametrize("case", golden("vote_example.json")["cases"], ids=lambda c: c["name"])
def test_vote_worked_example(case):
    acc, p = oracle.ss_vote_expected_accuracy(case["counts"], case["draws"])
    assert round(100 * acc) == case["accuracy_percent"]
    assert p[case["correct"]] == pytest.approx(case["p_correct"], abs=1e-12)
    # closed forms behind the printed numbers
    if case["name"] == "turing_1_draw":
        assert acc == pytest.approx(0.9 * 0.9 + 0.1 * 0.1, abs=1e-15)
    if case["name"] == "pascal_2_draws":
        assert acc == pytest.approx((1 - 0.2 ** 2) * 0.8 + 0.2 ** 2 * 0.2, abs=1e-15)


def test_purity_and_vote():
    assign = np.array([0, 0, 0, 1, 1, 2, 2, 2, 2])
    labels = np.array([2, 2, 0, 1, 3, 4, 4, 4, 0])
    pur, mean = oracle.ss_purity(assign, labels, 4)
    assert list(pur) == [2 / 3, 1 / 2, 3 / 4, 0.0]
    assert mean == pytest.approx((2 + 1 + 3) / 9, abs=1e-15)
    # vote with some members unbenchmarked (-1); cluster 1 tie (1 vs 3) -> lowest id; cluster 3 empty
    bench = np.array([2, -1, 0, 1, 3, 4, -1, -1, 0])
    cl = oracle.ss_vote(assign, bench, 4)
    assert list(cl) == [0, 1, 0, 0]  # c0: tie 2 vs 0 -> 0 ; c2: tie 4 vs 0 -> 0 ; c3: global majority (0: 2 votes)


def test_preprocess_closed_form():
    rng = np.random.default_rng(0)
    raw = rng.uniform(0, 1e6, size=(50, oracle.NFEAT))
    for j in range(oracle.NFEAT):
        if oracle._ss().or_ss_feature_kind(j) == 1:
            raw[:, j] = rng.uniform(0, 1, size=50)
    raw[:, 5] = 7.0  # constant column -> 0
    out, mins, maxs = oracle.ss_preprocess(raw)
    for j in range(oracle.NFEAT):
        t = np.log1p(raw[:, j]) if oracle._ss().or_ss_feature_kind(j) == 0 else np.sqrt(raw[:, j])
        assert mins[j] == t.min() and maxs[j] == t.max()
        if t.max() > t.min():
            assert np.allclose(out[:, j], (t - t.min()) / (t.max() - t.min()), rtol=0, atol=1e-15)
            assert out[:, j].min() == 0.0 and out[:, j].max() == 1.0
        else:
            assert (out[:, j] == 0).all()
    kinds = [oracle._ss().or_ss_feature_kind(j) for j in range(oracle.NFEAT)]
    fracs = [oracle.TABLE1[j] for j in range(oracle.NFEAT) if kinds[j] == 1]
    assert fracs == ["nnz_frac", "hyb_ell_frac", "dia_frac", "ell_frac"]


def test_pca_against_numpy_eigh():
    rng = np.random.default_rng(1)
    d, n = oracle.NFEAT, 400
    A = rng.normal(size=(d, d))
    X = rng.normal(size=(n, d)) @ A  # anisotropic cloud
    mean, basis, ev = oracle.ss_pca(X, 8)
    C = np.cov(X.T, bias=True)
    w, V = np.linalg.eigh(C)
    w, V = w[::-1], V[:, ::-1]
    assert np.allclose(mean, X.mean(0), atol=1e-12)
    assert np.allclose(ev, w[:8], rtol=1e-10)
    for c in range(8):
        cosang = abs(np.dot(basis[c], V[:, c]))
        assert cosang == pytest.approx(1.0, abs=1e-9)
        big = np.argmax(np.abs(basis[c]))
        assert basis[c][big] > 0  # sign convention (F3)
    assert np.allclose(basis @ basis.T, np.eye(8), atol=1e-12)
    Y = oracle.ss_project(X, mean, basis)
    assert np.allclose(Y, (X - mean) @ basis.T, atol=1e-10)


def test_pca_recovers_a_line():
    rng = np.random.default_rng(2)
    u = rng.normal(size=oracle.NFEAT)
    u /= np.linalg.norm(u)
    t = rng.normal(size=300)
    X = np.outer(t, u) * 10 + rng.normal(scale=1e-3, size=(300, oracle.NFEAT))
    mean, basis, ev = oracle.ss_pca(X, 8)
    assert abs(np.dot(basis[0], u)) > 0.999999
    assert ev[0] > 1e6 * ev[1]


def test_kmeans_against_sklearn():
    from sklearn.cluster import KMeans
    rng = np.random.default_rng(3)
    centers = rng.uniform(-10, 10, size=(6, 8))
    Y = np.concatenate([c + rng.normal(scale=0.5, size=(40, 8)) for c in centers])
    perm = rng.permutation(len(Y))
    Y = Y[perm]
    init = np.array([int(np.nonzero(perm == 40 * b)[0][0]) for b in range(6)], np.int32)  # one point per blob
    cent, assign, it = oracle.ss_kmeans(Y, init, max_iter=100)
    km = KMeans(n_clusters=6, init=Y[init], n_init=1, algorithm="lloyd", max_iter=100, tol=0.0).fit(Y)
    assert (km.labels_ == assign).all()
    assert np.allclose(km.cluster_centers_, cent, atol=1e-12)
    truth = perm // 40
    for b in range(6):
        assert len(set(assign[truth == b].tolist())) == 1  # blobs recovered
    assert it < 100
    # assignment = nearest centroid, ties to the lowest id
    tie = oracle.ss_assign(np.zeros((1, 8)), np.stack([np.ones(8), -np.ones(8)]))
    assert tie[0] == 0


FRACTIONS = {"nnz_frac", "hyb_ell_frac", "dia_frac", "ell_frac"}  # F1: sqrt; every other Table-1 feature log1p


def _np_transform(raw):
    """F1 written independently from the reading: sqrt for the four fractions, log1p otherwise."""
    out = np.empty_like(raw)
    for j, name in enumerate(oracle.TABLE1):
        out[:, j] = np.sqrt(raw[:, j]) if name in FRACTIONS else np.log1p(raw[:, j])
    return out


def _np_corpus(rng, n):
    """Table-1-shaped rows: counts / sizes spanning decades, fractions in (0, 1]."""
    raw = np.exp(rng.uniform(0, 14, size=(n, oracle.NFEAT)))
    for j, name in enumerate(oracle.TABLE1):
        if name in FRACTIONS:
            raw[:, j] = rng.uniform(1e-6, 1.0, size=n)
    return raw


def test_scale_against_numpy():
    """or_ss_scale (the prediction path's scaling, F2): queries transformed, then mapped with
    the TRAINING ranges, unclipped (queries may leave [0, 1]); a constant training column maps to 0."""
    rng = np.random.default_rng(11)
    train = _np_corpus(rng, 120)
    train[:, 4] = 3.0  # constant column
    q = _np_corpus(rng, 40)
    q[:3] *= 50.0  # beyond the training range
    X, mins, maxs = oracle.ss_preprocess(train)
    t = _np_transform(train)
    # numpy's log1p may differ from the C library's by an ulp: compare to 1e-15 relative
    assert np.allclose(mins, t.min(0), rtol=1e-15, atol=0) and np.allclose(maxs, t.max(0), rtol=1e-15, atol=0)
    got = oracle.ss_scale(q, mins, maxs)
    tq = _np_transform(q)
    rng_ = t.max(0) - t.min(0)
    want = np.where(rng_ > 0, (tq - t.min(0)) / np.where(rng_ > 0, rng_, 1.0), 0.0)
    assert np.allclose(got, want, rtol=1e-13, atol=1e-13)
    assert (got[:, 4] == 0).all()
    assert got.max() > 1.0  # unclipped
    # the training rows themselves map onto ss_preprocess's output
    assert np.allclose(oracle.ss_scale(train, mins, maxs), X, rtol=0, atol=1e-15)


def test_predict_against_numpy():
    """ss_predict (a new matrix gets its nearest centroid's cluster): numpy recomputes scale ->
    centre -> project on the fitted basis -> argmin squared distance (first index on ties) from the fit's
    parameters; the oracle's cluster ids match wherever the two nearest centroids are not within
    rounding of each other."""
    rng = np.random.default_rng(12)
    train = _np_corpus(rng, 300)
    q = _np_corpus(rng, 200)
    init = rng.choice(300, size=12, replace=False).astype(np.int32)
    fit = oracle.ss_fit(train, init, pcs=8)
    X = oracle.ss_scale(q, fit["mins"], fit["maxs"])
    Y = (X - fit["mean"]) @ fit["basis"].T
    d2 = ((Y[:, None, :] - fit["centroids"][None, :, :]) ** 2).sum(-1)
    want = np.argmin(d2, axis=1)
    srt = np.sort(d2, axis=1)
    clear = srt[:, 1] - srt[:, 0] > 1e-9 * (1 + srt[:, 0])
    got = oracle.ss_predict(fit, q)
    assert clear.sum() > 190
    assert (got[clear] == want[clear]).all()
    # the fitted training assignment is the same rule applied to the training rows
    Yt = (oracle.ss_scale(train, fit["mins"], fit["maxs"]) - fit["mean"]) @ fit["basis"].T
    d2t = ((Yt[:, None, :] - fit["centroids"][None, :, :]) ** 2).sum(-1)
    assert (np.argmin(d2t, axis=1) == fit["assign"]).mean() > 0.99
