"""GPU tests of the race harness beyond parity: the per-matrix race mask ("benchmark only
one matrix from each cluster", §4), the allocator hook (SURVEY §8(b) ownership:
library buffers from torch's caching allocator) and the binding's placement checks."""
import numpy as np
import pytest

import oracle
import paper_conf_icppw_dhandhaniadpbl21_b200 as sfs
import sfsgen
from gpu_util import assert_features_equal, check_spmv, to_dev

pytestmark = pytest.mark.gpu


def _mats():
    return {
        "laplace64": sfsgen.laplace2d(64),
        "band": sfsgen.generate(sfsgen.make_spec(sfsgen.BAND, seed=3, m=20011, ia=9, pa=0.7)),
        "uniform": sfsgen.generate(sfsgen.make_spec(sfsgen.UNIFORM, seed=5, m=12000, n=9000, pa=17.0)),
        "powerlaw32": sfsgen.generate(sfsgen.make_spec(sfsgen.POWERLAW, seed=6, m=30000, pa=2.15, dtype=sfsgen.F32)),
        "rmat14": sfsgen.rmat(14, seed=7),
    }


def test_race_mask_features_only_launches_no_spmv():
    """A matrix with race mask 0 is featurised (bit-exact) and nothing else: no conversion, no SpMV.
    Launch accounting: the launches of a masked corpus are the sum of the per-matrix feature passes, and
    racing one matrix adds exactly what racing it alone adds."""
    import torch
    A = _mats()
    names = list(A)
    mats = [to_dev(A[k]) for k in names]
    opts = sfs.default_opts(reps=4, warmup=1)

    def count(ms, mask):
        torch.cuda.synchronize()
        c0 = sfs.launch_count()
        out = sfs.label_corpus(ms, opts, race_mask=mask)
        torch.cuda.synchronize()
        return sfs.launch_count() - c0, out

    n0, (feats, labs) = count(mats, [0] * len(mats))
    for k, f, L in zip(names, feats, labs):
        assert_features_equal(f, oracle.features(A[k].m, A[k].n, A[k].rp, A[k].col), k)
        assert L["matrix_status"] == 0 and L["label"] == -1
        assert all(s == sfs.ERR_NOT_RUN for s in L["status"]) and all(t == 0 for t in L["t_spmv_us"])
    singles = [count([m], [0])[0] for m in mats]
    assert n0 == sum(singles), (n0, singles)
    # race only matrix 0 (all formats) and matrix 2 (CSR + COO)
    mask = [0x1F, 0, 0x03, 0, 0]
    n1, (_, labs1) = count(mats, mask)
    r0 = count([mats[0]], [0x1F])[0] - singles[0]
    r2 = count([mats[2]], [0x03])[0] - singles[2]
    assert n1 == n0 + r0 + r2
    for j, L in enumerate(labs1):
        ran = [f for f in range(5) if L["status"][f] == 0]
        adm = L["admissible_mask"]
        assert ran == [f for f in range(5) if (mask[j] >> f) & 1 and (adm >> f) & 1]
        assert (L["label"] >= 0) == bool(ran)


def test_race_mask_representative_labels_match_full_race():
    """Racing a subset gives the subset the same statuses as a full race, and the same label wherever the
    full race has a clear winner (>= 15 % ahead of the runner-up: the label is a timing result)."""
    A = _mats()
    mats = [to_dev(A[k]) for k in A]
    opts = sfs.default_opts(reps=50, warmup=5)
    _, full = sfs.label_corpus(mats, opts)
    mask = [0x1F if j % 2 == 0 else 0 for j in range(len(mats))]
    _, sub = sfs.label_corpus(mats, opts, race_mask=mask)
    for j, (Lf, Ls) in enumerate(zip(full, sub)):
        if not mask[j]:
            assert Ls["label"] == -1
            continue
        assert Ls["status"] == Lf["status"]
        t = sorted(v for f, v in enumerate(Lf["t_spmv_us"]) if Lf["status"][f] == 0)
        if len(t) > 1 and t[1] > 1.15 * t[0]:
            assert Ls["label"] == Lf["label"], (j, Lf["t_spmv_us"], Ls["t_spmv_us"])


def test_torch_allocator_hook_owns_library_buffers():
    """With the hook on, a converted matrix's buffers are torch caching-allocator blocks (memory_allocated
    grows by at least the handle's bytes and drops back after sfs_matrix_free); results are identical to the
    library's own pool."""
    import torch
    A = _mats()["band"]
    x = sfsgen.vector(11, A.n)
    dA = to_dev(A)
    was = sfs.torch_allocator_enabled()
    sfs.use_torch_allocator(True)
    torch.cuda.synchronize()
    before = torch.cuda.memory_allocated()
    M = sfs.convert(dA, sfs.ELL)
    torch.cuda.synchronize()
    grew = torch.cuda.memory_allocated() - before
    assert grew >= M.layout().bytes > 0
    y_hook = check_spmv(A, sfs.ELL, M, x, sfs.F64, "torch allocator")
    M.free()
    torch.cuda.synchronize()
    assert torch.cuda.memory_allocated() == before
    sfs.use_torch_allocator(False)
    try:
        M2 = sfs.convert(dA, sfs.ELL)
        y_pool = check_spmv(A, sfs.ELL, M2, x, sfs.F64, "library pool")
        M2.free()
    finally:
        sfs.use_torch_allocator(was)
    assert np.array_equal(y_hook, y_pool)
    # a handle keeps the allocator it was built with: built under the hook, freed after the hook is off
    sfs.use_torch_allocator(True)
    M3 = sfs.convert(dA, sfs.COO)
    sfs.use_torch_allocator(False)
    torch.cuda.synchronize()
    held = torch.cuda.memory_allocated()
    M3.free()
    torch.cuda.synchronize()
    assert torch.cuda.memory_allocated() < held  # returned to torch's pool, not to the library's
    sfs.use_torch_allocator(was)


def test_torch_allocator_host_inputs_cross_stream():
    """Host inputs are staged on the copy stream and freed on the compute stream: the hook orders the
    reuse; two back-to-back calls give identical features and statuses."""
    import torch
    A = _mats()
    pin = lambda a: torch.from_numpy(np.ascontiguousarray(a)).pin_memory()
    hm = [sfs.Csr(B.m, B.n, pin(B.rp), pin(B.col), pin(B.val)) for B in A.values()]
    opts = sfs.default_opts(reps=3, warmup=1)
    was = sfs.torch_allocator_enabled()
    sfs.use_torch_allocator(True)
    try:
        f1, l1 = sfs.label_corpus(hm, opts)
        f2, l2 = sfs.label_corpus(hm, opts)
    finally:
        sfs.use_torch_allocator(was)
    for k, a, b, L1, L2 in zip(A, f1, f2, l1, l2):
        assert_features_equal(a, oracle.features(A[k].m, A[k].n, A[k].rp, A[k].col), k)
        assert_features_equal(b, a, k)
        assert L1["status"] == L2["status"] and L1["matrix_status"] == 0


def test_mixed_placement_rejected():
    import torch
    A = _mats()["laplace64"]
    d = lambda a: torch.from_numpy(a).cuda()
    h = lambda a: torch.from_numpy(a)
    with pytest.raises(sfs.SfsError):
        sfs.features(sfs.Csr(A.m, A.n, d(A.rp), h(A.col), d(A.val)))
    with pytest.raises(sfs.SfsError):
        sfs.features(sfs.Csr(A.m, A.n, h(A.rp).pin_memory(), h(A.col).pin_memory(), d(A.val)))
    with pytest.raises(sfs.SfsError):  # pageable host memory
        sfs.features(sfs.Csr(A.m, A.n, h(A.rp), h(A.col), h(A.val)))


def test_subset_labelling_races_only_representatives():
    """f2 end to end: one representative per cluster is raced, every other matrix
    is featurised only; the predicted labels of the representatives are their own race labels when their
    cluster holds no other representative; the f4 scores are within their ranges."""
    from paper_conf_icppw_dhandhaniadpbl21_b200 import predictor as pr
    rng = np.random.default_rng(9)
    mats, hosts = [], []
    for i in range(24):
        cls = [sfsgen.BAND, sfsgen.UNIFORM, sfsgen.BLOCKDIAG, sfsgen.POWERLAW][i % 4]
        pa = 0.8 if cls in (sfsgen.BAND, sfsgen.BLOCKDIAG) else (12.0 if cls == sfsgen.UNIFORM else 2.4)
        A = sfsgen.generate(sfsgen.make_spec(cls, seed=100 + i, m=int(rng.integers(3000, 20000)), ia=6, pa=pa))
        hosts.append(A)
        mats.append(to_dev(A))
    opts = sfs.default_opts(reps=20, warmup=2)
    _, full = sfs.label_corpus(mats, opts)
    r = pr.subset_labelling(mats, opts, nc=6, k=1, truth=full)
    assert r["raced"] <= 6 and r["others_not_raced"]
    assert len(r["pred"]) == 24 and all(0 <= p < 5 for p in r["pred"])
    q = r["quality"]
    assert 0 < q["GT"] <= 1.0 and q["CSR"] > 0 and 0 <= q["Threshold"] <= 24 and 0 <= q["accuracy"] <= 1
    assert r["t_subset_race_s"] > 0 and r["t_features_s"] > 0
