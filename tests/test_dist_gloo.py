"""N > 1 host logic on CPU: world_size-2 gloo process groups (no GPU).  The labeller / local SpMV are
test doubles backed by the oracle; on a GPU box they are sfs.label_corpus / sfs.spmv."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_icppw_dhandhaniadpbl21_b200 import dist as sd


def test_lpt_assign():
    costs = [5, 1, 9, 3, 3, 7, 2]
    sh = sd.lpt_assign(costs, 3)
    assert sorted(sum(sh, [])) == list(range(7))
    loads = [sum(costs[i] for i in s) for s in sh]
    assert max(loads) - min(loads) <= max(costs)
    assert sd.lpt_assign(costs, 3) == sh  # deterministic
    assert sd.lpt_assign([1.0] * 4, 1) == [[0, 1, 2, 3]]
    assert sd.lpt_assign([], 2) == [[], []]


def test_row_blocks():
    assert sd.row_blocks(10, 4) == [0, 3, 6, 9, 10]
    assert sd.row_blocks(8, 8) == list(range(9))
    assert sd.row_blocks(3, 4) == [0, 1, 2, 3, 3]


def test_pack_roundtrip():
    import paper_conf_icppw_dhandhaniadpbl21_b200 as sfs
    feat = {k: i for i, k in enumerate(sfs.FEATURE_INT_FIELDS)}
    feat.update({k: 0.5 + i for i, k in enumerate(sfs.FEATURE_FLOAT_FIELDS)})
    lab = {"label": 3, "matrix_status": 0, "admissible_mask": 31, "csr_variant": 1, "t_spmv_us": [1, 2, 3, 4, 5],
           "t_convert_us": [0, 1, 1, 1, 1], "status": [0, 0, -3, 0, -7], "t_features_us": 9.0}
    r = sd.unpack_result(sd.pack_result(42, feat, lab))
    assert r["id"] == 42 and r["label"] == 3 and r["status"] == [0, 0, -3, 0, -7]
    assert all(r["features"][k] == feat[k] for k in feat)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _oracle_labeller(batch):
    import oracle
    feats, labs = [], []
    for (A, x) in batch:
        lab, f, ts, tc = oracle.label_matrix(A.m, A.n, A.rp, A.col, A.val.astype(np.float64), x, reps=1)
        f = dict(f)
        f["csr_variant"] = 0
        feats.append(f)
        labs.append({"label": lab, "matrix_status": 0, "admissible_mask": f["admissible_mask"], "csr_variant": 0,
                     "t_spmv_us": list(ts * 1e6), "t_convert_us": list(tc * 1e6),
                     "status": [0 if (f["admissible_mask"] >> k) & 1 else -3 for k in range(5)],
                     "t_features_us": 0.0})
    return feats, labs


def _make(i):
    import sfsgen
    s = sfsgen.make_spec(sfsgen.UNIFORM if i % 2 else sfsgen.BAND, seed=i + 1, m=300 + 37 * i, ia=3, pa=5.0)
    A = sfsgen.generate(s)
    return (A, sfsgen.vector(i, A.n))


def _worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        ids = list(range(9))
        costs = [float(_make(i)[0].nnz) for i in ids]
        res = sd.label_corpus_sharded(ids, costs, _make, _oracle_labeller, rank, world, batch_bytes=2e4,
                                      nbytes=lambda t: t[0].nbytes())
        # row partition of one square matrix, 3 power-iteration steps
        import oracle
        import sfsgen
        A = sfsgen.generate(sfsgen.make_spec(sfsgen.ST2D5, ia=13))
        part = sd.RowPartition(A.m, A.n, world, rank)
        b = part.bounds
        rp, col, val = sd.slice_rows(A.rp, A.col, A.val, b[rank], b[rank + 1])

        def local_spmv(xf, y):
            yy, _ = oracle.spmv_csr(len(rp) - 1, A.n, rp, col, val, xf.numpy())
            y.copy_(torch.from_numpy(yy))

        x = torch.from_numpy(sfsgen.vector(5, A.n))
        y = sd.rowpart_spmv_iterate(part, local_spmv, x[b[rank]:b[rank + 1]].clone(), iters=3)
        q.put((rank, [(r["id"], r["label"], r["features"]["nnz"]) for r in res], y.numpy()))
    except Exception as e:  # surface worker failures immediately
        import traceback
        q.put((rank, "ERROR", traceback.format_exc()))
        raise
    finally:
        dist.destroy_process_group()


def test_gloo_world2_corpus_and_rowpartition():
    import oracle
    import sfsgen
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    out = [q.get(timeout=240) for _ in range(world)]
    for o in out:
        assert o[1] != "ERROR", o[2]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    out.sort()
    (r0, res0, y0), (r1, res1, y1) = out
    assert res0 == res1  # every rank holds the whole corpus result
    assert [i for i, _, _ in res0] == list(range(9))
    for i, lab, nnz in res0:
        assert nnz == _make(i)[0].nnz and 0 <= lab < 5
    # row-partitioned power iteration == global oracle SpMV iterated
    A = sfsgen.generate(sfsgen.make_spec(sfsgen.ST2D5, ia=13))
    x = sfsgen.vector(5, A.n)
    for _ in range(3):
        x, _ = oracle.spmv_csr(A.m, A.n, A.rp, A.col, A.val, x)
    y = np.concatenate([y0, y1])
    assert np.allclose(y, x, rtol=1e-12, atol=0)


def test_weak_shard_balanced():
    """bench.py's weak scaling: the first 200·N corpus matrices, each exactly once over the ranks, with
    estimated race costs within 2 % of each other (LPT), and N = 1 the configs[1] ids in order."""
    import sfsgen
    assert sd.weak_shard(200, 200, 0, 1) == list(range(200))
    w = 4
    sh = [sd.weak_shard(200, 50, r, w) for r in range(w)]
    assert sorted(sum(sh, [])) == list(range(200))
    loads = [sum(sd.race_cost(sfsgen.corpus_spec(200, i)) for i in s) for s in sh]
    assert max(loads) / min(loads) < 1.02


def test_expected_nnz_tracks_generator():
    """The scheduling estimate is within ±25 % of the generated nnz for each corpus class."""
    import sfsgen
    for i in range(8):  # two of each class, small sizes only
        sp = sfsgen.corpus_spec(200, i)
        if sp.m > 200000:
            continue
        est, act = sd.expected_nnz(sp), sfsgen.generate(sp).nnz
        assert 0.75 * act <= est <= 1.25 * act, (i, est, act)


def _halo_case(kind):
    import sfsgen
    from helpers import random_csr
    if kind == "stencil":
        return sfsgen.stencil3d27(12)
    rng = np.random.default_rng(9)
    return random_csr(rng, 1500, 1500, 0.01, empty_rows=0.1, dense_rows=1)


@pytest.mark.parametrize("kind", ["stencil", "random"])
@pytest.mark.parametrize("world", [1, 3, 4])
def test_halo_plans_reproduce_the_row_blocks(kind, world):
    """Every rank's renumbered block applied to x_ext = [x[lo] | own slice | x[hi]] gives its rows of A·x
    exactly as the global-column block does; rank j sends rank k exactly the ghosts k receives from j;
    a stencil block keeps its diagonals (contiguous ghost runs keep offsets)."""
    import oracle
    A = _halo_case(kind)
    x = np.random.default_rng(1).uniform(-1, 1, A.n)
    blocks = []
    for k in range(world):
        b = sd.row_blocks(A.m, world)
        blocks.append(sd.slice_rows(A.rp, A.col, A.val, b[k], b[k + 1]))
    plans = sd.halo_plans_local(A.m, A.n, world, [c for _, c, _ in blocks])
    yg, _ = oracle.spmv_csr(A.m, A.n, A.rp, A.col, A.val, x)
    for k, (P, (rp, col, val)) in enumerate(zip(plans, blocks)):
        xe = np.concatenate([x[P.lo], x[P.r0:P.r1], x[P.hi]])
        assert P.n_ext == len(xe) and P.col_ext.max(initial=-1) < P.n_ext and P.col_ext.min(initial=0) >= 0
        y, _ = oracle.spmv_csr(len(rp) - 1, P.n_ext, rp, P.col_ext, val, xe)
        assert np.array_equal(y, yg[P.r0:P.r1])  # same entries in the same order: bitwise
        for j, o, c in P.recv:  # what k receives from j is what j packs for k
            Q = plans[j]
            so = [(oo, cc) for d, oo, cc in Q.send if d == k]
            assert len(so) == 1 and so[0][1] == c
            got = Q.send_idx[so[0][0]:so[0][0] + c] + Q.r0
            want = np.concatenate([P.lo, P.hi])[o - (0 if o < P.n_lo else P.n_local):][:c]
            assert np.array_equal(got, want)
        if kind == "stencil":
            d_glob = np.unique(col.astype(np.int64) - np.repeat(np.arange(P.r0, P.r1), np.diff(rp)))
            d_ext = np.unique(P.col_ext.astype(np.int64) - P.n_lo - np.repeat(np.arange(P.n_local), np.diff(rp)))
            assert np.array_equal(d_glob, d_ext)


def _halo_worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import oracle
        A = _halo_case("stencil")
        part = sd.RowPartition(A.m, A.n, world, rank)
        b = part.bounds
        rp, col, val = sd.slice_rows(A.rp, A.col, A.val, b[rank], b[rank + 1])
        plan = sd.halo_plan(part, col)  # collective: all_to_all of the requests

        def local_spmv(xe, y):
            yy, _ = oracle.spmv_csr(len(rp) - 1, plan.n_ext, rp, plan.col_ext, val, xe.numpy())
            y.copy_(torch.from_numpy(yy))

        def gather(src, idx, out):
            out.copy_(src[idx.long()])

        x = torch.from_numpy(np.random.default_rng(2).uniform(-1, 1, A.n))
        y = sd.rowpart_halo_iterate(plan, local_spmv, gather, x[b[rank]:b[rank + 1]].clone(), iters=3)
        dst_off = sd.exchange_recv_offsets(plan)  # collective: where this rank's pushes land
        q.put((rank, y.numpy().copy(), plan.recv_count, dst_off, sd.push_runs(plan, dst_off)))
    except Exception:
        import traceback
        q.put((rank, "ERROR", traceback.format_exc()))
        raise
    finally:
        dist.destroy_process_group()


def test_gloo_world2_halo_exchange_power_iteration():
    """Two ranks exchange only their ghost planes (batch_isend_irecv) and reproduce the global power
    iteration; each receives one 12^2 plane instead of half of x."""
    import oracle
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_halo_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    out = sorted([q.get(timeout=240) for _ in range(world)], key=lambda t: t[0])
    for o in out:
        assert not isinstance(o[1], str), o[2]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    A = _halo_case("stencil")
    x = np.random.default_rng(2).uniform(-1, 1, A.n)
    for _ in range(3):
        x, _ = oracle.spmv_csr(A.m, A.n, A.rp, A.col, A.val, x)
    assert np.array_equal(np.concatenate([out[0][1], out[1][1]]), x)
    assert out[0][2] == out[1][2] == 12 * 12
    # the push plan exchanged over gloo equals the one built from every rank's plan in one process
    blocks = [sd.slice_rows(A.rp, A.col, A.val, *sd.row_blocks(A.m, world)[k:k + 2]) for k in range(world)]
    plans = sd.halo_plans_local(A.m, A.n, world, [c for _, c, _ in blocks])
    offs = [sd.recv_offsets_by_source(P) for P in plans]
    for k in range(world):
        want = {j: offs[j][k] for j, _, _ in plans[k].send}
        assert out[k][3] == want
        assert out[k][4] == sd.push_runs(plans[k], want)
        assert len(out[k][4]) == 1  # one contiguous plane per neighbour


@pytest.mark.parametrize("kind", ["stencil", "random"])
@pytest.mark.parametrize("world", [2, 3, 5])
def test_push_runs_deliver_the_ghosts(kind, world):
    """The fused push (runs of own-slice rows stored into the neighbours' x_ext, include/sfs.h
    sfs_spmv_push) fills every rank's ghost region with exactly x[lo] and x[hi]: the same data the
    batch_isend_irecv exchange delivers; runs never overlap; a stencil needs one run per neighbour."""
    A = _halo_case(kind)
    x = np.random.default_rng(4).uniform(-1, 1, A.n)
    bnd = sd.row_blocks(A.m, world)
    blocks = [sd.slice_rows(A.rp, A.col, A.val, bnd[k], bnd[k + 1]) for k in range(world)]
    plans = sd.halo_plans_local(A.m, A.n, world, [c for _, c, _ in blocks])
    xs = []
    for P in plans:
        xe = np.full(P.n_ext, np.nan)
        xe[P.n_lo:P.n_lo + P.n_local] = x[P.r0:P.r1]
        xs.append(xe)
    sd.apply_push_host(plans, xs)
    offs = [sd.recv_offsets_by_source(P) for P in plans]
    for k, P in enumerate(plans):
        assert np.array_equal(xs[k], np.concatenate([x[P.lo], x[P.r0:P.r1], x[P.hi]]))
        runs = sd.push_runs(P, {j: offs[j][k] for j, _, _ in P.send})
        assert sum(e - b for _, b, e, _ in runs) == len(P.send_idx)
        for j, b, e, o in runs:
            assert 0 <= b < e <= P.n_local
        nb = sd.push_neighbours(P)
        assert set(j for j, _, _ in P.send) <= set(nb) and set(j for j, _, _ in P.recv) <= set(nb)
        if kind == "stencil":
            assert len(runs) == len(P.send) <= 2
            assert nb == [j for j in (k - 1, k + 1) if 0 <= j < world]


def test_push_struct_marshalling():
    """sfs_push_t as the binding fills it (host only): counts, runs, flag addresses and epochs; limits of
    include/sfs.h (SFS_MAX_PUSH runs, SFS_MAX_PEERS flags) are enforced before the C call."""
    import paper_conf_icppw_dhandhaniadpbl21_b200 as sfs
    p = sfs.push_struct([(0, 10, 0x1000), (90, 100, 0x2000)], [0x10, 0x14], 7, [0x30], 8, 0x40)
    assert p.nseg == 2 and (p.seg_begin[1], p.seg_end[1], p.seg_dst[1]) == (90, 100, 0x2000)
    assert p.nwait == 2 and p.wait_flag[1] == 0x14 and p.wait_value == 7
    assert p.nsig == 1 and p.sig_flag[0] == 0x30 and p.sig_value == 8 and p.counter == 0x40
    with pytest.raises(sfs.SfsError):
        sfs.push_struct([(i, i + 1, 0x1000) for i in range(sfs.MAX_PUSH + 1)], [], 0, [], 1, 0x40)
    with pytest.raises(sfs.SfsError):
        sfs.push_struct([], [0x10] * (sfs.MAX_PEERS + 1), 0, [], 1, 0x40)
    B = sd._PushBuffers(1000, 4, 8)  # x_ext double buffer, flags[world], counter: disjoint, in order
    assert B.x(0, 1) == 8000 and B.flag(0, 0) == 16000 and B.flag(0, 3) == 16012 and B.counter(0) == 16016
    assert B.nbytes >= 16020 and B.nbytes % 256 == 0
