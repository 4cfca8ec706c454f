"""Multi-GPU drivers on one GPU: the row partition (configs[3] shape) and the sharded corpus driver
with the real library (the N > 1 exchange is covered by the gloo tests)."""
import numpy as np
import pytest

import oracle
import paper_conf_icppw_dhandhaniadpbl21_b200 as sfs
import sfsgen
from gpu_util import TOL, to_dev
from paper_conf_icppw_dhandhaniadpbl21_b200 import dist as sd

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("world", [2, 4, 8])
@pytest.mark.parametrize("fmt", [sfs.CSR, sfs.DIA, sfs.ELL])
def test_row_partition_blocks_reassemble(world, fmt):
    """Each rank's row block (global column ids) through sfs_convert / sfs_spmv, x = the full vector
    (what all_gather_into_tensor delivers), blocks concatenated == oracle y within tolerance."""
    import torch
    A = sfsgen.generate(sfsgen.make_spec(sfsgen.ST3D27, ia=24))
    x = sfsgen.vector(11, A.n)
    xd = torch.from_numpy(x).cuda()
    ys = []
    for rank in range(world):
        part = sd.RowPartition(A.m, A.n, world, rank)
        b = part.bounds
        rp, col, val = sd.slice_rows(A.rp, A.col, A.val, b[rank], b[rank + 1])
        if part.local_rows == 0:
            continue
        t = lambda a: torch.from_numpy(a).cuda()
        Ak = sfs.Csr(part.local_rows, A.n, t(rp), t(col), t(val))
        M = sfs.convert(Ak, fmt)
        y = torch.empty(part.local_rows, dtype=torch.float64, device="cuda")
        sfs.spmv(fmt, M, xd, y)
        ys.append(y.cpu().numpy())
        M.free()
    y = np.concatenate(ys)
    yr, ay = oracle.spmv_csr(A.m, A.n, A.rp, A.col, A.val, x)
    assert np.all(np.abs(y - yr) <= TOL[sfs.F64] * ay)


def test_rowpart_iterate_single_rank_power_iteration():
    import torch
    A = sfsgen.generate(sfsgen.make_spec(sfsgen.ST2D5, ia=40))
    part = sd.RowPartition(A.m, A.n, 1, 0)
    t = lambda a: torch.from_numpy(a).cuda()
    M = sfs.convert(sfs.Csr(A.m, A.n, t(A.rp), t(A.col), t(A.val)), sfs.CSR)
    x0 = sfsgen.vector(3, A.n)
    y = sd.rowpart_spmv_iterate(part, lambda xf, yl: sfs.spmv(sfs.CSR, M, xf, yl), t(x0), iters=3)
    xr = x0
    for _ in range(3):
        xr, _ = oracle.spmv_csr(A.m, A.n, A.rp, A.col, A.val, xr)
    assert np.allclose(y.cpu().numpy(), xr, rtol=1e-11, atol=1e-12)


def test_sharded_corpus_driver_single_rank():
    import torch
    ids = list(range(6))

    def make(i):
        A = sfsgen.generate(sfsgen.make_spec(sfsgen.BAND if i % 2 else sfsgen.UNIFORM, seed=i + 3, m=2000 + 100 * i,
                                             ia=4, pa=9.0))
        t = lambda a: torch.from_numpy(a).cuda()
        return sfs.Csr(A.m, A.n, t(A.rp), t(A.col), t(A.val)), A

    cache = {}

    def mk(i):
        cache[i] = make(i)
        return cache[i][0]

    res = sd.label_corpus_sharded(ids, [1.0] * len(ids), mk, lambda b: sfs.label_corpus(b, sfs.default_opts(reps=5)),
                                  rank=0, world=1, batch_bytes=1e5, nbytes=lambda m: m.nbytes())
    assert [r["id"] for r in res] == ids
    for r in res:
        A = cache[r["id"]][1]
        fo = oracle.features(A.m, A.n, A.rp, A.col)
        assert r["features"]["nnz"] == fo["nnz"] and r["features"]["nnz_sig"] == fo["nnz_sig"]
        assert 0 <= r["label"] < 5 and r["matrix_status"] == 0


@pytest.mark.parametrize("scaling", ["strong", "weak"])
def test_bench_two_ranks_share_one_gpu(scaling):
    """bench.py's N > 1 path end to end (LPT shards of the identical corpus or weak shards, the timed result
    all-gather, max-over-ranks timing, summed launch counts, the configs[3]-shaped rowpart record at a small
    grid with its all-gather and push exchanges): torchrun with 2 ranks on this one GPU, gloo collectives."""
    import json
    import os
    import socket
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
           "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.join(root, "bench.py"),
           "--gpus", "2", "--steps", "1", "--warmup", "1", "--corpus", "6", "--e2e-steps", "1",
           "--no-cpu-baseline", "--dist-backend", "gloo", "--scaling", scaling, "--rowpart-N", "24",
           "--rowpart-iters", "5"]
    r = subprocess.run(cmd, cwd=root, capture_output=True, text=True, timeout=900)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, r.stdout[-2000:]
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["config"]["matrices_all_ranks"] == (6 if scaling == "strong" else 12)
    assert d["value"] > 0 and d["e2e"]["value"] > 0 and d["gpu_launches"] > 0
    assert d["scaling"] == scaling and d["config"]["gather_ok"]
    rp = d["rowpart"]
    assert "error" not in rp, rp
    for f in ("DIA", "CSR"):
        r = rp["formats"][f]
        assert r["allgather"]["t_iter_us"] > 0 and r["t_spmv_only_us"] > 0 and r["t_spmv_full_matrix_1gpu_us"] > 0
        assert r["push"].get("t_iter_us", 0) > 0, r["push"]
        assert "skipped" in r["halo"]


def test_gather_kernel():
    import torch
    rng = np.random.default_rng(3)
    for dt in (np.float64, np.float32):
        src = rng.uniform(-1, 1, 100_003).astype(dt)
        idx = rng.integers(0, len(src), 77_777).astype(np.int32)
        s, i = torch.from_numpy(src).cuda(), torch.from_numpy(idx).cuda()
        out = torch.empty(len(idx), dtype=s.dtype, device="cuda")
        sfs.gather(s, i, out)
        assert np.array_equal(out.cpu().numpy(), src[idx])
    empty = torch.empty(0, dtype=torch.int32, device="cuda")
    sfs.gather(s, empty, torch.empty(0, dtype=s.dtype, device="cuda"))  # n = 0: no launch, OK


@pytest.mark.parametrize("world", [2, 4, 8])
@pytest.mark.parametrize("fmt", [sfs.CSR, sfs.DIA, sfs.ELL])
def test_halo_exchange_power_iteration_simulated(world, fmt):
    """SURVEY §8(f) f3 on one GPU: the P ranks' renumbered row blocks through sfs_convert / sfs_spmv, the
    send buffers packed by sfs_gather and the point-to-point exchange done by device copies between the
    simulated ranks; 3 power-iteration steps == the oracle's global iteration within tolerance.  DIA of
    a stencil block keeps its 27 diagonals after the renumbering."""
    import torch
    A = sfsgen.generate(sfsgen.make_spec(sfsgen.ST3D27, ia=24))
    x0 = sfsgen.vector(11, A.n)
    b = sd.row_blocks(A.m, world)
    blocks = [sd.slice_rows(A.rp, A.col, A.val, b[k], b[k + 1]) for k in range(world)]
    plans = sd.halo_plans_local(A.m, A.n, world, [c for _, c, _ in blocks])
    t = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
    mats, bufs = [], []
    for k, (P, (rp, _, val)) in enumerate(zip(plans, blocks)):
        Ak = sfs.Csr(P.n_local, P.n_ext, t(rp), t(P.col_ext), t(val))
        if fmt == sfs.DIA:
            assert sfs.features(Ak)["diagonals"] == 27
        mats.append(sfs.convert(Ak, fmt))
        xa = torch.zeros(P.n_ext, dtype=torch.float64, device="cuda")
        xa[P.n_lo:P.n_lo + P.n_local] = t(x0[P.r0:P.r1])
        bufs.append([xa, torch.zeros_like(xa), t(P.send_idx.astype(np.int32)),
                     torch.empty(len(P.send_idx), dtype=torch.float64, device="cuda")])

    def exchange(which):
        for k, P in enumerate(plans):
            src = bufs[k][which]
            sfs.gather(src[P.n_lo:P.n_lo + P.n_local], bufs[k][2], bufs[k][3])
        for k, P in enumerate(plans):  # k receives from j: j's send segment addressed to k
            for j, o, c in P.recv:
                Q = plans[j]
                (so,) = [oo for d, oo, cc in Q.send if d == k]
                bufs[k][which][o:o + c] = bufs[j][3][so:so + c]

    cur = 0
    exchange(cur)
    for _ in range(3):
        for k, P in enumerate(plans):
            sfs.spmv(fmt, mats[k], bufs[k][cur], bufs[k][1 - cur][P.n_lo:P.n_lo + P.n_local])
        exchange(1 - cur)
        cur = 1 - cur
    y = np.concatenate([bufs[k][cur][P.n_lo:P.n_lo + P.n_local].cpu().numpy() for k, P in enumerate(plans)])
    x = x0
    for _ in range(3):
        x, ax = oracle.spmv_csr(A.m, A.n, A.rp, A.col, A.val, x)
    assert np.all(np.abs(y - x) <= 1e-11 * (np.abs(x) + ax))
    for M in mats:
        M.free()


@pytest.mark.parametrize("world", [2, 4, 8])
@pytest.mark.parametrize("fmt,variant", [(4, -1), (2, -1), (0, 2), (0, 4), (1, -1), (3, -1)])
@pytest.mark.parametrize("dtype", ["f64", "f32"])
def test_push_fused_power_iteration_simulated(world, fmt, variant, dtype):
    """sfs_spmv_push on one GPU with P simulated ranks (include/sfs.h): the ghost rows are
    stored into the neighbours' next x_ext by the SpMV kernel itself (DIA, ELL, CSR stream) or by the
    push kernel after it (CSR tile, COO, HYB), with the wait / signal flags; 3 power-iteration steps ==
    the oracle's global iteration within tolerance; flags end at the last epoch, counters at 0."""
    import torch
    A = sfsgen.generate(sfsgen.make_spec(sfsgen.ST3D27, ia=24))
    if dtype == "f32":
        A = sfsgen.CSR(A.m, A.n, A.rp, A.col, A.val.astype(np.float32))
    x0 = sfsgen.vector(11, A.n, 0 if dtype == "f32" else 1)
    b = sd.row_blocks(A.m, world)
    blocks = [sd.slice_rows(A.rp, A.col, A.val, b[k], b[k + 1]) for k in range(world)]
    plans = sd.halo_plans_local(A.m, A.n, world, [c for _, c, _ in blocks])
    t = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
    opts = sfs.default_opts(csr_variant=variant)
    mats = []
    for P, (rp, _, val) in zip(plans, blocks):
        M = sfs.convert(sfs.Csr(P.n_local, P.n_ext, t(rp), t(P.col_ext), t(val)), fmt, opts)
        if fmt == sfs.CSR:
            assert M.layout().variant == variant
        mats.append(M)
    iters = 3
    ys, mem = sd.rowpart_push_iterate_local(plans, mats, fmt, [t(x0[P.r0:P.r1]) for P in plans], iters)
    y = np.concatenate([v.cpu().numpy().astype(np.float64) for v in ys])
    x = x0.astype(np.float64)
    for _ in range(iters):
        x, ax = oracle.spmv_csr(A.m, A.n, A.rp, A.col, A.val.astype(np.float64), x)
        if dtype == "f32":  # each step's y is rounded to fp32 before the next
            x = x.astype(np.float32).astype(np.float64)
    tol = 1e-11 if dtype == "f64" else 3e-5
    assert np.all(np.abs(y - x) <= tol * (np.abs(x) + ax))
    B = sd._PushBuffers(max(P.n_ext for P in plans), world, ys[0].element_size())
    for k, P in enumerate(plans):
        raw = mem[k].cpu().numpy()
        flags = raw[B.flag_off:B.flag_off + 4 * world].view(np.uint32)
        for j in sd.push_neighbours(P):
            assert flags[j] == iters + 1
        assert raw[B.counter_off:B.counter_off + 4].view(np.uint32)[0] == 0
    for M in mats:
        M.free()


def test_push_argument_errors():
    import torch
    A = sfsgen.laplace2d(16)
    M = sfs.convert(to_dev(A), sfs.DIA)
    x = torch.ones(A.n, dtype=torch.float64, device="cuda")
    y = torch.empty(A.m, dtype=torch.float64, device="cuda")
    cnt = torch.zeros(1, dtype=torch.int32, device="cuda")
    dst = torch.empty(8, dtype=torch.float64, device="cuda")
    ok = sfs.push_struct([(0, 8, dst.data_ptr())], [], 0, [], 1, cnt.data_ptr())
    sfs.spmv_push(sfs.DIA, M, x, y, ok)
    torch.cuda.synchronize()
    assert np.array_equal(dst.cpu().numpy(), y[:8].cpu().numpy()) and cnt.item() == 0
    bad = [sfs.push_struct([(0, A.m + 1, dst.data_ptr())], [], 0, [], 1, cnt.data_ptr()),   # run past the block
           sfs.push_struct([(0, 8, dst.data_ptr()), (4, 12, dst.data_ptr())], [], 0, [], 1, cnt.data_ptr()),
           sfs.push_struct([(0, 8, dst.data_ptr())], [], 0, [], 1, 0)]                        # no counter
    for p in bad:
        with pytest.raises(sfs.SfsError) as ei:
            sfs.spmv_push(sfs.DIA, M, x, y, p)
        assert ei.value.status == sfs.ERR_INVALID_ARG
    with pytest.raises(sfs.SfsError):
        sfs.spmv_push(sfs.CSR, M, x, y, ok)  # format mismatch
    M.free()


def test_push_two_processes_share_one_gpu():
    """The push-fused row partition across two real processes (tools/push_2proc.py under torchrun): x_ext
    buffers and flags in CUDA IPC memory mapped into the other process, each rank's fused SpMV kernel
    storing its ghost rows into the other's buffer and waiting on the other's flag (the two contexts
    time-slice the GPU, so the waits are real); DIA, ELL, CSR, COO == the oracle's 3-step iteration."""
    import os
    import socket
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
           "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.join(root, "tools", "push_2proc.py")]
    r = subprocess.run(cmd, cwd=root, capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, (r.stdout[-2000:], r.stderr[-3000:])
    assert r.stdout.count("matches the oracle") == 8, r.stdout[-2000:]


@pytest.mark.parametrize("exchange", ["allgather", "halo", "push"])
def test_bench_rowpart_tool_runs(exchange):
    """tools/bench_rowpart.py (configs[3] row partition) end to end at a small grid, one rank: every
    exchange path prints its JSON line."""
    import json
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    r = subprocess.run([sys.executable, os.path.join(root, "tools", "bench_rowpart.py"), "--N", "24", "--iters", "5",
                        "--warmup", "2", "--exchange", exchange, "--fmt", "DIA"], cwd=root, capture_output=True,
                       text=True, timeout=600)
    assert r.returncode == 0, r.stderr[-2000:]
    d = json.loads([l for l in r.stdout.splitlines() if l.startswith("{")][-1])
    assert d["exchange"] == exchange and d["t_iter_us"] > 0 and d["agg_spmv_gbs"] > 0


def test_bench_corpus2000_tool_runs():
    """tools/bench_corpus2000.py (configs[4]) on its first 6 matrices, one rank: every matrix labelled."""
    import json
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    r = subprocess.run([sys.executable, os.path.join(root, "tools", "bench_corpus2000.py"), "--limit", "6", "--reps",
                        "5"], cwd=root, capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, r.stderr[-2000:]
    d = json.loads([l for l in r.stdout.splitlines() if l.startswith("{")][-1])
    assert d["matrices"] == 6 and d["ok"] and d["value"] > 0
