#!/usr/bin/env python
"""configs[3]: 3D 27-point stencil on 128^3 row-partitioned over N GPUs: an NCCL all-gather of x, or
(--exchange halo) NCCL send/recv of the ghost planes only, or (--exchange push) the
ghost rows stored into the neighbours' x by the SpMV kernel itself over symmetric memory (sfs_spmv_push).

    python -m torch.distributed.run --nproc-per-node N --master-addr 127.0.0.1 tools/bench_rowpart.py

Each rank holds rows [r_k, r_{k+1}) (equal blocks, global column ids) converted to --fmt by
sfs_convert; one iteration = all_gather_into_tensor(x_full, x_local) + sfs_spmv(A_k, x_full, y_local)
(+ y becomes the next x).  Reports per-iteration time (max over ranks, CUDA events), the all-gather
and SpMV parts measured separately, and the aggregate effective GB/s (sum of the ranks' algorithmic
SpMV bytes / iteration time).
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--N", type=int, default=128)
    ap.add_argument("--fmt", default="DIA")
    ap.add_argument("--dtype", default="f64")
    ap.add_argument("--iters", type=int, default=100)
    ap.add_argument("--warmup", type=int, default=10)
    ap.add_argument("--exchange", default="allgather", choices=["allgather", "halo", "push"])
    ap.add_argument("--backend", default="nccl")
    args = ap.parse_args()

    import torch
    import torch.distributed as dist

    import paper_conf_icppw_dhandhaniadpbl21_b200 as sfs
    import sfsgen
    from paper_conf_icppw_dhandhaniadpbl21_b200 import dist as sd

    rank, world, local = int(os.environ.get("RANK", 0)), int(os.environ.get("WORLD_SIZE", 1)), int(
        os.environ.get("LOCAL_RANK", 0))
    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group(args.backend, device_id=torch.device("cuda", local) if args.backend == "nccl" else None)
    dt = sfsgen.F64 if args.dtype == "f64" else sfsgen.F32
    A = sfsgen.stencil3d27(args.N, dtype=dt)
    part = sd.RowPartition(A.m, A.n, world, rank)
    b = part.bounds
    rp, col, val = sd.slice_rows(A.rp, A.col, A.val, b[rank], b[rank + 1])
    t = lambda a: torch.from_numpy(a).cuda()
    halo = args.exchange in ("halo", "push")
    plan = sd.halo_plan(part, col, device=torch.device("cuda", local)) if halo else None
    Ak = sfs.Csr(part.local_rows, plan.n_ext if halo else A.n, t(rp), t(plan.col_ext if halo else col), t(val))
    fmt = sfs.FORMAT_NAMES.index(args.fmt)
    M = sfs.convert(Ak, fmt)
    feats = sfs.features(Ak)
    nbytes = sfs.spmv_bytes(feats, fmt, dt)
    xs = torch.from_numpy(sfsgen.vector(5, A.n, dt)).cuda()
    x_local = xs[b[rank]:b[rank + 1]].clone()
    spmv = lambda xf, yl: sfs.spmv(fmt, M, xf, yl)
    push_t = {}
    if args.exchange == "push":
        iterate = lambda it: sd.rowpart_push_iterate(plan, M, fmt, x_local, it, timing=push_t)
    elif halo:
        iterate = lambda it: sd.rowpart_halo_iterate(plan, spmv, sfs.gather, x_local, iters=it)
    else:
        iterate = lambda it: sd.rowpart_spmv_iterate(part, spmv, x_local, iters=it)
    iterate(args.warmup)

    def timed(fn):
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        fn()
        e1.record()
        torch.cuda.synchronize()
        v = torch.tensor([e0.elapsed_time(e1) / 1000.0], device="cuda")
        if world > 1:
            dist.all_reduce(v, op=dist.ReduceOp.MAX)
        return float(v.item())

    t_iter = timed(lambda: iterate(args.iters)) / args.iters
    if args.exchange == "push":  # the iteration loop alone (symmetric-memory setup excluded), max over ranks
        v = torch.tensor([push_t["ms_per_iter"] / 1000.0], device="cuda")
        if world > 1:
            dist.all_reduce(v, op=dist.ReduceOp.MAX)
        t_iter = float(v.item())
    blk = part.block
    xp = torch.zeros(blk, dtype=xs.dtype, device="cuda")
    xf = torch.empty(blk * world, dtype=xs.dtype, device="cuda")
    yl = torch.empty(part.local_rows, dtype=xs.dtype, device="cuda")

    def ag():
        for _ in range(args.iters):
            if world > 1:
                dist.all_gather_into_tensor(xf, xp)
            else:
                xf.copy_(xp)

    xm = torch.zeros(plan.n_ext, dtype=xs.dtype, device="cuda") if halo else xs

    def mv():
        for _ in range(args.iters):
            spmv(xm, yl)

    t_ag = timed(ag) / args.iters if (world == 1 or args.backend == "nccl") else float("nan")
    t_mv = timed(mv) / args.iters
    tot_bytes = torch.tensor([float(nbytes)], device="cuda")
    if world > 1:
        dist.all_reduce(tot_bytes)
    if rank == 0:
        print(json.dumps({"config": f"configs[3] 3D27 {args.N}^3 {args.dtype} row-partitioned", "n_gpus": world,
                          "format": args.fmt, "exchange": args.exchange, "t_iter_us": t_iter * 1e6,
                          "t_allgather_us": t_ag * 1e6,
                          "halo_recv_entries_rank0": plan.recv_count if halo else None,
                          "t_spmv_us": t_mv * 1e6, "agg_spmv_gbs": float(tot_bytes.item()) / t_iter / 1e9,
                          "rows_per_rank": part.block}))
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
