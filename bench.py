#!/usr/bin/env python
"""bench.py — matrices labelled per second on the BASELINE configs[1] corpus (the headline metric).

One step = the whole hot path (SURVEY §8(a) a1–a15) over one batch: for every matrix of the
configs[1] corpus-200 (banded / uniform random / block-diagonal / power-law, 10K–1M rows, fp32 and
fp64 values) the Table-1 feature pass, every admissible conversion, the device-timed format race
(5 warm-up + 100 timed SpMVs per format) and the label, then the all-gather of every rank's
fixed-size result rows (inside the timed region).  At N GPUs the SAME 200 matrices are LPT-sharded
over the ranks on an estimated race cost (strong scaling: "Scaling = rate(P)/rate(1) on
the identical corpus and seeds"; --scaling weak gives every rank its own 200).  Inputs are resident in
HBM when the timed region starts (`value`); `e2e` repeats the step through the same C-ABI call with
pinned HOST buffers (H2D inside the call).  The `rowpart` record times BASELINE configs[3] (3D
27-point stencil, 128^3, fp64) row-partitioned over the N ranks with each exchange of SURVEY §8(e) 2 /
§8(f) f3 (NCCL all-gather of x, NCCL halo send/recv, push fused into the SpMV over peer memory).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]

`--impl reference` times the CPU oracle (the only reference that exists: the paper ships no code)
on the box's host cores, on a bounded sample of the same workload.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

# ncu hot-rep traffic of the race per format (tools/traffic_corpus.py); the newest round's file
TRAFFIC_JSON = next((p for p in (os.path.join(ROOT, "profiles", r, "traffic_corpus200.json") for r in ("r02", "r01"))
                     if os.path.exists(p)), os.path.join(ROOT, "profiles", "r01", "traffic_corpus200.json"))
METRIC = "matrices labelled/s (features + all-format conversion + 100-rep SpMV race + label), corpus-200"
UNIT = "matrices/s"
DAGGR_BYTES = 136  # device aggregate record copied back per matrix (internal.h DevAggr)
LABEL_BYTES = 4 * 4 + 5 * 4 * 3 + 5 * 8 + 4  # sfs_label_t


def parse():
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=3)
    p.add_argument("--warmup", type=int, default=3)
    p.add_argument("--impl", default="ours", choices=["ours", "reference"])
    p.add_argument("--corpus", type=int, default=200, help="matrices per rank (configs[1]: 200)")
    p.add_argument("--reps", type=int, default=100)
    p.add_argument("--race-warmup", type=int, default=5)
    p.add_argument("--graphs", action="store_true", help="capture the timed reps in CUDA graphs")
    p.add_argument("--e2e-steps", type=int, default=2)
    p.add_argument("--cpu-budget", type=float, default=15.0, help="seconds of oracle work for cpu_baseline")
    p.add_argument("--no-cpu-baseline", action="store_true")
    p.add_argument("--out", default=None, help="also append the JSON line to this file")
    p.add_argument("--dump", default=None, help="write per-matrix results of the last timed step (JSONL)")
    p.add_argument("--dist-backend", default="nccl", choices=["nccl", "gloo"],
                   help="gloo: host-side collectives, lets N ranks share one GPU (tests of the N > 1 path only)")
    p.add_argument("--scaling", default="strong", choices=["strong", "weak"],
                   help="strong: the identical corpus-200 sharded over the N ranks; weak: 200 matrices per rank")
    p.add_argument("--rowpart-N", type=int, default=128, help="configs[3] grid edge (0 = skip the rowpart record)")
    p.add_argument("--rowpart-iters", type=int, default=100)
    p.add_argument("--predictor-nc", type=int, default=20, help="clusters of the f2 subset-labelling record (0 = skip)")
    p.add_argument("--no-configs-record", dest="configs_record", action="store_false",
                   help="skip the configs[0] / configs[2] race record")
    return p.parse_args()


def dist_env():
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return rank, world, local


def corpus_ids(rank, per_rank, world=1, scaling="strong"):
    """strong: the first per_rank matrices of the configs[1] recipe (200: the whole corpus), LPT-sharded over
    the ranks on an estimated race cost (dist.race_cost; identical on every rank, no communication).
    weak: the first per_rank*world matrices, LPT-balanced so every rank gets ~per_rank (dist.weak_shard)."""
    import sfsgen
    from paper_conf_icppw_dhandhaniadpbl21_b200 import dist as sd
    if scaling == "weak":
        return sd.weak_shard(200, per_rank, rank, world)
    ids = list(range(per_rank))
    if world == 1:
        return ids
    return [ids[j] for j in sd.lpt_assign([sd.race_cost(sfsgen.corpus_spec(200, i)) for i in ids], world)[rank]]


def generate_host(ids):
    import sfsgen
    mats = []
    for i in ids:
        A = sfsgen.generate(sfsgen.corpus_spec(200, i))
        x = sfsgen.vector(sfsgen.corpus_spec(200, i).seed, A.n, A.dtype)
        mats.append((i, A, x))
    return mats


# ------------------------------------------------------------------ clocks (nvidia-smi during the timed region)
class ClockSampler:
    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, index):
        self.index = index
        self.proc = None
        self.lines = []

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", f"--id={self.index}", f"--query-gpu={self.Q}",
                                          "--format=csv,noheader,nounits", "-lms", "200"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self):
        if not self.proc:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        self.t.join(timeout=2)
        sm, mx, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            f = [v.strip() for v in ln.split(",")]
            if len(f) < 9:
                continue
            try:
                sm.append(float(f[1]))
                mx.append(float(f[2]))
            except ValueError:
                continue
            for nm, v in zip(names, f[5:9]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(sm)}


# ------------------------------------------------------------------ CPU oracle (cpu_baseline / reference arm)
def stratified(items, stride=9):
    """Corpus order interleaved with a stride (ids 0, 9, 18, ..., 1, 10, ...; 9 is coprime with the 4 classes
    of i mod 4): a bounded prefix spans the size range, the four classes and both value types of corpus-200
    instead of its first few matrices."""
    return [items[j] for r in range(stride) for j in range(r, len(items), stride)]


def oracle_sample(host_mats, budget_s, threads, reps_target=100, reps_cpu=3):
    """The oracle's whole labelling pass (features, every admissible conversion, `reps_cpu` timed SpMV reps
    per format, argmin) on the matrices in stratified order, `threads` matrices at a time (one thread
    each), dispatching until `budget_s` of wall time is spent.  Each matrix's time is its own measured
    wall time under that load, with the SpMV reps scaled to `reps_target` by its own measured per-rep
    times:  t_i = wall_i + (reps_target - reps_cpu) * sum_f t_spmv_f,i.
    Throughput = threads * done / sum_i t_i: the per-matrix times are MEASURED with `threads` jobs
    running concurrently (memory-bandwidth contention included); only a perfectly load-balanced long
    corpus is assumed.  Returns (matrices/s, done, threads, wall, nnz, per-matrix times in sample order)."""
    import oracle
    from concurrent.futures import ThreadPoolExecutor, FIRST_COMPLETED, wait

    t0 = time.perf_counter()
    done, nnz, tsum = 0, 0, 0.0
    order = stratified(host_mats)
    it = iter(enumerate(order))
    times = {}
    futs = set()

    def job(item):
        k, (_, A, x) = item
        w0 = time.perf_counter()
        _, _, ts, _ = oracle.label_matrix(A.m, A.n, A.rp, A.col, A.val.astype(np.float64), x.astype(np.float64),
                                          reps=reps_cpu)
        wall_i = time.perf_counter() - w0
        return k, A.nnz, wall_i + (reps_target - reps_cpu) * float(np.sum(ts))

    with ThreadPoolExecutor(max_workers=threads) as ex:
        for _ in range(threads):
            nxt = next(it, None)
            if nxt is None:
                break
            futs.add(ex.submit(job, nxt))
        while futs:
            fin, futs = wait(futs, return_when=FIRST_COMPLETED)
            for f in fin:
                k, z, ti = f.result()
                times[k] = ti
                nnz += z
                tsum += ti
                done += 1
            if time.perf_counter() - t0 < budget_s:
                for _ in range(len(fin)):
                    nxt = next(it, None)
                    if nxt is not None:
                        futs.add(ex.submit(job, nxt))
    wall = time.perf_counter() - t0
    return threads * done / tsum, done, threads, wall, nnz, [times[k] for k in sorted(times)]


def cpu_baseline_record(host_mats, budget_s, reps):
    """T = nproc (the reported value) and T = 1 (BASELINE.md CPU plan).  T = nproc as oracle_sample says.
    T = 1: the first matrices of the same stratified order, one job alone on the machine; its rate is put on
    the T = nproc sample by the measured ratio of single-job to under-load per-matrix times on the matrices
    both runs labelled (so both figures describe the same sample)."""
    nproc = os.cpu_count() or 1
    v, d, c, w, nnz, tn = oracle_sample(host_mats, budget_s, nproc, reps_target=reps)
    _, d1, _, w1, nnz1, t1 = oracle_sample(host_mats, max(3.0, budget_s / 3), 1, reps_target=reps)
    common = min(d1, len(tn))
    r = sum(t1[:common]) / sum(tn[:common]) if common else float("nan")  # single-job / under-load time
    v1 = (len(tn) / (r * sum(tn))) if common else None
    sample = (f"stratified sample (every 9th matrix first) of corpus-200: T={c}: {d} matrices ({nnz} nnz), "
              f"{w:.1f} s wall; T=1: the first {d1} of them ({nnz1} nnz) alone, {w1:.1f} s wall.  Oracle labelling "
              f"pass per matrix (features + every admissible conversion + 3 SpMV reps per format + argmin), each "
              f"matrix's SpMV reps scaled to {reps} by its own measured per-rep times; T={c}: per-matrix times "
              f"measured with {c} jobs running concurrently (one thread each), throughput = {c} x matrices / sum of "
              f"times (perfect load balance over a long corpus assumed, contention measured)")
    return {"value": v, "unit": UNIT, "cores": c, "kind": "oracle", "sample": sample,
            "t1": {"value": v1, "unit": UNIT, "cores": 1, "matrices_measured": d1,
                   "single_job_over_loaded_time": r,
                   "note": "T=1 rate on the T=nproc sample: matrices / (sum of under-load times x measured ratio)"},
            "speedup_t1_to_tn": v / v1 if v1 else None}


def run_reference(args):
    rank, world, _ = dist_env()
    if rank != 0:
        return 0
    host = generate_host(corpus_ids(0, args.corpus))
    threads = os.cpu_count() or 1
    budget = max(5.0, min(args.cpu_budget, 20.0))
    for _ in range(args.warmup):
        oracle_sample(host, budget / 4, threads, reps_target=args.reps)
    vals, walls, done = [], [], []
    for _ in range(args.steps):
        v, d, c, w, nnz, _ = oracle_sample(host, budget, threads, reps_target=args.reps)
        vals.append(v)
        walls.append(w)
        done.append(d)
    value = statistics.median(vals)
    sample = (f"{min(done)}-{max(done)} matrices of corpus-200 per step in stratified order (every 9th first), "
              f"oracle labelling pass (features + conversions + 3 SpMV reps/format + argmin), each matrix's SpMV "
              f"reps scaled to {args.reps} by its own measured per-rep times; {threads} concurrent single-thread "
              f"jobs, throughput = {threads} x matrices / sum of the measured per-matrix times")
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1000 * statistics.median(walls),
            "higher_is_better": True, "scaling": "strong" if args.scaling == "strong" else "weak",
            "vs_baseline": None, "dtype": "f64",
            "data": "synthetic", "config": {"workload": "corpus-200 (BASELINE configs[1])", "matrices": args.corpus},
            "cpu_baseline": {"value": value, "unit": UNIT, "cores": threads, "kind": "oracle", "sample": sample},
            "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


# ------------------------------------------------------------------ configs[3] row partition (rowpart record)
def rowpart_measure(N, iters, warmup, rank, world, dev, gloo, group=None, formats=("DIA", "CSR")):
    """BASELINE configs[3]: the 3D 27-point stencil on an N^3 grid (fp64), rows partitioned into `world`
    equal contiguous blocks.  Per format, per exchange, `warmup` untimed then `iters`
    timed power-iteration steps (y becomes the next x) between CUDA events on the launching stream, max
    over ranks (SURVEY §8(d) "Row partition (C4)"):
      allgather: all_gather_into_tensor(x_full, x_local) + sfs_spmv of the block (global column ids);
      halo:      NCCL send/recv of the ghost entries only (sfs_gather packs) + sfs_spmv of the renumbered
                 block;
      push:      sfs_spmv_push -- the ghost rows stored into the neighbours' next x by the SpMV kernel
                 itself over CUDA-IPC peer memory (NVLink), flags instead of NCCL (§8(f) f3).
    Also the all-gather alone, the block SpMV alone, and (rank 0) the whole matrix's SpMV on one GPU, so
    efficiency = t_spmv_full(1 GPU) / (P * t_iter(P)) is computed inside the run.  gloo (ranks sharing
    one GPU, tests only): the all-gather goes through host memory; halo is skipped."""
    import torch
    import torch.distributed as dist

    import paper_conf_icppw_dhandhaniadpbl21_b200 as sfs
    import sfsgen
    from paper_conf_icppw_dhandhaniadpbl21_b200 import dist as sd

    A = sfsgen.stencil3d27(N, dtype=sfsgen.F64)  # host, untimed (every rank: the slice needs row_ptr)
    part = sd.RowPartition(A.m, A.n, world, rank)
    b = part.bounds
    rp, col, val = sd.slice_rows(A.rp, A.col, A.val, b[rank], b[rank + 1])
    t = lambda a: torch.from_numpy(np.ascontiguousarray(a)).to(dev)
    x0 = sfsgen.vector(5, A.n)
    x_local = t(x0[b[rank]:b[rank + 1]])
    stream = torch.cuda.current_stream()
    cdev = torch.device("cpu") if gloo else dev

    def barrier():
        if world > 1:
            dist.barrier(group=group)
        torch.cuda.synchronize()

    def maxr(v):
        if world == 1:
            return v
        tt = torch.tensor([v], dtype=torch.float64, device=cdev)
        dist.all_reduce(tt, op=dist.ReduceOp.MAX, group=group)
        return float(tt.item())

    def sumr(v):
        if world == 1:
            return v
        tt = torch.tensor([v], dtype=torch.float64, device=cdev)
        dist.all_reduce(tt, op=dist.ReduceOp.SUM, group=group)
        return float(tt.item())

    def timed(fn, n):
        """seconds per iteration of fn(n), CUDA events on the launching stream, max over ranks"""
        fn(warmup)
        barrier()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        fn(n)
        e1.record(stream)
        barrier()
        return maxr(e0.elapsed_time(e1) / 1000.0 / n)

    blk = part.block
    x_pad = torch.zeros(blk, dtype=torch.float64, device=dev)
    x_full = torch.empty(blk * world, dtype=torch.float64, device=dev)

    def allgather(dst, src):
        if world == 1:
            dst.copy_(src)
        elif gloo:  # tests only: host staging
            h = torch.empty(dst.numel(), dtype=dst.dtype)
            dist.all_gather_into_tensor(h, src.cpu(), group=group)
            dst.copy_(h)
        else:
            dist.all_gather_into_tensor(dst, src, group=group)

    halo_ok = world == 1 or not gloo
    plan = sd.halo_plan(part, col, group=group, device=cdev)  # world 1: no ghosts
    out = {"config": f"BASELINE configs[3]: 3D 27-point stencil {N}^3 (m = {A.m}, nnz = {A.nnz}), fp64, "
                     f"{world} contiguous row blocks of {blk} rows", "n_gpus": world, "iters": iters,
           "warmup": warmup, "halo_entries_per_rank_max": int(maxr(float(plan.recv_count))),
           "allgather_entries_per_rank": int(blk * (world - 1)), "formats": {}}
    y_loc = torch.empty(part.local_rows, dtype=torch.float64, device=dev)
    for fname in formats:
        fmt = sfs.FORMAT_NAMES.index(fname)
        rec = {}
        # global-column block (all-gather path)
        Ak = sfs.Csr(part.local_rows, A.n, t(rp), t(col), t(val))
        M = sfs.convert(Ak, fmt)
        fk = sfs.features(Ak)
        nbytes = sfs.spmv_bytes(fk, fmt, sfs.F64)
        rec["kernel_variant"] = M.layout().variant

        def ag_iter(n):
            cur = x_local
            for _ in range(n):
                x_pad[:cur.numel()].copy_(cur)
                allgather(x_full, x_pad)
                sfs.spmv(fmt, M, x_full[:A.n], y_loc)
                cur = y_loc

        def ag_only(n):
            for _ in range(n):
                allgather(x_full, x_pad)

        def mv_only(n):
            for _ in range(n):
                sfs.spmv(fmt, M, x_full[:A.n], y_loc)

        x_pad[:x_local.numel()].copy_(x_local)
        allgather(x_full, x_pad)
        rec["allgather"] = {"t_iter_us": 1e6 * timed(ag_iter, iters)}
        rec["t_allgather_only_us"] = 1e6 * timed(ag_only, iters)
        rec["t_spmv_only_us"] = 1e6 * timed(mv_only, iters)
        M.free()
        # renumbered block (halo and push paths)
        Mh = sfs.convert(sfs.Csr(part.local_rows, plan.n_ext, t(rp), t(plan.col_ext), t(val)), fmt)
        if halo_ok:
            spmv_h = lambda xe, yv: sfs.spmv(fmt, Mh, xe, yv)
            rec["halo"] = {"t_iter_us": 1e6 * timed(
                lambda n: sd.rowpart_halo_iterate(plan, spmv_h, sfs.gather, x_local, n, group=group), iters)}
        else:
            rec["halo"] = {"skipped": "gloo test mode (NCCL send/recv of device buffers)"}
        try:
            tm = {}
            sd.rowpart_push_iterate(plan, Mh, fmt, x_local, warmup, group=group)
            barrier()
            sd.rowpart_push_iterate(plan, Mh, fmt, x_local, iters, group=group, timing=tm)
            rec["push"] = {"t_iter_us": 1e3 * maxr(tm["ms_per_iter"]), "transport": "CUDA IPC peer memory"}
        except Exception as ex:  # report, never hide
            rec["push"] = {"error": f"{type(ex).__name__}: {ex}"[:300]}
        Mh.free()
        tot_bytes = sumr(float(nbytes))
        rec["spmv_bytes_all_ranks"] = tot_bytes
        # whole matrix on one GPU (rank 0): the P = 1 reference of the efficiency
        t1 = 0.0
        if rank == 0:
            Af = sfs.Csr(A.m, A.n, t(A.rp), t(A.col), t(A.val))
            Mf = sfs.convert(Af, fmt)
            xf = t(x0)
            yf = torch.empty(A.m, dtype=torch.float64, device=dev)

            def full(n):
                for _ in range(n):
                    sfs.spmv(fmt, Mf, xf, yf)
            full(warmup)
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            full(iters)
            e1.record(stream)
            torch.cuda.synchronize()
            t1 = e0.elapsed_time(e1) / 1000.0 / iters
            Mf.free()
            del Af, xf, yf
        t1 = maxr(t1)
        rec["t_spmv_full_matrix_1gpu_us"] = 1e6 * t1
        for ex in ("allgather", "halo", "push"):
            ti = rec[ex].get("t_iter_us")
            if ti:
                rec[ex]["agg_gbs"] = tot_bytes / (ti / 1e6) / 1e9
                rec[ex]["efficiency"] = (1e6 * t1) / (world * ti)
        out["formats"][fname] = rec
    return out


# ------------------------------------------------------------------ configs[0] / configs[2] race lines
def configs_measure(dev):
    """BASELINE configs[0] (2D 5-point Laplacian 64x64, fp64, all formats) and configs[2] (R-MAT 2^22, fp32;
    CSR / COO / HYB, ELL and DIA inadmissible) through sfs_label_corpus: the race protocol (5 warm-ups +
    100 back-to-back reps between CUDA events) and, for configs[2], the cold protocol (L2 flushed
    before every rep, SURVEY §8(d) "Roofline timing"); GB/s on the algorithmic bytes of each format.  The
    R-MAT matrix is generated on the device (bit-identical to the host generator)."""
    import torch

    import paper_conf_icppw_dhandhaniadpbl21_b200 as sfs
    import sfsgen
    out = {}
    A = sfsgen.laplace2d(64)
    t = lambda a: torch.from_numpy(a).to(dev)
    c0 = sfs.Csr(A.m, A.n, t(A.rp), t(A.col), t(A.val), t(sfsgen.vector(5, A.n)))
    try:
        m, n, rp, col, val = sfsgen.generate_device(sfsgen.make_spec(sfsgen.RMAT, seed=1, ia=22, ib=16, dtype=sfsgen.F32))
        c2 = sfs.Csr(m, n, rp, col, val, sfsgen.vector_device(5, n, sfsgen.F32))
        gen = "device"
    except Exception:
        B = sfsgen.rmat(22, seed=1)
        c2 = sfs.Csr(B.m, B.n, t(B.rp), t(B.col), t(B.val), t(sfsgen.vector(5, B.n, sfsgen.F32)))
        gen = "host"
    for name, M, cold in (("configs[0] 2D 5-pt Laplacian 64x64 fp64", c0, False),
                          ("configs[2] R-MAT 2^22 fp32", c2, True)):
        rec = {"nrows": M.m, "nnz": M.nnz}
        modes = [("hot", 0)] + ([("cold", 1)] if cold else [])
        for mode, flag in modes:
            feats, labs = sfs.label_corpus([M], sfs.default_opts(cold=flag))
            L, F = labs[0], feats[0]
            rec[mode] = {sfs.FORMAT_NAMES[f]: {"t_spmv_us": L["t_spmv_us"][f], "gbs": L["bytes"][f] / L["t_spmv_us"][f] / 1e3}
                         for f in range(5) if L["status"][f] == 0}
            rec[mode + "_label"] = sfs.FORMAT_NAMES[L["label"]] if L["label"] >= 0 else None
        rec["admissible"] = [sfs.FORMAT_NAMES[f] for f in range(5) if (F["admissible_mask"] >> f) & 1]
        rec["csr_variant"] = F["csr_variant"]
        out[name] = rec
    out["generation"] = f"configs[2] generated on the {gen}"
    return out


# ------------------------------------------------------------------ our arm
def run_ours(args):
    import torch
    import torch.distributed as dist

    import paper_conf_icppw_dhandhaniadpbl21_b200 as sfs
    from paper_conf_icppw_dhandhaniadpbl21_b200 import dist as sd

    rank, world, local = dist_env()
    local = local % torch.cuda.device_count()
    torch.cuda.set_device(local)
    gloo = args.dist_backend == "gloo"
    if world > 1:
        if gloo:
            dist.init_process_group("gloo")
        else:
            # communicator set-up logged (NVLS / P2P transports), not per-call traffic
            os.environ.setdefault("NCCL_DEBUG", "INFO")
            os.environ.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    dev = torch.device("cuda", local)
    cdev = torch.device("cpu") if gloo else dev  # where the collectives' tensors live
    stream = torch.cuda.current_stream()

    host = generate_host(corpus_ids(rank, args.corpus, world, args.scaling))
    t = lambda a: torch.from_numpy(a).to(dev)
    mats = [sfs.Csr(A.m, A.n, t(A.rp), t(A.col), t(A.val), t(x)) for _, A, x in host]
    pin = lambda a: torch.from_numpy(a).pin_memory()
    hmats = [sfs.Csr(A.m, A.n, pin(A.rp), pin(A.col), pin(A.val), pin(x)) for _, A, x in host]
    torch.cuda.synchronize()
    opts = sfs.default_opts(reps=args.reps, warmup=args.race_warmup, use_graphs=1 if args.graphs else 0)
    n = len(mats)
    n_max = n
    if world > 1:  # LPT shards differ in length: pad the gathered result rows
        nt = torch.tensor([n], dtype=torch.int64, device=cdev)
        dist.all_reduce(nt, op=dist.ReduceOp.MAX)
        n_max = int(nt.item())
    RF = sd.RESULT_FIELDS
    gather_host = torch.full((max(n_max, 1), RF), -1.0, dtype=torch.float64).pin_memory()
    gather_buf = torch.empty(max(n_max, 1) * RF, dtype=torch.float64, device=cdev)
    all_buf = torch.zeros(world * max(n_max, 1) * RF, dtype=torch.float64, device=cdev)
    gathered = {}

    def step(batch):
        feats, labs = sfs.label_corpus(batch, opts)
        # a15: every rank's fixed-size result rows (id, label, statuses, times, 23 features) to every rank
        rows = np.stack([sd.pack_result(i, f, L) for (i, _, _), f, L in zip(host, feats, labs)]) if n else None
        if rows is not None:
            gather_host[:n].copy_(torch.from_numpy(rows))
        gather_buf.copy_(gather_host.reshape(-1), non_blocking=True)
        if world > 1:
            dist.all_gather_into_tensor(all_buf, gather_buf)
        else:
            all_buf.copy_(gather_buf)
        gathered["buf"] = all_buf
        return feats, labs

    def barrier():
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()

    def maxr(v):
        if world == 1:
            return v
        tt = torch.tensor([v], dtype=torch.float64, device=cdev)
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        return float(tt.item())

    def sumr(v):
        if world == 1:
            return v
        tt = torch.tensor([v], dtype=torch.float64, device=cdev)
        dist.all_reduce(tt, op=dist.ReduceOp.SUM)
        return float(tt.item())

    for _ in range(args.warmup):
        step(mats)
    # ---- timed region: K steps, inputs resident in HBM
    clocks = ClockSampler(local)
    clocks.start()
    barrier()
    l0 = sfs.launch_count()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ev_steps = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps)]
    e0.record(stream)
    results = []
    for k in range(args.steps):
        results.append(step(mats))
        ev_steps[k].record(stream)  # step boundaries on the same stream (per-step spread)
    e1.record(stream)
    barrier()
    clk = clocks.stop()
    launches = sfs.launch_count() - l0
    t_dev = e0.elapsed_time(e1) / 1000.0
    t_max = maxr(t_dev)
    step_ms = [maxr(ev_steps[k - 1].elapsed_time(ev_steps[k]) if k else e0.elapsed_time(ev_steps[0]))
               for k in range(args.steps)]  # per step, max over ranks (median and spread)
    n_all = int(sumr(float(n)))
    total_mats = n_all * args.steps
    value = total_mats / t_max
    launches_all = int(sumr(float(launches)))
    # the gathered rows hold every matrix of the job exactly once
    got = gathered["buf"].reshape(-1, RF)[:, 0].cpu().numpy()
    gathered_ids = sorted(int(v) for v in got if v >= 0)
    gather_ok = len(gathered_ids) == n_all and len(set(gathered_ids)) == n_all

    # ---- e2e: same call with pinned host inputs (H2D inside the call), result D2H inside; one untimed
    # warm-up step first (it grows the pool to hold the staged corpus)
    if args.e2e_steps > 0:
        step(hmats)
    barrier()
    e2 = torch.cuda.Event(enable_timing=True)
    e3 = torch.cuda.Event(enable_timing=True)
    e2.record(stream)
    for _ in range(args.e2e_steps):
        step(hmats)
    e3.record(stream)
    barrier()
    t_e2e = maxr(e2.elapsed_time(e3) / 1000.0)
    h2d = sum(m.nbytes() + m.x.numel() * m.x.element_size() for m in hmats)
    e2e = None
    if args.e2e_steps > 0:
        e2e = {"value": n_all * args.e2e_steps / t_e2e, "unit": UNIT, "h2d_bytes_per_step": h2d,
               "d2h_bytes_per_step": n * DAGGR_BYTES,
               "note": "per rank; H2D of the rank's CSR + x from pinned host memory inside sfs_label_corpus"}

    # ---- roofline of the dominant kernel (from the race's own CUDA events, inside the timed region)
    feats, labs = results[-1]
    if args.dump and rank == 0:
        import sfsgen
        with open(args.dump, "w") as fh:
            for (i, A, _), f, L in zip(host, feats, labs):
                fh.write(json.dumps({"id": i, "spec": sfsgen.corpus_spec(200, i).describe(), "m": A.m, "nnz": A.nnz,
                                     "features": f, "race": L}) + "\n")
    per_fmt = {}
    for f in range(sfs.NFMT):
        tt = sum(L["t_spmv_us"][f] for L in labs if L["status"][f] == 0) * args.reps
        bb = sum(L["bytes"][f] for L in labs if L["status"][f] == 0) * args.reps
        big = [(L["bytes"][f], L["t_spmv_us"][f]) for L in labs if L["status"][f] == 0 and L["bytes"][f] > 256e6]
        flops = sum(2.0 * feats[k]["nnz"] for k, L in enumerate(labs) if L["status"][f] == 0) * args.reps
        per_fmt[sfs.FORMAT_NAMES[f]] = {
            "matrices": sum(1 for L in labs if L["status"][f] == 0),
            "spmv_time_s": tt / 1e6, "gbs": (bb / (tt / 1e6) / 1e9) if tt else None,
            "gflops": (flops / (tt / 1e6) / 1e9) if tt else None,
            "gbs_footprint_gt_2xL2": (sum(b for b, _ in big) / (sum(t for _, t in big) / 1e6) / 1e9) if big else None,
            "labels": sum(1 for L in labs if L["label"] == f),
            "convert_over_csr_spmv": (statistics.median(
                [L["t_convert_us"][f] / L["t_spmv_us"][0] for L in labs
                 if L["status"][f] == 0 and L["status"][0] == 0 and L["t_spmv_us"][0] > 0]) if f else 0.0),
        }
    try:  # per-format L2-sector rate from the ncu sector counts of the same race (profiles/r01/traffic_corpus200.json)
        with open(TRAFFIC_JSON) as fh:
            tjall = json.load(fh)
        for k, v in per_fmt.items():
            tk = tjall.get(k)
            if tk and tk.get("l2_sectors_per_launch") and v["spmv_time_s"]:
                v["l2_gsectors_per_s"] = tk["l2_sectors_per_launch"] * v["matrices"] * args.reps / v["spmv_time_s"] / 1e9
    except Exception:
        pass
    dom = max(per_fmt, key=lambda k: per_fmt[k]["spmv_time_s"])
    peaks = {}
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as fh:
            peaks = json.load(fh)
    except Exception:
        pass
    peak = peaks.get("hbm_gbs")
    peak_src = "measured (MEASURED_PEAKS.json hbm_gbs)"
    if not peak:
        peak, peak_src = 6650.0, "fallback (B200_PROFILING.md)"
    kernels = {"CSR": "k_zero_rows + k_spmv_csr_tile<bitmap> (large or skewed) / k_spmv_csr_stream (small regular) / "
                      "k_zero + k_spmv_csr_tile<bitmap, row map> (empty rows)",
               "COO": "k_zero + k_spmv_coo", "ELL": "k_spmv_ell",
               "HYB": "k_spmv_ell<OVF> (short overflow) / k_zero + k_spmv_ell<ATOM> || k_spmv_coo<ACCUM,ATOM> "
                      "(long overflow, parts overlapped)",
               "DIA": "k_spmv_dia"}
    achieved = per_fmt[dom]["gbs"]
    launches_dom = sum(1 for L in labs if L["status"][sfs.FORMAT_NAMES.index(dom)] == 0) * args.reps
    bytes_per_launch = (per_fmt[dom]["gbs"] * 1e9 * per_fmt[dom]["spmv_time_s"] / launches_dom) if launches_dom else 0
    traffic, traffic_src = None, None
    try:  # ncu dram__bytes_read+write of this format's kernels on this workload, hot reps (tools/traffic_corpus.py)
        with open(TRAFFIC_JSON) as fh:
            tj = json.load(fh).get(dom)
        if tj:
            traffic = tj["ratio"] * bytes_per_launch
            traffic_src = (f"ncu dram__bytes_read.sum + dram__bytes_write.sum of {tj['kernel']} over the corpus-200 race "
                           f"(last of 2 back-to-back calls per matrix, --cache-control none) = {tj['ratio']:.3f} x "
                           f"the algorithmic bytes ({os.path.relpath(TRAFFIC_JSON, ROOT)}); < 1: the hot reps re-read "
                           f"part of each matrix from L2")
    except Exception:
        pass
    l2 = None
    try:  # the L2-sector view: gather-heavy SpMVs are bound by the SM <- L2 sector rate, not by HBM
        with open(os.path.join(ROOT, "profiles", "r01", "ceilings.json")) as fh:
            cj = json.load(fh)
        with open(TRAFFIC_JSON) as fh:
            tj = json.load(fh).get(dom)
        if tj and tj.get("l2_sectors_per_launch"):
            rate = tj["l2_sectors_per_launch"] * launches_dom / per_fmt[dom]["spmv_time_s"] / 1e9
            l2 = {"bound": "l2_sectors", "achieved": rate, "peak": cj["l2_random_sector_rate_gsps"],
                  "unit": "G sectors/s", "frac": rate / cj["l2_random_sector_rate_gsps"],
                  "sectors_per_launch": tj["l2_sectors_per_launch"],
                  "source": "ncu lts__t_sectors_srcunit_tex.sum of the same kernels on this workload "
                            f"({os.path.relpath(TRAFFIC_JSON, ROOT)}) over this run's event-timed race time; peak = "
                            "measured random-sector rate of tools/gather.cu (profiles/r01/ceilings.txt)"}
    except Exception:
        pass
    step_time = t_dev / args.steps
    roofline = {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                "frac": achieved / peak if achieved else None, "traffic": traffic, "traffic_source": traffic_src,
                "kernel": f"SpMV {dom}: {kernels[dom]}", "bytes_per_launch": bytes_per_launch,
                "launches": launches_dom, "peak_source": peak_src,
                "share_of_step": per_fmt[dom]["spmv_time_s"] / step_time,
                "achieved_footprint_gt_2xL2": per_fmt[dom]["gbs_footprint_gt_2xL2"], "l2": l2,
                "note": "achieved = sum over the step's matrices of algorithmic bytes (SURVEY 8(a) a9-a13) x reps / "
                        "sum of their event-timed race time (CUDA events on the launching stream); reps run "
                        "back-to-back (P:L217), so the many corpus matrices that fit the 126 MB L2 are latency- "
                        "and L2-bound rather than HBM-bound; achieved_footprint_gt_2xL2 restricts to footprints "
                        "> 256 MB"}

    # ---- f2 / f4: cluster-subset labelling of the same corpus (N = 1): features of all, K-Means on them,
    # race only one representative per cluster, vote, predict; scored against this step's full race
    predictor = None
    if world == 1 and args.predictor_nc > 0:
        from paper_conf_icppw_dhandhaniadpbl21_b200 import predictor as pr
        try:
            r = pr.subset_labelling(mats, opts, nc=args.predictor_nc, k=1, truth=labs)
            t_full = t_dev / args.steps
            predictor = {k: r[k] for k in ("n", "nc", "k", "raced", "t_features_s", "t_fit_s", "t_subset_race_s",
                                           "others_not_raced", "quality")}
            predictor["t_full_race_s"] = t_full
            predictor["race_time_saved"] = 1.0 - r["t_subset_race_s"] / t_full
            predictor["time_saved_incl_clustering"] = 1.0 - r["t_total_s"] / t_full
            predictor["note"] = ("PAPER.md L134/L167-169: only one matrix per cluster benchmarked; times device-measured "
                                 "(CUDA events); t_subset_race_s = features of all + race of the representatives; "
                                 "quality (P:L231 GT / CSR / Threshold, accuracy) against this run's full race")
        except Exception as ex:
            predictor = {"error": f"{type(ex).__name__}: {ex}"[:300]}

    # ---- configs[3] row partition over the same ranks (BASELINE configs[3])
    rowpart = None
    if args.rowpart_N > 0:
        try:
            rowpart = rowpart_measure(args.rowpart_N, args.rowpart_iters, 10, rank, world, dev, gloo)
        except Exception as ex:  # reported in the line, never silently dropped
            rowpart = {"error": f"{type(ex).__name__}: {ex}"[:400]}

    # ---- configs[0] / configs[2] race lines (rank 0, N = 1)
    configs = None
    if rank == 0 and world == 1 and args.configs_record:
        try:
            configs = configs_measure(dev)
        except Exception as ex:
            configs = {"error": f"{type(ex).__name__}: {ex}"[:300]}

    # ---- CPU oracle baseline (rank 0, N = 1 only)
    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        cpu = cpu_baseline_record(host, args.cpu_budget, args.reps)

    if rank == 0:
        line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
                "warmup": args.warmup, "ms_per_step": 1000 * t_max / args.steps,
                "step_ms": {"median": statistics.median(step_ms), "min": min(step_ms), "max": max(step_ms)},
                "higher_is_better": True,
                "scaling": args.scaling, "vs_baseline": None, "dtype": "f64", "data": "synthetic",
                "config": {"workload": "corpus-200 (BASELINE configs[1]): banded/uniform/block-diagonal/power-law, "
                                       "10K-1M rows, values fp32 and fp64 (half each); dtype = the SpMV arithmetic "
                                       "(fp64 products and sums for both value types, y rounded once)",
                           "matrices_rank0": n, "matrices_all_ranks": n_all,
                           "nnz_rank0": int(sum(m.nnz for m in mats)),
                           "reps": args.reps, "race_warmup": args.race_warmup,
                           "parallelism": (f"the identical {n_all}-matrix corpus LPT-sharded over {world} GPU(s) on "
                                           f"estimated race cost (strong scaling)" if args.scaling == "strong" else
                                           f"{n_all} matrices, ~{args.corpus} per GPU (weak scaling)") +
                                          "; one all_gather_into_tensor of 44-double result rows per step, timed",
                           "gather_ok": gather_ok,
                           "l2": "inputs larger than L2 (corpus >> 126 MB per step); in-race reps back-to-back (P:L217)"},
                "e2e": e2e, "gpu_launches": launches_all, "clocks": clk, "roofline": roofline,
                "cpu_baseline": cpu, "per_format": per_fmt,
                "label_histogram": {k: v["labels"] for k, v in per_fmt.items()},
                "predictor": predictor, "rowpart": rowpart, "configs_0_2": configs}
        s = json.dumps(line)
        print(s, flush=True)
        if args.out:
            with open(args.out, "a") as fh:
                fh.write(s + "\n")
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()
    return 0


def main():
    args = parse()
    # torchrun pins OMP_NUM_THREADS=1 per rank; the (untimed) host generation of each rank's corpus
    # shares the node's cores instead, set before the generator's OpenMP runtime loads
    lw = int(os.environ.get("LOCAL_WORLD_SIZE", "1"))
    if lw > 1:
        os.environ["OMP_NUM_THREADS"] = str(max(1, (os.cpu_count() or 1) // lw))
    if args.impl == "reference":
        return run_reference(args)
    return run_ours(args)


if __name__ == "__main__":
    sys.exit(main())
