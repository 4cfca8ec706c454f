#!/usr/bin/env python
"""bench.py — matrices labelled per second on the BASELINE configs[1] corpus (the headline metric).

One step = the whole hot path (SURVEY §8(a) a1–a15) over one batch: for every matrix of the rank's
corpus-200 (configs[1]: banded / uniform random / block-diagonal / power-law, 10K–1M rows, fp32 and
fp64 values) the Table-1 feature pass, every admissible conversion, the device-timed format race
(5 warm-up + 100 timed SpMVs per format) and the label; at N > 1 the labels/features are
gathered over NCCL.  Inputs are resident in HBM when the timed region starts (`value`); `e2e`
repeats the step through the same C-ABI call with pinned HOST buffers (H2D inside the call).

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
    return p.parse_args()


def dist_env():
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return rank, world, local


def corpus_ids(rank, per_rank, world=1):
    """Weak scaling: the job is the first per_rank*world matrices of the configs[1] recipe, LPT-balanced
    over the ranks on an estimated race cost (dist.weak_shard); N = 1 labels ids [0, per_rank)."""
    from paper_conf_icppw_dhandhaniadpbl21_b200 import dist as sd
    return sd.weak_shard(200, per_rank, rank, world)


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
def oracle_sample(host_mats, budget_s, threads, reps_target=100, reps_cpu=3):
    """The oracle's whole labelling pass (features, every admissible conversion, timed SpMV reps per
    format, argmin) on the matrices in corpus order, `threads` matrices at a time, dispatching until
    `budget_s` of wall time is spent.  Each matrix runs `reps_cpu` SpMV reps per format; its
    single-thread time is scaled to `reps_target` reps with its own measured per-rep SpMV times:
        t_i = wall_i + (reps_target - reps_cpu) * sum_f t_spmv_f,i
    and the throughput is threads * done / sum_i t_i (perfect scaling over cores: generous to the CPU).
    Returns (matrices/s, done, threads, wall, nnz, measured matrices/s at reps_cpu)."""
    import oracle
    from concurrent.futures import ThreadPoolExecutor, FIRST_COMPLETED, wait

    t0 = time.perf_counter()
    done, nnz, tsum = 0, 0, 0.0
    it = iter(host_mats)
    futs = set()

    def job(item):
        _, A, x = item
        w0 = time.perf_counter()
        _, _, ts, _ = oracle.label_matrix(A.m, A.n, A.rp, A.col, A.val.astype(np.float64), x.astype(np.float64),
                                          reps=reps_cpu)
        wall_i = time.perf_counter() - w0
        return A.nnz, wall_i + (reps_target - reps_cpu) * float(np.sum(ts))

    with ThreadPoolExecutor(max_workers=threads) as ex:
        for _ in range(threads):
            nxt = next(it, None)
            if nxt is None:
                break
            futs.add(ex.submit(job, nxt))
        while futs:
            fin, futs = wait(futs, return_when=FIRST_COMPLETED)
            for f in fin:
                z, ti = f.result()
                nnz += z
                tsum += ti
                done += 1
            if time.perf_counter() - t0 < budget_s:
                for _ in range(len(fin)):
                    nxt = next(it, None)
                    if nxt is not None:
                        futs.add(ex.submit(job, nxt))
    wall = time.perf_counter() - t0
    return threads * done / tsum, done, threads, wall, nnz, done / wall


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
    sample = (f"first {min(done)}-{max(done)} matrices (corpus order) of corpus-200 per step, oracle labelling "
              f"pass (features + conversions + 3 SpMV reps/format + argmin) with each matrix's time scaled to "
              f"{args.reps} reps by its own per-rep SpMV time; {threads} threads, perfect core scaling assumed")
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1000 * statistics.median(walls),
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64",
            "data": "synthetic", "config": {"workload": "corpus-200 (BASELINE configs[1])", "matrices_per_rank": args.corpus},
            "cpu_baseline": {"value": value, "unit": UNIT, "cores": threads, "kind": "oracle", "sample": sample},
            "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


# ------------------------------------------------------------------ our arm
def run_ours(args):
    import torch
    import torch.distributed as dist

    import paper_conf_icppw_dhandhaniadpbl21_b200 as sfs

    rank, world, local = dist_env()
    local = local % torch.cuda.device_count()
    torch.cuda.set_device(local)
    gloo = args.dist_backend == "gloo"
    if world > 1:
        if gloo:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    dev = torch.device("cuda", local)
    cdev = torch.device("cpu") if gloo else dev  # where the collectives' tensors live
    stream = torch.cuda.current_stream()

    host = generate_host(corpus_ids(rank, args.corpus, world))
    t = lambda a: torch.from_numpy(a).to(dev)
    mats = [sfs.Csr(A.m, A.n, t(A.rp), t(A.col), t(A.val), t(x)) for _, A, x in host]
    pin = lambda a: torch.from_numpy(a).pin_memory()
    hmats = [sfs.Csr(A.m, A.n, pin(A.rp), pin(A.col), pin(A.val), pin(x)) for _, A, x in host]
    torch.cuda.synchronize()
    opts = sfs.default_opts(reps=args.reps, warmup=args.race_warmup, use_graphs=1 if args.graphs else 0)
    n = len(mats)
    n_max = n
    if world > 1:  # LPT shards differ by a matrix or two: pad the gathered result rows
        nt = torch.tensor([n], dtype=torch.int64, device=cdev)
        dist.all_reduce(nt, op=dist.ReduceOp.MAX)
        n_max = int(nt.item())
    gather_buf = torch.full((n_max * 9,), -1.0, dtype=torch.float64, device=cdev)
    all_buf = torch.zeros(world * n_max * 9, dtype=torch.float64, device=cdev)

    def step(batch):
        feats, labs = sfs.label_corpus(batch, opts)
        if world > 1:  # a15: gather labels + timing summary to every rank (results, ~64 B / matrix)
            rows = [[i, L["label"]] + L["t_spmv_us"] + [L["t_features_us"], L["matrix_status"]]
                    for (i, _, _), L in zip(host, labs)]
            gather_buf[:n * 9].copy_(torch.tensor(rows, dtype=torch.float64).reshape(-1))
            dist.all_gather_into_tensor(all_buf, gather_buf)
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

    # ---- e2e: same call with pinned host inputs (H2D inside the call), result D2H inside; one untimed
    # warm-up step first (it grows the stream-ordered pool to hold the staged corpus)
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
               "d2h_bytes_per_step": n * DAGGR_BYTES}

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
        with open(os.path.join(ROOT, "profiles", "r01", "traffic_corpus200.json")) as fh:
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
    kernels = {"CSR": "k_spmv_csr_tile<bitmap> + fixup (large or skewed, no empty rows) / k_spmv_csr_stream "
                      "(small regular) / k_spmv_csr_merge + fixup (many empty rows)",
               "COO": "k_zero + k_spmv_coo", "ELL": "k_spmv_ell", "HYB": "k_spmv_ell + k_spmv_coo<ACCUM>",
               "DIA": "k_spmv_dia"}
    achieved = per_fmt[dom]["gbs"]
    launches_dom = sum(1 for L in labs if L["status"][sfs.FORMAT_NAMES.index(dom)] == 0) * args.reps
    bytes_per_launch = (per_fmt[dom]["gbs"] * 1e9 * per_fmt[dom]["spmv_time_s"] / launches_dom) if launches_dom else 0
    traffic, traffic_src = None, None
    try:  # ncu dram__bytes_read+write of this format's kernels on this workload, hot reps (tools/traffic_corpus.py)
        with open(os.path.join(ROOT, "profiles", "r01", "traffic_corpus200.json")) as fh:
            tj = json.load(fh).get(dom)
        if tj:
            traffic = tj["ratio"] * bytes_per_launch
            traffic_src = (f"ncu dram__bytes_read.sum + dram__bytes_write.sum of {tj['kernel']} over the corpus-200 race "
                           f"(last of 2 back-to-back calls per matrix, --cache-control none) = {tj['ratio']:.3f} x "
                           f"the algorithmic bytes (profiles/r01/traffic_corpus200.json); < 1: the hot reps re-read "
                           f"part of each matrix from L2")
    except Exception:
        pass
    l2 = None
    try:  # the L2-sector view: gather-heavy SpMVs are bound by the SM <- L2 sector rate, not by HBM
        with open(os.path.join(ROOT, "profiles", "r01", "ceilings.json")) as fh:
            cj = json.load(fh)
        with open(os.path.join(ROOT, "profiles", "r01", "traffic_corpus200.json")) as fh:
            tj = json.load(fh).get(dom)
        if tj and tj.get("l2_sectors_per_launch"):
            rate = tj["l2_sectors_per_launch"] * launches_dom / per_fmt[dom]["spmv_time_s"] / 1e9
            l2 = {"bound": "l2_sectors", "achieved": rate, "peak": cj["l2_random_sector_rate_gsps"],
                  "unit": "G sectors/s", "frac": rate / cj["l2_random_sector_rate_gsps"],
                  "sectors_per_launch": tj["l2_sectors_per_launch"],
                  "source": "ncu lts__t_sectors_srcunit_tex.sum of the same kernels on this workload "
                            "(profiles/r01/traffic_corpus200.json) over this run's event-timed race time; peak = "
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

    # ---- CPU oracle baseline (rank 0, N = 1 only)
    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        threads = os.cpu_count() or 1
        v, d, c, w, nnz, meas = oracle_sample(host, args.cpu_budget, threads, reps_target=args.reps)
        cpu = {"value": v, "unit": UNIT, "cores": c, "kind": "oracle",
               "sample": f"first {d} of this rank's {n} corpus-200 matrices in corpus order ({nnz} nnz): oracle "
                         f"labelling pass (features + conversions + 3 SpMV reps/format + argmin), each matrix's time "
                         f"scaled to {args.reps} reps by its own per-rep SpMV time; {c} threads, perfect core scaling "
                         f"assumed; {w:.1f} s wall ({meas:.1f} matrices/s measured at 3 reps)"}

    if rank == 0:
        line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
                "warmup": args.warmup, "ms_per_step": 1000 * t_max / args.steps,
                "step_ms": {"median": statistics.median(step_ms), "min": min(step_ms), "max": max(step_ms)},
                "higher_is_better": True,
                "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
                "config": {"workload": "corpus-200 (BASELINE configs[1]): banded/uniform/block-diagonal/power-law, "
                                       "10K-1M rows, values fp32 and fp64 (half each), SpMV accumulates in fp64",
                           "matrices_per_rank": n, "matrices_all_ranks": n_all,
                           "nnz_per_rank": int(sum(m.nnz for m in mats)),
                           "reps": args.reps, "race_warmup": args.race_warmup,
                           "parallelism": f"corpus of {n_all} matrices LPT-sharded over {world} GPU(s) on estimated race "
                                          f"cost (weak: {args.corpus} per GPU), no data-path collective",
                           "l2": "inputs larger than L2 (corpus >> 126 MB per step); in-race reps back-to-back (P:L217)"},
                "e2e": e2e, "gpu_launches": launches_all, "clocks": clk, "roofline": roofline,
                "cpu_baseline": cpu, "per_format": per_fmt,
                "label_histogram": {k: v["labels"] for k, v in per_fmt.items()}}
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
