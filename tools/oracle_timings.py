#!/usr/bin/env python
"""The CPU oracle timed on this host's cores on the BASELINE configs it can finish (BASELINE.md "CPU
plan"; SURVEY §8(d) "Oracle timing" column), T = 1 and T = nproc, next to the GPU numbers as a reported
baseline (not a target).  The oracle is run as it stands (plain single-threaded C); T = nproc runs T
copies of it concurrently on contiguous row blocks (global column ids) -- the row partition of
SURVEY §8(e) 2 applied to the CPU -- so every thread executes the unmodified oracle loop.

  C1  2D 5-point Laplacian 64x64 fp64: features + 5 conversions + 5 SpMVs (T = 1; T = nproc: nproc
      independent copies of the whole pass, throughput)
  C3  R-MAT 2^22 fp32: features (T = 1), CSR / COO / HYB SpMV (T = 1 and row-parallel T = nproc)
  C4  3D 27-point 128^3 fp64: one CSR SpMV and one DIA SpMV (T = 1 and row-parallel T = nproc)

  python tools/oracle_timings.py [--out profiles/r02/oracle_timings.jsonl]
"""
import argparse
import json
import os
import sys
import time
from concurrent.futures import ThreadPoolExecutor

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402


def best_of(fn, reps=3):
    ts = []
    for _ in range(reps):
        t0 = time.perf_counter()
        fn()
        ts.append(time.perf_counter() - t0)
    return min(ts)


def row_blocks_spmv(oracle, fmt, A, x, T):
    """T concurrent oracle SpMVs on contiguous row blocks (conversion done ahead, untimed)."""
    from paper_conf_icppw_dhandhaniadpbl21_b200 import dist as sd
    b = sd.row_blocks(A.m, T)
    cvs = []
    for k in range(T):
        rp, col, val = sd.slice_rows(A.rp, A.col, A.val, b[k], b[k + 1])
        if b[k + 1] > b[k]:
            cvs.append(oracle.convert(fmt, b[k + 1] - b[k], A.n, rp, col, val.astype(np.float64)))
    x64 = x.astype(np.float64)
    with ThreadPoolExecutor(max_workers=T) as ex:
        def run():
            list(ex.map(lambda cv: oracle.spmv(cv, x64, with_abs=False), cvs))
        return best_of(run)


def _c1_worker(k):
    import oracle
    import sfsgen
    A = sfsgen.laplace2d(64)
    x = sfsgen.vector(5, A.n)
    for _ in range(k):
        f = oracle.features(A.m, A.n, A.rp, A.col)
        for fmt in range(5):
            oracle.spmv(oracle.convert(fmt, A.m, A.n, A.rp, A.col, A.val, f), x, with_abs=False)
    return k


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default=None)
    ap.add_argument("--configs", default="C1,C3,C4")
    args = ap.parse_args()
    import oracle
    import sfsgen
    T = os.cpu_count() or 1
    cpu = ""
    try:
        cpu = [l.split(":", 1)[1].strip() for l in open("/proc/cpuinfo") if l.startswith("model name")][0]
    except Exception:
        pass
    out = {"what": "CPU oracle timings (BASELINE.md CPU plan)", "cores": T, "cpu": cpu, "configs": {}}
    names = args.configs.split(",")
    if "C1" in names:
        A = sfsgen.laplace2d(64)
        x = sfsgen.vector(5, A.n)

        def full_pass():
            f = oracle.features(A.m, A.n, A.rp, A.col)
            for fmt in range(5):
                oracle.spmv(oracle.convert(fmt, A.m, A.n, A.rp, A.col, A.val, f), x, with_abs=False)
        t1 = best_of(full_pass, 5)
        # T = nproc: T processes (a pass is ~1 ms: Python threads would measure the interpreter), 200 each
        import multiprocessing as mp
        with mp.get_context("spawn").Pool(T) as pool:
            pool.map(_c1_worker, [20] * T)  # warm
            t0 = time.perf_counter()
            pool.map(_c1_worker, [200] * T)
            tn = time.perf_counter() - t0
        out["configs"]["C1"] = {"workload": "2D 5-pt Laplacian 64x64 fp64 (m 4096, nnz 20224): features + 5 conversions "
                                            "+ 5 SpMVs", "t1_s": t1, "t1_passes_per_s": 1 / t1,
                                "tn_passes_per_s": 200 * T / tn, "tn_note": f"{T} processes x 200 passes"}
    if "C3" in names:
        A = sfsgen.rmat(22, seed=1)
        x = sfsgen.vector(5, A.n, A.dtype)
        t0 = time.perf_counter()
        f = oracle.features(A.m, A.n, A.rp, A.col)
        tf = time.perf_counter() - t0
        rec = {"workload": f"R-MAT 2^22 fp32 (m {A.m}, nnz {A.nnz})", "features_t1_s": tf, "spmv": {}}
        for name, fmt in (("CSR", oracle.CSR), ("COO", oracle.COO), ("HYB", oracle.HYB)):
            cv = oracle.convert(fmt, A.m, A.n, A.rp, A.col, A.val.astype(np.float64), f)
            t1 = best_of(lambda: oracle.spmv(cv, x.astype(np.float64), with_abs=False))
            del cv
            tn = row_blocks_spmv(oracle, fmt, A, x, T)
            rec["spmv"][name] = {"t1_s": t1, "tn_s": tn, "t1_gnnz_per_s": A.nnz / t1 / 1e9,
                                 "tn_gnnz_per_s": A.nnz / tn / 1e9}
        out["configs"]["C3"] = rec
    if "C4" in names:
        A = sfsgen.stencil3d27(128)
        x = sfsgen.vector(5, A.n)
        rec = {"workload": f"3D 27-pt 128^3 fp64 (m {A.m}, nnz {A.nnz}): one SpMV", "spmv": {}}
        f = oracle.features(A.m, A.n, A.rp, A.col)
        for name, fmt in (("CSR", oracle.CSR), ("DIA", oracle.DIA)):
            cv = oracle.convert(fmt, A.m, A.n, A.rp, A.col, A.val, f)
            t1 = best_of(lambda: oracle.spmv(cv, x, with_abs=False))
            del cv
            tn = row_blocks_spmv(oracle, fmt, A, x, T)
            rec["spmv"][name] = {"t1_s": t1, "tn_s": tn, "t1_gnnz_per_s": A.nnz / t1 / 1e9,
                                 "tn_gnnz_per_s": A.nnz / tn / 1e9}
        out["configs"]["C4"] = rec
    s = json.dumps(out)
    print(s, flush=True)
    if args.out:
        with open(args.out, "a") as fh:
            fh.write(s + "\n")


if __name__ == "__main__":
    main()
