#!/usr/bin/env python
"""Per-format SpMV / conversion / feature microbenchmark on one BASELINE-shaped matrix.

Reports effective GB/s (algorithmic bytes of SURVEY §8(a) a9–a13 / event time) per format, hot
(back-to-back, as the race) and cold (L2 flushed before every rep).  This is the "SpMV effective HBM
GB/s per format (% of B200 peak)" half of the BASELINE metric, on configs[2] (R-MAT 2^22 fp32) and
configs[3] (3D 27-point 128^3 fp64), and the target of the ncu captures under profiles/.

  python tools/micro.py --matrix rmat22 [--formats CSR,COO,HYB] [--reps 50] [--json out.jsonl]
"""
from __future__ import annotations

import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402


def make_matrix(name):
    import sfsgen
    if name == "rmat22":
        return sfsgen.rmat(22, seed=1)
    if name == "st3d27":
        return sfsgen.stencil3d27(128)
    if name == "st3d27f":
        return sfsgen.stencil3d27(128, dtype=sfsgen.F32)
    if name == "laplace64":
        return sfsgen.laplace2d(64)
    if name.startswith("corpus:") or name.startswith("corpus-"):
        return sfsgen.generate(sfsgen.corpus_spec(200, int(name[7:])))
    if name == "band_big":
        return sfsgen.generate(sfsgen.make_spec(sfsgen.BAND, seed=11, m=1_000_000, ia=24, pa=0.8))
    if name == "blockdiag_big":
        return sfsgen.generate(sfsgen.make_spec(sfsgen.BLOCKDIAG, seed=14, m=1_500_000, ia=40, pa=0.75))
    if name == "uniform_big":
        return sfsgen.generate(sfsgen.make_spec(sfsgen.UNIFORM, seed=12, m=1_000_000, pa=40.0))
    if name == "band_big_f32":
        return sfsgen.generate(sfsgen.make_spec(sfsgen.BAND, seed=11, m=1_000_000, ia=24, pa=0.8, dtype=sfsgen.F32))
    if name == "powerlaw_big":
        return sfsgen.generate(sfsgen.make_spec(sfsgen.POWERLAW, seed=13, m=2_000_000, pa=2.2, dtype=sfsgen.F32))
    raise ValueError(name)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--matrix", default="rmat22")
    ap.add_argument("--formats", default="CSR,COO,ELL,HYB,DIA")
    ap.add_argument("--reps", type=int, default=50)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--variant", type=int, default=-1, help="CSR kernel: -1 auto (Q17), 0 vector, 1 merge, 2 stream")
    ap.add_argument("--variants", default=None, help="comma list: time CSR once per variant (CSR/v keys)")
    ap.add_argument("--json", default=None)
    ap.add_argument("--no-cold", action="store_true")
    args = ap.parse_args()

    import torch

    import paper_conf_icppw_dhandhaniadpbl21_b200 as sfs
    import sfsgen

    from bench import ClockSampler  # nvidia-smi clocks and throttle reasons during the measurement
    for name in args.matrix.split(","):
        run_one(args, name, torch, sfs, sfsgen, ClockSampler(torch.cuda.current_device()))


def run_one(args, matrix, torch, sfs, sfsgen, clk=None):
    A = make_matrix(matrix)
    if clk:  # sampled from here: the (host) generation above leaves the GPU idle at low clocks
        clk.start()
    x = sfsgen.vector(3, A.n, A.dtype)
    t = lambda a: torch.from_numpy(a).cuda()
    dA = sfs.Csr(A.m, A.n, t(A.rp), t(A.col), t(A.val))
    xd = t(x)
    y = torch.empty(A.m, dtype=xd.dtype, device="cuda")
    opts = sfs.default_opts(csr_variant=args.variant)
    feats = sfs.features(dA, opts)
    l2 = torch.cuda.get_device_properties(0).L2_cache_size
    flush = torch.ones(2 * l2 // 4, dtype=torch.float32, device="cuda")
    peak = 6437.9
    try:
        peak = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"]
    except Exception:
        pass
    # feature pass time
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    out = {"matrix": matrix, "m": A.m, "n": A.n, "nnz": A.nnz, "dtype": "f64" if A.dtype else "f32",
           "peak_gbs": peak, "formats": {}}
    jobs = []
    for name in args.formats.split(","):
        if name == "CSR" and args.variants:
            jobs += [(f"CSR/{v}", int(v)) for v in args.variants.split(",")]
        else:
            jobs.append((name, args.variant))
    for name, variant in jobs:
        opts = sfs.default_opts(csr_variant=variant)
        fmt = sfs.FORMAT_NAMES.index(name.split("/")[0])
        if not (feats["admissible_mask"] >> fmt) & 1:
            out["formats"][name] = "inadmissible"
            continue
        sfs.convert(dA, fmt, opts).free()  # warm the memory pool
        torch.cuda.synchronize()
        e0.record()
        M = sfs.convert(dA, fmt, opts)
        e1.record()
        torch.cuda.synchronize()
        t_conv = e0.elapsed_time(e1) * 1e3  # includes the internal feature pass + one host sync
        nbytes = sfs.spmv_bytes(feats, fmt, A.dtype)
        for _ in range(args.warmup):
            sfs.spmv(fmt, M, xd, y)
        torch.cuda.synchronize()
        e0.record()
        for _ in range(args.reps):
            sfs.spmv(fmt, M, xd, y)
        e1.record()
        torch.cuda.synchronize()
        hot = e0.elapsed_time(e1) * 1e3 / args.reps
        res = {"bytes": nbytes, "hot_us": hot, "hot_gbs": nbytes / hot / 1e3, "convert_us_incl_features": t_conv,
               "variant": M.layout().variant}
        if not args.no_cold:
            ts = []
            for r in range(args.reps):
                flush.sum()  # read-only flush: L2 left holding clean lines
                e0.record()
                sfs.spmv(fmt, M, xd, y)
                e1.record()
                torch.cuda.synchronize()
                ts.append(e0.elapsed_time(e1) * 1e3)
            cold = float(np.median(ts))
            res.update(cold_us=cold, cold_gbs=nbytes / cold / 1e3, cold_frac=nbytes / cold / 1e3 / peak)
        out["formats"][name] = res
        M.free()
    out["clocks"] = clk.stop() if clk else None
    out["env"] = {k: v for k, v in os.environ.items() if k.startswith("SFS_")}
    s = json.dumps(out)
    print(f"{matrix:14s} m={A.m} nnz={A.nnz} " + "  ".join(
        f"{k} {v['hot_us']:.1f}us {v['hot_gbs']:.0f}GB/s" for k, v in out["formats"].items() if isinstance(v, dict)))
    if args.json:
        with open(args.json, "a") as fh:
            fh.write(s + "\n")


if __name__ == "__main__":
    main()
