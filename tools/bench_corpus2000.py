#!/usr/bin/env python
"""configs[4]: the SuiteSparse-shaped corpus of 2,000 synthetic matrices (10^4 - 5*10^7 nnz, fp64; sfsgen
corpus_spec(2000, i)) labelled across N GPUs -- strong scaling over one fixed corpus (SURVEY §8(d) C5,
§8(e) 1).

    python tools/bench_corpus2000.py [--limit K]                          # 1 GPU
    python -m torch.distributed.run --nproc-per-node 8 --master-addr 127.0.0.1 tools/bench_corpus2000.py

Matrices are LPT-assigned to ranks on dist.race_cost (estimated from the generator parameters; no rank
generates another's matrices), generated on the rank's GPU (--gen device, bit-identical to the host generator; --gen host: host +
H2D) and labelled in
memory-bounded batches by sfs_label_corpus (features + every admissible conversion + 5 warm-ups + 100
timed reps per format + argmin).  Timed: barrier, then the whole sharded labelling
including the result D2H and the final all-gather of the result rows, minus the interleaved (measured,
reported) generation time.
matrices/s = matrices / max over ranks of the timed seconds.
"""
import argparse
import json
import os
import sys
import time
from collections import Counter

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--limit", type=int, default=2000, help="first K matrices of the corpus")
    ap.add_argument("--reps", type=int, default=100)
    ap.add_argument("--batch-gb", type=float, default=40.0, help="device-resident CSR per label_corpus call")
    ap.add_argument("--backend", default="nccl")
    ap.add_argument("--out", default=None)
    ap.add_argument("--gen", default="device", choices=["device", "host"], help="where the corpus is generated (untimed)")
    args = ap.parse_args()

    import numpy as np
    import torch
    import torch.distributed as dist

    import paper_conf_icppw_dhandhaniadpbl21_b200 as sfs
    import sfsgen
    from paper_conf_icppw_dhandhaniadpbl21_b200 import dist as sd

    rank, world, local = (int(os.environ.get(k, d)) for k, d in (("RANK", 0), ("WORLD_SIZE", 1), ("LOCAL_RANK", 0)))
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        dist.init_process_group(args.backend, device_id=dev if args.backend == "nccl" else None)
    ids = list(range(args.limit))
    costs = [sd.race_cost(sfsgen.corpus_spec(2000, i)) for i in ids]
    opts = sfs.default_opts(reps=args.reps)
    stats = {"gen_s": 0.0, "label_s": 0.0, "nnz": 0, "matrices": 0, "batches": 0}

    def make(i):
        t0 = time.perf_counter()
        sp = sfsgen.corpus_spec(2000, i)
        if args.gen == "device":  # generated on device per rank (bit-identical to the host)
            m, n, rp, col, val = sfsgen.generate_device(sp)
            M = sfs.Csr(m, n, rp, col, val, sfsgen.vector_device(sp.seed, n, sp.dtype))
        else:
            A = sfsgen.generate(sp)
            x = sfsgen.vector(sp.seed, A.n, A.dtype)
            t = lambda a: torch.from_numpy(np.ascontiguousarray(a)).to(dev)
            M = sfs.Csr(A.m, A.n, t(A.rp), t(A.col), t(A.val), t(x))
        torch.cuda.synchronize()
        stats["gen_s"] += time.perf_counter() - t0
        stats["nnz"] += M.nnz
        return M

    def labeller(batch):
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        out = sfs.label_corpus(batch, opts)
        torch.cuda.synchronize()
        stats["label_s"] += time.perf_counter() - t0
        stats["matrices"] += len(batch)
        stats["batches"] += 1
        return out

    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    w0 = time.perf_counter()
    res = sd.label_corpus_sharded(ids, costs, make, labeller, rank, world, batch_bytes=args.batch_gb * 1e9,
                                  nbytes=lambda M: M.nbytes(), device=dev if args.backend == "nccl" else None)
    torch.cuda.synchronize()
    # timed = features + conversions + race + result D2H + the final all-gather; the
    # (interleaved) generation is measured and taken out
    timed_s = time.perf_counter() - w0 - stats["gen_s"]
    mine = torch.tensor([timed_s, stats["gen_s"], float(stats["nnz"]), float(stats["matrices"]), stats["label_s"]],
                        dtype=torch.float64, device=dev if args.backend == "nccl" else "cpu")
    allr = [torch.zeros_like(mine) for _ in range(world)]
    if world > 1:
        dist.all_gather(allr, mine)
    else:
        allr = [mine]
    per = [r.cpu().tolist() for r in allr]
    t_max = max(p[0] for p in per)
    if rank == 0:
        labels = Counter(sfs.FORMAT_NAMES[r["label"]] if r["label"] >= 0 else "none" for r in res)
        line = {"metric": "matrices labelled/s (features + all-format conversion + 100-rep SpMV race + label)",
                "config": f"configs[4] corpus-2000 (first {args.limit}), fp64, strong scaling", "n_gpus": world,
                "value": len(res) / t_max, "unit": "matrices/s", "matrices": len(res),
                "timed_s_max_over_ranks": t_max, "timed_s_per_rank": [round(p[0], 3) for p in per],
                "label_corpus_s_per_rank": [round(p[4], 3) for p in per],
                "matrices_per_rank": [int(p[3]) for p in per], "nnz_total": int(sum(p[2] for p in per)),
                "untimed_generation_s_per_rank": [round(p[1], 1) for p in per], "generation": args.gen,
                "label_histogram": dict(labels), "reps": args.reps,
                "ok": all(r["matrix_status"] == 0 for r in res)}
        s = json.dumps(line)
        print(s, flush=True)
        if args.out:
            with open(args.out, "a") as fh:
                fh.write(s + "\n")
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
