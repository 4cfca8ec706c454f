"""Two processes on ONE GPU run the push-fused row partition over torch symmetric memory (gloo process
group; kernels of the two processes time-slice, so each rank's flag waits are really waited on) and
compare 3 power-iteration steps with the single-process result.

    python -m torch.distributed.run --nproc-per-node 2 --master-addr 127.0.0.1 tools/push_2proc.py
"""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import torch
    import torch.distributed as dist
    import oracle
    import paper_conf_icppw_dhandhaniadpbl21_b200 as sfs
    import sfsgen
    from paper_conf_icppw_dhandhaniadpbl21_b200 import dist as sd
    rank, world = int(os.environ["RANK"]), int(os.environ["WORLD_SIZE"])
    torch.cuda.set_device(0)
    dist.init_process_group("gloo")  # two processes on one GPU: NCCL refuses, CUDA IPC does not
    A = sfsgen.generate(sfsgen.make_spec(sfsgen.ST3D27, ia=24))
    x0 = sfsgen.vector(11, A.n)
    part = sd.RowPartition(A.m, A.n, world, rank)
    b = part.bounds
    rp, col, val = sd.slice_rows(A.rp, A.col, A.val, b[rank], b[rank + 1])
    plan = sd.halo_plan(part, col)
    t = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
    ok = True
    for fname in ["DIA", "ELL", "CSR", "COO"]:
        fmt = sfs.FORMAT_NAMES.index(fname)
        M = sfs.convert(sfs.Csr(part.local_rows, plan.n_ext, t(rp), t(plan.col_ext), t(val)), fmt)
        y = sd.rowpart_push_iterate(plan, M, fmt, t(x0[b[rank]:b[rank + 1]]), 3).cpu().numpy()
        x = x0
        for _ in range(3):
            x, ax = oracle.spmv_csr(A.m, A.n, A.rp, A.col, A.val, x)
        good = bool(np.all(np.abs(y - x[b[rank]:b[rank + 1]]) <= 1e-11 * (np.abs(x) + ax)[b[rank]:b[rank + 1]]))
        ok = ok and good
        print(f"rank {rank} {fname}: push-fused 3-step power iteration {'matches' if good else 'DIFFERS FROM'} the oracle",
              flush=True)
        M.free()
    dist.destroy_process_group()
    sys.exit(0 if ok else 1)


if __name__ == "__main__":
    main()
