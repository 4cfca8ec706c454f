"""Worker of tests/test_gpu_push_full.py (run as a subprocess so that SFS_DIA_S, which the library reads
once per process, can force every diagonal-split instance of the DIA push kernels).

ONE push-fused SpMV of BASELINE configs[3] at full size -- the 3D 27-point stencil on a 128^3 grid
(2,097,152 rows, 55,742,968 nnz) -- row-partitioned over P = 2 / 4 / 8 ranks simulated on one GPU
(dist.rowpart_push_iterate_local, iters = 1: the initial ghost push, then each rank's sfs_spmv_push).
Checks, against the oracle's y = A x of the whole matrix (long-double accumulation, rounded once):
  * every row of every row block: |y - y_ref| <= tol * (|A||x|)_r, tol 1e-12 (fp64) / 1e-5 (fp32)
    (north_star; PAPER.md L31 y = A x split by rows);
  * the ghosts the kernel pushed into every neighbour's next x_ext equal, bit for bit, the y entries of
    the rows they copy (the push is a second store of the same value).
Prints one JSON line per case; exit code 1 if any case fails."""
import argparse
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--N", type=int, default=128)
    ap.add_argument("--worlds", default="2,4,8")
    ap.add_argument("--dtypes", default="f64,f32")
    ap.add_argument("--formats", default="DIA:-1,ELL:-1,CSR:2,CSR:4,COO:-1,HYB:-1")
    args = ap.parse_args()
    import torch

    import oracle
    import paper_conf_icppw_dhandhaniadpbl21_b200 as sfs
    import sfsgen
    from paper_conf_icppw_dhandhaniadpbl21_b200 import dist as sd

    torch.cuda.set_device(0)
    A64 = sfsgen.generate(sfsgen.make_spec(sfsgen.ST3D27, ia=args.N))
    worlds = [int(w) for w in args.worlds.split(",")]
    plans, blocks = {}, {}
    for w in worlds:
        b = sd.row_blocks(A64.m, w)
        blocks[w] = [sd.slice_rows(A64.rp, A64.col, A64.val, b[k], b[k + 1]) for k in range(w)]
        plans[w] = sd.halo_plans_local(A64.m, A64.n, w, [c for _, c, _ in blocks[w]])
    t = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
    ok = True
    for dt in args.dtypes.split(","):
        f32 = dt == "f32"
        x = sfsgen.vector(11, A64.n, sfsgen.F32 if f32 else sfsgen.F64)
        vals = A64.val.astype(np.float32) if f32 else A64.val
        yr, ay = oracle.spmv_csr(A64.m, A64.n, A64.rp, A64.col, vals.astype(np.float64), x.astype(np.float64))
        tol = 1e-5 if f32 else 1e-12
        for w in worlds:
            for spec in args.formats.split(","):
                name, var = spec.split(":")
                fmt, var = sfs.FORMAT_NAMES.index(name), int(var)
                opts = sfs.default_opts(csr_variant=var)
                mats, kinst = [], []
                for P, (rp, _, val) in zip(plans[w], blocks[w]):
                    v = val.astype(np.float32) if f32 else val
                    M = sfs.convert(sfs.Csr(P.n_local, P.n_ext, t(rp), t(P.col_ext), t(v)), fmt, opts)
                    kinst.append(M.layout().variant)
                    mats.append(M)
                ys, mem = sd.rowpart_push_iterate_local(plans[w], mats, fmt, [t(x[P.r0:P.r1]) for P in plans[w]], 1)
                torch.cuda.synchronize()
                y = np.concatenate([v.cpu().numpy().astype(np.float64) for v in ys])
                err = np.abs(y - yr)
                bad = ~(err <= tol * ay) | ((ay == 0) & (y != 0))
                # pushed ghosts: parity-1 x_ext of every rank, ghost regions vs the owners' y (bitwise)
                B = sd._PushBuffers(max(P.n_ext for P in plans[w]), w, ys[0].element_size())
                ynp = np.concatenate([v.cpu().numpy() for v in ys])
                gbad = 0
                for k, P in enumerate(plans[w]):
                    xe = mem[k][B.x_bytes:B.x_bytes + P.n_ext * B.elem].view(ys[0].dtype).cpu().numpy()
                    got = np.concatenate([xe[:P.n_lo], xe[P.n_lo + P.n_local:]])
                    want = ynp[np.concatenate([P.lo, P.hi]).astype(np.int64)]
                    gbad += int((got.view(np.uint8) != want.view(np.uint8)).sum())
                good = not bad.any() and gbad == 0
                ok = ok and good
                print(json.dumps({"dtype": dt, "world": w, "fmt": name, "csr_variant": var, "variants": sorted(set(kinst)),
                                  "dia_s": os.environ.get("SFS_DIA_S", "auto"), "rows": int(A64.m),
                                  "rows_out_of_tol": int(bad.sum()),
                                  "max_err_over_tol": float(np.max(np.where(ay > 0, err / (tol * np.maximum(ay, 1e-300)), 0))),
                                  "ghost_bytes_differ": gbad, "ok": good}), flush=True)
                for M in mats:
                    M.free()
                del mem
    sys.exit(0 if ok else 1)


if __name__ == "__main__":
    main()
