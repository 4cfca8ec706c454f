"""CSR race time of every corpus-200 matrix under each forced CSR kernel variant (the bench's protocol:
sfs_label_corpus, 5 warm-ups + 100 PDL-chained reps, CSR only), to re-fit the Q17 rule.

    python tools/csr_variant_race.py --variants 1,3,4,5 --out gpurun_out/csr_variants.jsonl"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--variants", default="-1,1,3,4,5")
    ap.add_argument("--corpus", type=int, default=200)
    ap.add_argument("--out", default=None)
    a = ap.parse_args()
    import torch
    import bench
    import paper_conf_icppw_dhandhaniadpbl21_b200 as sfs
    host = bench.generate_host(range(a.corpus))
    t = lambda v: torch.from_numpy(v).cuda()
    mats = [sfs.Csr(A.m, A.n, t(A.rp), t(A.col), t(A.val), t(x)) for _, A, x in host]
    res = {}
    for v in [int(s) for s in a.variants.split(",")]:
        opts = sfs.default_opts(formats_mask=1, csr_variant=v)
        sfs.label_corpus(mats, opts)  # warm
        feats, labs = sfs.label_corpus(mats, opts)
        res[v] = [L["t_spmv_us"][0] for L in labs]
        print(f"variant {v}: total {sum(res[v]):.1f} us/rep", flush=True)
        if v == -1:
            res["auto_variant"] = [L["csr_variant"] for L in labs]
            res["features"] = [{k: f[k] for k in ("nrows", "nnz", "nnz_min", "nnz_max")} for f in feats]
    if a.out:
        with open(a.out, "w") as fh:
            json.dump({"ids": [i for i, _, _ in host], **{str(k): v for k, v in res.items()}}, fh)


if __name__ == "__main__":
    main()
