"""Race timings (the bench's protocol: sfs_label_corpus, 5 warm-ups + 100 PDL-chained reps) of a few corpus
matrices, per format, for A/B builds (SFS_LIB).  python tools/race_probe.py --ids 0,1,122 [--mask 3]"""
import argparse, json, os, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--ids", default="0,1,2,3,5,9,11,14,57,64,88,122,123,126,152")
    ap.add_argument("--mask", type=int, default=31)
    ap.add_argument("--rounds", type=int, default=3)
    ap.add_argument("--tag", default=os.path.basename(os.environ.get("SFS_LIB", "libsfs.so")))
    ap.add_argument("--json", default=None)
    ap.add_argument("--quiet", action="store_true")
    ap.add_argument("--csr-variant", type=int, default=-1)
    ap.add_argument("--corpus", type=int, default=200, help="corpus_spec size: 200 (configs[1]) or 2000 (configs[4])")
    a = ap.parse_args()
    import torch
    import paper_conf_icppw_dhandhaniadpbl21_b200 as sfs
    import sfsgen
    ids = [int(v) for v in a.ids.split(",")]
    t = lambda v: torch.from_numpy(v).cuda()
    mats = []
    for i in ids:
        sp = sfsgen.corpus_spec(a.corpus, i)
        A = sfsgen.generate(sp)
        mats.append(sfs.Csr(A.m, A.n, t(A.rp), t(A.col), t(A.val), t(sfsgen.vector(sp.seed, A.n, A.dtype))))
    opts = sfs.default_opts(formats_mask=a.mask, csr_variant=a.csr_variant)
    best = None
    for _ in range(a.rounds):
        _, labs = sfs.label_corpus(mats, opts)
        cur = [L["t_spmv_us"] for L in labs]
        best = cur if best is None else [[min(p, q) for p, q in zip(b, c)] for b, c in zip(best, cur)]
    tot = [sum(r[f] for r in best) for f in range(5)]
    if a.json:
        with open(a.json, "a") as fh:
            fh.write(json.dumps({"tag": a.tag, "ids": ids, "t": best}) + "\n")
    print(a.tag, "total", [round(v, 1) for v in tot], flush=True)
    if not a.quiet:
        for i, M, r in zip(ids, mats, best):
            print(f"  {i:4d} nnz={M.nnz:9d}", " ".join(f"{sfs.FORMAT_NAMES[f]}:{r[f]:7.2f}" for f in range(5)))


if __name__ == "__main__":
    main()
