import sys, torch, numpy as np
sys.path.insert(0, '.')
import sfsgen, paper_conf_icppw_dhandhaniadpbl21_b200 as sfs
t = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
mats = []
for m in [1, 1000, 10000, 100000]:
    A = sfsgen.generate(sfsgen.make_spec(sfsgen.BAND, seed=3, m=max(m, 2), ia=2, pa=1.0))
    x = sfsgen.vector(1, A.n, A.dtype)
    mats.append(sfs.Csr(A.m, A.n, t(A.rp), t(A.col), t(A.val), t(x)))
for pdl in ["1"]:
    feats, labs = sfs.label_corpus(mats, sfs.default_opts())
    for M, L in zip(mats, labs):
        print(M.m, M.nnz, [round(v, 2) for v in L["t_spmv_us"]], L["csr_variant"])
print("graphs:")
feats, labs = sfs.label_corpus(mats, sfs.default_opts(use_graphs=1))
for M, L in zip(mats, labs):
    print(M.m, M.nnz, [round(v, 2) for v in L["t_spmv_us"]], L["csr_variant"])
