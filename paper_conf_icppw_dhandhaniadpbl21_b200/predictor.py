"""The paper's semi-supervised format predictor driven end to end on the GPU race.

Evaluation glue around the C ABI, off the hot path (BASELINE north_star: "the K-Means clustering over the
small feature matrix stays off the hot path"): the per-matrix work runs in libsfs (features, conversions,
SpMV race, clustering kernels); this module only chooses which matrices to race and scores the outcome.

* f2, cluster-subset labelling (§3 "we only need to benchmark a few matrices ... one
  matrix per cluster in an ideal case", L134 §4 "Example"): featurise every matrix (race mask
  0), fit the clusters on the Table-1 features (sfs_cluster_fit), race only k representatives per
  cluster (sfs_label_corpus with a per-matrix race mask: the other matrices launch no conversion and no
  SpMV), vote the cluster labels from the representatives, predict every matrix from its
  cluster.  The device time of that labelling is measured against a full race of the same corpus.
* f4, predictor quality (§5.3, Table 6): GT = geometric mean over matrices of
  t_best / t_pred (<= 1: "an oracle scheme, which always makes the correct prediction"), CSR =
  geometric mean of t_CSR / t_pred ("speedup ... over ... always using the CSR format"), Threshold =
  number of matrices with t_pred >= 1.5 t_CSR ("a significant slowdown of >= 1.5X over the CSR
  baseline").  A predicted format the matrix cannot be stored in (inadmissible, Q11) falls back to CSR
  and is counted (reading F6).  Accuracy = fraction of matrices whose predicted label is the race label.
"""
from __future__ import annotations

import math
from typing import Dict, List, Sequence

import numpy as np

CSR = 0
THRESHOLD_SLOWDOWN = 1.5


def splitmix64(x: int) -> int:
    """Counter-based choice of representatives (SURVEY App. B mixer): deterministic, seed-stable."""
    x = (x + 0x9E3779B97F4A7C15) & 0xFFFFFFFFFFFFFFFF
    z = ((x ^ (x >> 30)) * 0xBF58476D1CE4E5B9) & 0xFFFFFFFFFFFFFFFF
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & 0xFFFFFFFFFFFFFFFF
    return z ^ (z >> 31)


def race_times(labels: Sequence[dict]) -> np.ndarray:
    """n x 5 per-SpMV times from sfs_label_t records; formats that did not run -> inf."""
    return np.array([[L["t_spmv_us"][f] if L["status"][f] == 0 else np.inf for f in range(5)] for L in labels],
                    dtype=np.float64)


def quality(times: np.ndarray, pred: Sequence[int]) -> Dict[str, float]:
    """f4 metrics of predicted formats `pred` against full-race times (n x 5, inf = not run / inadmissible).
    The true label is the argmin with ties to the lowest format id (Q14)."""
    t = np.asarray(times, dtype=np.float64)
    p = np.asarray(pred, dtype=np.int64).copy()
    n = len(p)
    if n == 0:
        return {"n": 0, "accuracy": None, "GT": None, "CSR": None, "Threshold": 0, "fallbacks": 0}
    best = np.argmin(t, axis=1)  # first minimum: the lowest id on ties
    ok = (p >= 0) & (p < t.shape[1])
    ok[ok] = np.isfinite(t[np.nonzero(ok)[0], p[ok]])
    fallbacks = int(np.sum(~ok))
    p[~ok] = CSR  # F6: an unstorable prediction runs in CSR
    tp = t[np.arange(n), p]
    tb = t[np.arange(n), best]
    tc = t[:, CSR]
    return {"n": n, "accuracy": float(np.mean(p == best)),
            "GT": float(math.exp(np.mean(np.log(tb / tp)))),
            "CSR": float(math.exp(np.mean(np.log(tc / tp)))),
            "Threshold": int(np.sum(tp >= THRESHOLD_SLOWDOWN * tc)), "fallbacks": fallbacks}


def representatives(assign: Sequence[int], nc: int, k: int, seed: int = 0x5EED) -> List[int]:
    """k members of every cluster (all of a smaller one), chosen by a counter-based hash of
    (seed, cluster, matrix) -- the lowest k hashes -- so the choice does not depend on array order."""
    a = np.asarray(assign)
    out = []
    for c in range(nc):
        mem = np.nonzero(a == c)[0]
        if len(mem) == 0:
            continue
        h = [splitmix64(seed ^ splitmix64((c << 32) ^ int(i))) for i in mem]
        out += [int(mem[j]) for j in np.argsort(h, kind="stable")[:k]]
    return sorted(out)


def subset_labelling(mats, opts, nc: int, k: int = 1, pcs: int = 8, seed: int = 0x5EED, truth=None, stream=None):
    """f2 on the GPU.  mats: sfs.Csr list (device-resident).  truth: optional sfs_label_t records of a full
    race of the same matrices (for the f4 scores).  Returns a dict with the device-timed phases (s),
    the representatives, the predicted formats and, given truth, the quality against the full race."""
    import torch

    import paper_conf_icppw_dhandhaniadpbl21_b200 as sfs
    n = len(mats)
    st = stream or torch.cuda.current_stream()

    def timed(fn):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        e0.record(st)
        out = fn()
        e1.record(st)
        torch.cuda.synchronize()
        return out, e0.elapsed_time(e1) / 1e3

    (feats, _), t_feat = timed(lambda: sfs.label_corpus(mats, opts, stream=st, race_mask=[0] * n))
    table = sfs.features_table1(feats)
    nc = max(1, min(nc, n))
    init = np.array(representatives(np.zeros(n, int), 1, nc, seed), np.int32)  # nc distinct seeded points
    M, t_fit = timed(lambda: sfs.ClusterModel(table, init, pcs=pcs, stream=st))
    assign = M.info["assign"]
    reps = representatives(assign, nc, k, seed ^ 0xA5)
    mask = np.zeros(n, np.uint32)
    mask[reps] = opts.formats_mask
    (_, rlabs), t_race = timed(lambda: sfs.label_corpus(mats, opts, stream=st, race_mask=mask.tolist()))
    bench = np.full(n, -1, np.int32)
    for i in reps:
        bench[i] = rlabs[i]["label"]
    cl = M.vote(bench, stream=st)
    pred = cl[assign]
    M.free()
    out = {"n": n, "nc": nc, "k": k, "raced": len(reps), "t_features_s": t_feat, "t_fit_s": t_fit,
           "t_subset_race_s": t_race, "t_total_s": t_feat + t_fit + t_race, "pred": pred.tolist(),
           "representatives": reps,
           "others_not_raced": all(all(s == sfs.ERR_NOT_RUN for s in rlabs[i]["status"])
                                   for i in range(n) if i not in set(reps))}
    if truth is not None:
        out["quality"] = quality(race_times(truth), pred)
    return out
