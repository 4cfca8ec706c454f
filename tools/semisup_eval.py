#!/usr/bin/env python
"""The paper's semi-supervised predictor on our own B200 race.

Input: bench.py --dump output (Table-1 features + race times + labels of the corpus-200 matrices).
5-fold cross-validation: K-Means on the training fold's features (sfs_cluster_fit, GPU),
cluster labels by majority vote of
  (a) every training matrix ("all benchmarked"), or
  (b) only `k` randomly drawn members per cluster (f2: "we only need to benchmark a few matrices",
      P:L126) — the race time this saves is reported,
then nearest-centroid prediction of the test fold (sfs_cluster_predict) and the metrics of P:L223 /
P:L231: ACC, macro F1, MCC, GT speedup (geo-mean t_best / t_pred), CSR speedup (geo-mean t_CSR /
t_pred), Threshold (# test matrices with t_pred >= 1.5 t_CSR).

    python tools/semisup_eval.py gpurun_out/dump.jsonl [--nc 10,20,40] [--json out.json]
"""
import argparse
import json
import math
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

NAMES = ["CSR", "COO", "ELL", "HYB", "DIA"]


def mcc(y, p, K=5):
    """Multiclass Matthews correlation (Gorodkin's R_K) from the confusion matrix."""
    C = np.zeros((K, K))
    for a, b in zip(y, p):
        C[a, b] += 1
    t, pk, c, s = C.sum(1), C.sum(0), np.trace(C), C.sum()
    num = c * s - np.dot(t, pk)
    den = math.sqrt(max(s * s - np.dot(pk, pk), 0)) * math.sqrt(max(s * s - np.dot(t, t), 0))
    return num / den if den else 0.0


def f1_scores(y, p, K=5):
    """(support-weighted F1, macro F1) over the classes present in y or p (reading F4)."""
    f, w = [], []
    for k in range(K):
        tp = np.sum((y == k) & (p == k))
        fp = np.sum((y != k) & (p == k))
        fn = np.sum((y == k) & (p != k))
        if tp + fp + fn == 0:
            continue
        f.append(2 * tp / (2 * tp + fp + fn))
        w.append(np.sum(y == k))
    if not f:
        return 0.0, 0.0
    return float(np.dot(f, w) / max(np.sum(w), 1)), float(np.mean(f))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("dump")
    ap.add_argument("--nc", default="8,16,32,48")
    ap.add_argument("--draws", default="1,2")
    ap.add_argument("--folds", type=int, default=5)
    ap.add_argument("--seed", type=int, default=7)
    ap.add_argument("--json", default=None)
    args = ap.parse_args()

    import paper_conf_icppw_dhandhaniadpbl21_b200 as sfs

    rows = [json.loads(l) for l in open(args.dump)]
    rows = [r for r in rows if r["race"]["matrix_status"] == 0 and r["race"]["label"] >= 0]
    n = len(rows)
    T = sfs.features_table1([r["features"] for r in rows])
    y = np.array([r["race"]["label"] for r in rows])
    tt = np.array([[r["race"]["t_spmv_us"][f] if r["race"]["status"][f] == 0 else np.inf for f in range(5)]
                   for r in rows])
    t_race = np.array([sum(r["race"]["t_spmv_us"][f] for f in range(5) if r["race"]["status"][f] == 0) for r in rows])
    rng = np.random.default_rng(args.seed)
    perm = rng.permutation(n)
    folds = np.array_split(perm, args.folds)
    out = {"n": n, "label_histogram": {NAMES[f]: int(np.sum(y == f)) for f in range(5)}, "results": []}
    for nc in [int(v) for v in args.nc.split(",")]:
        for mode in ["all"] + [f"k={d}" for d in args.draws.split(",")]:
            ys, ps, tb, tc, tp, saved, fit_ms, pur = [], [], [], [], [], [], [], []
            nfall = 0
            for fi in range(args.folds):
                test = folds[fi]
                train = np.concatenate([folds[j] for j in range(args.folds) if j != fi])
                init = rng.choice(len(train), size=nc, replace=False).astype(np.int32)
                t0 = time.perf_counter()
                M = sfs.ClusterModel(T[train], init, pcs=8)
                fit_ms.append(1e3 * (time.perf_counter() - t0))
                assign = M.info["assign"]
                bench = y[train].copy()
                if mode != "all":
                    d = int(mode[2:])
                    keep = np.zeros(len(train), bool)
                    for c in range(nc):
                        mem = np.nonzero(assign == c)[0]
                        if len(mem):
                            keep[rng.choice(mem, size=min(d, len(mem)), replace=False)] = True
                    bench[~keep] = -1
                    saved.append(1.0 - t_race[train][keep].sum() / t_race[train].sum())
                cl = M.vote(bench)
                pred = cl[M.predict(T[test])]
                # a predicted format the matrix cannot be stored in (inadmissible, Q1/Q3/Q5) falls back
                # to CSR, the always-admissible default (reading F6)
                bad = ~np.isfinite(tt[test, pred])
                nfall += int(bad.sum())
                pred = np.where(bad, 0, pred)
                # purity of the training clusters w.r.t. the true labels
                sizes = np.bincount(assign, minlength=nc)
                mx = [np.max(np.bincount(y[train][assign == c], minlength=5)) if sizes[c] else 0 for c in range(nc)]
                pur.append(sum(mx) / len(train))
                ys.append(y[test])
                ps.append(pred)
                tb.append(tt[test, y[test]])
                tc.append(tt[test, 0])
                tp.append(tt[test, pred])
                M.free()
            ys, ps = np.concatenate(ys), np.concatenate(ps)
            tb, tc, tp = np.concatenate(tb), np.concatenate(tc), np.concatenate(tp)
            gt = float(np.exp(np.mean(np.log(tb / tp))))
            csr = float(np.exp(np.mean(np.log(tc / tp))))
            f1w, f1m = f1_scores(ys, ps)
            res = {"nc": nc, "labels_from": mode, "ACC": float(np.mean(ys == ps)), "F1": f1w, "F1_macro": f1m,
                   "MCC": mcc(ys, ps), "GT": gt, "CSR": csr, "Threshold": int(np.sum(tp >= 1.5 * tc)),
                   "purity": float(np.mean(pur)), "fit_ms": float(np.median(fit_ms)),
                   "race_time_saved": float(np.mean(saved)) if saved else 0.0,
                   "inadmissible_fallbacks": nfall}
            out["results"].append(res)
            print(f"NC={nc:3d} {mode:4s} ACC {res['ACC']:.3f} F1 {res['F1']:.3f} MCC {res['MCC']:.3f} "
                  f"GT {gt:.3f} CSR {csr:.3f} Thr {res['Threshold']:3d} purity {res['purity']:.3f} "
                  f"race saved {100 * res['race_time_saved']:.1f}% fallbacks {nfall} fit {res['fit_ms']:.1f} ms")
    if args.json:
        json.dump(out, open(args.json, "w"), indent=1)


if __name__ == "__main__":
    main()
