"""Analyse bench.py --dump output: where the race time goes (by size and class), per-format GB/s,
label histogram (Table-3 analog) and conversion / CSR-SpMV ratios (Table-8 analog)."""
import json
import math
import statistics
import sys

NAMES = ['CSR', 'COO', 'ELL', 'HYB', 'DIA']
rows = [json.loads(l) for l in open(sys.argv[1])]
tot = [0.0] * 5
for r in rows:
    for f in range(5):
        if r['race']['status'][f] == 0:
            tot[f] += r['race']['t_spmv_us'][f]
print(f"{len(rows)} matrices; race time per rep (sum over matrices, us):",
      {NAMES[f]: round(tot[f]) for f in range(5)}, 'total', round(sum(tot)))
bins = {}
for r in rows:
    k = int(math.log10(max(r['nnz'], 1)))
    b = bins.setdefault(k, [0, 0.0, 0.0, 0.0, 0.0])
    L = r['race']
    b[0] += 1
    b[1] += sum(L['t_spmv_us'][f] for f in range(5) if L['status'][f] == 0)
    b[2] += sum(L['t_convert_us'])
    b[3] += L['t_features_us']
    b[4] += sum(L['bytes'][f] for f in range(5) if L['status'][f] == 0)
for k in sorted(bins):
    n, t, c, f, by = bins[k]
    print(f"nnz ~1e{k}: {n:3d} matrices  spmv {t:8.0f} us/rep ({by / t / 1e3 if t else 0:6.0f} GB/s)  "
          f"convert {c:8.0f} us  features {f:7.0f} us")
print('per class (median GB/s per format):')
for cls in sorted(set(r['spec']['cls'] for r in rows)):
    sel = [r for r in rows if r['spec']['cls'] == cls]
    med = {}
    for f in range(5):
        v = [r['race']['bytes'][f] / r['race']['t_spmv_us'][f] / 1e3 for r in sel
             if r['race']['status'][f] == 0 and r['race']['t_spmv_us'][f] > 0]
        if v:
            med[NAMES[f]] = round(statistics.median(v))
    labels = {NAMES[f]: sum(1 for r in sel if r['race']['label'] == f) for f in range(5)}
    print(f"  {cls:10s} n={len(sel):3d} GB/s {med}  labels {labels}")
hist = {NAMES[f]: sum(1 for r in rows if r['race']['label'] == f) for f in range(5)}
print('label histogram (Table-3 analog):', hist)
ratio = {}
for f in range(1, 5):
    v = [r['race']['t_convert_us'][f] / r['race']['t_spmv_us'][0] for r in rows
         if r['race']['status'][f] == 0 and r['race']['t_spmv_us'][0] > 0]
    if v:
        ratio[NAMES[f]] = round(statistics.median(v), 2)
print('conversion / CSR SpMV, median (Table-8 analog; paper COO 9, ELL 102, HYB 147):', ratio)
if len(sys.argv) > 2:
    k = sys.argv[2]
    for r in sorted(rows, key=lambda r: r['nnz']):
        if r['spec']['cls'] == k:
            L = r['race']
            print(f"{r['m']:9d} {r['nnz']:10d} {r['spec']['dtype']} " + ' '.join(
                f"{NAMES[f]} {L['t_spmv_us'][f]:6.1f}" for f in range(5) if L['status'][f] == 0) + f" -> {NAMES[L['label']]}")
