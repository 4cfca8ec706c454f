#!/bin/bash
# Round-2 iteration: all GPU tests, DIA XV A/B, R-MAT CSR variants, bench (no rowpart / cpu baseline).
OUT=${OUT:-gpurun_out}
mkdir -p $OUT
timeout 2400 python -m pytest -q -p no:cacheprovider -m gpu tests > $OUT/pytest_iter.log 2>&1
echo "pytest rc=$?"; tail -4 $OUT/pytest_iter.log
for xv in 0 1; do
  SFS_DIA_XV=$xv timeout 600 python tools/micro.py --matrix st3d27f,band_big_f32 --formats DIA --reps 30 --json $OUT/dia_xv_$xv.jsonl
done
timeout 600 python tools/micro.py --matrix rmat22 --formats CSR,COO --variants 1,5 --reps 30 --json $OUT/rmat_csr5b.jsonl
timeout 900 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --rowpart-N 0 --predictor-nc 20 --out $OUT/bench_iter.jsonl 2>&1 | tail -1 | cut -c1-300
