#!/bin/bash
# Round-2 micro A/B: cp.async DIA (fp32 / fp64) and CSR variants on R-MAT; correctness of the touched kernels first.
OUT=${OUT:-gpurun_out}
mkdir -p $OUT
timeout 1500 python -m pytest -q -p no:cacheprovider -m gpu tests/test_gpu_parity.py tests/test_gpu_configs.py tests/test_gpu_race.py tests/test_gpu_push_full.py > $OUT/pytest_micro.log 2>&1
echo "pytest rc=$?"; tail -5 $OUT/pytest_micro.log
for mode in 0 1 2; do
  SFS_DIA_CPA=$mode timeout 600 python tools/micro.py --matrix st3d27f,st3d27,band_big --formats DIA --reps 30 --json $OUT/dia_cpa_$mode.jsonl
done
timeout 600 python tools/micro.py --matrix rmat22 --formats CSR,COO --variants 1,3 --reps 30 --json $OUT/rmat_csr.jsonl
timeout 900 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --rowpart-N 0 --out $OUT/bench_hook.jsonl 2>&1 | tail -1 | cut -c1-300
SFS_DIA_CPA=0 timeout 900 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --rowpart-N 0 --out $OUT/bench_nocpa.jsonl 2>&1 | tail -1 | cut -c1-300
