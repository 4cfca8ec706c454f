#!/bin/bash
# Per-format microbenchmarks + one ncu --set full capture per SpMV kernel (run under gpurun, 1 GPU).
set -x
OUT=${OUT:-gpurun_out}
mkdir -p $OUT
for M in st3d27 rmat22 band_big uniform_big powerlaw_big st3d27f; do
  timeout 300 python tools/micro.py --matrix $M --reps 30 --json $OUT/micro.jsonl 2>&1 | tail -1
done
NCU="ncu --set full --clock-control none --import-source on"
timeout 300 $NCU -k regex:k_spmv_dia -s 2 -c 1 -o $OUT/ncu_dia_st3d27 -f python tools/micro.py --matrix st3d27 --formats DIA --reps 3 --warmup 1 --no-cold > /dev/null 2>&1
timeout 300 $NCU -k regex:k_spmv_ell -s 2 -c 1 -o $OUT/ncu_ell_st3d27 -f python tools/micro.py --matrix st3d27 --formats ELL --reps 3 --warmup 1 --no-cold > /dev/null 2>&1
timeout 300 $NCU -k regex:k_spmv_csr -s 2 -c 1 -o $OUT/ncu_csrvec_st3d27 -f python tools/micro.py --matrix st3d27 --formats CSR --reps 3 --warmup 1 --no-cold > /dev/null 2>&1
timeout 300 $NCU -k regex:k_spmv_coo -s 2 -c 1 -o $OUT/ncu_coo_st3d27 -f python tools/micro.py --matrix st3d27 --formats COO --reps 3 --warmup 1 --no-cold > /dev/null 2>&1
timeout 300 $NCU -k regex:k_spmv_csr_merge -s 2 -c 1 -o $OUT/ncu_csrmerge_rmat22 -f python tools/micro.py --matrix rmat22 --formats CSR --reps 3 --warmup 1 --no-cold > /dev/null 2>&1
timeout 300 $NCU -k regex:k_spmv_coo -s 2 -c 1 -o $OUT/ncu_coo_rmat22 -f python tools/micro.py --matrix rmat22 --formats COO --reps 3 --warmup 1 --no-cold > /dev/null 2>&1
ls -la $OUT
