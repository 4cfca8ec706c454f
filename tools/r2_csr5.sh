#!/bin/bash
# CSR variant 5 (bitmap over the non-empty rows + row map): parity, R-MAT / power-law micro, corpus race A/B.
OUT=${OUT:-gpurun_out}
mkdir -p $OUT
timeout 1500 python -m pytest -q -p no:cacheprovider -m gpu tests/test_gpu_parity.py tests/test_gpu_configs.py -k "variant or tile or split or rmat or tolerance" > $OUT/pytest_csr5.log 2>&1
echo "pytest rc=$?"; tail -5 $OUT/pytest_csr5.log
timeout 600 python tools/micro.py --matrix rmat22,powerlaw_big,uniform_big,st3d27 --formats CSR,COO --variants 1,3,4,5 --reps 30 --json $OUT/csr5_micro.jsonl
# corpus race with every CSR variant forced (race_probe): per-matrix CSR time
timeout 1200 python tools/csr_variant_race.py --out $OUT/csr_variant_race.json
