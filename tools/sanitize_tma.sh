#!/bin/bash
# compute-sanitizer over the TMA DIA / ELL kernels at every size (the child bodies of tests/test_gpu_dia_tma.py
# and tests/test_gpu_ell_tma.py run directly, with the size gates set to 0).
OUT=${OUT:-gpurun_out}/san_tma
mkdir -p $OUT
SAN=/usr/local/cuda/bin/compute-sanitizer
for tool in memcheck synccheck initcheck racecheck; do
  SFS_DIA_SX_MIN=0 timeout 1200 $SAN --tool $tool --error-exitcode 9 --print-limit 20 python -c "import sys; sys.path.insert(0, 'tests'); import test_gpu_dia_tma as t; t.run_all()" > $OUT/dia_$tool.log 2>&1
  echo "dia $tool rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|DIA_TMA_OK' $OUT/dia_$tool.log | tail -2 | tr '\n' ' ')"
  SFS_ELL_TMA_MB=0 timeout 1200 $SAN --tool $tool --error-exitcode 9 --print-limit 20 python -c "import sys; sys.path.insert(0, 'tests'); import test_gpu_ell_tma as t; t.run_all()" > $OUT/ell_$tool.log 2>&1
  echo "ell $tool rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|ELL_TMA' $OUT/ell_$tool.log | tail -2 | tr '\n' ' ')"
done
