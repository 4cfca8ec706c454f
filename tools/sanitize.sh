#!/bin/bash
# compute-sanitizer over a fast subset of the GPU parity tests (small matrices, every CSR variant incl. 5), the halo gather,
# the fused push, the race mask / f2 subset labelling and the clustering kernels.
OUT=${OUT:-gpurun_out}
SAN=/usr/local/cuda/bin/compute-sanitizer
K="tiny4x4 or 1x1 or empty or laplace64 or rand_ragged or rand_zeros or rmat14 or st3d27_20 or st3d7_32f"
for tool in memcheck racecheck synccheck initcheck; do
  timeout 1200 $SAN --tool $tool --error-exitcode 9 --print-limit 20 python -m pytest tests/test_gpu_parity.py tests/test_gpu_dist.py tests/test_gpu_race.py tests/test_gpu_semisup.py -q -p no:cacheprovider -x -k "($K and not refine) or gather_kernel or (halo_exchange and 2-0) or (push_fused and f64) or push_argument or race_mask or subset_labelling or fit_vote or table1" > $OUT/san_$tool.log 2>&1
  echo "$tool rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|passed|failed' $OUT/san_$tool.log | tail -2 | tr '\n' ' ')"
done
