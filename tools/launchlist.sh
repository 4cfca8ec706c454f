#!/bin/bash
# Host-overhead profile + ncu launch list of one bench step (kernel shares; cold-cache, serialised).
OUT=${OUT:-gpurun_out}
SFS_PROFILE=1 timeout 600 python bench.py --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 0 2>&1 | grep -E "^\[sfs\]|value" | cut -c1-200 | tail -6
timeout 1500 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches_r01.csv \
  python bench.py --steps 1 --warmup 0 --no-cpu-baseline --e2e-steps 0 > $OUT/launches_bench.log 2>&1
echo "ncu rc=$?"; wc -l $OUT/launches_r01.csv; tail -2 $OUT/launches_bench.log | cut -c1-300
