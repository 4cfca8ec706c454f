#!/bin/bash
OUT=${OUT:-gpurun_out}
for G in "" "--no-graphs"; do
  echo "== graphs flag: '$G'"
  SFS_PROFILE=1 timeout 600 python bench.py --steps 1 --warmup 2 --no-cpu-baseline --e2e-steps 0 $G 2>&1 | grep -E "^\[sfs\]|value" | cut -c1-260 | tail -3
done
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches_small_r01.csv \
  python bench.py --corpus 8 --steps 1 --warmup 0 --reps 10 --race-warmup 1 --no-cpu-baseline --e2e-steps 0 > $OUT/launches_small.log 2>&1
echo "ncu rc=$?"
