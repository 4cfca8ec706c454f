#!/bin/bash
# A/B two builds of libsfs: default vs $ALT (env SFS_LIB).  Micro on large matrices + bench step.
OUT=${OUT:-gpurun_out}
ALT=${ALT:-paper_conf_icppw_dhandhaniadpbl21_b200/libsfs_ef.so}
for L in default $ALT; do
  if [ "$L" = default ]; then unset SFS_LIB; else export SFS_LIB=$PWD/$L; fi
  tag=$(basename $L .so)
  for M in ${MATS:-rmat22 st3d27 uniform_big band_big}; do
    timeout 300 python tools/micro.py --matrix $M --reps 30 --json $OUT/ab_micro_$tag.jsonl > /dev/null 2>&1
  done
  timeout 600 python bench.py --steps 2 --warmup 3 --no-cpu-baseline --e2e-steps 0 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$tag', round(d['value'],2), round(d['ms_per_step'],1))"
done
