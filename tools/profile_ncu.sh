#!/bin/bash
# ncu --set full captures of selected SpMV kernels (1 GPU). Usage: CAPS="name:matrix:fmt:variant:kregex ..." bash tools/profile_ncu.sh
OUT=${OUT:-gpurun_out}
mkdir -p $OUT
for c in $CAPS; do
  IFS=: read name mat fmt var kre <<< "$c"
  timeout 300 ncu --set full --clock-control none --import-source on -k regex:$kre -s 2 -c 1 -o $OUT/ncu_$name -f \
    python tools/micro.py --matrix $mat --formats $fmt --variant $var --reps 3 --warmup 1 --no-cold > $OUT/ncu_$name.log 2>&1
  echo "$name rc=$?"
done
