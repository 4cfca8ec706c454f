#!/bin/bash
OUT=${OUT:-gpurun_out}
mkdir -p $OUT
for lib in libsfs_p64.so libsfs.so; do
  SFS_LIB=paper_conf_icppw_dhandhaniadpbl21_b200/$lib timeout 600 python tools/micro.py --matrix rmat22,powerlaw_big,st3d27f --formats CSR,COO,HYB --reps 30 --no-cold --json $OUT/fp32b_micro_$lib.jsonl
done
IDS=$(python -c "print(','.join(str(i) for i in range(200) if (i>>2)&1))")
for lib in libsfs_p64.so libsfs.so; do
  SFS_LIB=paper_conf_icppw_dhandhaniadpbl21_b200/$lib timeout 900 python tools/race_probe.py --ids $IDS --rounds 2 --quiet --tag $lib --json $OUT/fp32b_race.jsonl
done
