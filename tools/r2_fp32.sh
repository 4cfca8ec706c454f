#!/bin/bash
# fp32 products / fp32 FMA chains (default) against fp64 products (libsfs_p64.so): parity, micro, race A/B.
OUT=${OUT:-gpurun_out}
mkdir -p $OUT
timeout 1800 python -m pytest -q -p no:cacheprovider -m gpu tests/test_gpu_parity.py tests/test_gpu_configs.py tests/test_gpu_push_full.py > $OUT/pytest_fp32.log 2>&1
echo "pytest rc=$?"; tail -4 $OUT/pytest_fp32.log
IDS=$(python -c "print(','.join(str(i) for i in range(200) if (i>>2)&1))")
for lib in libsfs_p64.so libsfs.so; do
  SFS_LIB=paper_conf_icppw_dhandhaniadpbl21_b200/$lib timeout 900 python tools/race_probe.py --ids $IDS --rounds 2 --quiet --tag $lib --json $OUT/fp32_race.jsonl
  SFS_LIB=paper_conf_icppw_dhandhaniadpbl21_b200/$lib timeout 600 python tools/micro.py --matrix st3d27f,rmat22,band_big_f32 --reps 30 --json $OUT/fp32_micro_$lib.jsonl
done
timeout 900 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --rowpart-N 0 --predictor-nc 0 --out $OUT/bench_fp32.jsonl 2>&1 | tail -1 | cut -c1-200
