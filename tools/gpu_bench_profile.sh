#!/bin/bash
# Bench line + the bench workload's own ncu evidence: per-format hot-rep DRAM traffic and the launch list.
OUT=${OUT:-gpurun_out}
mkdir -p $OUT
timeout 900 python bench.py --steps 3 --warmup 3 --out $OUT/bench.jsonl --dump $OUT/dump.jsonl 2>&1 | tail -1 | cut -c1-300
python tools/analyze_dump.py $OUT/dump.jsonl > $OUT/dump_summary.txt 2>&1
timeout 1500 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sectors_srcunit_tex.sum --cache-control none \
  --clock-control none -k regex:"k_spmv|k_zero" --csv --log-file $OUT/traffic_launches.csv \
  python bench.py --steps 1 --warmup 0 --reps 1 --race-warmup 1 --e2e-steps 0 --no-cpu-baseline --dump $OUT/dump_traffic.jsonl > $OUT/traffic_bench.log 2>&1
echo "ncu traffic rc=$?"
python tools/traffic_corpus.py $OUT/traffic_launches.csv $OUT/dump_traffic.jsonl 2 $OUT/traffic_corpus200.json | head -40
if [ -n "$LAUNCHLIST" ]; then
timeout 1500 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches_bench.csv \
  python bench.py --steps 1 --warmup 0 --no-cpu-baseline --e2e-steps 0 > $OUT/launches_bench.log 2>&1
echo "ncu launch list rc=$?"; python tools/launch_shares.py $OUT/launches_bench.csv > $OUT/launch_shares.txt; head -30 $OUT/launch_shares.txt
fi
