#!/bin/bash
# Hot-rep DRAM traffic and L2 sectors per format over the bench race itself (roofline.traffic / roofline.l2):
# the race with 1 warm-up + 1 rep per format under ncu --cache-control none (the last call of each
# (matrix, format) runs right after an identical one, as in the back-to-back reps).
OUT=${OUT:-gpurun_out}/r2tr
mkdir -p $OUT
timeout 2400 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sectors_srcunit_tex.sum \
  --cache-control none --clock-control none -k regex:"k_spmv|k_zero" --csv --log-file $OUT/traffic_launches.csv \
  python bench.py --steps 1 --warmup 0 --reps 1 --race-warmup 1 --e2e-steps 0 --no-cpu-baseline --rowpart-N 0 \
  --predictor-nc 0 --no-configs-record --dump $OUT/dump_traffic.jsonl > $OUT/traffic_bench.log 2>&1
echo "ncu traffic rc=$?"
python tools/traffic_corpus.py $OUT/traffic_launches.csv $OUT/dump_traffic.jsonl 2 $OUT/traffic_corpus200.json | tail -20
gzip -f $OUT/traffic_launches.csv; du -sh $OUT
