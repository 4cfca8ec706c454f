#!/bin/bash
# Round-end evidence on one B200: GPU tests, the hot-rep traffic / L2-sector pass over the bench race,
# the bench line (reads the fresh traffic file), the launch list of the bench command, and ncu --set
# full captures of the dominant format's kernels.  Everything lands in $OUT (gpurun_out/).
OUT=${OUT:-gpurun_out}
mkdir -p $OUT
if [ -z "$NOTESTS" ]; then
  timeout 1200 python -m pytest tests -m gpu -q -p no:cacheprovider -x > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 $OUT/pytest_gpu.log
fi
timeout 1500 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sectors_srcunit_tex.sum \
  --cache-control none --clock-control none -k regex:"k_spmv|k_zero" --csv --log-file $OUT/traffic_launches.csv \
  python bench.py --steps 1 --warmup 0 --reps 1 --race-warmup 1 --e2e-steps 0 --no-cpu-baseline --dump $OUT/dump_traffic.jsonl > $OUT/traffic_bench.log 2>&1
echo "ncu traffic rc=$?"
python tools/traffic_corpus.py $OUT/traffic_launches.csv $OUT/dump_traffic.jsonl 2 $OUT/traffic_corpus200.json > /dev/null && \
  cp $OUT/traffic_corpus200.json profiles/r01/traffic_corpus200.json
timeout 900 python bench.py --steps 3 --warmup 3 --out $OUT/bench.jsonl --dump $OUT/dump.jsonl 2>&1 | tail -1 | cut -c1-200
python tools/analyze_dump.py $OUT/dump.jsonl > $OUT/dump_summary.txt 2>&1
timeout 1500 ncu --metrics gpu__time_duration.sum --clock-control none -c ${LAUNCHES:-12000} --csv --log-file $OUT/launches_bench.csv \
  python bench.py --steps 1 --warmup 0 --no-cpu-baseline --e2e-steps 0 > $OUT/launches_bench.log 2>&1
echo "ncu launch list rc=$?"; python tools/launch_shares.py $OUT/launches_bench.csv > $OUT/launch_shares.txt; head -12 $OUT/launch_shares.txt
CAPS=${CAPS:-"hyb_uniform57:corpus-57:HYB:-1:k_spmv_ell hyb_powerlaw11:corpus-11:HYB:-1:k_spmv_coo ell_uniform57:corpus-57:ELL:-1:k_spmv_ell"} \
  bash tools/profile_ncu.sh
for f in $OUT/ncu_*.ncu-rep; do python tools/ncu_summary.py $f; done > $OUT/ncu_full_summary.txt 2>&1
head -60 $OUT/ncu_full_summary.txt
