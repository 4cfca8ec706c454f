#!/bin/bash
# The bench's ncu launch list (B200_PROFILING.md recipe: gpu__time_duration.sum, --clock-control none) on the
# first 8 matrices of corpus-200 (the full step is ~130K launches), and the N = 2 bench line (2 ranks sharing
# this GPU, gloo collectives) carrying the strong-scaling corpus and the rowpart record.
OUT=${OUT:-gpurun_out}/r2ll
mkdir -p $OUT
timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches_corpus8.csv \
  python bench.py --steps 1 --warmup 0 --corpus 8 --no-cpu-baseline --rowpart-N 0 --predictor-nc 0 --e2e-steps 0 > $OUT/ll_bench.log 2>&1
echo "launch list rc=$?"; wc -l $OUT/launches_corpus8.csv; gzip -f $OUT/launches_corpus8.csv
PORT=$((29500 + RANDOM % 1000))
timeout 1500 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port $PORT \
  bench.py --gpus 2 --steps 3 --warmup 3 --dist-backend gloo --rowpart-N 128 --out $OUT/bench_2rank_gloo.jsonl > $OUT/bench_2rank.log 2>&1
echo "2-rank bench rc=$?"; tail -c 600 $OUT/bench_2rank.log
timeout 300 python __graft_entry__.py smoke 2>&1 | tail -1
