#!/bin/bash
OUT=${OUT:-gpurun_out}
for M in laplace64 corpus:1 corpus:3 corpus:2 corpus:0 corpus:4; do
  timeout 300 python tools/micro.py --matrix $M --reps 100 --no-cold --json $OUT/micro_small.jsonl > /dev/null 2>&1
done
timeout 600 python bench.py --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 1 --dump $OUT/dump.jsonl | tail -1 | cut -c1-200
