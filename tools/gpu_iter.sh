#!/bin/bash
# One GPU iteration: parity tests, small-matrix + corpus micro timings, a bench line.
OUT=${OUT:-gpurun_out}
mkdir -p $OUT
timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider -x 2>&1 | tail -${TESTTAIL:-6}
for M in ${MATS:-laplace64 corpus:1 corpus:122 corpus:0 corpus:57 corpus:11 rmat22 st3d27}; do
  timeout 300 python tools/micro.py --matrix $M --reps 100 --no-cold --json $OUT/micro_iter.jsonl > /dev/null 2>&1
done
python tools/show_micro.py $OUT/micro_iter.jsonl 2>/dev/null | tail -40
if [ -z "$NOBENCH" ]; then timeout 900 python bench.py --steps 3 --warmup 3 --out $OUT/bench.jsonl --dump $OUT/dump.jsonl 2>&1 | tail -1 | cut -c1-400; python tools/analyze_dump.py $OUT/dump.jsonl | head -8; fi
