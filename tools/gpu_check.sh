#!/bin/bash
# One GPU round trip: parity tests, per-format micro (both CSR kernels), bench.
OUT=${OUT:-gpurun_out}
mkdir -p $OUT
timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider -x 2>&1 | tail -15
for M in ${MATS:-st3d27 rmat22 band_big uniform_big powerlaw_big st3d27f}; do
  timeout 300 python tools/micro.py --matrix $M --reps 30 --json $OUT/micro.jsonl > /dev/null 2>&1
  timeout 300 python tools/micro.py --matrix $M --reps 30 --formats CSR --variant $([ "$M" = rmat22 -o "$M" = powerlaw_big ] && echo 2 || echo 1) --json $OUT/micro_csr_alt.jsonl > /dev/null 2>&1
done
if [ -z "$NOBENCH" ]; then timeout 900 python bench.py --steps 3 --warmup 3 --out $OUT/bench.jsonl --dump $OUT/dump.jsonl 2>&1 | tail -3; fi
