#!/bin/bash
# Full GPU suite + smoke + the driver's bench command (N = 1) + the reference arm, as the round end runs them.
OUT=${OUT:-gpurun_out}/r2final
mkdir -p $OUT
timeout 2700 python -m pytest tests -m gpu -q -p no:cacheprovider > $OUT/pytest_gpu.log 2>&1
echo "pytest rc=$?"; tail -3 $OUT/pytest_gpu.log
timeout 300 python __graft_entry__.py smoke > $OUT/smoke.log 2>&1; tail -1 $OUT/smoke.log
timeout 1500 python bench.py --impl reference --gpus 1 --steps 20 --warmup 5 > $OUT/ref.log 2>&1; echo "ref rc=$?"; tail -c 300 $OUT/ref.log
timeout 1500 python bench.py --gpus 1 --steps 20 --warmup 5 --out $OUT/bench.jsonl > $OUT/bench.log 2>&1
echo "bench rc=$?"; python -c "
import json; d=json.loads(open('$OUT/bench.jsonl').readlines()[-1])
print(d['value'], d['e2e']['value'], d['roofline']['frac'], d['clocks'])"
