#!/bin/bash
# configs[4] (corpus-2000) on one GPU with device-side generation, and a bench line with the configs[0]/[2] record.
OUT=${OUT:-gpurun_out}/r2c5
mkdir -p $OUT
timeout 1800 python tools/bench_corpus2000.py --out $OUT/corpus2000_1gpu.jsonl > $OUT/c5.log 2>&1
echo "c5 rc=$?"; tail -c 1200 $OUT/c5.log
timeout 1200 python bench.py --steps 5 --warmup 3 --out $OUT/bench.jsonl > $OUT/bench.log 2>&1
echo "bench rc=$?"; python -c "
import json; d=json.loads(open('$OUT/bench.jsonl').readlines()[-1]); print(d['value'], d['e2e']['value']); print(json.dumps(d['configs_0_2'])[:1500])"
