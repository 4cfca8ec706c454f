#!/bin/bash
OUT=${OUT:-gpurun_out}
run() { SFS_PROFILE=1 timeout 600 python bench.py --steps 1 --warmup 2 --no-cpu-baseline --e2e-steps 0 --dump $OUT/dump_$1.jsonl $2 2>&1 | grep -E "^\[sfs\]|value" | cut -c1-230 | tail -2; }
echo "== graphs + side upload"; run gup ""
echo "== graphs, implicit upload"; SFS_GRAPH_UPLOAD=0 run gimp ""
echo "== direct launches"; run direct "--no-graphs"
