#!/bin/bash
# Round-2 GPU round trip: build check, GPU tests, smoke, bench A/B of the allocator hook.
OUT=${OUT:-gpurun_out}
mkdir -p $OUT
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > $OUT/smi.txt 2>&1
timeout 2400 python -m pytest tests -m gpu -q -p no:cacheprovider ${PYTEST_ARGS} > $OUT/pytest_gpu.log 2>&1
echo "pytest rc=$?" >> $OUT/pytest_gpu.log
tail -30 $OUT/pytest_gpu.log
timeout 300 python __graft_entry__.py smoke > $OUT/smoke.log 2>&1; tail -2 $OUT/smoke.log
if [ -z "$NOBENCH" ]; then
  timeout 900 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --out $OUT/bench.jsonl 2>&1 | tail -1 | cut -c1-400
  SFS_TORCH_ALLOC=0 timeout 900 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --out $OUT/bench_pool.jsonl 2>&1 | tail -1 | cut -c1-400
fi
