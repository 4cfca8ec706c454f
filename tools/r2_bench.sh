#!/bin/bash
# Round-2: targeted GPU tests + the default bench line (N=1) + the full-size push parity evidence.
OUT=${OUT:-gpurun_out}
mkdir -p $OUT
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider ${PYTEST_ARGS:-tests/test_gpu_race.py tests/test_gpu_dist.py tests/test_gpu_semisup.py} > $OUT/pytest_gpu.log 2>&1
echo "pytest rc=$?" >> $OUT/pytest_gpu.log
tail -15 $OUT/pytest_gpu.log
if [ -n "$PUSHFULL" ]; then timeout 900 python tests/push_parity_worker.py > $OUT/push_full_parity.jsonl 2>&1; echo "push worker rc=$?"; fi
timeout 1200 python bench.py ${BENCH_ARGS} --out $OUT/bench.jsonl > $OUT/bench.log 2>&1
echo "bench rc=$?"; tail -c 3000 $OUT/bench.log
