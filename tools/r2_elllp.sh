#!/bin/bash
# ELL slot-parts as lanes of one warp (shuffle reduction) vs parts in different warps (smem + barriers).
OUT=${OUT:-gpurun_out}
mkdir -p $OUT
timeout 1800 python -m pytest -q -p no:cacheprovider -m gpu tests/test_gpu_parity.py tests/test_gpu_configs.py tests/test_gpu_dist.py tests/test_gpu_push_full.py > $OUT/pytest_elllp.log 2>&1
echo "pytest rc=$?"; tail -3 $OUT/pytest_elllp.log
for v in 0 1; do SFS_ELL_LP=$v timeout 900 python tools/race_probe.py --ids $(python -c "print(','.join(map(str,range(200))))") --mask 12 --rounds 2 --quiet --tag lp$v --json $OUT/elllp_race.jsonl; done
