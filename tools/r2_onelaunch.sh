#!/bin/bash
# One-launch COO / CSR tile: parity first, then the corpus race A/B (SFS_ONE_LAUNCH=0/1) and the bench.
OUT=${OUT:-gpurun_out}
mkdir -p $OUT
timeout 1800 python -m pytest -q -p no:cacheprovider -m gpu tests/test_gpu_parity.py tests/test_gpu_configs.py tests/test_gpu_race.py tests/test_gpu_sfsgen_device.py > $OUT/pytest_ol.log 2>&1
echo "pytest rc=$?"; tail -6 $OUT/pytest_ol.log
for ol in 0 1; do SFS_ONE_LAUNCH=$ol timeout 900 python tools/race_probe.py --ids $(python -c "print(','.join(map(str,range(0,200,2))))") --rounds 2 --quiet --tag ol$ol --json $OUT/ol_race.jsonl; done
for ol in 0 1; do SFS_ONE_LAUNCH=$ol timeout 900 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --rowpart-N 0 --predictor-nc 0 --out $OUT/bench_ol$ol.jsonl 2>&1 | tail -1 | cut -c1-200; done
