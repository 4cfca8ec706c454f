#!/bin/bash
# COO with split-row zeroing (no full zero pass) for matrices without empty rows vs the full zero pass.
OUT=${OUT:-gpurun_out}
mkdir -p $OUT
timeout 1800 python -m pytest -q -p no:cacheprovider -m gpu tests/test_gpu_parity.py tests/test_gpu_configs.py tests/test_gpu_dist.py tests/test_gpu_race.py > $OUT/pytest_coosz.log 2>&1
echo "pytest rc=$?"; tail -3 $OUT/pytest_coosz.log
for v in 0 1; do SFS_COO_SPLIT_ZERO=$v timeout 900 python tools/race_probe.py --ids $(python -c "print(','.join(map(str,range(200))))") --mask 2 --rounds 2 --quiet --tag coosz$v --json $OUT/coosz_race.jsonl; done
rm -f $OUT/coosz.jsonl
for v in 0 1; do SFS_COO_SPLIT_ZERO=$v timeout 600 python tools/micro.py --matrix st3d27,uniform_big,powerlaw_big --formats COO --reps 30 --json $OUT/coosz.jsonl > /dev/null 2>&1; done
python - <<'PY'
import json
for l in open('gpurun_out/coosz.jsonl'):
    d=json.loads(l); r=d['formats']['COO']
    print(d['env'].get('SFS_COO_SPLIT_ZERO','1'), d['matrix'], round(r['hot_us'],1), round(r['cold_us'],1))
PY
