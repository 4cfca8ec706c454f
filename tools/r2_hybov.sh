#!/bin/bash
# Overlapped HYB (zero -> ELL part atomics -> COO part atomics, concurrent) vs the ELL -> COO<ACCUM> pair.
OUT=${OUT:-gpurun_out}
mkdir -p $OUT
timeout 1800 python -m pytest -q -p no:cacheprovider -m gpu tests/test_gpu_parity.py tests/test_gpu_configs.py tests/test_gpu_dist.py tests/test_gpu_push_full.py > $OUT/pytest_hybov.log 2>&1
echo "pytest rc=$?"; tail -3 $OUT/pytest_hybov.log
rm -f $OUT/hybov.jsonl
for ov in 0 1; do SFS_HYB_OVERLAP=$ov timeout 600 python tools/micro.py --matrix rmat22,powerlaw_big,corpus-91,corpus-3 --formats HYB --reps 30 --json $OUT/hybov.jsonl > /dev/null 2>&1; done
python - <<'PY'
import json
for l in open('gpurun_out/hybov.jsonl'):
    d=json.loads(l); r=d['formats']['HYB']
    print(d['env'].get('SFS_HYB_OVERLAP','1'), d['matrix'], round(r['hot_us'],1), round(r['cold_us'],1))
PY
for ov in 0 1; do SFS_HYB_OVERLAP=$ov timeout 900 python tools/race_probe.py --ids $(python -c "print(','.join(map(str,range(3,200,4))))") --mask 8 --rounds 2 --quiet --tag ov$ov --json $OUT/hybov_race.jsonl; done
