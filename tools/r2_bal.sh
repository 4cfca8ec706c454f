#!/bin/bash
# Balanced grids (equal row blocks per CTA) vs min(items, resident CTAs): parity, micro, corpus race.
OUT=${OUT:-gpurun_out}
mkdir -p $OUT
timeout 1800 python -m pytest -q -p no:cacheprovider -m gpu tests/test_gpu_parity.py tests/test_gpu_configs.py tests/test_gpu_push_full.py -k "not S" > $OUT/pytest_bal.log 2>&1
echo "pytest rc=$?"; tail -2 $OUT/pytest_bal.log
rm -f $OUT/bal.jsonl
for b in 0 1; do SFS_BALANCED_GRID=$b timeout 600 python tools/micro.py --matrix st3d27f,st3d27,band_big,band_big_f32,blockdiag_big,uniform_big --formats CSR,ELL,DIA --reps 30 --json $OUT/bal.jsonl > /dev/null 2>&1; done
python - <<'PY'
import json
rows=[json.loads(l) for l in open('gpurun_out/bal.jsonl')]
for d in rows:
    e=d.get('env',{}).get('SFS_BALANCED_GRID','1')
    print(e, d['matrix'], {k:(round(r['hot_us'],1), round(r['cold_us'],1)) for k,r in d['formats'].items() if isinstance(r,dict)})
PY
for b in 0 1; do SFS_BALANCED_GRID=$b timeout 900 python tools/race_probe.py --ids $(python -c "print(','.join(map(str,range(200))))") --rounds 1 --quiet --tag bal$b --json $OUT/bal_race.jsonl; done
