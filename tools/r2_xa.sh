#!/bin/bash
OUT=${OUT:-gpurun_out}
mkdir -p $OUT
timeout 1800 python -m pytest -q -p no:cacheprovider -m gpu tests/test_gpu_parity.py tests/test_gpu_configs.py tests/test_gpu_push_full.py > $OUT/pytest_xa.log 2>&1
echo "pytest rc=$?"; tail -3 $OUT/pytest_xa.log
rm -f $OUT/xa.jsonl
for xa in 0 1; do SFS_DIA_XA=$xa timeout 300 python tools/micro.py --matrix st3d27f,band_big_f32 --formats DIA --reps 30 --json $OUT/xa.jsonl > /dev/null 2>&1; done
python - <<'PY'
import json
for l in open('gpurun_out/xa.jsonl'):
    d=json.loads(l); r=d['formats']['DIA']; e=d.get('env',{})
    print(d['matrix'], e, round(r['hot_us'],1), round(r['cold_us'],1), round(r['cold_frac'],3), d['clocks']['sm_mhz'])
PY
IDS=$(python -c "print(','.join(str(i) for i in range(200) if (i>>2)&1))")
for xa in 0 1; do SFS_DIA_XA=$xa timeout 900 python tools/race_probe.py --ids $IDS --mask 16 --rounds 2 --quiet --tag xa$xa --json $OUT/xa_race.jsonl; done
