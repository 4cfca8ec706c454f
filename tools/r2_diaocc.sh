#!/bin/bash
# fp32 DIA occupancy / batch A/B builds: default (4 diagonals x 4 CTAs/SM), kb2c5, kb2c6, kb4c5.
OUT=${OUT:-gpurun_out}
mkdir -p $OUT
rm -f $OUT/diaocc.jsonl
IDS=$(python -c "print(','.join(str(i) for i in range(200) if (i>>2)&1))")
for v in "" _kb2c5 _kb2c6 _kb4c5; do
  SFS_LIB=paper_conf_icppw_dhandhaniadpbl21_b200/libsfs$v.so timeout 300 python tools/micro.py --matrix st3d27f,band_big_f32 --formats DIA --reps 30 --json $OUT/diaocc.jsonl > /dev/null 2>&1
  SFS_LIB=paper_conf_icppw_dhandhaniadpbl21_b200/libsfs$v.so timeout 600 python tools/race_probe.py --ids $IDS --mask 16 --rounds 2 --quiet --tag "lib$v" --json $OUT/diaocc_race.jsonl
done
python - <<'PY'
import json
for l in open('gpurun_out/diaocc.jsonl'):
    d=json.loads(l); r=d['formats']['DIA']
    print(d['env'].get('SFS_LIB','default').split('/')[-1], d['matrix'], round(r['hot_us'],1), round(r['cold_us'],1), round(r['cold_frac'],3))
PY
