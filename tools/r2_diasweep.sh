#!/bin/bash
# fp32 DIA sweep on the bandwidth-bound matrices: diagonal split S, L2 prefetch distance, strided vs v4 kernel.
OUT=${OUT:-gpurun_out}
mkdir -p $OUT
rm -f $OUT/diasweep.jsonl
for S in 1 2 4; do for PF in 0 1 2; do
  SFS_DIA_S=$S SFS_DIA_PF=$PF timeout 300 python tools/micro.py --matrix st3d27f,band_big_f32 --formats DIA --reps 30 --json $OUT/diasweep.jsonl > /dev/null 2>&1
done; done
for S in 1 2 4; do SFS_DIA_F4=0 SFS_DIA_S=$S timeout 300 python tools/micro.py --matrix st3d27f,band_big_f32 --formats DIA --reps 30 --json $OUT/diasweep.jsonl > /dev/null 2>&1; done
python - <<'PY'
import json
for l in open('gpurun_out/diasweep.jsonl'):
    d=json.loads(l); r=d['formats']['DIA']; e=d.get('env',{})
    print(d['matrix'], e, round(r['hot_us'],1), round(r['cold_us'],1), round(r['cold_frac'],3))
PY
