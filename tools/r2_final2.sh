#!/bin/bash
# After the overlapped HYB: the race traffic / L2 sectors per format, then the driver's bench command.
bash tools/r2_traffic.sh
cp gpurun_out/r2tr/traffic_corpus200.json profiles/r02/traffic_corpus200.json 2>/dev/null
OUT=gpurun_out/r2final2
mkdir -p $OUT
timeout 1500 python bench.py --gpus 1 --steps 20 --warmup 5 --out $OUT/bench.jsonl > $OUT/bench.log 2>&1
echo "bench rc=$?"; python -c "
import json; d=json.loads(open('$OUT/bench.jsonl').readlines()[-1])
print(d['value'], d['e2e']['value'], d['roofline']['frac'], d['roofline']['kernel'], d['roofline'].get('l2',{}).get('frac'), d['clocks'])
print({k:(round(v['spmv_time_s'],4), round(v['gbs'])) for k,v in d['per_format'].items()})"
