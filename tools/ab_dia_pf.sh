#!/bin/bash
# A/B of the L2 slab prefetch distance in the fp32 DIA kernel (SFS_DIA_PF = 0 off, 1, 2, 3 batches ahead).
cd ${GRAFT_REPO_ROOT:-.}
O=gpurun_out
for PF in 0 1 2 3; do
  export SFS_DIA_PF=$PF
  rm -f $O/pf_micro_$PF.jsonl
  for M in st3d27f; do
    timeout 300 python tools/micro.py --matrix $M --formats DIA --reps 30 --json $O/pf_micro_$PF.jsonl > /dev/null 2>&1
  done
  echo "PF=$PF"; python tools/show_micro.py $O/pf_micro_$PF.jsonl 2>&1 | grep DIA
done
for PF in 0 2 0 2; do
  export SFS_DIA_PF=$PF
  timeout 600 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 0 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('PF=$PF', round(d['value'],2), round(d['ms_per_step'],1), {k:round(v['spmv_time_s'],5) for k,v in d['per_format'].items()})"
done
