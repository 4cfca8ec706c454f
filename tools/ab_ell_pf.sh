#!/bin/bash
# A/B of the next-batch L2 prefetch in the ELL kernel: SFS_ELL_PF_MB=-1 (never) vs the default gate (slab > 256 MB).
cd ${GRAFT_REPO_ROOT:-.}
O=gpurun_out
for PF in -1 256; do
  export SFS_ELL_PF_MB=$PF
  rm -f $O/epf_micro$PF.jsonl
  for M in st3d27f st3d27 blockdiag_big uniform_big band_big; do
    timeout 300 python tools/micro.py --matrix $M --formats ELL --reps 30 --json $O/epf_micro$PF.jsonl > /dev/null 2>&1
  done
  echo "SFS_ELL_PF_MB=$PF"; python tools/show_micro.py $O/epf_micro$PF.jsonl 2>&1 | grep -E "^[a-z]|ELL"
done
for PF in -1 256 -1 256; do
  export SFS_ELL_PF_MB=$PF
  timeout 600 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 0 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('PF_MB=$PF', round(d['value'],2), round(d['ms_per_step'],1), {k:round(v['spmv_time_s'],5) for k,v in d['per_format'].items()})"
done
