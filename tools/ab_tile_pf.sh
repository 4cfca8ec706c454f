#!/bin/bash
# A/B of the next-chunk L2 prefetch in the CSR tile kernel (libsfs_pf.so built with -DSFS_TILE_PF) vs default.
cd ${GRAFT_REPO_ROOT:-.}
O=gpurun_out
for L in "" _pf; do
  export SFS_LIB=$PWD/paper_conf_icppw_dhandhaniadpbl21_b200/libsfs$L.so
  rm -f $O/tpf_micro$L.jsonl
  for M in st3d27 st3d27f band_big blockdiag_big uniform_big powerlaw_big; do
    timeout 300 python tools/micro.py --matrix $M --formats CSR --reps 30 --json $O/tpf_micro$L.jsonl > /dev/null 2>&1
  done
  echo "lib$L"; python tools/show_micro.py $O/tpf_micro$L.jsonl 2>&1 | grep -E "^[a-z]|CSR"
done
for L in "" _pf "" _pf; do
  export SFS_LIB=$PWD/paper_conf_icppw_dhandhaniadpbl21_b200/libsfs$L.so
  timeout 600 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 0 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('lib$L', round(d['value'],2), round(d['ms_per_step'],1), {k:round(v['spmv_time_s'],5) for k,v in d['per_format'].items()})"
done
