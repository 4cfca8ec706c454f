#!/bin/bash
# A/B of the TMA-staged fp32 DIA kernel: GPU parity subset, micro (fp32 / fp64 stencil, band), corpus DIA race, bench.
cd ${GRAFT_REPO_ROOT:-.}
O=gpurun_out
timeout 900 python -m pytest tests -m gpu -q -x -k "dia or DIA or config3" > $O/tma_pytest.log 2>&1; tail -3 $O/tma_pytest.log
for L in _old ""; do
  export SFS_LIB=$PWD/paper_conf_icppw_dhandhaniadpbl21_b200/libsfs$L.so
  for M in st3d27f; do
    timeout 300 python tools/micro.py --matrix $M --formats DIA --reps 30 --json $O/tma_micro$L.jsonl > /dev/null 2>&1
  done
  python tools/show_micro.py $O/tma_micro$L.jsonl 2>&1 | tail -6
  timeout 300 python tools/race_probe.py --tag "lib$L" --mask 16 --json $O/tma_race.jsonl 2>&1 | tail -6
done
for L in _old ""; do
  export SFS_LIB=$PWD/paper_conf_icppw_dhandhaniadpbl21_b200/libsfs$L.so
  timeout 600 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 0 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('lib$L', round(d['value'],2), round(d['ms_per_step'],1), {k:round(v['spmv_time_s'],5) for k,v in d['per_format'].items()})"
done
