#!/bin/bash
cd ${GRAFT_REPO_ROOT:-.}
O=gpurun_out
timeout 600 python -m pytest tests -m gpu -q -x -k "dia or DIA or parity" > $O/xvec_pytest.log 2>&1; tail -2 $O/xvec_pytest.log
for L in _old ""; do
  export SFS_LIB=$PWD/paper_conf_icppw_dhandhaniadpbl21_b200/libsfs$L.so
  for M in st3d27f st3d27; do
    timeout 300 python tools/micro.py --matrix $M --formats DIA,ELL --reps 30 --json $O/xvec_micro$L.jsonl > /dev/null 2>&1
  done
  python tools/show_micro.py $O/xvec_micro$L.jsonl 2>&1 | tail -8
  timeout 300 python tools/race_probe.py --tag "lib$L" --mask 16 --json $O/xvec_race.jsonl 2>&1 | tail -5
done
for L in _old "" _old ""; do
  export SFS_LIB=$PWD/paper_conf_icppw_dhandhaniadpbl21_b200/libsfs$L.so
  timeout 600 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 0 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('lib$L', round(d['value'],2), round(d['ms_per_step'],1), {k:round(v['spmv_time_s'],5) for k,v in d['per_format'].items()})"
done
