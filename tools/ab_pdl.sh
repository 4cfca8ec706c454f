#!/bin/bash
# A/B: PDL on/off on the bench workload (1 timed step) + ncu of DIA fp32 st3d27
OUT=${OUT:-gpurun_out}
for P in 0 1; do
  SFS_PDL=$P timeout 600 python bench.py --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 0 --dump $OUT/dump_pdl$P.jsonl | python -c "import json,sys; d=json.loads(sys.stdin.readlines()[-1]); print('PDL=$P', d['value'], d['ms_per_step'])"
done
CAPS="dia3_st3d27f:st3d27f:DIA:-1:k_spmv_dia dia3_corpus8:corpus:8:DIA:-1:k_spmv_dia stream3_corpus5:corpus:5:CSR:-1:k_spmv_csr_stream" bash tools/profile_ncu.sh
