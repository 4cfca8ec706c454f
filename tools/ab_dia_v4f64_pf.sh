#!/bin/bash
# fp64 DIA: strided k_spmv_dia (default) vs consecutive-row k_spmv_dia_v4<double> with the L2 slab prefetch
# (SFS_DIA_V4_F64=1, SFS_DIA_PF=0/1/2).
cd ${GRAFT_REPO_ROOT:-.}
O=gpurun_out
run() { rm -f $O/v4f64_$1.jsonl; for M in st3d27 band_big; do timeout 300 python tools/micro.py --matrix $M --formats DIA --reps 30 --json $O/v4f64_$1.jsonl > /dev/null 2>&1; done; echo "$1"; python tools/show_micro.py $O/v4f64_$1.jsonl 2>&1 | grep -E "^[a-z]|DIA"; }
run default
SFS_DIA_V4_F64=1 SFS_DIA_PF=0 run v4pf0
SFS_DIA_V4_F64=1 SFS_DIA_PF=1 run v4pf1
SFS_DIA_V4_F64=1 SFS_DIA_PF=2 run v4pf2
