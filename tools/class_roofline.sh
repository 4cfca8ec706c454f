#!/bin/bash
# Best kernel per structure class at footprints >> L2: per-format hot / cold GB/s (tools/micro.py) and an
# ncu --set full capture of each class's best kernel (dram / L2 throughput, stalls).
OUT=${OUT:-gpurun_out}
mkdir -p $OUT
rm -f $OUT/class_micro.jsonl
for M in st3d27 st3d27f band_big blockdiag_big uniform_big powerlaw_big rmat22; do
  timeout 300 python tools/micro.py --matrix $M --reps 30 --json $OUT/class_micro.jsonl > /dev/null 2>&1
done
python tools/show_micro.py $OUT/class_micro.jsonl > $OUT/class_micro.txt 2>&1
CAPS="cls_st3d27_dia:st3d27:DIA:-1:k_spmv_dia cls_band_dia:band_big:DIA:-1:k_spmv_dia cls_blockdiag_ell:blockdiag_big:ELL:-1:k_spmv_ell cls_uniform_ell:uniform_big:ELL:-1:k_spmv_ell cls_powerlaw_coo:powerlaw_big:COO:-1:k_spmv_coo cls_rmat_coo:rmat22:COO:-1:k_spmv_coo" \
  bash tools/profile_ncu.sh
for f in $OUT/ncu_cls_*.ncu-rep; do python tools/ncu_summary.py $f; done > $OUT/class_ncu.txt 2>&1
cat $OUT/class_micro.txt; grep -E "^==|dram_throughput|lts__throughput|duration" $OUT/class_ncu.txt
