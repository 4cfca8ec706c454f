#!/bin/bash
# ncu --set full (hot: --cache-control none) of the kernels named in VERDICT r01: CSR variant 5 and COO on
# R-MAT 2^22, fp32 DIA on the 128^3 stencil (cold and hot), ELL on the 1M-row band, and the mid-size corpus
# matrices of the ~1e6-nnz decade (CSR tile / COO / ELL / DIA), each one launch after warm-up.
OUT=${OUT:-gpurun_out}/ncu_r2
mkdir -p $OUT
cap() {  # name, matrix, formats, kernel regex, cache-control, extra micro args
  timeout 600 ncu --set full --import-source on --clock-control none --cache-control $5 -k regex:$4 -s 8 -c 1 \
    -o $OUT/$1 -f python tools/micro.py --matrix $2 --formats $3 --reps 12 --warmup 2 --no-cold $6 > $OUT/$1.log 2>&1
  echo "$1 rc=$?"
}
cap rmat_csr5 rmat22 CSR k_spmv_csr_tile none "--variant 5"
cap rmat_coo rmat22 COO k_spmv_coo none ""
cap st3d27f_dia_cold st3d27f DIA k_spmv_dia all ""
cap st3d27f_dia_hot st3d27f DIA k_spmv_dia none ""
cap band_ell band_big ELL k_spmv_ell all ""
cap c89_csr corpus-89 CSR k_spmv_csr none ""
cap c89_ell corpus-89 ELL k_spmv_ell none ""
cap c91_csr corpus-91 CSR k_spmv_csr_tile none ""
cap c91_coo corpus-91 COO k_spmv_coo none ""
cap c64_dia corpus-64 DIA k_spmv_dia none ""
cap c64_ell corpus-64 ELL k_spmv_ell none ""
cap c14_ell corpus-14 ELL k_spmv_ell none ""
for f in $OUT/*.ncu-rep; do
  ncu -i $f --page raw --csv > ${f%.ncu-rep}.raw.csv 2>/dev/null
  ncu -i $f --page details --csv > ${f%.ncu-rep}.details.csv 2>/dev/null
  ncu -i $f --page source --csv --print-source sass > ${f%.ncu-rep}.sass.csv 2>/dev/null
  gzip -f ${f%.ncu-rep}.sass.csv
done
rm -f $OUT/*.ncu-rep  # the reports are ~9 MB each; gpurun_out must stay < 64 MiB
du -sh $OUT; ls -la $OUT | head -60
