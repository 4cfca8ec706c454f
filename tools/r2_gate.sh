#!/bin/bash
# Round-2 ncu gate after the TMA DIA / ELL kernels: best kernel per structure class at footprint >> L2, one
# launch after warm-up, cold (--cache-control all), clocks free; per-class hot / cold micro with clocks; the
# bench launch list; ncu --set full of the TMA kernels (SASS source page: UBLKCP / SYNCS evidence).
OUT=${OUT:-gpurun_out}/r2gate
mkdir -p $OUT
M="gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,dram__throughput.avg.pct_of_peak_sustained_elapsed,lts__t_sector_hit_rate.pct,l1tex__t_sector_hit_rate.pct,lts__t_sectors_srcunit_tex.sum,sm__warps_active.avg.pct_of_peak_sustained_active"
gate() {  # name matrix format regex
  timeout 600 ncu --metrics $M --cache-control all --clock-control none -k regex:$4 -s 8 -c 1 --csv \
    python tools/micro.py --matrix $2 --formats $3 --reps 10 --warmup 2 --no-cold > $OUT/gate_$1.csv 2>/dev/null
  echo "gate $1 rc=$?"
}
gate st3d27_dia st3d27 DIA k_spmv_dia
gate st3d27_ell st3d27 ELL k_spmv_ell
gate st3d27f_dia st3d27f DIA k_spmv_dia
gate st3d27f_ell st3d27f ELL k_spmv_ell
gate band_dia band_big DIA k_spmv_dia
gate band_ell band_big ELL k_spmv_ell
gate band32_dia band_big_f32 DIA k_spmv_dia
gate blockdiag_ell blockdiag_big ELL k_spmv_ell
gate blockdiag_csr blockdiag_big CSR k_spmv_csr
gate uniform_ell uniform_big ELL k_spmv_ell
gate uniform_coo uniform_big COO k_spmv_coo
gate powerlaw_csr powerlaw_big CSR k_spmv_csr
gate powerlaw_coo powerlaw_big COO k_spmv_coo
gate rmat_coo rmat22 COO k_spmv_coo
gate rmat_csr rmat22 CSR k_spmv_csr
timeout 900 python tools/micro.py --matrix st3d27,st3d27f,band_big,band_big_f32,blockdiag_big,uniform_big,powerlaw_big,rmat22 --reps 30 --json $OUT/class_micro.jsonl > $OUT/class_micro.log 2>&1
echo "micro rc=$?"
for c in "st3d27f DIA k_spmv_dia_tma" "st3d27 ELL k_spmv_ell_tma" "uniform_big COO k_spmv_coo"; do
  set -- $c
  timeout 600 ncu --set full --import-source on --clock-control none --cache-control all -k regex:$3 -s 8 -c 1 \
    -o $OUT/full_$1_$2 -f python tools/micro.py --matrix $1 --formats $2 --reps 10 --warmup 2 --no-cold > /dev/null 2>&1
  echo "full $1 $2 rc=$?"
done
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 9000 --csv --log-file $OUT/launches_first9k.csv \
  python bench.py --steps 1 --warmup 0 --no-cpu-baseline --rowpart-N 0 --predictor-nc 0 --e2e-steps 0 > /dev/null 2>&1
echo "launch list rc=$?"; gzip -f $OUT/launches_first9k.csv; du -sh $OUT
