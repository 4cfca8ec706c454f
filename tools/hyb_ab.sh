cd ${GRAFT_REPO_ROOT:-.}
[ -z "$NOTEST" ] && timeout 1200 python -m pytest tests -m gpu -q -p no:cacheprovider -x 2>&1 | tail -4
IDS=1,9,17,33,45,57,73,77,85,89,97,101,113,129,133,137,145,149,153,165,169,173,185,14,22,46,74,86,98,102,118,126,158,174,186,190,0,28,40,48,52,60,80,84,144,148,152,156,164,184
P="--ids $IDS --mask 12 --rounds 2"
SFS_LIB=$PWD/paper_conf_icppw_dhandhaniadpbl21_b200/libsfs_old.so python tools/race_probe.py $P --tag old --json gpurun_out/hyb_ab.jsonl --quiet
for T in default 32,4 32,8 32,16 64,32 1000,1000 0,0; do
  if [ $T = default ]; then unset SFS_HYB_ROWWISE; else export SFS_HYB_ROWWISE=$T; fi
  python tools/race_probe.py $P --tag new_$T --json gpurun_out/hyb_ab.jsonl --quiet
done
