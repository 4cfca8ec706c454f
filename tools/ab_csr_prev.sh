#!/bin/bash
cd ${GRAFT_REPO_ROOT:-.}
[ -z "$NOTEST" ] && timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider -x -k "tolerance or tile or split_rows or bitmap or x_ones or unit_vector or configs" 2>&1 | tail -3
IDS=$(python -c "print(','.join(str(i) for i in range(200)))")
for L in _prev ""; do SFS_LIB=$PWD/paper_conf_icppw_dhandhaniadpbl21_b200/libsfs$L.so python tools/race_probe.py --ids $IDS --mask 1 --rounds 1 --tag lib$L --json gpurun_out/ab_csr_prev.jsonl --quiet; done
for L in _prev ""; do for M in st3d27 band_big uniform_big; do SFS_LIB=$PWD/paper_conf_icppw_dhandhaniadpbl21_b200/libsfs$L.so python tools/micro.py --matrix $M --formats CSR --reps 30 --json gpurun_out/ab_csr_prev_micro$L.jsonl > /dev/null 2>&1; done; python tools/show_micro.py gpurun_out/ab_csr_prev_micro$L.jsonl | grep -v "^ *COO\|ELL\|HYB\|DIA"; done
