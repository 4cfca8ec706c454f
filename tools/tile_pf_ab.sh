#!/bin/bash
# A/B: CSR tile kernel with next-chunk prefetch (SFS_TILE_PF=<min nnz>) vs without, race + micro.
cd ${GRAFT_REPO_ROOT:-.}
[ -z "$NOTEST" ] && SFS_TILE_PF=0 timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider -x -k "tolerance or tile_edges or split_rows" 2>&1 | tail -3
IDS=$(python -c "print(','.join(str(i) for i in range(200)))")
for T in -1 0 1000000 4000000; do
  SFS_TILE_PF=$T python tools/race_probe.py --ids $IDS --mask 1 --rounds 1 --csr-variant 3 --tag pf$T --json gpurun_out/tile_pf.jsonl --quiet
done
for T in -1 0; do for M in st3d27 band_big uniform_big; do SFS_TILE_PF=$T python tools/micro.py --matrix $M --formats CSR --variant 3 --reps 30 --json gpurun_out/tile_pf_micro$T.jsonl > /dev/null 2>&1; done; python tools/show_micro.py gpurun_out/tile_pf_micro$T.jsonl; done
