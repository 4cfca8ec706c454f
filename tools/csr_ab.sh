#!/bin/bash
# CSR variants 3 (tile) vs 4 (TMA-staged tile) on the race, plus the parity tests that cover them.
cd ${GRAFT_REPO_ROOT:-.}
[ -z "$NOTEST" ] && timeout 1200 python -m pytest tests -m gpu -q -p no:cacheprovider -x -k "tolerance or tile_edges or split_rows" 2>&1 | tail -4
IDS=${IDS:-0,1,2,5,9,10,11,14,22,34,40,46,52,57,64,74,81,86,88,98,102,113,118,120,121,122,126,137,145,149,152,165,174,178,184}
for V in 3 4; do python tools/race_probe.py --ids $IDS --mask 1 --rounds 2 --csr-variant $V --tag v$V --json gpurun_out/csr_ab.jsonl --quiet; done
for M in st3d27 rmat22 uniform_big band_big; do python tools/micro.py --matrix $M --formats CSR --variants 3,4 --reps 30 --json gpurun_out/csr_ab_micro.jsonl > /dev/null 2>&1; done
python tools/show_micro.py gpurun_out/csr_ab_micro.jsonl
