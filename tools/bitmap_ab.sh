#!/bin/bash
# CSR tile (3) vs bitmap tile (4): parity subset, whole-corpus CSR race, large-matrix micro.
cd ${GRAFT_REPO_ROOT:-.}
[ -z "$NOTEST" ] && timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider -x -k "tolerance or tile or split_rows or bitmap" 2>&1 | tail -3
IDS=$(python -c "print(','.join(str(i) for i in range(200)))")
for V in 3 4; do python tools/race_probe.py --ids $IDS --mask 1 --rounds 1 --csr-variant $V --tag v$V --json gpurun_out/bitmap_ab.jsonl --quiet; done
for M in st3d27 band_big uniform_big blockdiag_big powerlaw_big; do python tools/micro.py --matrix $M --formats CSR --variants 3,4 --reps 30 --json gpurun_out/bitmap_micro.jsonl > /dev/null 2>&1; done
python tools/show_micro.py gpurun_out/bitmap_micro.jsonl
