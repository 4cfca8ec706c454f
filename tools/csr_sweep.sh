#!/bin/bash
# CSR race time of every corpus-200 matrix under each CSR kernel (Q17 rule study).
cd ${GRAFT_REPO_ROOT:-.}
IDS=$(python -c "print(','.join(str(i) for i in range(200)))")
for V in 0 1 2 3; do python tools/race_probe.py --ids $IDS --mask 1 --rounds 1 --csr-variant $V --tag v$V --json gpurun_out/csr_sweep.jsonl --quiet; done
