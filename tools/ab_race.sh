#!/bin/bash
# A/B race timings of libsfs builds (libsfs$L.so for L in $LIBS) on a few corpus matrices.
cd ${GRAFT_REPO_ROOT:-.}
[ -n "$TESTS" ] && timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider -x ${TESTS/all/} 2>&1 | tail -4
for L in ${LIBS:-_old ""}; do
  SFS_LIB=$PWD/paper_conf_icppw_dhandhaniadpbl21_b200/libsfs$L.so timeout 300 python tools/race_probe.py --tag "lib$L" ${PROBE_ARGS} --json gpurun_out/ab_race.jsonl 2>&1 | tail -${TAIL:-17}
done
