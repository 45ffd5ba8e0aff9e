#!/usr/bin/env bash
# device search time per config with and without the query sort
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/../..}"
for v in 0 1000000000; do
  echo "== DTS_QSORT_MIN=$v"
  DTS_QSORT_MIN=$v timeout 600 python scripts/probes/search_overhead.py ${CFGS:-C1 C2 C3 S1 S2 S3} 2>&1 | grep "time_kernels False"
done
