#!/usr/bin/env bash
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out
echo "== pytest subset"; timeout 1500 python -m pytest tests -m gpu -q -x --timeout=600 -k "${PYTEST_K:-sorted or layout or c4 or adversarial or deferred or spill or heavy or c0}" > gpurun_out/pytest_j.log 2>&1; echo "pytest rc=$?"
tail -3 gpurun_out/pytest_j.log
VARIANTS="${VARIANTS:-multi|DTS_QSORT_DROP=19|tree;one|X=1|tree}" AB_ARGS="${AB_ARGS:---points C4:0.005 C4:0.02 C2:8 S2:1}" AB_OUT=abj bash scripts/ab_env.sh
DTS_TRACE=1 NPTS=1 python scripts/overhead_probe.py 2> gpurun_out/trace_j.err | head -2; sed -n '10,12p' gpurun_out/trace_j.err
