#!/usr/bin/env bash
# split pass 1: correctness subset, then A/B against the fused kernel
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out
echo "== pytest subset"; timeout 1200 python -m pytest tests -m gpu -q -x --timeout=600 -k "${PYTEST_K:-c0 or adversarial or c4 or crowded or exclude or spill or distinct or count or heavy}" > gpurun_out/pytest_g.log 2>&1; echo "pytest rc=$?"
tail -3 gpurun_out/pytest_g.log
VARIANTS="${VARIANTS:-fused|DTS_SPLIT=0|tree;split|X=1|tree;so8|X=1|ab/libdts_so8.so;ro12|X=1|ab/libdts_ro12.so}" AB_ARGS="--points C4:0.005 C4:0.02 C2:2 C2:8 C1:0.005" AB_OUT=abg bash scripts/ab_env.sh
