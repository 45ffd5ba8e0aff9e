#!/usr/bin/env bash
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out
echo "== pytest subset"; timeout 1800 python -m pytest tests -m gpu -q -x --timeout=900 -k "${PYTEST_K:-count or budget or spill or c0 or adversarial or distinct or exclude or costs or concurrent or multirank}" > gpurun_out/pytest_gpu_e.log 2>&1; echo "pytest rc=$?"
tail -3 gpurun_out/pytest_gpu_e.log
echo "== s2 d=5"; timeout 1500 python scripts/s2_d5.py 5.0 > gpurun_out/s2_d5.json 2> gpurun_out/s2_d5.err; echo "s2 rc=$?"; cat gpurun_out/s2_d5.json; tail -3 gpurun_out/s2_d5.err
