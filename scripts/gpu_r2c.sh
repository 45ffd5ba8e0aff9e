#!/usr/bin/env bash
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out
echo "== pytest subset"; timeout 1800 python -m pytest tests -m gpu -q --timeout=900 -k "${PYTEST_K:-spill or heavy or huge or crowded or non_distinct or c0 or adversarial}" > gpurun_out/pytest_gpu_c.log 2>&1; echo "pytest rc=$?"
tail -3 gpurun_out/pytest_gpu_c.log
echo "== heavy"; timeout 900 python scripts/heavy_points.py --points ${POINTS:-C2:8 S2:1 C2:2 S3:0.09} > gpurun_out/heavy.jsonl 2> gpurun_out/heavy.err; echo "heavy rc=$?"; cut -c1-420 gpurun_out/heavy.jsonl; tail -3 gpurun_out/heavy.err
