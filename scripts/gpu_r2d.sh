#!/usr/bin/env bash
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out
echo "== pytest subset"; timeout 1800 python -m pytest tests -m gpu -q -x --timeout=900 -k "${PYTEST_K:-c0 or adversarial or spill or crowded or methods or huge or distinct or exclude or heavy or pipelined or stationary or merge or golden or paper_example}" > gpurun_out/pytest_gpu_d.log 2>&1; echo "pytest rc=$?"
tail -3 gpurun_out/pytest_gpu_d.log
echo "== ab"; bash scripts/ab.sh
echo "== heavy"; timeout 900 python scripts/heavy_points.py --points ${POINTS:-C2:8 S2:1} > gpurun_out/heavy.jsonl 2> gpurun_out/heavy.err; echo "heavy rc=$?"; cut -c1-420 gpurun_out/heavy.jsonl; tail -3 gpurun_out/heavy.err
