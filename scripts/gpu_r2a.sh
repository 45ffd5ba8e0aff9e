#!/usr/bin/env bash
# round 2, call A: GPU tests, smoke, bench (default args as the driver runs
# them), sanitizers on the current kernels.
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out
nvidia-smi > gpurun_out/smi.txt 2>&1
nproc > gpurun_out/nproc.txt
echo "== pytest -m gpu"; timeout 2400 python -m pytest tests -m gpu -q -x --timeout=1200 -rA ${PYTEST_ARGS:-} > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"
tail -5 gpurun_out/pytest_gpu.log
echo "== smoke"; timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"
echo "== bench"; timeout 1200 python bench.py --gpus 1 --steps 20 --warmup 5 > gpurun_out/bench.log 2>&1; echo "bench rc=$?"
tail -c 600 gpurun_out/bench.log
if [ -n "${SANITIZE:-}" ]; then bash scripts/gpu_sanitize.sh; fi
