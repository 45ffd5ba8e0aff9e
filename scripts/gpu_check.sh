#!/usr/bin/env bash
# One gpurun call: GPU tests, smoke, a short bench, logs to gpurun_out/.
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out
nvidia-smi > gpurun_out/smi.txt 2>&1
echo "== pytest -m gpu" ; timeout ${PYTEST_TIMEOUT:-1500} python -m pytest tests -m gpu -q --timeout=600 ${PYTEST_ARGS:-} > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"
tail -8 gpurun_out/pytest_gpu.log
echo "== smoke" ; timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"
tail -2 gpurun_out/smoke.log
echo "== bench" ; timeout ${BENCH_TIMEOUT:-900} python bench.py ${BENCH_ARGS:---steps 5 --warmup 3 --cpu-seconds 5} > gpurun_out/bench.log 2>&1; echo "bench rc=$?"
tail -2 gpurun_out/bench.log
if [ -n "${PROFILE:-}" ]; then bash scripts/gpu_profile.sh; fi
