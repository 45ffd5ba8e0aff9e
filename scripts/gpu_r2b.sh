#!/usr/bin/env bash
# round 2, call B: GPU tests, output-heavy points, bench, racecheck.
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out
echo "== pytest -m gpu"; timeout 2400 python -m pytest tests -m gpu -q --timeout=1200 ${PYTEST_ARGS:-} > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"
tail -5 gpurun_out/pytest_gpu.log
echo "== heavy"; timeout 900 python scripts/heavy_points.py > gpurun_out/heavy.jsonl 2> gpurun_out/heavy.err; echo "heavy rc=$?"; cat gpurun_out/heavy.jsonl | cut -c1-400
echo "== bench"; timeout 1200 python bench.py --gpus 1 --steps 20 --warmup 5 > gpurun_out/bench.log 2>&1; echo "bench rc=$?"
tail -c 300 gpurun_out/bench.log
if [ -n "${SANITIZE:-}" ]; then
  timeout 900 compute-sanitizer --tool racecheck --error-exitcode 9 python scripts/sanitize_run.py > gpurun_out/sanitize_racecheck.log 2>&1; echo "racecheck rc=$?"; tail -3 gpurun_out/sanitize_racecheck.log
  timeout 900 compute-sanitizer --tool memcheck --error-exitcode 9 python scripts/sanitize_run.py > gpurun_out/sanitize_memcheck.log 2>&1; echo "memcheck rc=$?"; tail -3 gpurun_out/sanitize_memcheck.log
fi
