#!/usr/bin/env bash
# Full verification call: every -m gpu test, smoke, the bench as the driver
# runs it, sanitizers on the current kernels, ncu launch list + pass-1 capture.
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out
TAG=${TAG:-r02}
nvidia-smi > gpurun_out/${TAG}_smi.txt 2>&1
echo "== pytest -m gpu"; timeout 2400 python -m pytest tests -m gpu -q --timeout=1200 -rA > gpurun_out/${TAG}_pytest_gpu.log 2>&1; echo "pytest rc=$?"
tail -3 gpurun_out/${TAG}_pytest_gpu.log
cp gpurun_out/parity_summary.json gpurun_out/${TAG}_parity_summary.json 2>/dev/null
echo "== smoke"; timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${TAG}_smoke.log 2>&1; echo "smoke rc=$?"; tail -1 gpurun_out/${TAG}_smoke.log
echo "== bench"; timeout 1200 python bench.py --gpus 1 --steps 20 --warmup 5 > gpurun_out/${TAG}_bench.log 2>&1; echo "bench rc=$?"
tail -c 400 gpurun_out/${TAG}_bench.log
echo "== reference arm"; timeout 600 python bench.py --impl reference --gpus 1 --steps 20 --warmup 5 > gpurun_out/${TAG}_ref.log 2>&1; echo "ref rc=$?"
if [ -z "${NO_SANITIZE:-}" ]; then
for tool in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool --error-exitcode 9 python scripts/sanitize_run.py > gpurun_out/${TAG}_sanitize_$tool.log 2>&1
  echo "$tool rc=$?"; tail -1 gpurun_out/${TAG}_sanitize_$tool.log
done
fi
TAG=$TAG KERNELS="${KERNELS:-k_wtile_count}" bash scripts/gpu_prof.sh
echo "== outliers"; timeout 900 python scripts/outlier_bench.py --plain --reps 20 > gpurun_out/${TAG}_outliers.jsonl 2> gpurun_out/${TAG}_outliers.err; echo "outliers rc=$?"; cut -c1-160 gpurun_out/${TAG}_outliers.jsonl
