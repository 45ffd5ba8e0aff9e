#!/usr/bin/env bash
# One gpurun call: bench line, launch list and full ncu captures of the top
# kernels of one C4 step (summarised locally into profiles/ afterwards).
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out
timeout 900 python bench.py ${BENCH_ARGS:-} > gpurun_out/bench_full.log 2>&1; echo "bench rc=$?"
tail -1 gpurun_out/bench_full.log > gpurun_out/bench_line.json
KERNELS="${KERNELS:-k_wtile_count k_onesweep k_gather_cells k_insert_blocks_lane k_bounds_keys}" \
  bash scripts/gpu_profile.sh
