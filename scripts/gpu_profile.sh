#!/usr/bin/env bash
# ncu launch list of one step + one full capture per listed kernel (one GPU).
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out
CFG=${CFG:-C4}
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file gpurun_out/launches_${CFG}.csv python scripts/profile_step.py --config $CFG --warmup 1 --steps 1 > gpurun_out/launches_${CFG}.log 2>&1
echo "launch list rc=$?"
for k in ${KERNELS:-k_tile_count k_gather k_rs_scatter k_insert k_count_cells}; do
  timeout 600 ncu --set full --clock-control none --import-source on \
    -k "regex:${k}" -c 1 -o gpurun_out/prof_${CFG}_${k} -f \
    python scripts/profile_step.py --config $CFG --warmup 0 --steps 1 > gpurun_out/prof_${CFG}_${k}.log 2>&1
  echo "full $k rc=$?"
done
