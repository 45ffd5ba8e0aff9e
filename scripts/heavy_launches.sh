#!/usr/bin/env bash
# ncu launch list (gpu__time_duration per launch) of one search at each
# output-heavy point; summarised per kernel for the last search call.
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out
for P in ${POINTS:-C2:8 S2:1}; do
  f=gpurun_out/heavy_$(echo $P | tr : _)
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $f.csv \
    python scripts/heavy_points.py --points $P --reps 1 > $f.log 2>&1
  echo "$P rc=$?"
done
