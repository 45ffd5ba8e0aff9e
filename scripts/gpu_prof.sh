#!/usr/bin/env bash
# ncu: launch list of one C4 search step + one --set full capture of each
# kernel in $KERNELS (one GPU; reports stay in gpurun_out/ for reading here).
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out
CFG=${CFG:-C4}
TAG=${TAG:-r02}
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --profile-from-start off \
  --log-file gpurun_out/${TAG}_launches_${CFG}.csv python scripts/traffic_probe.py --config $CFG --warm 2 > gpurun_out/${TAG}_launches_${CFG}.log 2>&1
echo "launch list rc=$?"
for k in ${KERNELS:-k_wtile_count}; do
  timeout 900 ncu --set full --clock-control none --import-source on \
    -k "regex:${k}" -c 1 -o gpurun_out/${TAG}_prof_${CFG}_${k} -f \
    python scripts/traffic_probe.py --config $CFG > gpurun_out/${TAG}_prof_${CFG}_${k}.log 2>&1
  echo "full $k rc=$?"
done
