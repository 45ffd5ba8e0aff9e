#!/usr/bin/env bash
# ncu launch list of one step + full captures of the top kernels (one GPU).
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out
CFG=${CFG:-C4}
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file gpurun_out/launches_${CFG}.csv python scripts/profile_step.py --config $CFG --warmup 1 --steps 1 > gpurun_out/launches_${CFG}.log 2>&1
echo "launch list rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on \
  -k "regex:${KREGEX:-k_pass|k_gather|k_rs_scatter|k_keys|k_bounds}" -s ${SKIP:-0} -c ${COUNT:-8} \
  -o gpurun_out/prof_${CFG} -f python scripts/profile_step.py --config $CFG --warmup 0 --steps 1 > gpurun_out/prof_${CFG}.log 2>&1
echo "full rc=$?"
