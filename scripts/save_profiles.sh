#!/usr/bin/env bash
# Copy the summaries of a scripts/gpu_full.sh run (TAG) from gpurun_out/ into
# profiles/ (tracked): bench and reference lines, parity summary, sanitizer
# tails, launch list, ncu summary of pass 1, outlier and heavy-point lines.
cd "$(dirname "$0")/.."
T=${1:?tag}
G=gpurun_out
tail -1 $G/${T}_bench.log > profiles/${T}_bench_C4.json
grep '^{' $G/${T}_ref.log | tail -1 > profiles/${T}_ref_C4.json
cp $G/${T}_parity_summary.json profiles/${T}_parity_summary.json 2>/dev/null
{
  for tool in memcheck racecheck synccheck; do
    echo "== compute-sanitizer --tool $tool python scripts/sanitize_run.py"
    grep -E "workload|SUMMARY" $G/${T}_sanitize_$tool.log
  done
  echo "commit: $(git rev-parse --short HEAD), $(date -u)"
} > profiles/${T}_sanitizer.txt
python scripts/launch_summary.py $G/${T}_launches_C4.csv > profiles/${T}_launches_C4.txt
R=$G/${T}_prof_C4_k_wtile_count.ncu-rep
(python scripts/ncu_summary.py $R; python scripts/ncu_lines.py $R 22) > profiles/${T}_ncu_C4_k_wtile_count.txt 2>&1
[ -f $G/${T}_outliers.jsonl ] && cp $G/${T}_outliers.jsonl profiles/${T}_outliers.jsonl
[ -f $G/${T}_heavy.jsonl ] && cp $G/${T}_heavy.jsonl profiles/${T}_heavy.jsonl
[ -s $G/${T}_s2_d5.json ] && cp $G/${T}_s2_d5.json profiles/${T}_s2_d5.json
grep -E "passed|failed" $G/${T}_pytest_gpu.log | tail -1 > profiles/${T}_pytest_gpu.txt
ls profiles/${T}_*
