#!/usr/bin/env bash
# A/B of env toggles inside ONE gpurun call (box-to-box variance is ~15%):
#   AB="DTS_PREFETCH=0|DTS_PREFETCH=1" bash scripts/ab.sh
# Each variant runs bench.py twice (interleaved); prints ms/step and phases.
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out
IFS='|' read -ra VARS <<< "${AB:-X=0}"
for rep in 1 2; do
  for v in "${VARS[@]}"; do
    line=$(env $v timeout 600 python bench.py --steps ${STEPS:-20} --warmup 3 --no-cpu-baseline \
           --e2e-steps 0 ${BENCH_EXTRA:-} 2>/dev/null | tail -1)
    echo "$line" > gpurun_out/ab_last.json
    python - "$v" "$rep" <<'EOF'
import json, sys
try:
    r = json.load(open("gpurun_out/ab_last.json"))
    ph = {k: round(x, 3) for k, x in r.get("phases_ms", {}).items()}
    print(f"{sys.argv[1]:<40} rep{sys.argv[2]} ms/step={r['ms_per_step']:.3f} frac={r['roofline']['frac']:.3f} {ph}")
except Exception as e:
    print(sys.argv[1], "failed", e)
EOF
  done
done | tee gpurun_out/ab.txt
