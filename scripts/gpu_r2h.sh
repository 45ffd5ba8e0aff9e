#!/usr/bin/env bash
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out
echo "== pytest -m gpu"; timeout 2000 python -m pytest tests -m gpu -q -x --timeout=900 > gpurun_out/pytest_h.log 2>&1; echo "pytest rc=$?"
tail -3 gpurun_out/pytest_h.log
echo "== bench"; timeout 900 python bench.py --steps 20 --warmup 5 --no-cpu-baseline > gpurun_out/bench_h.log 2>&1; echo "bench rc=$?"
python - <<'PY'
import json
l=[x for x in open('gpurun_out/bench_h.log') if x.startswith('{')][-1]
d=json.loads(l)
print(d['ms_per_step'], d['phases_ms'], d['roofline']['frac'], d['e2e']['value'])
PY
VARIANTS="tile|DTS_EMIT=tile|tree;gather|X=1|tree" AB_ARGS="--points C4:0.005 C4:0.02 C2:8 C1:0.005" AB_OUT=abh bash scripts/ab_env.sh
