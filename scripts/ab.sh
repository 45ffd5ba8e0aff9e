#!/usr/bin/env bash
# A/B of the in-tree libdts against ab/libdts_*.so, interleaved (one gpurun call).
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out
for rep in 1 2; do
  for lib in ${LIBS:-ab/libdts_base.so tree}; do
    if [ "$lib" = tree ]; then unset DTS_LIB; else export DTS_LIB=$PWD/$lib; fi
    timeout 600 python scripts/ab_search.py --tag "$lib" ${AB_ARGS:-} >> gpurun_out/ab.jsonl 2>> gpurun_out/ab.err
  done
done
unset DTS_LIB
python - <<'PY'
import json, collections
rows = [json.loads(l) for l in open("gpurun_out/ab.jsonl")]
agg = collections.defaultdict(list)
for r in rows: agg[(r["config"], r["d"], r["lib"])].append(r)
for k in sorted(agg):
    v = agg[k]
    print(k, "search %.4f count %.4f prep %.4f emit %.4f canon %.4f" % tuple(
        min(x[f] for x in v) for f in ("search_ms", "count_ms", "prep_ms", "emit_ms", "canon_ms")))
PY
