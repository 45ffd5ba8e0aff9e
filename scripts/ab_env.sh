#!/usr/bin/env bash
# A/B of runtime variants: each entry of VARIANTS is "tag|ENV=VAL ...|lib or tree";
# two interleaved repetitions, one JSON line per point.
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out
OUT=gpurun_out/${AB_OUT:-abenv}.jsonl
rm -f $OUT
IFS=';' read -ra VS <<< "$VARIANTS"
for rep in 1 2; do
  for v in "${VS[@]}"; do
    tag=$(echo "$v" | cut -d'|' -f1); envs=$(echo "$v" | cut -d'|' -f2); lib=$(echo "$v" | cut -d'|' -f3)
    if [ "$lib" = tree ] || [ -z "$lib" ]; then libenv=""; else libenv="DTS_LIB=$PWD/$lib"; fi
    env $envs $libenv timeout 600 python scripts/ab_search.py --tag "$tag" ${AB_ARGS:-} >> $OUT 2>> gpurun_out/abenv.err
  done
done
python - "$OUT" <<'PY'
import json, sys, collections
rows = [json.loads(l) for l in open(sys.argv[1])]
agg = collections.defaultdict(list)
for r in rows: agg[(r["config"], r["d"], r["lib"])].append(r)
for k in sorted(agg):
    v = agg[k]
    print(k, "search %.4f count %.4f prep %.4f emit %.4f canon %.4f build %.4f" % tuple(
        min(x.get(f, 0) for x in v) for f in ("search_ms", "count_ms", "prep_ms", "emit_ms", "canon_ms", "build_ms")),
        "insert %.4f" % min(x.get("build_phases", [0]*5)[4] for x in v))
PY
