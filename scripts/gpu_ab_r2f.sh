#!/usr/bin/env bash
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out
for rep in 1 2; do for lib in ${LIBS}; do
  if [ "$lib" = tree ]; then unset DTS_LIB; else export DTS_LIB=$PWD/$lib; fi
  timeout 300 python scripts/ab_build.py --tag $lib >> gpurun_out/abb.jsonl 2>>gpurun_out/abb.err
done; done
unset DTS_LIB
cat gpurun_out/abb.jsonl
LIBS="${LIBS}" AB_ARGS="${AB_ARGS:---points C4:0.005 C4:0.02 C2:2}" bash scripts/ab.sh
if [ -n "$PROF" ]; then TAG=r02f KERNELS=k_wtile_count bash scripts/gpu_prof.sh; fi
