#!/usr/bin/env bash
# The GPU test suite against the checked build (device invariants compiled
# in: DTS_DCHECK traps on a violation), for use where compute-sanitizer is
# unavailable.  Build it first: scripts/build_variant.sh checked -DDTS_CHECKED
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out
TAG=${TAG:-r02}
export DTS_LIB=$PWD/ab/libdts_checked.so
echo "== pytest -m gpu (checked build)"; timeout 2400 python -m pytest tests -m gpu -q --timeout=1200 ${PYTEST_K:+-k "$PYTEST_K"} > gpurun_out/${TAG}_pytest_checked.log 2>&1; echo "pytest rc=$?"
tail -3 gpurun_out/${TAG}_pytest_checked.log
grep -c "DTS_DCHECK failed" gpurun_out/${TAG}_pytest_checked.log
echo "== sanitize workload (checked build)"; timeout 600 python scripts/sanitize_run.py > gpurun_out/${TAG}_checked_workload.log 2>&1; echo "workload rc=$?"; tail -2 gpurun_out/${TAG}_checked_workload.log
