#!/usr/bin/env bash
# Build compile-time variants of libdts into ab/libdts_<tag>.so, then rebuild
# the in-tree library: build_variant.sh tag "-DFLAG ..." [tag "-D..."]...
cd "$(dirname "$0")/.."
mkdir -p ab
while [ $# -ge 2 ]; do
  DTS_NVCC_EXTRA="$2" python -m paper_conf_ipps_gowanlockc15_b200.build --force >/dev/null || exit 1
  cp paper_conf_ipps_gowanlockc15_b200/libdts.so ab/libdts_$1.so
  echo "built ab/libdts_$1.so ($2)"
  shift 2
done
python -m paper_conf_ipps_gowanlockc15_b200.build --force >/dev/null && echo "rebuilt in-tree"
