#!/bin/bash
# Build experimental variants of liblcf.so (build/variants/*.so) for A/B timing.
# Usage: scripts/build_variants.sh <<'LIST'
#   name -DFLAG ...
# LIST
set -e
cd "$(dirname "$0")/.."
mkdir -p build/variants
rm -f build/variants/*.so
F="-gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC -shared -Iinclude"
while read name defs; do
  [ -z "$name" ] && continue
  nvcc $F $defs -o build/variants/$name.so paper_conf_asplos_azamifb25_b200/csrc/*.cu &
done
wait
ls build/variants
