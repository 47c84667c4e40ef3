#!/bin/bash
# Build alternate liblmo.so variants (experiments) into build/variants/<name>.so.
# usage: scripts/build_variants.sh name1 "-DFOO=1 -DBAR=2" name2 "-D..." ...
# Load one with LMO_LIB=build/variants/<name>.so.
set -e
cd "$(dirname "$0")/.."
mkdir -p build/variants
PKG=paper_conf_ipps_wurypgll25_b200
pids=()
while [ $# -ge 2 ]; do
  name=$1; defs=$2; shift 2
  /usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 \
    -Xcompiler -fPIC,-O2 -Xptxas -v --shared -cudart static $defs -I include -I $PKG/csrc \
    -o build/variants/$name.so $PKG/csrc/*.cu > build/variants/$name.log 2>&1 &
  pids+=($!)
done
for p in "${pids[@]}"; do wait $p; done
ls -la build/variants/*.so
