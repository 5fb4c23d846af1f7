#!/bin/bash
# Build libpagoda variants for A/B runs: build/variants/libpagoda_v<name>.so, selected at run time
# with PAGODA_LIB=<path> (scripts/var_ab.sh).   usage: bash scripts/build_variants.sh name "-DFOO=1" [name "-D..."]
set -e
cd "$(dirname "$0")/.."
mkdir -p build/variants
ARCH="-gencode arch=compute_100a,code=sm_100a"
while [ $# -ge 2 ]; do
  v=$1; flags=$2; shift 2
  d=build/variants/v$v; mkdir -p $d
  for f in paper_conf_ppopp_yehsser17_b200/csrc/*.cu; do
    n=$(basename $f .cu)
    nvcc $ARCH -O3 -lineinfo -std=c++17 -Xcompiler -fPIC,-O2 -Iinclude -Ipaper_conf_ppopp_yehsser17_b200/csrc \
      $flags -c $f -o $d/$n.o &
  done
  wait
  nvcc $ARCH -shared -o build/variants/libpagoda_v$v.so $d/*.o -lpthread -lrt -ldl
done
