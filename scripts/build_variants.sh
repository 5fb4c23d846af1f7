#!/bin/bash
# Build libpagoda variants with -DPAGODA_TDES_VARIANT=v into build/variants/libpagoda_v<v>.so
# (experiments; select one at run time with PAGODA_LIB=<path>).
set -e
cd "$(dirname "$0")/.."
mkdir -p build/variants
ARCH="-gencode arch=compute_100a,code=sm_100a"
for v in "$@"; do
  d=build/variants/v$v; mkdir -p $d
  for f in paper_conf_ppopp_yehsser17_b200/csrc/*.cu; do
    n=$(basename $f .cu)
    nvcc $ARCH -O3 -lineinfo -std=c++17 -Xcompiler -fPIC,-O2 -Iinclude -Ipaper_conf_ppopp_yehsser17_b200/csrc \
      -DPAGODA_TDES_VARIANT=$v -c $f -o $d/$n.o &
  done
  wait
  nvcc $ARCH -shared -o build/variants/libpagoda_v$v.so $d/*.o -lpthread -lrt -ldl
done
