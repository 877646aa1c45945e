#!/bin/bash
# Build A/B variants of libhirace.so into build/variants/<name>.so.
# usage: scripts/build_variants.sh name1:"-DFLAG ..." name2:"" ...
set -e
cd "$(dirname "$0")/.."
mkdir -p build/variants
rm -f build/variants/*.so
SRC=$(ls paper_conf_sc_jacobsonbg24_b200/csrc/*.cu paper_conf_sc_jacobsonbg24_b200/csrc/*.cpp)
for spec in "$@"; do
  name=${spec%%:*}; flags=${spec#*:}
  /usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -lineinfo -O3 -std=c++17 \
    -Xcompiler -fPIC,-O2 -shared -I include -I paper_conf_sc_jacobsonbg24_b200/csrc $flags \
    -o build/variants/$name.so $SRC &
done
wait
for spec in "$@"; do n=${spec%%:*}; test -f build/variants/$n.so || { echo "variant $n failed"; exit 1; }; done
ls -la build/variants
