#!/bin/bash
# Build library variants with extra nvcc -D flags (all translation units) on the GPU box and run a
# command against each through CDSCREEN_LIB.  usage:
#   tools/lib_variants.sh "<cmd>" "-DA=1" "-DA=2 -DB=3" ...
set -e
P=paper_conf_ipps_hellwigcmbw23_b200
F="-gencode arch=compute_100a,code=sm_100a -lineinfo -O3 -std=c++17 -Xcompiler -fPIC -shared -Iinclude"
CMD=$1; shift
mkdir -p build/variants
i=0
for v in "$@"; do
  out=build/variants/v$i.so
  nvcc $F $v -o $out $P/csrc/*.cu &
  i=$((i+1))
done
wait
i=0
for v in "$@"; do
  echo "== variant [$v]"
  CDSCREEN_LIB=$PWD/build/variants/v$i.so bash -c "$CMD"
  i=$((i+1))
done
