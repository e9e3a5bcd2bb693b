#!/bin/bash
# Build the library with different -D options for cd_kernels.cu and run the sweep for each.
# usage: tools/variant_sweep.sh "-DCD_STEP_MINB=4" "-DCD_STEP_MINB=6" ...
set -e
P=paper_conf_ipps_hellwigcmbw23_b200
F="-gencode arch=compute_100a,code=sm_100a -lineinfo -O3 -std=c++17 -Xcompiler -fPIC -Iinclude"
mkdir -p /tmp/vb
for f in cd_sort cd_hybrid; do nvcc $F -c -o /tmp/vb/$f.o $P/csrc/$f.cu & done; wait
cp $P/libcdscreen.so /tmp/vb/orig.so
for v in "$@"; do
  nvcc $F $v -c -o /tmp/vb/k.o $P/csrc/cd_kernels.cu &
  nvcc $F $v -c -o /tmp/vb/cd_api.o $P/csrc/cd_api.cu &
  wait
  nvcc -gencode arch=compute_100a,code=sm_100a -shared -o $P/libcdscreen.so /tmp/vb/*.o
  echo "== variant $v"
  timeout ${VTIMEOUT:-150} python tools/sweep.py --steps 400 --cell ${CELLS:-4} --persist ${PERSIST:-0} --table ${TABLE:-0} 2>&1 | tail -${NCELL:-1}
done
cp /tmp/vb/orig.so $P/libcdscreen.so
