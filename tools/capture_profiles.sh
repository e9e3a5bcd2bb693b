#!/bin/bash
# GPU-box capture for profiles/: launch list of one bench-shaped call and one ncu --set full
# capture of the dominant kernel.  Output under gpurun_out/$1/.
set -e
OUT=gpurun_out/${1:-prof}
mkdir -p $OUT
# launch list (cold-cache, serialised: compare shares, not absolutes)
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches.csv \
    python tools/profile_step.py --steps 200 > $OUT/launches.log 2>&1 || true
# full section set of the fused step kernel (steady state launches)
ncu --set full --clock-control none --import-source on -k regex:k_step -s 20 -c 3 \
    -o $OUT/k_step python tools/profile_step.py --steps 40 > $OUT/full.log 2>&1 || true
