#!/bin/bash
# GPU-box capture of the hybrid variant (1M objects, config 4, 200 coarse steps): launch list and
# ncu --set full of its kernels.  Output under gpurun_out/$1/.
OUT=gpurun_out/${1:-hyb}
mkdir -p $OUT
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/hyb_launches.csv \
    python tools/profile_step.py --variant hybrid --steps 200 > $OUT/hyb_launches.log 2>&1 || true
ncu --set full --clock-control none --import-source on -k regex:"k_step|k_hybrid_filter|k_brent" -s 40 -c 6 \
    -o $OUT/hyb python tools/profile_step.py --variant hybrid --steps 200 > $OUT/hyb_full.log 2>&1 || true
