#!/bin/bash
# GPU-box capture for profiles/ (round 2, second pass): launch list of the bench command, ncu
# --set full of the grid k_step (1M, steady state), of the hybrid kernels (1M, 200 coarse steps)
# and of the 8M refinement.  Output under gpurun_out/$1/.
OUT=gpurun_out/${1:-r2b}
mkdir -p $OUT
ncu --metrics gpu__time_duration.sum --clock-control none -c 3000 --csv --log-file $OUT/launches.csv \
    python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-hybrid --e2e-steps 0 --no-profile > $OUT/launches.log 2>&1 || true
ncu --set full --clock-control none --import-source on -k regex:k_step -s 60 -c 2 \
    -o $OUT/k_step python tools/profile_step.py --steps 400 > $OUT/full.log 2>&1 || true
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/hyb_launches.csv \
    python tools/profile_step.py --variant hybrid --steps 200 > $OUT/hyb_launches.log 2>&1 || true
ncu --set full --clock-control none --import-source on -k regex:"k_step" -s 40 -c 2 \
    -o $OUT/hyb python tools/profile_step.py --variant hybrid --steps 200 > $OUT/hyb_full.log 2>&1 || true
ncu --set full --clock-control none --import-source on -k regex:"k_hybrid_filter|k_brent" -s 2 -c 2 \
    -o $OUT/hybf python tools/profile_step.py --variant hybrid --steps 200 > $OUT/hybf_full.log 2>&1 || true
ncu --set full --clock-control none --import-source on -k regex:"k_prefilter|k_brent" -s 2 -c 2 \
    -o $OUT/ref8 python tools/profile_step.py --config 5 --steps 200 > $OUT/ref8_full.log 2>&1 || true
ncu --set full --clock-control none --import-source on -k regex:"k_step" -s 150 -c 1 \
    -o $OUT/k8 python tools/profile_step.py --config 5 --steps 200 > $OUT/k8_full.log 2>&1 || true
