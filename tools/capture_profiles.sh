#!/bin/bash
# GPU-box capture for profiles/: launch list of the bench command (cold-cache, serialised:
# compare shares, not absolutes), ncu --set full of the dominant kernel (grid k_step, steady
# state), of the hybrid variant's kernels and of the legacy chain's kernels.  Output under
# gpurun_out/$1/.
set -e
OUT=gpurun_out/${1:-prof}
mkdir -p $OUT
ncu --metrics gpu__time_duration.sum --clock-control none -c 3000 --csv --log-file $OUT/launches.csv \
    python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-hybrid --e2e-steps 0 --no-profile > $OUT/launches.log 2>&1 || true
ncu --set full --clock-control none --import-source on -k regex:k_step -s 60 -c 3 \
    -o $OUT/k_step python tools/profile_step.py --steps 400 > $OUT/full.log 2>&1 || true
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/hyb_launches.csv \
    python tools/profile_step.py --variant hybrid --steps 200 > $OUT/hyb_launches.log 2>&1 || true
ncu --set full --clock-control none --import-source on -k regex:"k_step" -s 30 -c 3 \
    -o $OUT/hyb python tools/profile_step.py --variant hybrid --steps 200 > $OUT/hyb_full.log 2>&1 || true
ncu --set full --clock-control none --import-source on -k regex:"k_hybrid_filter|k_brent" -s 2 -c 2 \
    -o $OUT/hybf python tools/profile_step.py --variant hybrid --steps 200 > $OUT/hybf_full.log 2>&1 || true
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/leg_launches.csv \
    python tools/profile_step.py --config 2 --variant legacy --t0 0 --steps 86401 > $OUT/leg_launches.log 2>&1 || true
ncu --set full --clock-control none --import-source on -k regex:"k_legacy" -c 2 \
    -o $OUT/leg python tools/profile_step.py --config 2 --variant legacy --t0 0 --steps 86401 > $OUT/leg_full.log 2>&1 || true
