#!/bin/bash
# A/B of library builds (CDSCREEN_LIB) on the per-step sweep: config 4 (1M, grid, auto cell),
# config 2 (30k, grid) and config 4 hybrid.  usage: tools/ab_libs.sh lib1.so lib2.so ...
for L in "$@"; do
  for args in "--config 4 --steps 1000" "--config 2 --steps 3000" "--config 4 --variant hybrid --steps 300"; do
    CDSCREEN_LIB=$PWD/$L timeout 200 python tools/sweep.py $args --cell 0 2>&1 | python -c "
import sys, json
for l in sys.stdin:
    try: d = json.loads(l)
    except Exception: continue
    print('$L', '$args', round(d['ms_per_step_total'] * 1e3, 2), round(d['us_scan'], 2))
"
  done
done
