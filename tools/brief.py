"""Condense tools/sweep.py JSON lines to 'scan refine' per line (GPU-box log helper)."""
import json
import sys

for line in sys.stdin:
    try:
        d = json.loads(line)
    except ValueError:
        print(line.rstrip())
        continue
    print(f"table {d['table']} cell {d['cell']} resort {d['resort']} rounds {d.get('rounds', 0)}: scan {d['us_scan']:.1f} us, refine {d['us_refine']:.2f} us, cand {d['cand']}, conj {d['conj']}")
