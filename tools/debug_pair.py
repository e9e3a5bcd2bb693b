"""Debug helper: one pair of a BASELINE population screened alone and inside the full population."""
import sys
from pathlib import Path
sys.path.insert(0, str(Path(__file__).resolve().parent.parent))
import numpy as np
import paper_conf_ipps_hellwigcmbw23_b200 as cds
from tools import popgen

cfgk, i, j, t0, t1, dt, mode = int(sys.argv[1]), int(sys.argv[2]), int(sys.argv[3]), float(sys.argv[4]), float(sys.argv[5]), float(sys.argv[6]), sys.argv[7]
pop, cfg, _ = popgen.make_config(cfgk)
sub = {k: np.array([v[i], v[j]]) for k, v in pop.items()}
for m in ("grid", "hybrid"):
    r, st = cds.screen(sub, t0, t1, dt, cfg.d, mode=m, return_stats=True)
    print("pair alone", m, r, {k: st[k] for k in ("candidates", "refined", "hybrid_ap_rejected", "hybrid_coplanar", "hybrid_path_rejected", "hybrid_time_rejected")})
K = cds.candidates(pop, t0, t1, dt, cfg.d)
print("full candidates", len(K), "pair present:", bool(np.any((K["i"] == i) & (K["j"] == j))))
r, st = cds.screen(pop, t0, t1, dt, cfg.d, mode=mode, return_stats=True)
print("full screen", len(r), st, r[(r["i"] == i) & (r["j"] == j)])
