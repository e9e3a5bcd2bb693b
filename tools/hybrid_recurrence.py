"""How often a hybrid coarse candidate pair recurs across consecutive coarse steps (decides
whether caching time-independent filter verdicts per pair can pay).

    python tools/hybrid_recurrence.py [--config 4] [--steps 40] [--t0 3600]
"""
import argparse
import json
import sys
from pathlib import Path

sys.path.insert(0, str(Path(__file__).resolve().parent.parent))

import numpy as np  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", type=int, default=4)
    ap.add_argument("--steps", type=int, default=40)
    ap.add_argument("--t0", type=float, default=3600.0)
    args = ap.parse_args()
    import paper_conf_ipps_hellwigcmbw23_b200 as cds
    from tools import popgen
    pop, cfg, _ = popgen.make_config(args.config)
    dt = cfg.dt_hybrid
    K = cds.candidates(pop, args.t0, args.t0 + (args.steps - 1) * dt, dt, cfg.d)
    key = K["i"].astype(np.uint64) << np.uint64(32) | K["j"].astype(np.uint64)
    u, inv, cnt = np.unique(key, return_inverse=True, return_counts=True)
    a, e = pop["a"], pop["e"]
    q, Q = a * (1 - e), a * (1 + e)
    i, j = K["i"], K["j"]
    ap_rej = np.maximum(q[i], q[j]) - np.minimum(Q[i], Q[j]) > cfg.d
    per_pair = cnt[inv]
    out = {"steps": args.steps, "candidates": int(len(K)), "per_step": len(K) / args.steps,
           "unique_pairs": int(len(u)), "candidates_per_pair": len(K) / max(1, len(u)),
           "frac_candidates_in_recurring_pairs": float(np.mean(per_pair > 1)),
           "frac_candidates_in_pairs_seen_ge_4": float(np.mean(per_pair >= 4)),
           "ap_rejected_frac": float(np.mean(ap_rej)),
           "candidates_per_pair_non_ap": float(np.sum(~ap_rej) / max(1, len(np.unique(key[~ap_rej])))),
           "recurrence_hist": np.bincount(np.minimum(cnt, 41)).tolist()}
    print(json.dumps(out))


if __name__ == "__main__":
    main()
