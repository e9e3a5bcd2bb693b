"""The hybrid variant's coarse step dt_h (the paper's s_ps, 9 s by default, reduced automatically
when memory binds) against the screen's cost at 1M objects over a 2 h window:
device time per simulated hour and conjunctions (the set of minima below d does not depend on
dt_h; only the owner step label does).

    python tools/hybrid_dt_sweep.py [--config 4] [--hours 2] [--dts 1,2,3,4.5,6,9]
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
    ap.add_argument("--hours", type=float, default=2.0)
    ap.add_argument("--dts", default="1,2,3,4.5,6,9")
    args = ap.parse_args()
    import torch
    import paper_conf_ipps_hellwigcmbw23_b200 as cds
    from tools import popgen
    pop, cfg, _ = popgen.make_config(args.config)
    dpop = {k: torch.from_numpy(v).cuda() for k, v in pop.items()}
    t0, t1 = 3600.0, 3600.0 + 3600.0 * args.hours
    ref = None
    for dt in [float(x) for x in args.dts.split(",")]:
        cds.screen(dpop, t0, t0 + 20 * dt, dt, cfg.d, mode="hybrid")   # warm
        torch.cuda.synchronize()
        res, st = cds.screen(dpop, t0, t1, dt, cfg.d, mode="hybrid", return_stats=True)
        key = set(zip(res["i"].tolist(), res["j"].tolist(), np.round(res["tca"], 2).tolist()))
        inner = {k for k in key if t0 + 10 < k[2] < t1 - 10}
        if ref is None:
            ref = inner
        print(json.dumps({"dt_h": dt, "ms_per_hour": st["ms_total"] / args.hours,
                          "candidates": st["candidates"], "refined": st["refined"],
                          "conjunctions": len(res), "same_minima_as_first": inner == ref}), flush=True)


if __name__ == "__main__":
    main()
