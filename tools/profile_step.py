"""One screening call on a BASELINE config population (for ncu / nsight captures).

    python tools/profile_step.py [--config 4] [--steps 64] [--variant grid] [--cell-factor 1]
"""
import argparse
import sys
from pathlib import Path

sys.path.insert(0, str(Path(__file__).resolve().parent.parent))

import numpy as np  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", type=int, default=4)
    ap.add_argument("--n", type=int, default=None)
    ap.add_argument("--steps", type=int, default=64)
    ap.add_argument("--t0", type=float, default=3600.0)
    ap.add_argument("--variant", default="grid")
    ap.add_argument("--cell-factor", type=float, default=None)
    ap.add_argument("--repeat", type=int, default=1)
    args = ap.parse_args()
    import torch
    import paper_conf_ipps_hellwigcmbw23_b200 as cds
    from tools import popgen
    pop, cfg, _ = popgen.make_config(args.config, n=args.n)
    dt = cfg.dt_hybrid if args.variant == "hybrid" else (cfg.dt_grid or 1.0)
    dpop = {k: torch.from_numpy(v).cuda() for k, v in pop.items()}
    kw = {}
    if args.cell_factor is not None:
        kw["cell_factor"] = args.cell_factor
    for _ in range(args.repeat):
        res, st = cds.screen(dpop, args.t0, args.t0 + (args.steps - 1) * dt, dt, cfg.d,
                             mode=args.variant, return_stats=True, **kw)
    print({k: st[k] for k in ("steps", "candidates", "refined", "conjunctions", "ms_total",
                              "kernel_launches", "retries")})


if __name__ == "__main__":
    main()
