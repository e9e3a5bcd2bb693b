"""One screening call with the sort + segment grid (grid_table 3), for ncu captures.

    python tools/profile_csr.py [--config 4] [--variant grid] [--steps 200]
"""
import argparse
import sys
from pathlib import Path

sys.path.insert(0, str(Path(__file__).resolve().parent.parent))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", type=int, default=4)
    ap.add_argument("--variant", default="grid")
    ap.add_argument("--steps", type=int, default=200)
    ap.add_argument("--table", type=int, default=3)
    args = ap.parse_args()
    import torch
    import paper_conf_ipps_hellwigcmbw23_b200 as cds
    from tools import popgen
    pop, cfg, _ = popgen.make_config(args.config)
    dt = cfg.dt_hybrid if args.variant == "hybrid" else cfg.dt_grid
    d = {k: torch.from_numpy(v).cuda() for k, v in pop.items()}
    t0 = 3600.0
    cds.screen(d, t0, t0 + (args.steps - 1) * dt, dt, cfg.d, mode=args.variant, grid_table=args.table)


if __name__ == "__main__":
    main()
