"""Library radial L2 shards (cd_options.shards) on one GPU: device time of one screening call for
several shard counts (device-resident inputs).  python tools/shard_sweep.py [--config 5] [--steps 1200] [--shards 1,2,3]"""
import argparse
import sys
from pathlib import Path

sys.path.insert(0, str(Path(__file__).resolve().parent.parent))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", type=int, default=5)
    ap.add_argument("--steps", type=int, default=1200)
    ap.add_argument("--shards", default="1,2,3")
    ap.add_argument("--variant", default="grid")
    args = ap.parse_args()
    import torch
    import paper_conf_ipps_hellwigcmbw23_b200 as cds
    from tools import popgen
    pop, cfg, _ = popgen.make_config(args.config)
    dt = cfg.dt_grid if args.variant == "grid" else cfg.dt_hybrid
    dpop = {k: torch.from_numpy(v).cuda() for k, v in pop.items()}
    t0 = 3 * 86400.0
    t1 = t0 + (args.steps - 1) * dt
    for S in [int(x) for x in args.shards.split(",")]:
        cds.screen(dpop, t0, t0 + 20 * dt, dt, cfg.d, mode=args.variant, shards=S)
        res, st = cds.screen(dpop, t0, t1, dt, cfg.d, mode=args.variant, shards=S, return_stats=True)
        print(f"shards {S}: {st['ms_total']:.1f} ms for {args.steps} steps, "
              f"{st['ms_total'] / args.steps * 1e3:.1f} us/step, {len(res)} conjunctions, "
              f"candidates {st['candidates']}", flush=True)


if __name__ == "__main__":
    main()
