"""Per-phase device time per step for a sweep of options (GPU tuning aid)."""
import argparse
import json
import sys
from pathlib import Path

sys.path.insert(0, str(Path(__file__).resolve().parent.parent))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", type=int, default=4)
    ap.add_argument("--n", type=int, default=None)
    ap.add_argument("--steps", type=int, default=400)
    ap.add_argument("--variant", default="grid")
    ap.add_argument("--cell", default="1,2,3,4,5,6,8")
    ap.add_argument("--batch", default="0")
    ap.add_argument("--persist", default="0")
    ap.add_argument("--table", default="0")
    ap.add_argument("--resort", default="0", help="cd_options.resort_steps values (0 auto, -1 off)")
    ap.add_argument("--t0", type=float, default=3600.0)
    ap.add_argument("--rounds", default="0", help="cd_options.round_steps values (0 = auto)")
    args = ap.parse_args()
    import torch
    import paper_conf_ipps_hellwigcmbw23_b200 as cds
    from tools import popgen
    pop, cfg, _ = popgen.make_config(args.config, n=args.n)
    dt = cfg.dt_grid if args.variant == "grid" else cfg.dt_hybrid
    dpop = {k: torch.from_numpy(v).cuda() for k, v in pop.items()}
    t0 = args.t0
    t1 = t0 + (args.steps - 1) * dt
    ref = None
    import itertools
    ints = lambda x: [int(v) for v in x.split(",")]
    for rs, pers, tbl, b, cf, rd in itertools.product(ints(args.resort), ints(args.persist), ints(args.table),
                                                      ints(args.batch), [float(v) for v in args.cell.split(",")],
                                                      ints(args.rounds)):
            kw = dict(cell_factor=cf, profile_phases=True, l2_persist=pers, grid_table=tbl,
                      resort_steps=rs)
            if b:
                kw["batch_object_steps"] = b
            if rd:
                kw["round_steps"] = rd
            cds.screen(dpop, t0, t0 + 20 * dt, dt, cfg.d, mode=args.variant, **kw)  # warm
            res, st = cds.screen(dpop, t0, t1, dt, cfg.d, mode=args.variant, return_stats=True, **kw)
            if ref is None:
                ref = res
            same = bool(len(res) == len(ref) and (res[["i", "j", "step"]] == ref[["i", "j", "step"]]).all())
            k = st["steps"]
            out = {"resort": rs, "rounds": rd, "cell": cf, "table": tbl, "batch": b, "persist": pers,
                   "ms_per_step_total": st["ms_total"] / k,
                   "us_clear": 1e3 * st["ms_clear"] / k, "us_prop": 1e3 * st["ms_propagate"] / k,
                   "us_insert": 1e3 * st["ms_insert"] / k, "us_scan": 1e3 * st["ms_scan"] / k,
                   "us_refine": 1e3 * st["ms_refine"] / k, "cand": st["candidates"],
                   "conj": st["conjunctions"], "same_as_first": same}
            print(json.dumps(out), flush=True)


if __name__ == "__main__":
    main()
