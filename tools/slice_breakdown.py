"""Per-phase breakdown of one bench-shaped slice call (1M objects, 1/24 of the day)."""
import sys
import time
from pathlib import Path

sys.path.insert(0, str(Path(__file__).resolve().parent.parent))


def main():
    import torch
    import paper_conf_ipps_hellwigcmbw23_b200 as cds
    from tools import popgen
    import argparse
    ap = argparse.ArgumentParser()
    ap.add_argument("--mode", default="grid")
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--table", type=int, default=0)
    ap.add_argument("--cell", type=float, default=0.0)
    args = ap.parse_args()
    pop, cfg, _ = popgen.make_config(4)
    dt = 1.0 if args.mode == "grid" else cfg.dt_hybrid
    dpop = {k: torch.from_numpy(v).cuda() for k, v in pop.items()}
    for rep in range(args.reps):
        torch.cuda.synchronize()
        t = time.perf_counter()
        res, st = cds.screen(dpop, cfg.t0, cfg.t1, dt, cfg.d, rank=5, n_ranks=24, return_stats=True,
                             profile_phases=1, mode=args.mode, grid_table=args.table,
                             cell_factor=args.cell)
        torch.cuda.synchronize()
        wall = time.perf_counter() - t
        keys = ["steps", "candidates", "refined", "conjunctions", "retries", "kernel_launches",
                "hybrid_ap_rejected", "hybrid_path_rejected", "hybrid_time_rejected", "hybrid_coplanar",
                "ms_total", "ms_precompute", "ms_propagate", "ms_scan", "ms_refine", "ms_finalize",
                "launches_scan", "launches_refine", "step_launches"]
        print(f"wall {1e3 * wall:.1f} ms", {k: (round(st[k], 3) if isinstance(st[k], float) else st[k]) for k in keys})


if __name__ == "__main__":
    main()
