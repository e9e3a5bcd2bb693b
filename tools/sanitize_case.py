"""Config 1 through every mode of the library, for compute-sanitizer (memcheck / racecheck /
synccheck / initcheck; SURVEY 4 "compute-sanitizer on config 1").  Prints the result sizes.

    compute-sanitizer --tool memcheck python tools/sanitize_case.py
"""
import sys
from pathlib import Path

sys.path.insert(0, str(Path(__file__).resolve().parent.parent))

import numpy as np  # noqa: E402

import paper_conf_ipps_hellwigcmbw23_b200 as cds  # noqa: E402
from tools import popgen  # noqa: E402


def main():
    pop, cfg, _ = popgen.make_config(1)
    t1 = 120.0
    out = {}
    out["grid"] = len(cds.screen(pop, cfg.t0, t1, 1.0, cfg.d))
    out["grid_open"] = len(cds.screen(pop, cfg.t0, t1, 1.0, cfg.d, grid_table=1, cell_factor=1.0))
    out["grid_csr"] = len(cds.screen(pop, cfg.t0, t1, 1.0, cfg.d, grid_table=3))
    out["grid_resort"] = len(cds.screen(pop, cfg.t0, t1, 1.0, cfg.d, resort_steps=5))
    out["grid_j2"] = len(cds.screen(dict(pop, propagator="j2"), cfg.t0, t1, 1.0, cfg.d))
    out["grid_halfshell"] = len(cds.screen(pop, cfg.t0, t1, 1.0, cfg.d, grid_table=2, cell_factor=1.0))
    out["hybrid"] = len(cds.screen(pop, cfg.t0, cfg.t1, 9.0, cfg.d, mode="hybrid"))
    out["hybrid_open"] = len(cds.screen(pop, cfg.t0, cfg.t1, 9.0, cfg.d, mode="hybrid", grid_table=1))
    out["hybrid_csr"] = len(cds.screen(pop, cfg.t0, cfg.t1, 9.0, cfg.d, mode="hybrid", grid_table=3))
    # a dense compact shell: full warps through every stage of the hybrid filter's queues
    rng = np.random.default_rng(8)
    n = 4000
    dense = {"a": rng.uniform(6900, 6904, n), "e": rng.uniform(0, 0.0003, n),
             "inc": 0.9 + rng.normal(0, 2e-4, n), "raan": rng.normal(1.0, 2e-4, n),
             "argp": rng.uniform(0, 2 * np.pi, n), "nu0": rng.uniform(0, 2 * np.pi, n)}
    dense = popgen.concat(dense, popgen.random_population(4000, 3))
    out["hybrid_dense"] = len(cds.screen(dense, 0.0, 180.0, 9.0, 5.0, mode="hybrid"))
    out["legacy"] = len(cds.screen(pop, cfg.t0, t1, 1.0, cfg.d, mode="legacy"))
    out["candidates"] = len(cds.candidates(pop, cfg.t0, t1, 1.0, cfg.d))
    out["shards"] = len(cds.screen(pop, cfg.t0, t1, 1.0, cfg.d, shards=3))
    print(out)


if __name__ == "__main__":
    main()
