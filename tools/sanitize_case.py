"""Config 1 through every mode of the library, for compute-sanitizer (memcheck / racecheck /
synccheck / initcheck; SURVEY 4 "compute-sanitizer on config 1").  Prints the result sizes.

    compute-sanitizer --tool memcheck python tools/sanitize_case.py
"""
import sys
from pathlib import Path

sys.path.insert(0, str(Path(__file__).resolve().parent.parent))

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
    out["hybrid"] = len(cds.screen(pop, cfg.t0, cfg.t1, 9.0, cfg.d, mode="hybrid"))
    out["legacy"] = len(cds.screen(pop, cfg.t0, t1, 1.0, cfg.d, mode="legacy"))
    out["candidates"] = len(cds.candidates(pop, cfg.t0, t1, 1.0, cfg.d))
    out["shards"] = len(cds.screen(pop, cfg.t0, t1, 1.0, cfg.d, shards=3))
    print(out)


if __name__ == "__main__":
    main()
