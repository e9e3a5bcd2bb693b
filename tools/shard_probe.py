"""Radial shards screened one after another on ONE GPU versus the unsharded call (large n: a
shard's per-step grid fits in L2).  python tools/shard_probe.py [--config 5] [--steps 150] [--shards 4,8,16]"""
import argparse
import sys
import time
from pathlib import Path

sys.path.insert(0, str(Path(__file__).resolve().parent.parent))

import numpy as np  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", type=int, default=5)
    ap.add_argument("--steps", type=int, default=150)
    ap.add_argument("--shards", default="4,8,16")
    args = ap.parse_args()
    import torch
    import paper_conf_ipps_hellwigcmbw23_b200 as cds
    from paper_conf_ipps_hellwigcmbw23_b200 import dist as cdist
    from tools import popgen
    pop, cfg, _ = popgen.make_config(args.config)
    dt, d = cfg.dt_grid, cfg.d
    t0 = 3 * 86400.0
    t1 = t0 + (args.steps - 1) * dt

    def timed(fn):
        torch.cuda.synchronize()
        t = time.perf_counter()
        r = fn()
        torch.cuda.synchronize()
        return time.perf_counter() - t, r
    cds.screen(pop, t0, t0 + 10 * dt, dt, d)
    w_full, full = timed(lambda: cds.screen(pop, t0, t1, dt, d))
    print(f"unsharded: {w_full:.3f} s, {len(full)} conjunctions", flush=True)
    for S in [int(x) for x in args.shards.split(",")]:
        b = cdist.shell_bounds(pop, S)
        tot, parts, mem = 0.0, [], []
        for s in range(S):
            w, (r, m) = timed(lambda: cdist.screen_shard(pop, t0, t1, dt, d, b, s))
            tot += w
            parts.append(r)
            mem.append(m)
        u = np.concatenate(parts)
        u = u[np.lexsort((u["step"], u["j"], u["i"]))]
        print(f"{S} shards: {tot:.3f} s total, max members {max(mem)}, sum members {sum(mem)}, "
              f"equal {np.array_equal(u, full)}", flush=True)


if __name__ == "__main__":
    main()
