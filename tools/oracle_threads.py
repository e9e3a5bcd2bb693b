"""CPU oracle thread scaling on BASELINE config 2 ("single-thread time is also
reported on config 2 for a speedup-vs-1-thread comparable to P:312"; the paper's CPU thread
study).  Each thread count runs in its own process (OpenMP reads OMP_NUM_THREADS at
start-up); the grid and hybrid oracles screen a fixed contiguous sample of the 24 h window.

    python tools/oracle_threads.py [--threads 1,2,4,8,16] > profiles/round1_oracle_threads.jsonl
"""
import argparse
import json
import os
import subprocess
import sys
import time
from pathlib import Path

ROOT = Path(__file__).resolve().parent.parent


def child(variant, steps):
    sys.path.insert(0, str(ROOT))
    import oracle
    from tools import popgen
    pop, cfg, _ = popgen.make_config(2)
    dt = cfg.dt_grid if variant == "grid" else cfg.dt_hybrid
    K = oracle.num_steps(cfg.t0, cfg.t1, dt)
    k0 = K // 2
    t = time.perf_counter()
    if variant == "grid":
        gc = oracle.cell_size(cfg.d, dt)
        C = oracle.candidates_grid(pop, cfg.t0, cfg.t1, dt, gc, k_begin=k0, k_end=k0 + steps)
        oracle.conjunctions(pop, cfg.t0, cfg.t1, dt, cfg.d, gc, C)
    else:
        oracle.hybrid(pop, cfg.t0, cfg.t1, dt, cfg.d, k_begin=k0, k_end=k0 + steps)
    sec = time.perf_counter() - t
    print(json.dumps({"variant": variant, "threads": oracle.num_threads(), "steps": steps,
                      "seconds": sec, "object_steps_per_s": len(pop["a"]) * steps / sec}))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--threads", default="1,2,4,8,16")
    ap.add_argument("--child", default=None)
    ap.add_argument("--steps", type=int, default=0)
    args = ap.parse_args()
    if args.child:
        return child(args.child, args.steps)
    base = {}
    for variant, steps in (("grid", 512), ("hybrid", 256)):
        for th in [int(x) for x in args.threads.split(",")]:
            env = dict(os.environ, OMP_NUM_THREADS=str(th))
            out = subprocess.run([sys.executable, __file__, "--child", variant, "--steps", str(steps)],
                                 env=env, capture_output=True, text=True, check=True).stdout
            d = json.loads(out.strip().splitlines()[-1])
            base.setdefault(variant, d["seconds"])
            d["speedup_vs_1_thread"] = base[variant] / d["seconds"]
            print(json.dumps(d), flush=True)


if __name__ == "__main__":
    main()
