"""All five BASELINE.json configs on one B200, with the oracle timed beside each (SURVEY.md 8(d)
table; build plan step 10).  Not the driver's bench line (that is bench.py, config 4 grid);
this records the per-config table under profiles/.

Per config and variant: the CUDA path over the config's window (device-resident inputs, CUDA
events on the call's stream, median of `--repeat` runs after one warm-up) -> object-steps/s and
wall time; config 5 (8M x 7 d) screens a contiguous sub-window and extrapolates the 7-day wall
time (labelled).  Oracle: the plain C oracle on the host cores over a bounded sample of steps of
the same window, plus a sampled-step parity check (candidate set and conjunction set of a few
steps compared element by element, tests/parity.py rules).

    python tools/bench_configs.py [--configs 1,2,3,4,5] [--repeat 3] > gpurun_out/configs.jsonl
"""
import argparse
import json
import sys
import time
from pathlib import Path

sys.path.insert(0, str(Path(__file__).resolve().parent.parent))
sys.path.insert(0, str(Path(__file__).resolve().parent.parent / "tests"))

import numpy as np  # noqa: E402

# (config, variant) -> sub-window in steps for the GPU timing (None = the config's full window)
GPU_STEPS = {(5, "grid"): 3600, (5, "hybrid"): 400}
VARIANTS = {1: ("grid",), 2: ("grid", "hybrid"), 3: ("hybrid",), 4: ("grid", "hybrid"),
            5: ("grid", "hybrid")}


def log(*a):
    print(*a, file=sys.stderr, flush=True)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--configs", default="1,2,3,4,5")
    ap.add_argument("--repeat", type=int, default=3)
    ap.add_argument("--cpu-seconds", type=float, default=10.0)
    args = ap.parse_args()
    import torch

    import oracle
    import paper_conf_ipps_hellwigcmbw23_b200 as cds
    import parity
    from tools import popgen

    dev = torch.device("cuda", 0)
    stream = torch.cuda.current_stream(dev)
    for k in [int(x) for x in args.configs.split(",")]:
        pop, cfg, _ = popgen.make_config(k)
        n = len(pop["a"])
        dpop = {f: torch.from_numpy(v).to(dev) for f, v in pop.items()}
        for var in VARIANTS[k]:
            dt = cfg.dt_grid if var == "grid" else cfg.dt_hybrid
            K = oracle.num_steps(cfg.t0, cfg.t1, dt)
            ks = GPU_STEPS.get((k, var))
            t0 = cfg.t0
            t1 = cfg.t1 if ks is None else cfg.t0 + (ks - 1) * dt
            Kt = oracle.num_steps(t0, t1, dt)
            times, st = [], None
            for r in range(args.repeat + 1):
                torch.cuda.synchronize()
                e0 = torch.cuda.Event(enable_timing=True)
                e1 = torch.cuda.Event(enable_timing=True)
                e0.record(stream)
                res, st = cds.screen(dpop, t0, t1, dt, cfg.d, mode=var, return_stats=True,
                                     stream=stream.cuda_stream)
                e1.record(stream)
                torch.cuda.synchronize()
                if r:
                    times.append(e0.elapsed_time(e1) / 1e3)
            wall = float(np.median(times))
            rate = n * Kt / wall
            line = {"config": k, "name": cfg.name, "variant": var, "n": n, "d_km": cfg.d,
                    "dt_s": dt, "window_steps": K, "timed_steps": Kt,
                    "gpu": {"object_steps_per_s": rate, "wall_s": wall,
                            "wall_s_window": wall * K / Kt, "extrapolated": Kt != K,
                            "candidates": int(st["candidates"]), "conjunctions": int(len(res)),
                            "retries": int(st["retries"])}}
            # oracle: bounded contiguous sample from the middle of the window, ~cpu-seconds
            gc = oracle.cell_size(cfg.d, dt)
            per = 1
            kmid = Kt // 2
            while True:
                t = time.perf_counter()
                if var == "grid":
                    Ko = oracle.candidates_grid(pop, t0, t1, dt, gc, k_begin=kmid, k_end=kmid + per)
                    Co = oracle.conjunctions(pop, t0, t1, dt, cfg.d, gc, Ko)
                else:
                    Co = oracle.hybrid(pop, t0, t1, dt, cfg.d, k_begin=kmid, k_end=kmid + per)
                sec = time.perf_counter() - t
                if sec * 2 > args.cpu_seconds or per * 2 > Kt - kmid:
                    break
                per *= 2
            line["cpu_oracle"] = {"object_steps_per_s": n * per / sec, "cores": oracle.num_threads(),
                                  "sample_steps": [kmid, kmid + per], "seconds": sec}
            # sampled parity on the oracle's sample steps (candidates: grid only)
            Cg = res[(res["step"] >= kmid) & (res["step"] < kmid + per)]
            if var == "grid":
                Kg = cds.candidates(dpop, t0, t1, dt, cfg.d, stream=stream.cuda_stream) if n * Kt <= 4e9 else None
                if Kg is not None:
                    Kg = Kg[(Kg["step"] >= kmid) & (Kg["step"] < kmid + per)]
                    parity.compare_candidates(pop, Kg, Ko, t0, dt, gc)
                co = Co
            else:
                co = Co[0] if isinstance(Co, tuple) else Co
            cmp = parity.compare_conjunctions(pop, Cg, co, t0, t1, dt, cfg.d, gc)
            line["parity_sample"] = {"steps": [kmid, kmid + per], "gpu_rows": int(len(Cg)),
                                     "oracle_rows": int(len(co)), **{k2: int(v) for k2, v in cmp.items()}}
            print(json.dumps(line), flush=True)
            log(json.dumps(line))
        del dpop
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
