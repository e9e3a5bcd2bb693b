"""Measurements of the SURVEY 8(f) rows beyond the north-star path, on one B200, with the oracle
timed beside each (not the driver's bench line -- that is bench.py, config 4 grid):

* legacy   mode CD_LEGACY (row 4) on BASELINE configs 1-3 over the config's window: device wall
           time (CUDA events on the call's stream, median of --repeat after a warm-up), pairs/s,
           filter-stage counts, and the recall cross-check against the grid variant on the same
           window (rows the grid misses; every grid row must be in the legacy set).  Oracle O5
           on a bounded sample: m objects drawn at random (seeded) from the same population over
           the same window (m chosen for ~cpu-seconds), scaled by the pair count.
* j2       CD_PROP_J2 (row 3) against CD_PROP_KEPLER, grid variant, BASELINE config 4 (1M objects)
           over a 1-hour slice: the cost of the rotating-frame propagator in the fused step
           kernel (average k_step launch period from the library's phase timers).

    python tools/bench_next_rows.py [--legacy-configs 1,2,3] [--repeat 2] > gpurun_out/rows.jsonl
"""
import argparse
import json
import sys
import time
from pathlib import Path

sys.path.insert(0, str(Path(__file__).resolve().parent.parent))

import numpy as np  # noqa: E402


def log(*a):
    print(*a, file=sys.stderr, flush=True)


def timed(fn, repeat, stream):
    import torch
    times, out = [], None
    for r in range(repeat + 1):
        torch.cuda.synchronize()
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        out = fn()
        e1.record(stream)
        torch.cuda.synchronize()
        if r:
            times.append(e0.elapsed_time(e1) / 1e3)
    return float(np.median(times)), out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--legacy-configs", default="1,2,3")
    ap.add_argument("--repeat", type=int, default=2)
    ap.add_argument("--cpu-seconds", type=float, default=10.0)
    ap.add_argument("--no-j2", action="store_true")
    args = ap.parse_args()
    import torch

    import oracle
    import paper_conf_ipps_hellwigcmbw23_b200 as cds
    from tools import popgen

    dev = torch.device("cuda", 0)
    stream = torch.cuda.current_stream(dev)
    s = stream.cuda_stream
    for k in [int(x) for x in args.legacy_configs.split(",") if x]:
        pop, cfg, _ = popgen.make_config(k)
        n = len(pop["a"])
        dpop = {f: torch.from_numpy(v).to(dev) for f, v in pop.items()}
        dt, d, t0, t1 = cfg.dt_grid or 1.0, cfg.d, cfg.t0, cfg.t1   # config 3 is hybrid-only: 1 s
        K = oracle.num_steps(t0, t1, dt)
        wall, (L, st) = timed(lambda: cds.screen(dpop, t0, t1, dt, d, mode="legacy", return_stats=True,
                                                 stream=s), args.repeat, stream)
        gwall, G = timed(lambda: cds.screen(dpop, t0, t1, dt, d, stream=s), 1, stream)
        lk = set(zip(L["i"].tolist(), L["j"].tolist(), L["step"].tolist()))
        Gn = G[(G["flags"] & cds.CD_FLAG_DEGENERATE) == 0]
        gk = set(zip(Gn["i"].tolist(), Gn["j"].tolist(), Gn["step"].tolist()))
        pairs = n * (n - 1) // 2
        line = {"row": "legacy", "config": k, "name": cfg.name, "n": n, "d_km": d, "dt_s": dt,
                "window_steps": K,
                "gpu": {"wall_s": wall, "pairs_per_s": pairs / wall, "object_steps_per_s": n * K / wall,
                        "conjunctions": int(len(L)), "intervals": int(st["refined"]),
                        "ap_rejected": int(st["hybrid_ap_rejected"]), "coplanar": int(st["hybrid_coplanar"]),
                        "path_rejected": int(st["hybrid_path_rejected"]),
                        "time_rejected": int(st["hybrid_time_rejected"]), "retries": int(st["retries"])},
                "grid_same_window": {"wall_s": gwall, "conjunctions_non_degenerate": int(len(Gn)),
                                     "grid_rows_missing_from_legacy": len(gk - lk),
                                     "legacy_rows_grid_missed": len(lk - gk)}}
        # oracle O5 on a seeded random subset of m objects of the same population, scaled by pairs
        rng = np.random.default_rng(1234 + k)
        m = min(n, 400)
        while True:
            sub = popgen.subset(pop, np.sort(rng.choice(n, m, replace=False)))
            t = time.perf_counter()
            oracle.legacy(sub, t0, t1, dt, d)
            sec = time.perf_counter() - t
            if sec * 4 > args.cpu_seconds or m * 2 > n:
                break
            m *= 2
        sp = m * (m - 1) // 2
        line["cpu_oracle"] = {"pairs_per_s": sp / sec, "cores": oracle.num_threads(),
                              "sample": f"{m} objects drawn at random (seeded) from the same "
                                        f"population, same window ({sp} pairs, {sec:.1f} s), "
                                        f"scaled by pairs",
                              "extrapolated_wall_s": sec * pairs / sp}
        print(json.dumps(line), flush=True)
        log(json.dumps(line))
        del dpop
        torch.cuda.empty_cache()
    if not args.no_j2:
        pop, cfg, _ = popgen.make_config(4)
        n = len(pop["a"])
        dpop = {f: torch.from_numpy(v).to(dev) for f, v in pop.items()}
        t0, t1, dt, d = 12 * 3600.0, 13 * 3600.0, cfg.dt_grid, cfg.d
        K = oracle.num_steps(t0, t1, dt)
        line = {"row": "j2", "config": 4, "n": n, "window": [t0, t1], "steps": K}
        for prop in ("kepler", "j2"):
            wall, (C, st) = timed(lambda: cds.screen(dpop, t0, t1, dt, d, return_stats=True, stream=s,
                                                     propagator=prop, profile_phases=1), args.repeat, stream)
            line[prop] = {"wall_s": wall, "object_steps_per_s": n * K / wall,
                          "k_step_period_us": 1e3 * st["ms_scan"] / max(1, st["launches_scan"]),
                          "candidates": int(st["candidates"]), "conjunctions": int(len(C))}
        print(json.dumps(line), flush=True)
        log(json.dumps(line))


if __name__ == "__main__":
    main()
