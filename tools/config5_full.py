"""BASELINE config 5 (8,000,000 objects, 7 days at 1 s = 604,801 steps, grid variant) screened in
full on one GPU -- not extrapolated.  The ~4e9 conjunction records (~130 GB) do not fit the device
or the host, so the library runs with cd_options.digest_only: every round's records
are folded on the device into a count, an order-independent digest (cdscreen.h cd_stats.digest)
and the smallest PCA, and the buffer is reused.  The window is still cut into time slices (owner
rule: they partition the result; digests add) so progress is visible.  Prints one JSON line.

    python tools/config5_full.py [--slices 168] [--variant grid] [--max-slices 0]
"""
import argparse
import ctypes as C
import json
import sys
import time
from pathlib import Path

sys.path.insert(0, str(Path(__file__).resolve().parent.parent))

import numpy as np  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", type=int, default=5)
    ap.add_argument("--slices", type=int, default=168)
    ap.add_argument("--variant", default="grid")
    ap.add_argument("--max-slices", type=int, default=0, help="stop after this many (testing)")
    args = ap.parse_args()
    import torch
    import paper_conf_ipps_hellwigcmbw23_b200 as cds
    from tools import popgen
    pop, cfg, _ = popgen.make_config(args.config)
    n = len(pop["a"])
    dt = cfg.dt_grid if args.variant == "grid" else cfg.dt_hybrid
    mode = cds.CD_GRID if args.variant == "grid" else cds.CD_HYBRID
    K = int(np.floor((cfg.t1 - cfg.t0) / dt)) + 1
    dev = torch.device("cuda", 0)
    dpop = {k: torch.from_numpy(v).to(dev) for k, v in pop.items()}
    stream = torch.cuda.current_stream(dev)
    talloc = cds.TorchAllocator(0, stream.cuda_stream)
    total_ms, count, steps, digest = 0.0, 0, 0, 0
    pmin = float("inf")
    cell = None
    wall0 = time.time()
    S = args.slices
    for q in range(S if not args.max_slices else min(S, args.max_slices)):
        E = cds._Elements(dpop)
        st = cds.cd_stats()
        opt = cds.make_options(rank=q, n_ranks=S, device=0, stream=stream.cuda_stream,
                               inputs_on_device=True, allocator=talloc, cell_factor=cell,
                               digest_only=True)
        opt.stats = C.pointer(st)
        out = cds.cd_conjunctions()
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        cds._check(cds.cd_screen_ex(E.s, E.n, cfg.t0, cfg.t1, dt, cfg.d, mode, opt, out))
        e1.record(stream)
        cds.cd_conjunctions_free(out)
        torch.cuda.synchronize()
        total_ms += e0.elapsed_time(e1)
        if cell is None and st.cell_factor > 0:
            cell = float(st.cell_factor)
        count += int(st.digest_conjunctions)
        digest = (digest + int(st.digest)) % (1 << 64)
        pmin = min(pmin, float(st.min_pca))
        steps += int(st.steps)
        print(json.dumps({"slice": q, "ms": round(total_ms, 1), "records": count}), file=sys.stderr, flush=True)
    print(json.dumps({"config": args.config, "variant": args.variant, "n": n, "dt_s": dt,
                      "steps_window": K, "steps_screened": steps, "slices": S,
                      "device_s": total_ms / 1e3, "object_steps_per_s": n * steps / (total_ms / 1e3),
                      "conjunctions": count, "digest": digest, "min_pca_km": pmin,
                      "host_wall_s": time.time() - wall0}), flush=True)


if __name__ == "__main__":
    main()
