"""Fixed cost of one library call (strong scaling cuts the day into many calls): device time of
cd_screen_ex over a 1-step and a 541-step slice of config 4, repeated; the difference per step
is the step cost, the intercept the per-call cost.

    python tools/call_overhead.py [--reps 30]
"""
import argparse
import ctypes as C
import json
import sys
from pathlib import Path

sys.path.insert(0, str(Path(__file__).resolve().parent.parent))

import numpy as np  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--reps", type=int, default=30)
    args = ap.parse_args()
    import torch
    import paper_conf_ipps_hellwigcmbw23_b200 as cds
    from paper_conf_ipps_hellwigcmbw23_b200 import dist as cdist
    from tools import popgen
    pop, cfg, _ = popgen.make_config(4)
    dev = torch.device("cuda", 0)
    dpop = {k: torch.from_numpy(v).to(dev) for k, v in pop.items()}
    stream = torch.cuda.current_stream(dev)
    talloc = cds.TorchAllocator(0, stream.cuda_stream)
    cell = None
    out = {}
    for steps in (1, 541):
        times = []
        for r in range(args.reps + 3):
            E = cds._Elements(dpop)
            st = cds.cd_stats()
            opt = cds.make_options(device=0, stream=stream.cuda_stream, inputs_on_device=True,
                                   outputs_on_device=True, allocator=talloc, cell_factor=cell)
            opt.stats = C.pointer(st)
            res = cds.cd_conjunctions()
            t0 = 40000.0 + 1000.0 * r
            torch.cuda.synchronize()
            e0 = torch.cuda.Event(enable_timing=True)
            e1 = torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            cds._check(cds.cd_screen_ex(E.s, E.n, t0, t0 + steps - 1, 1.0, cfg.d, cds.CD_GRID, opt, res))
            recs = cdist.device_records_to_tensor(res, dev)
            cds.cd_conjunctions_free(res)
            e1.record(stream)
            torch.cuda.synchronize()
            if cell is None and st.cell_factor > 0:
                cell = float(st.cell_factor)
            if r >= 3:
                times.append(e0.elapsed_time(e1))
        out[steps] = float(np.median(times))
    step = (out[541] - out[1]) / 540.0
    print(json.dumps({"ms_call_1_step": out[1], "ms_call_541_steps": out[541], "ms_per_step": step,
                      "ms_fixed_per_call": out[1] - step}))


if __name__ == "__main__":
    main()
