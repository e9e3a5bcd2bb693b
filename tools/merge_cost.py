"""Cost of the record merge (dist.merge_conjunctions: count + record all-gather over the
process group, device sort) for a given record count, at the world size it is launched with.

    torchrun --nproc-per-node N tools/merge_cost.py [--records 538000] [--reps 20]
"""
import argparse
import json
import os
import sys
from pathlib import Path

sys.path.insert(0, str(Path(__file__).resolve().parent.parent))

import numpy as np  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--records", type=int, default=538000)
    ap.add_argument("--reps", type=int, default=20)
    args = ap.parse_args()
    import torch
    import torch.distributed as dist
    from paper_conf_ipps_hellwigcmbw23_b200 import dist as cdist
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    world, rank = dist.get_world_size(), dist.get_rank()
    m = args.records // world
    rng = np.random.default_rng(rank)
    rec = np.zeros(m, dtype=[("i", "<u4"), ("j", "<u4"), ("step", "<u4"), ("flags", "<u4"),
                             ("tca", "<f8"), ("pca", "<f8")])
    rec["i"] = rng.integers(0, 500000, m)
    rec["j"] = rec["i"] + 1 + rng.integers(0, 500000, m)
    rec["step"] = rng.integers(0, 4000, m) + 4000 * rank
    local_t = torch.from_numpy(np.frombuffer(rec.tobytes(), dtype=np.uint8).reshape(-1, 32).copy()).cuda()
    st = torch.cuda.current_stream()
    times = []
    for r in range(args.reps + 3):
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(st)
        out = cdist.merge_conjunctions(local_t, stream=st.cuda_stream)
        e1.record(st)
        torch.cuda.synchronize()
        if r >= 3:
            times.append(e0.elapsed_time(e1))
    if rank == 0:
        print(json.dumps({"world": world, "records": int(out.shape[0]), "ms_median": float(np.median(times)),
                          "ms_min": float(np.min(times))}))
    dist.destroy_process_group()


if __name__ == "__main__":
    main()
