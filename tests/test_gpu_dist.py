"""The multi-GPU data plane on a GPU (north star: "the per-GPU conjunction
lists are merged with an NCCL all-gather over NVLink, then deduplicated").  The round-end GPU
box has one device, so the NCCL path runs at world size 1 -- the same code (process group, count
+ record all-gather, device sort, duplicate check, max-over-ranks timing) as at 8 ranks; the
world-size 2/3 logic is covered on CPU with gloo (tests/test_dist_cpu.py)."""
import json
import os
import socket
import subprocess
import sys
from pathlib import Path

import numpy as np
import pytest

from tools import popgen

pytestmark = pytest.mark.gpu
cds = pytest.importorskip("paper_conf_ipps_hellwigcmbw23_b200")
from paper_conf_ipps_hellwigcmbw23_b200 import dist as cdist  # noqa: E402

ROOT = Path(__file__).resolve().parent.parent


@pytest.fixture(scope="module", autouse=True)
def _need_gpu():
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def test_nccl_merge_of_time_slices_equals_whole_window():
    """Four time slices screened on the device (cd_screen_ex, device results), their records
    merged through the NCCL process group (all-gather + cd_conjunctions_sort_device): identical,
    row for row and field for field, to the whole-window screen, and free of duplicates."""
    import torch
    import torch.distributed as dist
    torch.cuda.set_device(0)
    dist.init_process_group("nccl", init_method=f"tcp://127.0.0.1:{_port()}", rank=0, world_size=1,
                            device_id=torch.device("cuda", 0))
    try:
        assert dist.get_backend() == "nccl"
        pop = popgen.random_population(30000, 91, "catalog", 6000)
        t0, t1, dt, d = 100.0, 1300.0, 1.0, 5.0
        whole = cds.screen(pop, t0, t1, dt, d)
        dev = torch.device("cuda", 0)
        parts = []
        for q in range(4):
            E = cds._Elements(pop)
            opt = cds.make_options(rank=q, n_ranks=4, device=0, outputs_on_device=True)
            out = cds.cd_conjunctions()
            cds._check(cds.cd_screen_ex(E.s, E.n, t0, t1, dt, d, cds.CD_GRID, opt, out))
            parts.append(cdist.device_records_to_tensor(out, dev))
            cds.cd_conjunctions_free(out)
        # slice 2's rows arrive first: the merge must restore the (i, j, step) order
        local = torch.cat([parts[2], parts[0], parts[3], parts[1]])
        merged = cdist.merge_conjunctions(local, stream=torch.cuda.current_stream().cuda_stream)
        torch.cuda.synchronize()
        assert cdist.count_duplicates(merged) == 0
        got = cdist.records_to_numpy(merged)
        assert len(whole) > 50
        assert np.array_equal(got, whole)
        # a duplicated row is detected
        assert cdist.count_duplicates(torch.cat([merged[:1], merged])) == 1
    finally:
        dist.destroy_process_group()


def test_bench_distributed_path_under_torchrun():
    """bench.py's NCCL path (torchrun, --dist at one rank): the process group, the merge of
    every timed step, the settled cell edge fed to the next slices, and the e2e leg with the
    merge inside; the merged result of the last step has no duplicates."""
    cmd = [sys.executable, "-m", "torch.distributed.run", "--standalone", "--nnodes=1",
           "--nproc-per-node=1", str(ROOT / "bench.py"), "--dist", "--config", "2", "--steps", "4",
           "--warmup", "3", "--no-cpu-baseline", "--no-hybrid", "--e2e-steps", "2"]
    env = dict(os.environ, MASTER_ADDR="127.0.0.1")
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=900, cwd=ROOT, env=env)
    assert r.returncode == 0, r.stderr[-3000:]
    line = json.loads([x for x in r.stdout.splitlines() if x.startswith("{")][-1])
    assert line["merge"]["backend"] == "nccl" and line["merge"]["ranks"] == 1
    assert line["merge"]["duplicates_last_step"] == 0
    assert line["merge"]["records_last_step"] > 0
    assert line["value"] > 0 and line["e2e"]["value"] > 0 and line["e2e"]["d2h_bytes_per_step"] > 0
    assert line["config"]["conjunctions"] > 0


def test_nccl_merge_of_shards_times_slices():
    """The two sharding axes (SURVEY 8(e) time slices x 8(f) radial object-space shards) through
    the NCCL merge: 3 radial shards x 2 time slices screened on the device (shard members only,
    R21), ids mapped to the caller's, gathered and sorted over the process group -- identical to
    the whole screen, without duplicates."""
    import torch
    import torch.distributed as dist
    torch.cuda.set_device(0)
    dist.init_process_group("nccl", init_method=f"tcp://127.0.0.1:{_port()}", rank=0, world_size=1,
                            device_id=torch.device("cuda", 0))
    try:
        pop = popgen.random_population(30000, 92, "catalog", 6000)
        t0, t1, dt, d = 500.0, 1099.0, 1.0, 5.0
        whole = cds.screen(pop, t0, t1, dt, d)
        bounds = cdist.shell_bounds(pop, 3)
        parts = []
        for s in range(len(bounds) - 1):
            for q in range(2):
                r, _ = cdist.screen_shard(pop, t0, t1, dt, d, bounds, s, rank=q, n_ranks=2)
                parts.append(torch.from_numpy(np.frombuffer(r.tobytes(), dtype=np.uint8).reshape(-1, 32).copy()))
        local = torch.cat(parts[::-1]).cuda()
        merged = cdist.merge_conjunctions(local, stream=torch.cuda.current_stream().cuda_stream)
        torch.cuda.synchronize()
        assert cdist.count_duplicates(merged) == 0
        assert len(whole) > 50
        assert np.array_equal(cdist.records_to_numpy(merged), whole)
    finally:
        dist.destroy_process_group()


def test_bench_two_ranks_share_one_gpu():
    """bench.py's multi-rank logic (slices per rank, max-over-ranks time, summed units and counts,
    the per-step merge, the e2e leg with the merge) at world size 2 on the one-GPU box, through
    the gloo backend (CD_BENCH_BACKEND, testing only; the product path is NCCL, one rank per
    GPU): the day's conjunctions over both ranks equal the stored oracle count of config 2."""
    import json as _json
    z = np.load(ROOT / "tests" / "golden" / "fullwindow_cfg2_grid.npz")
    want = _json.loads(str(z["meta"]))["conjunctions"]
    cmd = [sys.executable, "-m", "torch.distributed.run", "--standalone", "--nnodes=1",
           "--nproc-per-node=2", str(ROOT / "bench.py"), "--config", "2", "--steps", "4",
           "--warmup", "3", "--no-cpu-baseline", "--e2e-steps", "2"]
    env = dict(os.environ, MASTER_ADDR="127.0.0.1", CD_BENCH_BACKEND="gloo")
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=900, cwd=ROOT, env=env)
    assert r.returncode == 0, r.stderr[-3000:]
    line = json.loads([x for x in r.stdout.splitlines() if x.startswith("{")][-1])
    assert line["n_gpus"] == 2 and line["config"]["slices"] == 8
    assert line["config"]["conjunctions"] == want
    assert line["merge"]["ranks"] == 2 and line["merge"]["duplicates_last_step"] == 0
    assert line["hybrid"]["steps_in_window"] == 9601
    assert line["e2e"]["value"] > 0
