"""Multi-process (world size 2, gloo, CPU) tests of the time-slice sharding and the record merge
(paper_conf_ipps_hellwigcmbw23_b200/dist.py).  Each rank screens its slice with the oracle
(stand-in for the GPU call on a CPU-only box); the gathered union must equal the whole-window
result exactly (owner rule: slices partition the conjunctions)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_ipps_hellwigcmbw23_b200 import dist as cdist


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _pop():
    rng = np.random.default_rng(5)
    n = 1200
    return {"a": rng.uniform(6900, 6915, n), "e": rng.uniform(0, 0.001, n),
            "inc": rng.uniform(0, np.pi, n), "raan": rng.uniform(0, 2 * np.pi, n),
            "argp": rng.uniform(0, 2 * np.pi, n), "nu0": rng.uniform(0, 2 * np.pi, n)}


def _worker(rank, world, port, t1, d, ret):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import oracle
        pop = _pop()
        K = oracle.num_steps(0.0, t1, 1.0)
        k0, k1 = cdist.slice_range(K, rank, world)
        gc = oracle.cell_size(d, 1.0)
        Kc = oracle.candidates_grid(pop, 0.0, t1, 1.0, gc, k_begin=k0, k_end=k1)
        C = oracle.conjunctions(pop, 0.0, t1, 1.0, d, gc, Kc)
        local = torch.from_numpy(np.frombuffer(C.tobytes(), dtype=np.uint8).reshape(-1, 32).copy())
        allrec = cdist.gather_records(local)
        if rank == 0:
            ret.put(allrec.numpy().tobytes())
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_slices_gather_equals_whole_window(orc, world):
    t1, d = 80.0, 10.0
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, t1, d, q)) for r in range(world)]
    for p in procs:
        p.start()
    data = q.get(timeout=300)
    for p in procs:
        p.join(timeout=300)
        assert p.exitcode == 0
    got = np.frombuffer(data, dtype=orc.CONJ_DTYPE)
    got = np.sort(got, order=["i", "j", "step"])
    pop = _pop()
    gc = orc.cell_size(d, 1.0)
    K = orc.candidates_grid(pop, 0.0, t1, 1.0, gc)
    whole = orc.conjunctions(pop, 0.0, t1, 1.0, d, gc, K)
    assert len(whole) > 10
    assert np.array_equal(got[["i", "j", "step"]], whole[["i", "j", "step"]])
    assert np.array_equal(got["tca"], whole["tca"])


def test_slice_range_partitions():
    for K in (1, 2, 7, 86401, 604801):
        for S in (1, 2, 3, 8, 24, 192):
            r = [cdist.slice_range(K, q, S) for q in range(S)]
            assert r[0][0] == 0 and r[-1][1] == K
            assert all(a[1] == b[0] for a, b in zip(r, r[1:]))
