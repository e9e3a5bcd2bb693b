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


def test_count_duplicates():
    """The merge's dedupe check (dist.count_duplicates) on sorted 32-byte records."""
    recs = np.zeros(5, dtype=[("i", "<u4"), ("j", "<u4"), ("step", "<u4"), ("flags", "<u4"),
                              ("tca", "<f8"), ("pca", "<f8")])
    recs["i"] = [1, 1, 1, 2, 2]
    recs["j"] = [3, 3, 4, 5, 5]
    recs["step"] = [7, 8, 8, 9, 9]
    t = torch.from_numpy(np.frombuffer(recs.tobytes(), dtype=np.uint8).reshape(-1, 32).copy())
    assert cdist.count_duplicates(t) == 1
    assert cdist.count_duplicates(t[:4]) == 0
    assert cdist.count_duplicates(t[:1]) == 0


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


# ----------------------------------------------------------------------------------------
# radial object-space shards: host logic on CPU
# ----------------------------------------------------------------------------------------

def _shard_worker(rank, world, port, t1, d, ret):
    """Each rank: its shard's members (the library's host helper cd_shell_members), the oracle's
    candidate set on the member subset, the shard rule (smaller radius in the band) applied as
    a plain definition, ids mapped back; gathered over gloo."""
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import oracle
        from tools import popgen
        pop = popgen.random_population(1500, 21, "catalog", 300)
        gc = oracle.cell_size(d, 1.0)
        bounds = cdist.shell_bounds(pop, world)
        lo, hi = bounds[rank], bounds[rank + 1]
        import paper_conf_ipps_hellwigcmbw23_b200 as cds
        idx = cds.shell_members(pop, lo, hi, gc)
        sub = popgen.subset(pop, idx)
        K = oracle.candidates_grid(sub, 0.0, t1, 1.0, gc)
        keep = np.zeros(len(K), dtype=bool)
        for q, c in enumerate(K):
            x = oracle.propagate(popgen.subset(sub, [c["i"], c["j"]]), [float(c["step"])])[0]
            rmin = np.min(np.linalg.norm(x, axis=1))
            keep[q] = lo <= rmin < hi
        K = K[keep]
        K["i"], K["j"] = idx[K["i"]], idx[K["j"]]
        rec = np.zeros((len(K), 32), dtype=np.uint8)
        rec[:, :12] = np.frombuffer(K.tobytes(), dtype=np.uint8).reshape(-1, 12)
        allrec = cdist.gather_records(torch.from_numpy(rec))
        if rank == 0:
            ret.put((allrec.numpy()[:, :12].tobytes(), len(idx)))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_radial_shards_partition_candidates(orc, world):
    from tools import popgen
    t1, d = 40.0, 20.0
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_shard_worker, args=(r, world, port, t1, d, q)) for r in range(world)]
    for p in procs:
        p.start()
    data, nmem = q.get(timeout=300)
    for p in procs:
        p.join(timeout=300)
        assert p.exitcode == 0
    got = np.sort(np.frombuffer(data, dtype=orc.CAND_DTYPE), order=["i", "j", "step"])
    pop = popgen.random_population(1500, 21, "catalog", 300)
    whole = orc.candidates_grid(pop, 0.0, t1, 1.0, orc.cell_size(d, 1.0))
    assert len(whole) > 50
    assert np.array_equal(got, whole)     # disjoint shards, union = the unsharded set
    assert nmem < 1500                    # rank 0 holds a strict subset


def test_shell_bounds_and_members():
    import paper_conf_ipps_hellwigcmbw23_b200 as cds
    from tools import popgen
    pop = popgen.random_population(5000, 22, "catalog", 1000)
    for S in (1, 2, 4, 8):
        b = cdist.shell_bounds(pop, S)
        assert len(b) == S + 1 and b[0] == 0.0 and all(x < y for x, y in zip(b, b[1:]))
        own = np.histogram(pop["a"], bins=b)[0]
        assert own.max() <= 5000 // S + 2            # balanced by mean radius
        gc = 9.8
        for s in range(S):
            idx = cds.shell_members(pop, b[s], b[s + 1], gc)
            q, Q = pop["a"] * (1 - pop["e"]), pop["a"] * (1 + pop["e"])
            want = np.where((Q >= b[s]) & (q < b[s + 1] + gc))[0]
            assert np.array_equal(idx, want.astype(np.uint32))
    with pytest.raises(cds.CdError):
        cds.shell_members(pop, 7000.0, 7000.0, 1.0)


def test_shell_bounds_merge_duplicate_quantiles():
    """Many objects with one a (a shell): coinciding quantiles merge bands instead of producing an
    empty band [b, b) (which cd_shell_members rejects); the bands still partition [0, inf)."""
    import paper_conf_ipps_hellwigcmbw23_b200 as cds
    from tools import popgen
    pop = popgen.random_population(2000, 23, "catalog", 0)
    pop["a"][:1400] = 7000.0
    b = cdist.shell_bounds(pop, 8)
    assert b[0] == 0.0 and b[-1] == cdist.FAR_KM
    assert all(x < y for x, y in zip(b, b[1:]))
    assert len(b) - 1 < 8
    own = np.histogram(pop["a"], bins=b)[0]
    assert own.sum() == 2000
    for s in range(len(b) - 1):
        cds.shell_members(pop, b[s], b[s + 1], 9.8)   # no CD_EINVAL


def test_elements_validation():
    """The binding checks the layout cdscreen.h assumes before any pointer reaches C."""
    import paper_conf_ipps_hellwigcmbw23_b200 as cds
    from tools import popgen
    pop = popgen.random_population(100, 24, "catalog", 0)
    bad = dict(pop, e=pop["e"][:50])
    with pytest.raises(ValueError, match="different lengths"):
        cds._Elements(bad)
    bad = dict(pop, inc=np.stack([pop["inc"], pop["inc"]]))
    with pytest.raises(ValueError, match="1-D"):
        cds._Elements(bad)
    E = cds._Elements(dict(pop, a=pop["a"].astype(np.float32)))   # host arrays are converted
    assert E.n == 100 and E.keep[0].dtype == np.float64
