"""Radial object-space shards on the device (cd_options.shell_lo/hi +
cd_shell_members): shard s holds only its members and keeps the candidates whose smaller radius
at t_k lies in its band.  The shards of a partition must report disjoint sets whose union is the
unsharded result -- exactly (same positions, same refinement arithmetic on every shard)."""
import numpy as np
import pytest

from tools import popgen

pytestmark = pytest.mark.gpu

cds = pytest.importorskip("paper_conf_ipps_hellwigcmbw23_b200")
from paper_conf_ipps_hellwigcmbw23_b200 import dist as cdist  # noqa: E402


@pytest.fixture(scope="module", autouse=True)
def _need_gpu():
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")


def _union(parts):
    u = np.concatenate(parts)
    return u[np.lexsort((u["step"], u["j"], u["i"]))]


@pytest.mark.parametrize("S,mode,prop", [(2, "grid", "kepler"), (5, "grid", "kepler"),
                                         (3, "hybrid", "kepler"), (4, "grid", "j2")])
def test_shards_union_equals_unsharded(S, mode, prop):
    pop = dict(popgen.random_population(30000, 77, "catalog", 6000), propagator=prop)
    dt = 1.0 if mode == "grid" else 9.0
    t0, t1, d = 1000.0, 1000.0 + 300 * dt, 5.0
    whole = cds.screen(pop, t0, t1, dt, d, mode=mode)
    b = cdist.shell_bounds(pop, S)
    parts, members = [], []
    for s in range(S):
        r, m = cdist.screen_shard(pop, t0, t1, dt, d, b, s, mode=mode)
        parts.append(r)
        members.append(m)
    got = _union(parts)
    assert len(whole) > 50
    assert len(got) == len(whole)
    assert np.array_equal(got, whole)
    assert max(members) < len(pop["a"])
    if mode == "grid":
        Kw = cds.candidates(pop, t0, t1, dt, d)
        Ku = _union([cdist.candidates_shard(pop, t0, t1, dt, d, b, s) for s in range(S)])
        assert np.array_equal(Ku, Kw)


def test_shards_full_size_config4():
    """1M objects (BASELINE config 4), 8 shards, 2 minutes of the day: union == unsharded, and
    every shard holds well under the whole population (the point of the row)."""
    pop, cfg, _ = popgen.make_config(4)
    t0, t1, dt, d = 40000.0, 40120.0, cfg.dt_grid, cfg.d
    whole = cds.screen(pop, t0, t1, dt, d)
    b = cdist.shell_bounds(pop, 8)
    parts, members = [], []
    for s in range(8):
        r, m = cdist.screen_shard(pop, t0, t1, dt, d, b, s)
        parts.append(r)
        members.append(m)
    assert np.array_equal(_union(parts), whole)
    assert max(members) < 0.35 * len(pop["a"]), members


def test_shard_option_errors():
    pop = popgen.random_population(200, 3)
    for bad in ((7000.0, 6000.0), (-1.0, 7000.0)):
        with pytest.raises(cds.CdError) as ei:
            cds.screen(pop, 0.0, 10.0, 1.0, 2.0, shell=bad)
        assert ei.value.status == cds.CD_EINVAL
    with pytest.raises(cds.CdError) as ei:
        cds.screen(pop, 0.0, 10.0, 1.0, 2.0, mode="legacy", shell=(0.0, 7000.0))
    assert ei.value.status == cds.CD_EINVAL


def test_shards_times_slices():
    """The two sharding axes combine (rank = (shard, time slice)): 3 radial shards x 4 time
    slices partition the result exactly."""
    pop = popgen.random_population(20000, 78, "catalog", 4000)
    t0, t1, dt, d = 500.0, 899.0, 1.0, 5.0
    whole = cds.screen(pop, t0, t1, dt, d)
    b = cdist.shell_bounds(pop, 3)
    parts = [cdist.screen_shard(pop, t0, t1, dt, d, b, s, rank=q, n_ranks=4)[0]
             for s in range(3) for q in range(4)]
    assert len(whole) > 50
    assert np.array_equal(_union(parts), whole)


@pytest.mark.parametrize("mode,dt,prop,S", [("grid", 1.0, "kepler", 2), ("grid", 1.0, "kepler", 5),
                                            ("hybrid", 9.0, "kepler", 3), ("grid", 1.0, "j2", 3)])
def test_library_l2_shards_equal_unsharded(mode, dt, prop, S):
    """cd_options.shards: the library screens S radial bands in turn on one device; the result is
    identical, field by field, to the unsharded call (and the default auto mode is off here)."""
    import torch
    pop = dict(popgen.random_population(30000, 79, "catalog", 6000), propagator=prop)
    t0, t1, d = 2000.0, 2000.0 + 250 * dt, 5.0
    one = cds.screen(pop, t0, t1, dt, d, mode=mode, shards=1)
    auto = cds.screen(pop, t0, t1, dt, d, mode=mode)
    many, st = cds.screen(pop, t0, t1, dt, d, mode=mode, shards=S, return_stats=True)
    assert len(one) > 50
    assert np.array_equal(auto, one)
    assert np.array_equal(many, one)
    tp = {k: torch.from_numpy(v).cuda() for k, v in pop.items() if k != "propagator"}
    tp["propagator"] = prop
    dev = cds.screen(tp, t0, t1, dt, d, mode=mode, shards=S, allocator="torch")
    assert np.array_equal(dev, one)
