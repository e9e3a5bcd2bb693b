"""Radial object-space shards on the device (cd_options.shell_lo/hi +
cd_shell_members; reading R21): shard s holds only its members and keeps the candidates whose
smaller radius at t_k lies in its band.  Each CUDA shard is compared with the oracle's shard --
R21 written out on the oracle side (member rule, oracle screen of the subset, band rule) --
element by element; the shards of a partition must also report disjoint sets whose union is the
unsharded CUDA result, exactly."""
import numpy as np
import pytest

import oracle
from tools import popgen
from tests import parity

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


EDGE_KM = 1e-6   # band-edge ambiguity: min radius within 1 mm of a band edge (either side)


def _rmin(pop, rows, t0, dt):
    """min(|r_i(t_k)|, |r_j(t_k)|) of every row (i, j, step), from the oracle's propagator."""
    out = np.zeros(len(rows))
    for k in np.unique(rows["step"]):
        sel = np.nonzero(rows["step"] == k)[0]
        ids = np.unique(np.concatenate([rows["i"][sel], rows["j"][sel]]))
        x = oracle.propagate(popgen.subset(pop, ids), [t0 + float(k) * dt])[0]
        r = dict(zip(ids.tolist(), np.linalg.norm(x, axis=1)))
        out[sel] = [min(r[int(a)], r[int(b)]) for a, b in zip(rows["i"][sel], rows["j"][sel])]
    return out


def oracle_shard(pop, t0, t1, dt, d, lo, hi, mode="grid"):
    """The oracle's result for radial shard [lo, hi) as the plain definition of R21 states it:
    the members (cd_shell_members' rule, written out here: radius range [a(1-e), a(1+e)] meets
    [lo, hi + g_c)), the oracle screen on that subset (O2+O3 grid, O4 hybrid), the rows whose
    smaller radius at t_k lies in [lo, hi), ids mapped back.  Also returns the rows whose smaller
    radius is within 1 mm of a band edge (either side; excused, counted)."""
    gc = oracle.cell_size(d, dt)
    q, Q = pop["a"] * (1 - pop["e"]), pop["a"] * (1 + pop["e"])
    idx = np.nonzero((Q >= lo) & (q < hi + gc))[0]
    sub = popgen.subset(pop, idx)
    if "propagator" in pop:
        sub["propagator"] = pop["propagator"]
    if mode == "grid":
        K = oracle.candidates_grid(sub, t0, t1, dt, gc)
        C = oracle.conjunctions(sub, t0, t1, dt, d, gc, K)
    else:
        C, _ = oracle.hybrid(sub, t0, t1, dt, d)
    rm = _rmin(sub, C, t0, dt)
    keep = (rm >= lo) & (rm < hi)
    amb = (np.abs(rm - lo) < EDGE_KM) | (np.abs(rm - hi) < EDGE_KM)
    C = C.copy()
    C["i"], C["j"] = idx[C["i"]], idx[C["j"]]
    return C[keep & ~amb], C[amb], len(idx)


def _drop(rows, amb):
    if len(amb) == 0 or len(rows) == 0:
        return rows
    bad = set(zip(amb["i"].tolist(), amb["j"].tolist(), amb["step"].tolist()))
    m = np.array([(a, b, c) not in bad for a, b, c in zip(rows["i"].tolist(), rows["j"].tolist(),
                                                          rows["step"].tolist())], dtype=bool)
    return rows[m]


@pytest.mark.parametrize("S,mode,prop", [(2, "grid", "kepler"), (5, "grid", "kepler"),
                                         (3, "hybrid", "kepler"), (4, "grid", "j2")])
def test_shards_against_oracle(S, mode, prop):
    """Every CUDA shard against the oracle's shard (R21 written out on the oracle side), element
    by element; then the union of the CUDA shards against the unsharded CUDA screen."""
    pop = dict(popgen.random_population(30000, 77, "catalog", 6000), propagator=prop)
    dt = 1.0 if mode == "grid" else 9.0
    t0, t1, d = 1000.0, 1000.0 + 300 * dt, 5.0
    gc = oracle.cell_size(d, dt)
    b = cdist.shell_bounds(pop, S)
    parts, members, matched, amb_total = [], [], 0, 0
    for s in range(len(b) - 1):
        r, m = cdist.screen_shard(pop, t0, t1, dt, d, b, s, mode=mode)
        o, amb, mo = oracle_shard(pop, t0, t1, dt, d, b[s], b[s + 1], mode)
        assert m == mo                                   # same member set
        res = parity.compare_conjunctions(pop, _drop(r, amb), o, t0, t1, dt, d, gc)
        assert res["one_sided"] == 0
        matched += res["matched"]
        amb_total += len(amb)
        parts.append(r)
        members.append(m)
    assert matched > 50 and amb_total <= 2, (matched, amb_total)
    whole = cds.screen(pop, t0, t1, dt, d, mode=mode)
    assert np.array_equal(_union(parts), whole)
    assert max(members) < len(pop["a"])
    if mode == "grid":
        Kw = cds.candidates(pop, t0, t1, dt, d)
        Ku = _union([cdist.candidates_shard(pop, t0, t1, dt, d, b, s) for s in range(len(b) - 1)])
        assert np.array_equal(Ku, Kw)


def test_shards_full_size_config4():
    """1M objects (BASELINE config 4), 8 shards, 2 minutes of the day: each shard against the
    oracle's shard on two sampled steps, the union equal to the unsharded screen, and every shard
    well under the whole population (the point of the row)."""
    pop, cfg, _ = popgen.make_config(4)
    t0, t1, dt, d = 40000.0, 40120.0, cfg.dt_grid, cfg.d
    gc = oracle.cell_size(d, dt)
    whole = cds.screen(pop, t0, t1, dt, d)
    b = cdist.shell_bounds(pop, 8)
    parts, members = [], []
    for s in range(len(b) - 1):
        r, m = cdist.screen_shard(pop, t0, t1, dt, d, b, s)
        parts.append(r)
        members.append(m)
        for k in (17, 101):
            tk = t0 + k * dt
            # oracle window [t_k - dt, t_k + dt]: its middle step is step k of the screen
            o, amb, _ = oracle_shard(pop, tk - dt, tk + dt, dt, d, b[s], b[s + 1])
            o, amb = o[o["step"] == 1].copy(), amb[amb["step"] == 1].copy()
            o["step"] += k - 1
            amb["step"] += k - 1
            rs = _drop(r[r["step"] == k], amb)
            res = parity.compare_conjunctions(pop, rs, o, t0, t1, dt, d, gc)
            assert res["one_sided"] == 0
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
