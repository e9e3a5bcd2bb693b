"""GPU parity: the CUDA path (through the C ABI) against the oracle, element by element.

Tolerances (BASELINE.json north star): positions 1e-9 relative; identical (i, j, k) candidate
and (i, j, step) conjunction sets except within 1 mm of the thresholds (and the other
exclusions of SURVEY.md 8(c)); TCA within 1e-3 s and PCA within 1 m."""
import math

import numpy as np
import pytest

import oracle
from tools import popgen
from tests import parity

pytestmark = pytest.mark.gpu

cds = pytest.importorskip("paper_conf_ipps_hellwigcmbw23_b200")


@pytest.fixture(scope="module", autouse=True)
def _need_gpu():
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")


def _mix(n, seed, incl="paper", shells=0):
    return popgen.random_population(n, seed, incl, shells)


# ----------------------------------------------------------------------------------------
# a1-a2: propagation
# ----------------------------------------------------------------------------------------

def test_propagate_positions_1e9():
    rng = np.random.default_rng(7)
    pop = _mix(20000, 1)
    # include every eccentricity class and the Contour edge cases
    extra = {"a": np.full(12, 26000.0), "e": np.array([0.0, 1e-13, 0.005, 0.05, 0.2, 0.45, 0.7, 0.8,
                                                     0.85, 0.9, 0.95, 0.99]),
             "inc": np.full(12, 1.0), "raan": np.full(12, 0.3), "argp": np.full(12, 0.2),
             "nu0": np.zeros(12)}
    pop = popgen.concat(pop, extra)
    times = np.concatenate([[0.0, 1.0, 86400.0, 604800.0], rng.uniform(0, 86400, 6)])
    xg, vg = cds.propagate(pop, times, velocity=True)
    xo, vo = oracle.propagate(pop, times, velocity=True)
    rel = np.linalg.norm(xg - xo, axis=2) / np.linalg.norm(xo, axis=2)
    assert rel.max() < 1e-9, rel.max()
    relv = np.linalg.norm(vg - vo, axis=2) / np.linalg.norm(vo, axis=2)
    assert relv.max() < 1e-9, relv.max()


def test_propagate_kepler_edges():
    """Mean anomaly exactly at / next to 0, pi, 2pi and the contour-node case sin(M+e) = 1."""
    mu = oracle.mu()
    rows = []
    for e in (0.0025, 0.05, 0.2, 0.5, 0.75):
        a = 8000.0
        nm = math.sqrt(mu / a ** 3)
        for M in (0.0, math.pi, math.pi / 2 - e, 1.5 * math.pi + e, 2 * math.pi - 1e-12, 1e-12,
                  math.pi - 1e-12, math.pi + 1e-12):
            rows.append((a, e, M / nm))
    n = len(rows)
    pop = {"a": np.array([r[0] for r in rows]), "e": np.array([r[1] for r in rows]),
           "inc": np.full(n, 0.5), "raan": np.full(n, 1.0), "argp": np.full(n, 2.0),
           "nu0": np.zeros(n)}
    for q, r in enumerate(rows):
        xg = cds.propagate(popgen.subset(pop, [q]), [r[2]])
        xo = oracle.propagate(popgen.subset(pop, [q]), [r[2]])
        assert np.all(np.isfinite(xg))
        assert np.linalg.norm(xg - xo) / np.linalg.norm(xo) < 1e-9, (r, xg, xo)


# ----------------------------------------------------------------------------------------
# a3-a6: candidate set K
# ----------------------------------------------------------------------------------------

def test_candidates_config1_brute_force():
    pop, cfg, _ = popgen.make_config(1)
    gc = oracle.cell_size(cfg.d, cfg.dt_grid)
    Kg = cds.candidates(pop, cfg.t0, cfg.t1, cfg.dt_grid, cfg.d)
    Ko = oracle.candidates_brute(pop, cfg.t0, cfg.t1, cfg.dt_grid, gc)
    assert parity.is_sorted(Kg)
    assert parity.compare_candidates(pop, Kg, Ko, cfg.t0, cfg.dt_grid, gc) == 0
    assert len(Kg) > 500


@pytest.mark.parametrize("n,steps,d", [(5037, 300, 2.0), (20011, 120, 10.0)])
def test_candidates_ragged_sizes(n, steps, d):
    pop = _mix(n, 100 + n, "catalog", shells=n // 5)
    gc = oracle.cell_size(d, 1.0)
    Kg = cds.candidates(pop, 0.0, steps - 1.0, 1.0, d)
    Ko = oracle.candidates_grid(pop, 0.0, steps - 1.0, 1.0, gc)
    parity.compare_candidates(pop, Kg, Ko, 0.0, 1.0, gc)
    assert len(Ko) > 0


@pytest.mark.parametrize("kw", [dict(grid_origin=(1234.5, -987.25, 55.125)), dict(cell_factor=1.0),
                                dict(grid_table=1), dict(grid_table=1, cell_factor=1.0),
                                dict(grid_table=2, cell_factor=1.0), dict(grid_table=1, round_steps=5),
                                dict(cell_factor=2.0), dict(cell_factor=1.5, grid_origin=(-3e3, 7.5, 1e4)),
                                dict(cell_factor=3.7), dict(batch_object_steps=1),
                                dict(round_steps=7), dict(batch_object_steps=10 ** 7),
                                dict(grid_table=3), dict(grid_table=3, cell_factor=1.0),
                                dict(grid_table=3, batch_object_steps=1), dict(grid_table=3, round_steps=5),
                                dict(grid_table=2, cell_factor=1.5, grid_origin=(-3e3, 7.5, 1e4)),
                                dict(grid_table=2, cell_factor=1.9, grid_origin=(11.0, -2.5, 0.75)),
                                dict(grid_table=1, cell_factor=1.9)])
def test_candidates_invariance(kw):
    pop = _mix(8000, 5)
    d = 20.0
    gc = oracle.cell_size(d, 1.0)
    Ko = oracle.candidates_grid(pop, 0.0, 59.0, 1.0, gc)
    Kg = cds.candidates(pop, 0.0, 59.0, 1.0, d, **kw)
    parity.compare_candidates(pop, Kg, Ko, 0.0, 1.0, gc)


@pytest.mark.parametrize("table", [1, 2, 3])
def test_halfshell_reach_swarm(table):
    """Half-shell scans skip the neighbour cells out of reach of the object (halfshell_reach):
    a compact swarm puts thousands of pairs across cell faces, edges and corners at distances
    around g_c; every cell edge in half-shell mode (g_c <= L < 2 g_c) must give the brute-force
    candidate set."""
    rng = np.random.default_rng(21)
    n = 2500
    pop = {"a": 7000.0 + rng.uniform(-40, 40, n), "e": rng.uniform(0, 2e-3, n),
           "inc": 0.9 + rng.normal(0, 4e-3, n), "raan": 1.0 + rng.normal(0, 4e-3, n),
           "argp": rng.uniform(0, 0.2, n), "nu0": rng.uniform(0, 0.2, n)}
    d, dt = 20.0, 1.0
    gc = oracle.cell_size(d, dt)
    Ko = oracle.candidates_brute(pop, 0.0, 4.0, dt, gc)
    assert len(Ko) > 50000
    for cf, org in ((1.0, (0.0, 0.0, 0.0)), (1.0, (13.1, -7.7, 2.9)), (1.3, (5.0, 5.0, 5.0)),
                    (1.999, (-1.0, 2.0, -3.0))):
        Kg = cds.candidates(pop, 0.0, 4.0, dt, d, cell_factor=cf, grid_origin=org, grid_table=table)
        parity.compare_candidates(pop, Kg, Ko, 0.0, dt, gc)


def test_worst_case_colocated_and_overflow_retry():
    """all objects co-located -> every pair a candidate.  3000 objects give 4.5M pairs
    in one step, above the initial queue capacity (forces the overflow retry)."""
    n = 3000
    pop = {"a": np.full(n, 7000.0), "e": np.zeros(n), "inc": np.linspace(0.1, 3.0, n),
           "raan": np.full(n, 1.0), "argp": np.zeros(n), "nu0": np.zeros(n)}
    Kg, st = cds.candidates(pop, 0.0, 0.0, 1.0, 10.0, return_stats=True)
    assert len(Kg) == n * (n - 1) // 2
    assert st["retries"] >= 1
    assert np.all(Kg["step"] == 0)


def test_best_case_far_apart():
    n = 500
    far = {"a": 7000.0 + 100.0 * np.arange(n), "e": np.zeros(n), "inc": np.full(n, 0.7),
           "raan": np.linspace(0, 6, n), "argp": np.zeros(n), "nu0": np.linspace(0, 6, n)}
    assert len(cds.candidates(far, 0.0, 600.0, 1.0, 10.0)) == 0
    assert len(cds.screen(far, 0.0, 600.0, 1.0, 10.0)) == 0


def test_time_slices_union():
    pop = _mix(6000, 9)
    d = 15.0
    whole = cds.candidates(pop, 0.0, 99.0, 1.0, d)
    parts = [cds.candidates(pop, 0.0, 99.0, 1.0, d, rank=r, n_ranks=3) for r in range(3)]
    u = np.sort(np.concatenate(parts), order=["i", "j", "step"])
    assert np.array_equal(u, whole)
    C = cds.screen(pop, 0.0, 99.0, 1.0, d)
    Cp = np.sort(np.concatenate([cds.screen(pop, 0.0, 99.0, 1.0, d, rank=r, n_ranks=3)
                                 for r in range(3)]), order=["i", "j", "step"])
    assert np.array_equal(C[["i", "j", "step"]], Cp[["i", "j", "step"]])


# ----------------------------------------------------------------------------------------
# a7: conjunctions
# ----------------------------------------------------------------------------------------

def test_screen_config1_planted_and_parity():
    pop, cfg, planted = popgen.make_config(1)
    gc = oracle.cell_size(cfg.d, cfg.dt_grid)
    Cg, st = cds.screen(pop, cfg.t0, cfg.t1, cfg.dt_grid, cfg.d, return_stats=True)
    Ko = oracle.candidates_brute(pop, cfg.t0, cfg.t1, cfg.dt_grid, gc)
    Co = oracle.conjunctions(pop, cfg.t0, cfg.t1, cfg.dt_grid, cfg.d, gc, Ko)
    assert parity.is_sorted(Cg)
    res = parity.compare_conjunctions(pop, Cg, Co, cfg.t0, cfg.t1, cfg.dt_grid, cfg.d, gc)
    assert res["matched"] >= len(Co) - 5 and res["one_sided"] == 0
    assert st["candidates"] == len(Ko)
    # planted closed form A
    mu = oracle.mu()
    for pa in planted.case_a:
        pca = 2 * pa.r * abs(math.cos(pa.delta / 2) * math.sin(pa.phi / 2))
        tca = (pa.u0 - pa.phi / 2) / math.sqrt(mu / pa.r ** 3)
        rows = Cg[(Cg["i"] == pa.ia) & (Cg["j"] == pa.ib)]
        if pca < cfg.d:
            assert len(rows) == 1 and abs(rows["tca"][0] - tca) < 1e-3 and abs(rows["pca"][0] - pca) < 1e-3
    (ia, ib), = planted.twins
    tw = Cg[(Cg["i"] == ia) & (Cg["j"] == ib)]
    assert len(tw) == 601 and np.all(tw["flags"] & cds.CD_FLAG_DEGENERATE)


@pytest.mark.parametrize("n,steps,d", [(4099, 400, 2.0), (30000, 90, 5.0)])
def test_screen_ragged_parity(n, steps, d):
    pop = _mix(n, 300 + n, "catalog", shells=n // 4)
    t1 = steps - 1.0
    gc = oracle.cell_size(d, 1.0)
    Cg = cds.screen(pop, 0.0, t1, 1.0, d)
    Ko = oracle.candidates_grid(pop, 0.0, t1, 1.0, gc)
    Co = oracle.conjunctions(pop, 0.0, t1, 1.0, d, gc, Ko)
    res = parity.compare_conjunctions(pop, Cg, Co, 0.0, t1, 1.0, d, gc)
    assert res["matched"] > 0 and res["one_sided"] == 0


@pytest.mark.parametrize("table", [1, 2])
def test_screen_dense_shell_many_conjunctions(table):
    """A compact shell with many encounters per step (exercises queue growth and refinement)."""
    rng = np.random.default_rng(3)
    n = 6000
    pop = {"a": rng.uniform(6900, 6905, n), "e": rng.uniform(0, 0.0005, n),
           "inc": rng.uniform(0, math.pi, n), "raan": rng.uniform(0, 2 * math.pi, n),
           "argp": rng.uniform(0, 2 * math.pi, n), "nu0": rng.uniform(0, 2 * math.pi, n)}
    d, t1 = 5.0, 200.0
    gc = oracle.cell_size(d, 1.0)
    Cg = cds.screen(pop, 0.0, t1, 1.0, d, round_steps=13, grid_table=table)
    Ko = oracle.candidates_grid(pop, 0.0, t1, 1.0, gc)
    Co = oracle.conjunctions(pop, 0.0, t1, 1.0, d, gc, Ko)
    res = parity.compare_conjunctions(pop, Cg, Co, 0.0, t1, 1.0, d, gc)
    assert res["matched"] > 100 and res["one_sided"] == 0


def test_edge_cases_and_errors():
    pop = _mix(50, 2)
    assert len(cds.screen(popgen.subset(pop, []), 0.0, 10.0, 1.0, 2.0)) == 0
    assert len(cds.screen(popgen.subset(pop, [0]), 0.0, 10.0, 1.0, 2.0)) == 0
    assert len(cds.candidates(pop, 5.0, 5.0, 1.0, 2.0)) == 0 or True   # K = 1 must not fail
    bad = dict(pop)
    bad["e"] = pop["e"].copy()
    bad["e"][3] = 1.2
    with pytest.raises(cds.CdError) as ei:
        cds.screen(bad, 0.0, 10.0, 1.0, 2.0)
    assert ei.value.status == cds.CD_EINVAL
    with pytest.raises(cds.CdError) as ei:
        cds.screen(pop, 0.0, 10.0, -1.0, 2.0)
    assert ei.value.status == cds.CD_EINVAL
    with pytest.raises(cds.CdError) as ei:
        cds.screen(pop, 10.0, 0.0, 1.0, 2.0)
    assert ei.value.status == cds.CD_EINVAL
    geo = {"a": np.array([42164.0, 42165.0]), "e": np.zeros(2), "inc": np.zeros(2),
           "raan": np.zeros(2), "argp": np.zeros(2), "nu0": np.array([0.0, 1.0])}
    with pytest.raises(cds.CdError) as ei:
        cds.screen(geo, 0.0, 10.0, 1.0, 0.01, v_margin=0.0)
    assert ei.value.status == cds.CD_ERANGE


def test_device_inputs_match_host_inputs():
    import torch
    pop = _mix(3000, 4)
    tp = {k: torch.from_numpy(v).cuda() for k, v in pop.items()}
    a = cds.screen(pop, 0.0, 120.0, 1.0, 10.0)
    b = cds.screen(tp, 0.0, 120.0, 1.0, 10.0)
    assert np.array_equal(a, b)


# ----------------------------------------------------------------------------------------
# full size (BASELINE.json config 4: 1M objects), bench launch configuration, sampled steps
# ----------------------------------------------------------------------------------------

@pytest.fixture(scope="module")
def cfg4():
    pop, cfg, _ = popgen.make_config(4)
    return pop, cfg


def test_full_size_sampled_steps(cfg4):
    """1M objects, the 1-hour window bench.py times; oracle on sampled steps one by one."""
    pop, cfg = cfg4
    d, dt = cfg.d, cfg.dt_grid
    t0, t1 = 7200.0, 7200.0 + 3600.0        # bench step 2 (hour 2 of 24)
    gc = oracle.cell_size(d, dt)
    Kg = cds.candidates(pop, t0, t1, dt, d)
    Cg = cds.screen(pop, t0, t1, dt, d)
    for k in (0, 1, 1800, 3599, 3600):
        Ko = oracle.candidates_grid(pop, t0, t1, dt, gc, k_begin=k, k_end=k + 1)
        Ks = Kg[Kg["step"] == k]
        parity.compare_candidates(pop, Ks, Ko, t0, dt, gc)
        assert len(Ko) > 1000
        Co = oracle.conjunctions(pop, t0, t1, dt, d, gc, Ko)
        Cs = Cg[Cg["step"] == k]
        parity.compare_conjunctions(pop, Cs, Co, t0, t1, dt, d, gc)


@pytest.mark.gpu
def test_config5_8m_sampled_steps():
    """BASELINE config 5 (8,000,000 objects, the stress population): a few steps of the 7-day
    window screened at full size, candidates and conjunctions compared with the oracle step by
    step (the same launch configuration as any other call: auto cell edge, pipelined rounds)."""
    pop, cfg = popgen.make_config(5)[:2]
    d, dt = cfg.d, cfg.dt_grid
    t0 = 3 * 86400.0 + 1234.0
    t1 = t0 + 2 * dt
    gc = oracle.cell_size(d, dt)
    Kg = cds.candidates(pop, t0, t1, dt, d)
    Cg = cds.screen(pop, t0, t1, dt, d)
    Ko = oracle.candidates_grid(pop, t0, t1, dt, gc)
    assert len(Ko) > 3 * 100000      # n^2 growth: ~64x the 1M population's rate per step
    parity.compare_candidates(pop, Kg, Ko, t0, dt, gc)
    Co = oracle.conjunctions(pop, t0, t1, dt, d, gc, Ko)
    # rows on one side only (a minimum just outside [t0, t1] taken for one) would hide here as
    # window-edge exclusions: the 2-s window has thousands of encounters straddling its ends
    assert parity.compare_conjunctions(pop, Cg, Co, t0, t1, dt, d, gc)["one_sided"] == 0


@pytest.mark.parametrize("mode,dt,R", [("grid", 1.0, 1), ("grid", 1.0, 7), ("hybrid", 9.0, 2),
                                       ("grid", 1.0, 3)])
def test_spatial_resort_is_invisible(mode, dt, R):
    """cd_options.resort_steps: renumbering the slots in Morton order every R steps (pipeline
    double-buffered: a launch builds in the new order while it scans in the old) changes nothing
    -- candidates and conjunctions identical to the unsorted screen and to the oracle."""
    pop = _mix(20000, 31, "paper", 3000)
    d = 8.0
    t0, t1 = 200.0, 200.0 + 90 * dt
    gc = oracle.cell_size(d, dt)
    kw = dict(batch_object_steps=40000) if R == 3 else {}   # B = 2 steps per batch
    K0 = cds.candidates(pop, t0, t1, dt, d, resort_steps=-1)
    K1 = cds.candidates(pop, t0, t1, dt, d, resort_steps=R, **kw)
    assert np.array_equal(K0, K1)
    C0 = cds.screen(pop, t0, t1, dt, d, mode=mode, resort_steps=-1)
    C1 = cds.screen(pop, t0, t1, dt, d, mode=mode, resort_steps=R, **kw)
    assert np.array_equal(C0, C1)
    if mode == "grid":
        Ko = oracle.candidates_grid(pop, t0, t1, dt, gc)
        parity.compare_candidates(pop, K1, Ko, t0, dt, gc)
        Co = oracle.conjunctions(pop, t0, t1, dt, d, gc, Ko)
        parity.compare_conjunctions(pop, C1, Co, t0, t1, dt, d, gc)


def test_raw_counts_and_grids_in_flight():
    """emit_raw_counts with the paper's cell (cell_factor 1) and map (grid_table 1): raw_pairs is
    the number of object pairs in the same or neighbouring cells of edge g_c, each unordered pair
    once per step -- counted here by brute force from the oracle's positions.
    grids_in_flight reports the batch B (the paper's p)."""
    pop = _mix(3000, 41, "paper", 500)
    d, dt, t0, t1 = 30.0, 1.0, 0.0, 9.0
    gc = oracle.cell_size(d, dt)
    K, st = cds.candidates(pop, t0, t1, dt, d, cell_factor=1.0, grid_table=1, emit_raw_counts=True,
                           return_stats=True)
    want = 0
    x = oracle.propagate(pop, t0 + dt * np.arange(10))
    # the library's cell edge for cell_factor 1 is g_c (1 + 1e-12), origin 0
    L = gc * (1.0 + 1e-12)
    for q in range(10):
        c = np.floor(x[q] / L).astype(np.int64)
        diff = np.abs(c[:, None, :] - c[None, :, :]).max(axis=2)
        want += int(np.count_nonzero(np.triu(diff <= 1, 1)))
    assert st["raw_pairs"] == want, (st["raw_pairs"], want)
    assert st["raw_pairs"] > len(K) > 0
    assert st["grids_in_flight"] >= 1
    _, st2 = cds.candidates(pop, t0, t1, dt, d, return_stats=True)
    assert st2["raw_pairs"] == 0


def test_memory_bounded_batch():
    """the number of grids in flight p is bounded by the free device memory.  With a
    huge requested batch and most of the device memory taken, the call still runs, with fewer
    steps per batch, and returns the same result as a small batch."""
    import torch
    pop = _mix(8000, 43)
    d, t0, t1 = 20.0, 0.0, 3999.0
    ref = cds.screen(pop, t0, t1, 1.0, d, batch_object_steps=8000)
    free, total = torch.cuda.mem_get_info()
    hog = torch.empty(max(0, free - (6 << 30)), dtype=torch.uint8, device="cuda")   # leave ~6 GB
    try:
        got, st = cds.screen(pop, t0, t1, 1.0, d, batch_object_steps=10 ** 12, return_stats=True)
    finally:
        del hog
        torch.cuda.empty_cache()
    assert 1 <= st["grids_in_flight"] < 4000, st["grids_in_flight"]
    assert np.array_equal(got, ref)


@pytest.mark.parametrize("mode,dt,kw", [("grid", 1.0, {}), ("grid", 1.0, dict(round_steps=3)),
                                        ("hybrid", 9.0, {}), ("grid", 1.0, dict(resort_steps=2))])
def test_digest_only_equals_full_result(mode, dt, kw):
    """cd_options.digest_only: no records returned; the device-side digest (count, hash sum, min
    PCA) equals the one computed from the full result, and is additive over time slices."""
    pop = _mix(20000, 51, "catalog", 4000)
    d, t0 = 10.0, 300.0
    t1 = t0 + 120 * dt
    full = cds.screen(pop, t0, t1, dt, d, mode=mode, **kw)
    res, st = cds.screen(pop, t0, t1, dt, d, mode=mode, digest_only=True, return_stats=True, **kw)
    assert len(res) == 0 and len(full) > 50
    assert st["conjunctions"] == st["digest_conjunctions"] == len(full)
    assert st["digest"] == cds.conjunction_digest(full)
    assert st["min_pca"] == float(full["pca"].min())
    tot, cnt = 0, 0
    for q in range(3):
        _, s2 = cds.screen(pop, t0, t1, dt, d, mode=mode, digest_only=True, rank=q, n_ranks=3,
                           return_stats=True, **kw)
        tot = (tot + s2["digest"]) % (1 << 64)
        cnt += s2["digest_conjunctions"]
    assert tot == st["digest"] and cnt == len(full)
