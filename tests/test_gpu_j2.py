"""GPU parity of the J2 secular propagator ("other propagators
instead of the Kepler Contour solver"; rates from Vallado & McClain [41] Sec. 9.6, reading R19)
through the C ABI (cd_options.propagator = CD_PROP_J2) against the oracle's O1'.

Same tolerances as the Kepler path: positions and velocities 1e-9 relative; identical candidate
and conjunction sets except within 1 mm of the thresholds; TCA 1e-3 s, PCA 1 m."""
import math

import numpy as np
import pytest

import oracle
from tools import popgen
from tests import parity

pytestmark = pytest.mark.gpu

cds = pytest.importorskip("paper_conf_ipps_hellwigcmbw23_b200")

DAY = 86400.0


@pytest.fixture(scope="module", autouse=True)
def _need_gpu():
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")


def _j2(pop):
    return dict(pop, propagator="j2")


def test_j2_positions_velocities_1e9():
    rng = np.random.default_rng(17)
    pop = popgen.random_population(20000, 5, "catalog", 2000)
    extra = {"a": np.full(12, 26000.0), "e": np.array([0.0, 1e-13, 0.005, 0.05, 0.2, 0.45, 0.7,
                                                     0.8, 0.85, 0.9, 0.95, 0.99]),
             "inc": np.linspace(0.0, math.pi, 12), "raan": np.full(12, 0.3),
             "argp": np.full(12, 0.2), "nu0": np.zeros(12)}
    pop = _j2(popgen.concat(pop, extra))
    times = np.concatenate([[0.0, 1.0, DAY, 7 * DAY], rng.uniform(0, 7 * DAY, 6)])
    xg, vg = cds.propagate(pop, times, velocity=True)
    xo, vo = oracle.propagate(pop, times, velocity=True)
    rel = np.linalg.norm(xg - xo, axis=2) / np.linalg.norm(xo, axis=2)
    assert rel.max() < 1e-9, rel.max()
    relv = np.linalg.norm(vg - vo, axis=2) / np.linalg.norm(vo, axis=2)
    assert relv.max() < 1e-9, relv.max()
    # the model is really in use: after a day LEO positions differ from two-body by many km
    xk = cds.propagate(dict(pop, propagator="kepler"), [DAY])
    assert np.median(np.linalg.norm(xk[0] - xg[2], axis=1)) > 1.0


@pytest.mark.parametrize("table", [1, 2])
def test_j2_candidates_config1_brute_force(table):
    pop, cfg, _ = popgen.make_config(1)
    pop = _j2(pop)
    t0, t1 = 2 * DAY, 2 * DAY + 300.0
    gc = oracle.cell_size(cfg.d, cfg.dt_grid)
    Kg = cds.candidates(pop, t0, t1, cfg.dt_grid, cfg.d, grid_table=table)
    Ko = oracle.candidates_brute(pop, t0, t1, cfg.dt_grid, gc)
    assert len(Ko) > 100
    parity.compare_candidates(pop, Kg, Ko, t0, cfg.dt_grid, gc)


@pytest.mark.parametrize("n,steps,d,t0", [(4099, 400, 2.0, 0.0), (30000, 90, 5.0, 5 * DAY)])
def test_j2_screen_ragged_parity(n, steps, d, t0):
    pop = _j2(popgen.random_population(n, 700 + n, "catalog", n // 4))
    t1 = t0 + steps - 1.0
    gc = oracle.cell_size(d, 1.0)
    Cg, st = cds.screen(pop, t0, t1, 1.0, d, return_stats=True)
    Ko = oracle.candidates_grid(pop, t0, t1, 1.0, gc)
    assert st["candidates"] == len(Ko)
    Co = oracle.conjunctions(pop, t0, t1, 1.0, d, gc, Ko)
    res = parity.compare_conjunctions(pop, Cg, Co, t0, t1, 1.0, d, gc)
    assert res["matched"] > 0


def test_j2_dense_shell():
    """Many encounters per step under J2 (the prefilter's acceleration bound includes the rotating
    frame's terms: nothing the oracle finds may be dropped)."""
    rng = np.random.default_rng(31)
    n = 6000
    pop = _j2({"a": rng.uniform(6900, 6905, n), "e": rng.uniform(0, 0.0005, n),
               "inc": rng.uniform(0, math.pi, n), "raan": rng.uniform(0, 2 * math.pi, n),
               "argp": rng.uniform(0, 2 * math.pi, n), "nu0": rng.uniform(0, 2 * math.pi, n)})
    d, t0 = 5.0, 3 * DAY
    t1 = t0 + 200.0
    gc = oracle.cell_size(d, 1.0)
    Cg = cds.screen(pop, t0, t1, 1.0, d, round_steps=13)
    Ko = oracle.candidates_grid(pop, t0, t1, 1.0, gc)
    Co = oracle.conjunctions(pop, t0, t1, 1.0, d, gc, Ko)
    res = parity.compare_conjunctions(pop, Cg, Co, t0, t1, 1.0, d, gc)
    assert res["matched"] > 100


def test_j2_full_size_sampled_steps():
    """1M objects (BASELINE config 4) under J2, hour 12 of the day, sampled steps."""
    pop, cfg, _ = popgen.make_config(4)
    pop = _j2(pop)
    d, dt = cfg.d, cfg.dt_grid
    t0, t1 = 12 * 3600.0, 12 * 3600.0 + 600.0
    gc = oracle.cell_size(d, dt)
    Kg = cds.candidates(pop, t0, t1, dt, d)
    Cg = cds.screen(pop, t0, t1, dt, d)
    for k in (0, 333, 600):
        Ko = oracle.candidates_grid(pop, t0, t1, dt, gc, k_begin=k, k_end=k + 1)
        parity.compare_candidates(pop, Kg[Kg["step"] == k], Ko, t0, dt, gc)
        assert len(Ko) > 1000
        Co = oracle.conjunctions(pop, t0, t1, dt, d, gc, Ko)
        parity.compare_conjunctions(pop, Cg[Cg["step"] == k], Co, t0, t1, dt, d, gc)


def test_j2_errors():
    pop = _j2(popgen.random_population(100, 3))
    with pytest.raises(cds.CdError) as ei:
        cds.screen(pop, 0.0, 90.0, 9.0, 2.0, mode="hybrid")
    assert ei.value.status == cds.CD_EINVAL
    with pytest.raises(cds.CdError) as ei:
        cds.screen(pop, 0.0, 10.0, 1.0, 2.0, propagator=7)
    assert ei.value.status == cds.CD_EINVAL
