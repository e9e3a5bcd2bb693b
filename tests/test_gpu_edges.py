"""Degenerate inputs through every mode (grid, hybrid, legacy) and option path: empty and
single-object populations, a one-step window (t1 = t0), a window shorter than one step, two
co-located objects, and the oracle's answer for each."""
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


MODES = [("grid", 1.0), ("hybrid", 9.0), ("legacy", 1.0)]


@pytest.mark.parametrize("mode,dt", MODES)
def test_empty_and_single(mode, dt):
    pop = popgen.random_population(10, 4)
    for idx in ([], [3]):
        assert len(cds.screen(popgen.subset(pop, idx), 0.0, 100.0, dt, 5.0, mode=mode)) == 0


@pytest.mark.parametrize("mode,dt", MODES)
def test_one_step_window_and_short_window(mode, dt):
    """K = 1 (t1 = t0) and t1 - t0 < dt: a single sampling step; results match the oracle."""
    pop, cfg, _ = popgen.make_config(1)
    for t0, t1 in ((300.0, 300.0), (300.0, 300.0 + 0.4 * dt)):
        g = cds.screen(pop, t0, t1, dt, cfg.d, mode=mode)
        if mode == "legacy":
            o, _ = oracle.legacy(pop, t0, t1, dt, cfg.d)
            parity.compare_legacy(pop, g, o, t0, t1, dt, cfg.d)
        elif mode == "hybrid":
            o, _ = oracle.hybrid(pop, t0, t1, dt, cfg.d)
            parity.compare_conjunctions(pop, g, o, t0, t1, dt, cfg.d, oracle.cell_size(cfg.d, dt))
        else:
            gc = oracle.cell_size(cfg.d, dt)
            K = oracle.candidates_brute(pop, t0, t1, dt, gc)
            o = oracle.conjunctions(pop, t0, t1, dt, cfg.d, gc, K)
            parity.compare_conjunctions(pop, g, o, t0, t1, dt, cfg.d, gc)
        assert np.all(g["step"] == 0)


def test_two_objects_crossing():
    """n = 2: the planted closed-form crossing pair alone, every mode finds the same minimum."""
    pop, cfg, planted = popgen.make_config(1)
    pa = next(p for p in planted.case_a if 2 * p.r * abs(np.cos(p.delta / 2) * np.sin(p.phi / 2)) < cfg.d)
    two = popgen.subset(pop, [pa.ia, pa.ib])
    rows = {}
    for mode, dt in (("grid", 1.0), ("legacy", 1.0), ("hybrid", 9.0)):
        r = cds.screen(two, cfg.t0, cfg.t1, dt, cfg.d, mode=mode)
        assert len(r) == 1, (mode, r)
        rows[mode] = r[0]
    assert abs(rows["grid"]["tca"] - rows["legacy"]["tca"]) < 1e-6
    assert abs(rows["grid"]["tca"] - rows["hybrid"]["tca"]) < 1e-3
    assert abs(rows["grid"]["pca"] - rows["hybrid"]["pca"]) < 1e-6


def test_geo_at_small_cell_fits_21bit_keys():
    """Cell keys pack 21 bits per axis (cdscreen.h CD_ERANGE): GEO objects at g_c = 0.1 km with
    the paper's cell edge (L = g_c) sit ~421,640 cells from the origin -- beyond the 2^18 of a
    19-bit key, inside 2^20 - 2.  Both grid structures, against brute force."""
    rng = np.random.default_rng(11)
    n = 400
    # a GEO-belt cluster with close neighbours (small offsets in longitude and radius)
    pop = {"a": 42164.0 + rng.uniform(-0.05, 0.05, n), "e": rng.uniform(0, 1e-7, n),
           "inc": rng.uniform(0, 1e-6, n), "raan": np.zeros(n),
           "argp": np.zeros(n), "nu0": rng.uniform(0, 2e-4, n)}
    d, dt = 0.1, 1.0
    gc = oracle.cell_size(d, dt, v_margin=0.0)
    Ko = oracle.candidates_brute(pop, 0.0, 20.0, dt, gc)
    assert len(Ko) > 0
    for table in (1, 2):
        Kg = cds.candidates(pop, 0.0, 20.0, dt, d, v_margin=0.0, cell_factor=1.0, grid_table=table)
        parity.compare_candidates(pop, Kg, Ko, 0.0, dt, gc)


def test_kepler_points_option():
    """cd_options.kepler_points: a minimum Contour point count for every object -- the same
    positions (1e-9) and candidate set; an unsupported count is CD_EINVAL."""
    pop = popgen.random_population(3000, 12, "paper", 200)
    times = np.array([0.0, 517.25, 86400.0])
    xo = oracle.propagate(pop, times)
    for kp in (8, 16):
        xg = cds.propagate(pop, times, kepler_points=kp)
        rel = np.linalg.norm(xg - xo, axis=2) / np.linalg.norm(xo, axis=2)
        assert rel.max() < 1e-9, (kp, rel.max())
    gc = oracle.cell_size(20.0, 1.0)
    Ko = oracle.candidates_grid(pop, 0.0, 30.0, 1.0, gc)
    Kg = cds.candidates(pop, 0.0, 30.0, 1.0, 20.0, kepler_points=12)
    parity.compare_candidates(pop, Kg, Ko, 0.0, 1.0, gc)
    with pytest.raises(cds.CdError) as ei:
        cds.propagate(pop, times, kepler_points=5)
    assert ei.value.status == cds.CD_EINVAL


def test_device_inputs_validation_and_streams():
    """CUDA-tensor inputs: fp64 / 1-D / one device are required (ValueError before C); inputs
    written on a side stream are screened on that stream (the binding passes torch's current
    stream), so the result equals the host-input result."""
    import torch
    pop = popgen.random_population(2000, 13)
    host = cds.screen(pop, 0.0, 60.0, 1.0, 20.0)
    bad = {k: torch.from_numpy(v).cuda() for k, v in pop.items()}
    bad["a"] = bad["a"].float()
    with pytest.raises(ValueError, match="float64"):
        cds.screen(bad, 0.0, 60.0, 1.0, 20.0)
    side = torch.cuda.Stream()
    with torch.cuda.stream(side):
        dev = {k: torch.empty(len(v), dtype=torch.float64, device="cuda") for k, v in pop.items()}
        for k, v in pop.items():
            dev[k].copy_(torch.from_numpy(v), non_blocking=True)
        got = cds.screen(dev, 0.0, 60.0, 1.0, 20.0)
    assert np.array_equal(got, host)


def test_release_caches():
    pop = popgen.random_population(2000, 14)
    a = cds.screen(pop, 0.0, 60.0, 1.0, 20.0)
    cds.release_caches()
    cds.release_caches(0)
    b = cds.screen(pop, 0.0, 60.0, 1.0, 20.0)
    assert np.array_equal(a, b)
    with pytest.raises(cds.CdError):
        cds.release_caches(4096)
