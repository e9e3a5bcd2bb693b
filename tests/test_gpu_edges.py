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
