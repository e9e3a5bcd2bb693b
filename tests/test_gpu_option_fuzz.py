"""Seeded random combinations of every option that must not change the result (cell edge, grid
structure, spatial re-sort, batch and round sizes, Contour point count, grid origin, PyTorch
allocator, time slices) on random small populations, each compared with the oracle (candidates
triple by triple, conjunctions element by element).  The options are performance knobs; the
result set is defined by the paper's quantities alone (R4-R14)."""
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


def _options(rng):
    kw = {}
    if rng.random() < 0.5:
        kw["cell_factor"] = float(rng.choice([1.0, 1.3, 2.0, 2.5, 4.0]))
    kw["grid_table"] = int(rng.choice([0, 1, 2, 3]))
    if rng.random() < 0.4:
        kw["resort_steps"] = int(rng.choice([-1, 1, 3, 8]))
    if rng.random() < 0.4:
        kw["batch_object_steps"] = int(rng.choice([1, 5000, 40000, 10 ** 7]))
    if rng.random() < 0.3:
        kw["round_steps"] = int(rng.choice([1, 4, 13]))
    if rng.random() < 0.3:
        kw["kepler_points"] = int(rng.choice([0, 6, 8, 16]))
    if rng.random() < 0.3:
        kw["grid_origin"] = tuple(rng.uniform(-5000, 5000, 3))
    if rng.random() < 0.3:
        kw["allocator"] = "torch"
    return kw


@pytest.mark.parametrize("seed", range(24))
def test_random_options_match_oracle(seed):
    rng = np.random.default_rng(4000 + seed)
    n = int(rng.integers(1000, 12000))
    pop = popgen.random_population(n, 5000 + seed, "catalog" if seed % 2 else "paper",
                                   int(rng.integers(0, n // 3)))
    d = float(rng.choice([5.0, 20.0, 40.0]))
    dt = float(rng.choice([0.5, 1.0, 3.0]))
    t0 = float(rng.uniform(0, 5000))
    t1 = t0 + dt * int(rng.integers(10, 80))
    kw = _options(rng)
    gc = oracle.cell_size(d, dt)
    Kg = cds.candidates(pop, t0, t1, dt, d, **kw)
    Ko = oracle.candidates_grid(pop, t0, t1, dt, gc)
    parity.compare_candidates(pop, Kg, Ko, t0, dt, gc)
    S = int(rng.choice([1, 1, 3]))
    parts = [cds.screen(pop, t0, t1, dt, d, rank=q, n_ranks=S, **kw) for q in range(S)]
    Cg = np.concatenate(parts)
    Cg = Cg[np.lexsort((Cg["step"], Cg["j"], Cg["i"]))]
    Co = oracle.conjunctions(pop, t0, t1, dt, d, gc, Ko)
    res = parity.compare_conjunctions(pop, Cg, Co, t0, t1, dt, d, gc)
    assert res["one_sided"] == 0, (kw, res)


@pytest.mark.parametrize("seed", range(10))
def test_random_options_hybrid_match_oracle(seed):
    rng = np.random.default_rng(6000 + seed)
    n = int(rng.integers(1000, 8000))
    pop = popgen.random_population(n, 7000 + seed, "catalog", int(rng.integers(0, n // 2)))
    d = float(rng.choice([2.0, 5.0, 10.0]))
    dt = float(rng.choice([3.0, 9.0, 15.0]))
    t0 = float(rng.uniform(0, 5000))
    t1 = t0 + dt * int(rng.integers(10, 60))
    kw = _options(rng)
    kw.pop("kepler_points", None)
    gc = oracle.cell_size(d, dt)
    Cg, st = cds.screen(pop, t0, t1, dt, d, mode="hybrid", return_stats=True, **kw)
    Co, cnt = oracle.hybrid(pop, t0, t1, dt, d)
    res = parity.compare_conjunctions(pop, Cg, Co, t0, t1, dt, d, gc)
    assert res["one_sided"] == 0, (kw, res)
    assert st["candidates"] == cnt["candidates"]


@pytest.mark.parametrize("seed", range(6))
def test_random_j2_and_legacy_match_oracle(seed):
    rng = np.random.default_rng(8000 + seed)
    n = int(rng.integers(300, 1500))
    pop = popgen.random_population(n, 9000 + seed, "catalog", int(rng.integers(0, n // 3)))
    d = float(rng.choice([10.0, 30.0]))
    t0, dt = float(rng.uniform(0, 3000)), 1.0
    t1 = t0 + int(rng.integers(20, 60))
    gc = oracle.cell_size(d, dt)
    kw = _options(rng)
    kw.pop("kepler_points", None)
    pj = dict(pop, propagator="j2")
    Kg = cds.candidates(pj, t0, t1, dt, d, **kw)
    Ko = oracle.candidates_grid(pj, t0, t1, dt, gc)
    parity.compare_candidates(pj, Kg, Ko, t0, dt, gc)
    Cg = cds.screen(pj, t0, t1, dt, d, **kw)
    Co = oracle.conjunctions(pj, t0, t1, dt, d, gc, Ko)
    assert parity.compare_conjunctions(pj, Cg, Co, t0, t1, dt, d, gc)["one_sided"] == 0
    # legacy chain on a dense swarm (its pairs split over two ranks for odd seeds)
    m = 800
    pop = {"a": rng.uniform(7000, 7010, m), "e": rng.uniform(0, 0.001, m),
           "inc": 0.9 + rng.uniform(-0.05, 0.05, m), "raan": 0.3 + rng.uniform(-0.05, 0.05, m),
           "argp": np.zeros(m), "nu0": rng.uniform(0, 0.5, m)}
    t1 = t0 + 300.0
    Lg = cds.screen(pop, t0, t1, dt, d, mode="legacy", rank=seed % 2, n_ranks=1 + seed % 2)
    Lo, _ = oracle.legacy(pop, t0, t1, dt, d)
    if seed % 2:
        Lg2 = cds.screen(pop, t0, t1, dt, d, mode="legacy", rank=0, n_ranks=2)
        Lg = np.concatenate([Lg2, Lg])
        Lg = Lg[np.lexsort((Lg["step"], Lg["j"], Lg["i"]))]
    assert len(Lo) > 5
    parity.compare_legacy(pop, Lg, Lo, t0, t1, dt, d)
