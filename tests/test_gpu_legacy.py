"""GPU parity of the legacy full-window filter chain (mode CD_LEGACY; SURVEY 8(f) row 4;
PAPER.md:43 filters, P:189 legacy variant, P:315-318 accuracy comparison) through the C ABI
against the oracle's O5, plus its relation to the grid variant (a superset: no Eq. 1 speed
assumption)."""
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


def _check_counts(st, cnt):
    assert st["candidates"] == cnt["pairs"]
    assert st["hybrid_ap_rejected"] == cnt["ap_rejected"]
    assert st["hybrid_coplanar"] == cnt["coplanar"]
    # node geometry in fp64 on both sides: stage counts agree up to boundary rounding
    for a, b in (("hybrid_path_rejected", "path_rejected"), ("hybrid_time_rejected", "time_rejected")):
        assert abs(st[a] - cnt[b]) <= max(2, 1e-5 * cnt[b]), (a, st[a], cnt[b])


def test_legacy_config1():
    pop, cfg, _ = popgen.make_config(1)
    Lg, st = cds.screen(pop, cfg.t0, cfg.t1, cfg.dt_grid, cfg.d, mode="legacy", return_stats=True)
    Lo, cnt = oracle.legacy(pop, cfg.t0, cfg.t1, cfg.dt_grid, cfg.d)
    _check_counts(st, cnt)
    assert parity.is_sorted(Lg)
    res = parity.compare_legacy(pop, Lg, Lo, cfg.t0, cfg.t1, cfg.dt_grid, cfg.d)
    assert res["matched"] >= len(Lo) - 2
    # the grid variant's non-degenerate rows are all there
    G = cds.screen(pop, cfg.t0, cfg.t1, cfg.dt_grid, cfg.d)
    G = G[(G["flags"] & cds.CD_FLAG_DEGENERATE) == 0]
    assert set(zip(G["i"].tolist(), G["j"].tolist(), G["step"].tolist())) <= \
        set(zip(Lg["i"].tolist(), Lg["j"].tolist(), Lg["step"].tolist()))


def test_legacy_counter_rotating_coplanar():
    """Thousands of coplanar pairs (whole-window search) and head-on encounters."""
    pop = popgen.counter_rotating(200, 5)
    t0, t1, dt, d = 0.0, 1200.0, 1.0, 5.0
    Lg, st = cds.screen(pop, t0, t1, dt, d, mode="legacy", return_stats=True)
    Lo, cnt = oracle.legacy(pop, t0, t1, dt, d)
    _check_counts(st, cnt)
    assert cnt["coplanar"] > 1000
    res = parity.compare_legacy(pop, Lg, Lo, t0, t1, dt, d)
    assert res["matched"] > 1000


@pytest.mark.parametrize("n,seed,t1,d", [(3000, 11, 3600.0, 5.0), (1237, 12, 1800.0, 20.0)])
def test_legacy_ragged(n, seed, t1, d):
    pop = popgen.random_population(n, seed, "catalog", n // 6)
    Lg, st = cds.screen(pop, 0.0, t1, 1.0, d, mode="legacy", return_stats=True)
    Lo, cnt = oracle.legacy(pop, 0.0, t1, 1.0, d)
    _check_counts(st, cnt)
    res = parity.compare_legacy(pop, Lg, Lo, 0.0, t1, 1.0, d)
    assert res["matched"] > 20


def test_legacy_rank_split_and_small_chunks():
    """Pairs split across ranks: the union is the full result."""
    pop = popgen.random_population(2000, 13, "catalog", 400)
    full = cds.screen(pop, 0.0, 1800.0, 1.0, 10.0, mode="legacy")
    parts = [cds.screen(pop, 0.0, 1800.0, 1.0, 10.0, mode="legacy", rank=r, n_ranks=3) for r in range(3)]
    merged = np.sort(np.concatenate(parts), order=["i", "j", "step"])
    assert np.array_equal(merged[["i", "j", "step"]], full[["i", "j", "step"]])
    assert np.array_equal(merged["tca"], full["tca"])


def test_legacy_contains_grid_30k():
    """BASELINE config 2 population (30,000 catalog-like objects), one hour: every grid-variant
    conjunction is in the legacy set with the same TCA/PCA; legacy-only rows have their nearest
    step outside the grid's candidate gate g_c."""
    pop, cfg, _ = popgen.make_config(2)
    t0, t1, dt, d = 3600.0, 7200.0, 1.0, cfg.d
    G = cds.screen(pop, t0, t1, dt, d)
    L, st = cds.screen(pop, t0, t1, dt, d, mode="legacy", return_stats=True)
    assert st["candidates"] == 30000 * 29999 // 2
    lk = {(int(r["i"]), int(r["j"]), int(r["step"])): r for r in L}
    for r in G:
        k = (int(r["i"]), int(r["j"]), int(r["step"]))
        if r["flags"] & cds.CD_FLAG_DEGENERATE:
            continue
        assert k in lk, k
        assert abs(lk[k]["tca"] - r["tca"]) < 1e-3 and abs(lk[k]["pca"] - r["pca"]) < 1e-3
    gc = oracle.cell_size(d, dt)
    gk = {(int(r["i"]), int(r["j"]), int(r["step"])) for r in G}
    for k in [k for k in lk if k not in gk]:
        D, _ = oracle.pair_distance(pop, k[0], k[1], [t0 + k[2] * dt])
        assert D[0] >= gc - 1e-6, (k, D[0])


def test_legacy_errors():
    pop = popgen.random_population(100, 3)
    with pytest.raises(cds.CdError) as ei:
        cds.screen(dict(pop, propagator="j2"), 0.0, 90.0, 1.0, 2.0, mode="legacy")
    assert ei.value.status == cds.CD_EINVAL
    with pytest.raises(cds.CdError) as ei:
        cds.candidates(pop, 0.0, 90.0, 1.0, 2.0, mode="legacy")
    assert ei.value.status == cds.CD_EINVAL
    assert len(cds.screen(popgen.subset(pop, [3]), 0.0, 90.0, 1.0, 2.0, mode="legacy")) == 0


def test_legacy_config2_full_window():
    """BASELINE config 2 at full size (30,000 objects, the whole 24 h at 1 s): the legacy chain on
    the device against oracle O5 element by element, and the filter-stage counts."""
    pop, cfg, _ = popgen.make_config(2)
    Lg, st = cds.screen(pop, cfg.t0, cfg.t1, cfg.dt_grid, cfg.d, mode="legacy", return_stats=True)
    Lo, cnt = oracle.legacy(pop, cfg.t0, cfg.t1, cfg.dt_grid, cfg.d)
    _check_counts(st, cnt)
    res = parity.compare_legacy(pop, Lg, Lo, cfg.t0, cfg.t1, cfg.dt_grid, cfg.d)
    assert res["matched"] > 7000
