"""Pins for the oracle's legacy full-window filter chain (O5; the paper's
grid-free comparison baseline: "classical orbital filters" P:43, legacy variant P:189, accuracy
comparison P:315-318).

The legacy chain has no sampling assumption (no Eq. 1 speed bound), so it must (a) agree with
dense-sampling brute force, (b) contain every grid-variant conjunction, and (c) add only
encounters the grid could not see (nearest sample farther than g_c -- relative speed beyond the
Eq. 1 bound).  Closed-form coplanar and crossing encounters pin TCA/PCA."""
import math

import numpy as np
import pytest

from tools import popgen


def _one_row(a, e, inc, raan, argp, nu0):
    return {k: np.array([v], dtype=np.float64) for k, v in zip(popgen.FIELDS, (a, e, inc, raan, argp, nu0))}


def test_legacy_equals_dense_sampling_brute_force(orc):
    """Every local minimum of D below d, found by 50 ms sampling of every pair of a compact
    shell (no filter at all), is reported once with its TCA/PCA; nothing else is."""
    rng = np.random.default_rng(41)
    n = 50
    pop = {"a": rng.uniform(6900, 6904, n), "e": rng.uniform(0, 3e-4, n),
           "inc": rng.uniform(0, math.pi, n), "raan": rng.uniform(0, 2 * math.pi, n),
           "argp": rng.uniform(0, 2 * math.pi, n), "nu0": rng.uniform(0, 2 * math.pi, n)}
    t0, t1, dt, d = 0.0, 1200.0, 1.0, 300.0
    C, cnt = orc.legacy(pop, t0, t1, dt, d)
    assert cnt["pairs"] == n * (n - 1) // 2
    t = np.arange(t0, t1 + 1e-9, 0.05)
    expect = []
    for i in range(n):
        for j in range(i + 1, n):
            D, _ = orc.pair_distance(pop, i, j, t)
            m = np.where((D[1:-1] < D[:-2]) & (D[1:-1] <= D[2:]) & (D[1:-1] < d))[0] + 1
            expect += [(i, j, t[q], D[q]) for q in m]
    assert len(expect) > 8
    assert len(C) == len(expect)
    for (i, j, tq, Dq), r in zip(sorted(expect), C):
        assert (i, j) == (int(r["i"]), int(r["j"]))
        assert abs(r["tca"] - tq) < 0.05
        assert r["pca"] <= Dq + 1e-12 and Dq - r["pca"] < 0.02
        assert r["step"] == int(math.floor((r["tca"] - t0) / dt + 0.5))


def test_legacy_contains_grid_and_explains_extras(orc):
    """Counter-rotating plane (head-on encounters near 15 km/s), grid screened with a reduced
    Eq. 1 speed (v_margin = 3 km/s, so the grid's speed assumption is violated on purpose): the
    legacy set contains every grid-variant conjunction (same TCA/PCA), and every extra row is an
    encounter whose nearest sample is not a grid candidate (distance >= g_c there)."""
    pop = popgen.counter_rotating(200, 5)
    t0, t1, dt, d, vm = 0.0, 1200.0, 1.0, 5.0, 3.0
    gc = orc.cell_size(d, dt, vm)
    K, G = orc.screen_grid(pop, t0, t1, dt, d, v_margin=vm)
    L, cnt = orc.legacy(pop, t0, t1, dt, d)
    assert len(G) > 10
    lk = {(int(r["i"]), int(r["j"]), int(r["step"])): r for r in L}
    for r in G:
        k = (int(r["i"]), int(r["j"]), int(r["step"]))
        assert k in lk, k
        assert abs(lk[k]["tca"] - r["tca"]) < 1e-3 and abs(lk[k]["pca"] - r["pca"]) < 1e-3
    gk = {(int(r["i"]), int(r["j"]), int(r["step"])) for r in G}
    extra = [k for k in lk if k not in gk]
    assert len(extra) > 10
    for k in extra:
        D, _ = orc.pair_distance(pop, k[0], k[1], [t0 + k[2] * dt])
        assert D[0] >= gc, (k, D[0], gc)
    # with the paper's 7.8 km/s (every encounter here is slower than 15.6 km/s) nothing is missed
    K, G = orc.screen_grid(pop, t0, t1, dt, d)
    assert np.array_equal(G[["i", "j", "step"]], L[["i", "j", "step"]])


def test_legacy_config1_equals_grid(orc):
    """The paper-mode config 1 has no encounter beyond the Eq. 1 bound: legacy == grid (minus the
    degenerate twins, which have no isolated minimum)."""
    pop, cfg, planted = popgen.make_config(1)
    L, cnt = orc.legacy(pop, cfg.t0, cfg.t1, cfg.dt_grid, cfg.d)
    K, G = orc.screen_grid(pop, cfg.t0, cfg.t1, cfg.dt_grid, cfg.d)
    G = G[(G["flags"] & 2) == 0]
    assert len(L) == len(G)
    assert np.array_equal(L[["i", "j", "step"]], G[["i", "j", "step"]])
    assert np.max(np.abs(L["tca"] - G["tca"])) < 1e-6
    # closed form A (two circular orbits through a common node)
    mu = orc.mu()
    for pa in planted.case_a:
        pca = 2 * pa.r * abs(math.cos(pa.delta / 2) * math.sin(pa.phi / 2))
        tca = (pa.u0 - pa.phi / 2) / math.sqrt(mu / pa.r ** 3)
        rows = L[(L["i"] == pa.ia) & (L["j"] == pa.ib)]
        if pca < cfg.d:
            assert len(rows) == 1 and abs(rows["tca"][0] - tca) < 1e-6 and abs(rows["pca"][0] - pca) < 1e-6


def test_legacy_coplanar_closed_form(orc):
    """Two circular orbits in one plane (mutual inclination 0: coplanar path, whole window
    searched), radii r and r + 3 km, phases aligned at t* = 3000 s: PCA = 3 km exactly at t*."""
    mu = orc.mu()
    r1, r2, ts = 7000.0, 7003.0, 3000.0
    n1, n2 = math.sqrt(mu / r1 ** 3), math.sqrt(mu / r2 ** 3)
    u10 = 0.4
    u20 = u10 + (n1 - n2) * ts
    pop = popgen.concat(_one_row(r1, 0.0, 0.5, 1.0, 0.0, u10), _one_row(r2, 0.0, 0.5, 1.0, 0.0, u20))
    L, cnt = orc.legacy(pop, 0.0, 6000.0, 1.0, 5.0)
    assert cnt["coplanar"] == 1
    assert len(L) == 1 and L["flags"][0] & 4
    assert abs(L["tca"][0] - ts) < 1e-6 and abs(L["pca"][0] - 3.0) < 1e-9


def test_legacy_filter_stage_cases(orc):
    """Disjoint shells are AP-rejected; a crossing pair whose node passages never coincide is
    time-rejected; both leave no output."""
    shells = popgen.concat(_one_row(7000.0, 0.0, 0.3, 0.0, 0.0, 0.0),
                           _one_row(7100.0, 0.0, 1.2, 1.0, 0.0, 0.5))
    L, cnt = orc.legacy(shells, 0.0, 3000.0, 1.0, 5.0)
    assert cnt["ap_rejected"] == 1 and len(L) == 0
    # same radius, planes crossing at 60 deg, A passes the node a quarter orbit after B
    mu = orc.mu()
    cross = popgen.concat(_one_row(7000.0, 0.0, 0.0, 0.0, 0.0, 0.0),
                          _one_row(7000.0, 0.0, math.radians(60.0), 0.0, 0.0, math.pi / 2))
    L, cnt = orc.legacy(cross, 0.0, 600.0, 1.0, 5.0)
    assert cnt["time_rejected"] == 1 and len(L) == 0
