"""Pins for the oracle's J2 secular propagator (O1'; "other
propagators instead of the Kepler Contour solver"; rates from Vallado & McClain [41] Sec. 9.6).

Each test measures the propagated positions -- not the rate formulas -- against something
outside the oracle: published sun-synchronous mission orbits and the ISS node regression
(tests/golden/j2_orbits.txt), the critical inclination of the perigee, the special inclination
where the mean-anomaly rate equals the Kepler rate, the derivative of the position, and the
grid/brute-force and dense-sampling constructions of the Kepler pins re-run under J2."""
import math
from pathlib import Path

import numpy as np
import pytest

from tools import popgen

GOLDEN = Path(__file__).resolve().parent / "golden" / "j2_orbits.txt"
RE = 6378.137
DAY = 86400.0


def _rows(kind):
    out = []
    for line in GOLDEN.read_text().splitlines():
        f = line.split()
        if f and not line.startswith("#") and f[0] == kind:
            out.append([f[1]] + [float(x) for x in f[2:]])
    assert out, kind
    return out


def _one(a, e, inc_deg, raan=0.3, argp=0.0, nu0=0.0, prop="j2"):
    p = {k: np.array([v], dtype=np.float64) for k, v in
         zip(popgen.FIELDS, (a, e, math.radians(inc_deg), raan, argp, nu0))}
    p["propagator"] = prop
    return p


def _node(orc, pop, t):
    """Right ascension of the ascending node from two positions 60 s apart (plane normal)."""
    x = orc.propagate(pop, [t, t + 60.0])
    h = np.cross(x[0, 0], x[1, 0])
    return math.atan2(h[0], -h[1]), h / np.linalg.norm(h)


@pytest.mark.parametrize("row", _rows("node_rate"), ids=lambda r: r[0])
def test_published_node_rates(orc, row):
    name, alt, inc, rate, tol = row
    pop = _one(RE + alt, 0.0, inc)
    w0, _ = _node(orc, pop, 0.0)
    w1, _ = _node(orc, pop, DAY)
    got = math.degrees(math.remainder(w1 - w0, 2 * math.pi))
    assert abs(got - rate) <= tol * abs(rate), (name, got, rate)
    # the Kepler propagator keeps the plane fixed
    kep = dict(pop, propagator="kepler")
    k0, _ = _node(orc, kep, 0.0)
    k1, _ = _node(orc, kep, DAY)
    assert abs(math.remainder(k1 - k0, 2 * math.pi)) < 1e-12


def _perigee_arg(orc, pop, t_center, period):
    """Argument of perigee measured from the positions: the time of minimum |r| within one orbit
    around t_center (1 s sampling + parabola), then its angle from the current ascending node."""
    ts = t_center + np.arange(0.0, period, 1.0)
    r = orc.propagate(pop, ts)[:, 0]
    R = np.linalg.norm(r, axis=1)
    q = int(np.argmin(R[1:-1])) + 1
    y0, y1, y2 = R[q - 1], R[q], R[q + 1]
    tp = ts[q] + 0.5 * (y0 - y2) / (y0 - 2 * y1 + y2)
    rp = orc.propagate(pop, [tp])[0, 0]
    node, h = _node(orc, pop, tp)
    nhat = np.array([math.cos(node), math.sin(node), 0.0])
    return math.atan2(np.dot(np.cross(nhat, rp), h), np.dot(nhat, rp))


def test_critical_inclination_freezes_perigee(orc):
    (name, icrit), = _rows("perigee_frozen")
    a, e, argp0 = 8000.0, 0.1, 0.7
    period = 2 * math.pi * math.sqrt(a ** 3 / orc.mu())
    drift = {}
    for inc in (30.0, icrit, 80.0):
        pop = _one(a, e, inc, argp=argp0)
        w = _perigee_arg(orc, pop, 10 * DAY, period)
        drift[inc] = math.degrees(math.remainder(w - argp0, 2 * math.pi))
    assert abs(drift[icrit]) < 0.01, drift
    assert drift[30.0] > 5.0, drift          # perigee advances below the critical inclination
    assert drift[80.0] < -5.0, drift         # and regresses above it
    # Kepler: no perigee motion at all
    w = _perigee_arg(orc, _one(a, e, 30.0, argp=argp0, prop="kepler"), 10 * DAY, period)
    assert abs(math.remainder(w - argp0, 2 * math.pi)) < 1e-4


def test_radius_unchanged_at_mean_motion_neutral_inclination(orc):
    """The J2 mean-anomaly rate equals the two-body rate where 1 - (3/2) sin^2 i = 0
    (i = 54.7356 deg) [41]: the plane and perigee rotate, but |r(t)| is the two-body radius.
    At other inclinations the radius histories separate (the along-track drift)."""
    ineutral = math.degrees(math.asin(math.sqrt(2.0 / 3.0)))
    t = np.linspace(0.0, 2 * DAY, 97)
    for inc, same in ((ineutral, True), (20.0, False)):
        pj = _one(7200.0, 0.02, inc)
        pk = dict(pj, propagator="kepler")
        Rj = np.linalg.norm(orc.propagate(pj, t)[:, 0], axis=1)
        Rk = np.linalg.norm(orc.propagate(pk, t)[:, 0], axis=1)
        err = np.max(np.abs(Rj - Rk))
        if same:
            assert err < 1e-8, err
        else:
            assert err > 1.0, err


def test_j2_velocity_is_derivative_of_position(orc):
    rng = np.random.default_rng(15)
    pop = dict(popgen.base_mixture(rng, 60), propagator="j2")
    for t in (3000.0, 5 * DAY):
        h = 1e-3
        r = orc.propagate(pop, [t - h, t + h])
        _, v = orc.propagate(pop, [t], velocity=True)
        fd = (r[1] - r[0]) / (2 * h)
        assert np.max(np.abs(fd - v[0]) / np.linalg.norm(v[0], axis=1)[:, None]) < 1e-7


def test_j2_epoch_state_equals_kepler(orc):
    """At t = 0 the secular angles have not moved: the J2 and two-body positions coincide."""
    rng = np.random.default_rng(16)
    pop = popgen.base_mixture(rng, 200)
    xk = orc.propagate(pop, [0.0])
    xj = orc.propagate(dict(pop, propagator="j2"), [0.0])
    assert np.max(np.abs(xk - xj)) < 1e-9


def test_j2_grid_equals_brute_and_dense_sampling(orc):
    """The candidate constructions and the conjunction search do not depend on the
    force model: grid == brute force, and every minimum below d found by 1 ms dense sampling of
    each candidate pair is reported once by its owner step."""
    pop, cfg, _ = popgen.make_config(1)
    pop = dict(pop, propagator="j2")
    t1 = 60.0
    gc = orc.cell_size(cfg.d, cfg.dt_grid)
    Kb = orc.candidates_brute(pop, cfg.t0, t1, cfg.dt_grid, gc)
    Kg = orc.candidates_grid(pop, cfg.t0, t1, cfg.dt_grid, gc)
    assert len(Kb) > 20 and np.array_equal(Kb, Kg)
    C = orc.conjunctions(pop, cfg.t0, t1, cfg.dt_grid, cfg.d, gc, Kb)
    assert len(C) > 5
    t = np.arange(cfg.t0, t1 + 1e-9, 1e-3)
    expect = []
    for (i, j) in sorted(set(zip(Kb["i"].tolist(), Kb["j"].tolist()))):
        D, _ = orc.pair_distance(pop, i, j, t)
        m = np.where((D[1:-1] < D[:-2]) & (D[1:-1] <= D[2:]) & (D[1:-1] < cfg.d))[0] + 1
        steps = set(Kb["step"][(Kb["i"] == i) & (Kb["j"] == j)].tolist())
        for q in m:
            k = int(math.floor((t[q] - cfg.t0) / cfg.dt_grid + 0.5))
            if k in steps:
                expect.append((i, j, k, t[q]))
    got = [r for r in C if not (r["flags"] & 2)]
    assert len(got) == len(expect)
    for (i, j, k, tq), r in zip(sorted(expect), got):
        assert (i, j, k) == (int(r["i"]), int(r["j"]), int(r["step"]))
        assert abs(r["tca"] - tq) < 1e-3


def test_hybrid_rejects_j2(orc):
    pop, cfg, _ = popgen.make_config(1, n=50)
    with pytest.raises(ValueError):
        orc.hybrid(dict(pop, propagator="j2"), 0.0, 30.0, 9.0, 10.0)
