"""Magnitude pin of the oracle's J2 secular propagator (O1', R19; "other
propagators instead of the Kepler Contour solver"; the rates are those of Vallado & McClain [41]
Sec. 9.6, the paper's own reference).

tests/test_oracle_j2.py pins O1' through published node regressions, the critical inclination
and the zero of the mean-anomaly correction.  This module pins all three secular rates --
including the *magnitude* of the dM/dt correction -- by deriving them here from first
principles, with none of the oracle's formulas:

1. the J2 disturbing function of Earth's zonal potential,
       R(r) = -(mu J2 R_E^2 / |r|^3) P2(z / |r|),   P2(x) = (3 x^2 - 1) / 2
   (U = mu/r [1 - J2 (R_E/r)^2 P2(sin phi)], R = U - mu/r);
2. its average over one orbit, R_bar(a, e, i, omega) = (1/2pi) integral R dM, evaluated
   numerically (trapezoid rule in M, spectrally accurate for a periodic integrand; Kepler's
   equation solved here by numpy Newton iterations);
3. Lagrange's planetary equations (e.g. Vallado & McClain [41] Sec. 9.3; Roy, Orbital Motion):
       dOmega/dt = dR/di / (n a^2 sqrt(1-e^2) sin i)
       domega/dt = sqrt(1-e^2) / (n a^2 e) dR/de - cot i / (n a^2 sqrt(1-e^2)) dR/di
       dM/dt     = n - (1-e^2) / (n a^2 e) dR/de - 2 / (n a) dR/da
   with the partial derivatives of R_bar taken by five-point central differences.

The oracle's J2 position at t must then equal the two-body (already pinned) position of the
elements advanced at these rates.  A wrong coefficient anywhere (3/4 for 3/2 in dM/dt, a
dropped sqrt(1-e^2), a sign) moves the position by tens to hundreds of km over a day, against a
1 m tolerance.
"""
import math

import numpy as np
import pytest

from tools import popgen

MU = 398600.4418           # km^3/s^2 (R1)
J2 = 1.08262668e-3         # EGM-96 (R19)
RE = 6378.137              # km, WGS-84 equatorial radius (R19)


def _kepler_E(M, e):
    E = M.copy() if e < 0.8 else np.full_like(M, math.pi)
    for _ in range(60):
        E = E - (E - e * np.sin(E) - M) / (1.0 - e * np.cos(E))
    return E


def _rbar(a, e, inc, argp, nquad=2048):
    """Orbit average of the J2 disturbing function (Omega = 0: R_bar does not depend on it)."""
    M = 2 * math.pi * np.arange(nquad) / nquad
    E = _kepler_E(M, e)
    nu = 2 * np.arctan2(math.sqrt(1 + e) * np.sin(E / 2), math.sqrt(1 - e) * np.cos(E / 2))
    r = a * (1 - e * np.cos(E))
    u = argp + nu
    sin_lat = math.sin(inc) * np.sin(u)          # z / r
    R = -(MU * J2 * RE ** 2 / r ** 3) * 0.5 * (3 * sin_lat ** 2 - 1)
    return float(np.mean(R))


def _d5(f, x, h):
    """Five-point central difference (truncation O(h^4))."""
    return (-f(x + 2 * h) + 8 * f(x + h) - 8 * f(x - h) + f(x - 2 * h)) / (12 * h)


def _rates(a, e, inc, argp):
    dRa = _d5(lambda x: _rbar(x, e, inc, argp), a, 1e-4 * a)
    dRe = _d5(lambda x: _rbar(a, x, inc, argp), e, min(1e-4, 0.25 * e))
    dRi = _d5(lambda x: _rbar(a, e, x, argp), inc, 1e-4)
    n = math.sqrt(MU / a ** 3)
    eta = math.sqrt(1 - e * e)
    dO = dRi / (n * a * a * eta * math.sin(inc))
    dw = eta / (n * a * a * e) * dRe - math.cos(inc) / math.sin(inc) / (n * a * a * eta) * dRi
    dM = n - (1 - e * e) / (n * a * a * e) * dRe - 2 / (n * a) * dRa
    return n, dO, dw, dM


def _mean_of_true(nu, e):
    E = 2 * math.atan2(math.sqrt(1 - e) * math.sin(nu / 2), math.sqrt(1 + e) * math.cos(nu / 2))
    return E - e * math.sin(E)


CASES = [  # a [km], e, i [deg], Omega0, omega0, nu0 [rad]
    (7000.0, 0.01, 30.0, 0.4, 1.0, 0.2),
    (6900.0, 0.002, 97.8, 2.0, 0.3, 4.0),
    (7500.0, 0.05, 63.4349, 5.0, 2.2, 1.3),
    (12000.0, 0.3, 45.0, 1.0, 4.0, 0.7),
    (26560.0, 0.01, 55.0, 3.0, 0.5, 2.5),
    (24400.0, 0.72, 7.0, 0.1, 3.0, 5.5),     # GTO-like
    (7200.0, 0.02, 140.0, 4.5, 5.0, 3.0),    # retrograde
]


@pytest.mark.parametrize("case", CASES, ids=[f"a{c[0]:.0f}_e{c[1]}_i{c[2]}" for c in CASES])
def test_j2_positions_follow_lagrange_rates(orc, case):
    a, e, inc_deg, O0, w0, nu0 = case
    inc = math.radians(inc_deg)
    n0, dO, dw, dM = _rates(a, e, inc, w0)
    pop = {k: np.array([v], dtype=np.float64) for k, v in zip(popgen.FIELDS, (a, e, inc, O0, w0, nu0))}
    pop["propagator"] = "j2"
    times = np.array([0.0, 3600.0, 43200.0, 86400.0])
    xj2 = orc.propagate(pop, times)[:, 0]
    M0 = _mean_of_true(nu0, e)
    for q, t in enumerate(times):
        # two-body position of the advanced elements: the Kepler propagator at time t' whose
        # mean anomaly n0 t' equals the J2-advanced M - M0
        kep = {k: np.array([v], dtype=np.float64) for k, v in
               zip(popgen.FIELDS, (a, e, inc, O0 + dO * t, w0 + dw * t, nu0))}
        tp = (dM * t) / n0
        xk = orc.propagate(kep, [tp])[0, 0]
        err = np.linalg.norm(xj2[q] - xk)
        assert err < 1e-3, (case, t, err)
    # the J2 part of each rate is material (not a vanishing correction the test cannot see):
    # over the day it moves the position by far more than the tolerance
    kep0 = {k: np.array([v], dtype=np.float64) for k, v in zip(popgen.FIELDS, (a, e, inc, O0, w0, nu0))}
    assert np.linalg.norm(orc.propagate(kep0, [86400.0])[0, 0] - xj2[-1]) > 10.0


def test_lagrange_rates_match_closed_form_limits():
    """The numerical derivation itself against two textbook limits it must reproduce: the
    node rate -1.5 n J2 (R_E/p)^2 cos i, p = a (1 - e^2), and the vanishing perigee rate at
    the critical inclination asin(sqrt(4/5)) -- so a failure above is the oracle's, not the
    quadrature's."""
    a, inc = 7000.0, math.radians(51.6)
    e = 1e-3
    n, dO, dw, dM = _rates(a, e, inc, 0.7)
    assert abs(dO - (-1.5 * n * J2 * (RE / (a * (1 - e * e))) ** 2 * math.cos(inc))) < 1e-6 * abs(dO)
    _, _, dw_c, _ = _rates(a, 0.05, math.asin(math.sqrt(0.8)), 1.2)
    assert abs(dw_c) < 1e-9 * n
