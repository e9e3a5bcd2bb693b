"""Pins for the oracle's MULTI predicate -- the one parity exclusion rule that depends on the
oracle's own judgement (SURVEY 8(c) parity rules).

P:57 (Section III) defines a PCA as *a* local minimum of D(t); the paper's Brent search on
[t_k - t_w, t_k + t_w] finds one of them.  O3 flags a candidate MULTI when
g(t) = (r_i - r_j).(v_i - v_j) = (1/2) dD^2/dt changes sign more than once (either direction) on
[t_k - t_w, t_k + t_w], t_w = 2 g_c / min(|v_i|, |v_j|) (R10); O5 (legacy chain) flags a minimum
MULTI when another minimum of the pair lies within 2 dt of it.  Both predicates are pinned here
against the closed-form extrema of SURVEY Appendix A.4 case A, independent of the oracle:

  two circular orbits of radius r, common node, inclinations i and i + Delta, phase offset phi:
      D^2(t) = 2 r^2 (1 - cos theta),
      cos theta = (1/2) [cos phi (1 + cos Delta) + cos(2 u_A + phi) (1 - cos Delta)],
  u_A = n (t - t_node): D^2 is a function of cos(2 u_A + phi) alone, so its extrema (the sign
  changes of g) sit at 2 u_A + phi = m pi -- minima for even m, maxima for odd m -- i.e. every
  pi / (2n) seconds, at t_m = t_node + (m pi / 2 - phi / 2) / n.

A predicate that never fires, fires everywhere, looks at a window of the wrong width or centre,
or counts only one direction of sign change fails one of these tests.
"""
import math

import numpy as np
import pytest

from tools import popgen

MU = 398600.4418          # R1 (WGS-84 / EGM-96 GM)


def _case_a(r=7000.0, delta=1.0, phi=1e-3, u0=0.3, inc=0.4, raan=1.1):
    """Case-A pair: A at argument of latitude -u0 at t = 0 (node passage at t = u0 / n)."""
    tp = 2 * math.pi
    rows = [(r, 0.0, inc, raan, 0.0, (-u0) % tp), (r, 0.0, inc + delta, raan, 0.0, (-u0 + phi) % tp)]
    arr = np.array(rows, dtype=np.float64)
    pop = {k: np.ascontiguousarray(arr[:, c]) for c, k in enumerate(popgen.FIELDS)}
    n = math.sqrt(MU / r ** 3)
    v = math.sqrt(MU / r)
    t_node = u0 / n

    def extremum(m):   # m even: minimum, m odd: maximum
        return t_node + (m * math.pi / 2 - phi / 2) / n

    return pop, n, v, extremum


def _extrema_in(extremum, lo, hi):
    ms = range(-8, 40)
    return [m for m in ms if lo < extremum(m) < hi]


def test_closed_form_extrema_are_the_sign_changes_of_g(orc):
    """Sanity of the construction itself: g changes sign at the closed-form times, D^2 is
    minimal at even m and maximal at odd m (so the predicate tests below test the oracle,
    not the fixture)."""
    pop, n, v, ext = _case_a()
    for m in range(0, 6):
        t = ext(m)
        D, g = orc.pair_distance(pop, 0, 1, [t - 1.0, t, t + 1.0])
        if m % 2 == 0:
            assert g[0] < 0 < g[2] and D[1] < D[0] and D[1] < D[2], (m, g, D)
        else:
            assert g[0] > 0 > g[2] and D[1] > D[0] and D[1] > D[2], (m, g, D)


def _cand(step):
    return np.array([(0, 1, step)], dtype=[("i", "<u4"), ("j", "<u4"), ("step", "<u4")])


@pytest.mark.parametrize("seed", range(6))
def test_o3_multi_flag_counts_sign_changes_in_tw_window(orc, seed):
    """orc_candidate_flags: MULTI iff the closed-form extrema inside [t_k - t_w, t_k + t_w]
    number more than one; t_k and t_w drawn at random (away from the window edges, where the
    64-sample count is ambiguous)."""
    rng = np.random.default_rng(1234 + seed)
    pop, n, v, ext = _case_a(r=float(rng.uniform(6800, 7400)), delta=float(rng.uniform(0.3, 2.0)),
                             u0=float(rng.uniform(0.1, 1.0)))
    quarter = math.pi / (2 * n)                      # spacing of the extrema
    checked = {True: 0, False: 0}
    tries = 0
    while min(checked.values()) < 6 and tries < 400:
        tries += 1
        k = int(rng.integers(0, int(6 * quarter)))   # dt = 1 s, t0 = 0: t_k = k
        tw = float(rng.uniform(0.2, 2.6)) * quarter
        lo, hi = k - tw, k + tw
        spacing = 2 * tw / 64
        if any(abs(ext(m) - e) < 2 * spacing for m in range(-8, 40) for e in (lo, hi)):
            continue
        want = len(_extrema_in(ext, lo, hi)) > 1
        gc = 0.5 * tw * v                             # t_w = 2 g_c / v (both speeds equal)
        f = orc.candidate_flags(pop, 0.0, 1.0, gc, _cand(k))
        assert bool(f[0] & orc.MULTI) == want, (k, tw / quarter, _extrema_in(ext, lo, hi))
        assert not f[0] & orc.DEGENERATE
        checked[want] += 1
    assert min(checked.values()) >= 6, checked


def test_o3_conjunction_rows_carry_the_flag(orc):
    """A conjunction row (minimum owned by step k = round(t_min)) is MULTI exactly when t_w
    reaches the neighbouring maxima at t_min +- pi / (2n); flag set and clear on either side."""
    pop, n, v, ext = _case_a()
    quarter = math.pi / (2 * n)
    tmin = ext(2)
    k = int(math.floor(tmin + 0.5))
    d = 10.0
    for frac, want in ((0.5, False), (0.9, False), (1.05, True), (1.6, True), (2.3, True)):
        tw = frac * quarter
        gc = 0.5 * tw * v
        C = orc.conjunctions(pop, 0.0, 2 * tmin, 1.0, d, gc, _cand(k))
        assert len(C) == 1, C
        assert abs(C["tca"][0] - tmin) < 1e-6
        assert bool(C["flags"][0] & orc.MULTI) == want, (frac, C)


def test_o3_crossing_pair_at_paper_scale_is_not_multi(orc):
    """At the paper's scale (d = 10 km, dt = 1 s, g_c = d + 7.8 dt: t_w ~ 5 s, far below the
    extrema spacing of ~1500 s) a case-A crossing has a single minimum: never MULTI.  This is
    the regime of every parity test, where the predicate must not fire."""
    import oracle
    pop, n, v, ext = _case_a()
    gc = oracle.cell_size(10.0, 1.0)
    tmin = ext(0)
    ks = np.arange(int(tmin) - 3, int(tmin) + 4)
    cands = np.array([(0, 1, int(k)) for k in ks], dtype=[("i", "<u4"), ("j", "<u4"), ("step", "<u4")])
    f = orc.candidate_flags(pop, 0.0, 1.0, gc, cands)
    assert not np.any(f & orc.MULTI), f
    C = orc.conjunctions(pop, 0.0, 2 * tmin, 1.0, 10.0, gc, cands)
    assert len(C) == 1 and not C["flags"][0] & orc.MULTI, C


@pytest.mark.parametrize("ratio,want", [(0.80, False), (0.95, False), (1.05, True), (1.30, True)])
def test_o5_legacy_multi_is_second_minimum_within_2dt(orc, ratio, want):
    """O5 flags a minimum MULTI iff another minimum of the pair lies within 2 dt.  Case A has
    minima every pi / n (at the two mutual nodes): dt = ratio * pi / (2n) puts the neighbouring
    minimum just outside (ratio < 1) or inside (ratio > 1) the 2 dt reach."""
    pop, n, v, ext = _case_a(phi=1e-3)
    half = math.pi / n                                  # minimum spacing
    dt = ratio * half / 2
    t_last = ext(6)
    K = int(math.floor(t_last / dt)) + 3
    t1 = (K - 1) * dt
    d = 10.0
    C, counts = orc.legacy(pop, 0.0, t1, dt, d)
    mins = [ext(m) for m in (0, 2, 4, 6) if ext(m) > 0]
    got = sorted(C["tca"].tolist())
    assert len(got) == len(mins), (got, mins)
    for t, tm in zip(got, mins):
        assert abs(t - tm) < 1e-6
    # every minimum has a neighbour at pi / n; only the 2 dt reach decides
    assert all(bool(f & orc.MULTI) == want for f in C["flags"]), (ratio, C["flags"])


def test_o5_isolated_minimum_is_not_multi(orc):
    """A window holding a single minimum of the pair: no MULTI whatever dt."""
    pop, n, v, ext = _case_a()
    tmin = ext(2)
    for dt in (1.0, 30.0, 600.0):
        t0 = tmin - 0.25 * math.pi / n
        t1 = tmin + 0.25 * math.pi / n
        C, _ = orc.legacy(pop, t0, t1, dt, 10.0)
        assert len(C) == 1 and abs(C["tca"][0] - tmin) < 1e-6, (dt, C)
        assert not C["flags"][0] & orc.MULTI
