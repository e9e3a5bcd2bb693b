"""Pins for the CPU oracle (-m "not gpu").  Each test ties the oracle to something other than
itself: textbook values, closed forms, invariants, brute force, and geometric constructions.
A plausible mistake anywhere in the oracle (a dropped term, a wrong sign, a transposed
operand, a wrong index) fails at least one of these."""
import math
from pathlib import Path

import numpy as np
import pytest

from tools import popgen

GOLDEN = Path(__file__).resolve().parent / "golden"
MU = 398600.4418


def _one(a, e, inc=0.0, raan=0.0, argp=0.0, nu0=0.0):
    return {k: np.array([v], dtype=np.float64)
            for k, v in zip(popgen.FIELDS, (a, e, inc, raan, argp, nu0))}


def _rot(axis, ang):
    c, s = math.cos(ang), math.sin(ang)
    if axis == 1:
        return np.array([[1, 0, 0], [0, c, -s], [0, s, c]])
    return np.array([[c, -s, 0], [s, c, 0], [0, 0, 1]])


def _perifocal_to_eci(raan, inc, argp):
    """Rotation matrix R3(raan) R1(inc) R3(argp) (Curtis Sec. 4.6) -- an independent
    formulation of the perifocal unit vectors P (column 0) and Q (column 1)."""
    return _rot(3, raan) @ _rot(1, inc) @ _rot(3, argp)


def _golden(kind):
    rows = []
    for line in (GOLDEN / "kepler_textbook.txt").read_text().splitlines():
        if line.strip() and not line.startswith("#"):
            f = line.split()
            if f[0] == kind:
                rows.append([f[1]] + [float(x) for x in f[2:]])
    assert rows, kind
    return rows


# ---------------------------------------------------------------------------------------
# Kepler's equation (the paper's solver [43] solves E - e sin E = M)
# ---------------------------------------------------------------------------------------

def test_kepler_vallado_example(orc):
    for _, M_deg, e, E_deg in _golden("kepler_E_deg"):
        E = orc.kepler(math.radians(M_deg), e)
        assert abs(math.degrees(E) - E_deg) < 1e-9


def test_kepler_residual_and_special_cases(orc):
    rng = np.random.default_rng(1)
    for _ in range(4000):
        e = float(rng.choice([rng.uniform(0, 0.05), rng.uniform(0, 0.99)]))
        M = float(rng.uniform(0, 2 * math.pi))
        E = orc.kepler(M, e)
        assert abs(E - e * math.sin(E) - M) <= 4 * np.spacing(max(1.0, M))
    for M in (0.0, 1.0, math.pi, 5.0):
        assert orc.kepler(M, 0.0) == M
    for e in (0.0, 0.1, 0.5, 0.9):
        assert abs(orc.kepler(0.0, e)) < 1e-15
        assert abs(orc.kepler(math.pi, e) - math.pi) < 1e-15


# ---------------------------------------------------------------------------------------
# propagation (Fig. 7/8)
# ---------------------------------------------------------------------------------------

def test_curtis_time_of_flight(orc):
    """Curtis Ex. 3.1 / 3.2 (perigee 9600 km, apogee 21000 km)."""
    for _, rp, ra, nu_deg, t_expect in _golden("time_to_nu_s"):
        pop = _one(0.5 * (rp + ra), (ra - rp) / (ra + rp))
        r = orc.propagate(pop, [t_expect])[0, 0]
        nu = math.degrees(math.atan2(r[1], r[0])) % 360.0
        assert abs(nu - nu_deg) < 0.01
    for _, rp, ra, t, nu_expect in _golden("nu_after_t_deg"):
        pop = _one(0.5 * (rp + ra), (ra - rp) / (ra + rp))
        r = orc.propagate(pop, [t])[0, 0]
        nu = math.degrees(math.atan2(r[1], r[0])) % 360.0
        assert abs(nu - nu_expect) < 0.05


def test_circular_closed_form(orc):
    """e = 0: r = a (cos u P0 + sin u Q0), u = omega + nu0 + n t."""
    rng = np.random.default_rng(2)
    for _ in range(20):
        a = rng.uniform(6600, 42000)
        inc, raan, argp, nu0 = rng.uniform(0, math.pi), *rng.uniform(0, 2 * math.pi, 3)
        R = _perifocal_to_eci(raan, inc, 0.0)
        t = rng.uniform(0, 86400, 5)
        r = orc.propagate(_one(a, 0.0, inc, raan, argp, nu0), t)[:, 0]
        n = math.sqrt(MU / a ** 3)
        u = argp + nu0 + n * t
        ref = a * (np.cos(u)[:, None] * R[:, 0] + np.sin(u)[:, None] * R[:, 1])
        assert np.max(np.abs(r - ref)) <= 1e-9 * a


def test_epoch_geometry(orc):
    """At t = 0 the object sits at true anomaly nu0 on the conic r = p / (1 + e cos nu)."""
    rng = np.random.default_rng(3)
    for _ in range(50):
        a, e = rng.uniform(6600, 40000), rng.uniform(0, 0.9)
        inc, raan, argp, nu0 = rng.uniform(0, math.pi), *rng.uniform(0, 2 * math.pi, 3)
        r = orc.propagate(_one(a, e, inc, raan, argp, nu0), [0.0])[0, 0]
        R = _perifocal_to_eci(raan, inc, argp)
        rp = R.T @ r          # perifocal coordinates
        assert abs(rp[2]) < 1e-9 * a
        assert abs((math.atan2(rp[1], rp[0]) - nu0 + math.pi) % (2 * math.pi) - math.pi) < 1e-11
        assert abs(np.linalg.norm(r) - a * (1 - e * e) / (1 + e * math.cos(nu0))) < 1e-9 * a


def test_invariants_vis_viva_momentum_period(orc):
    rng = np.random.default_rng(4)
    pop = popgen.base_mixture(rng, 300)
    t = np.array([0.0, 1234.5, 86400.0])
    r, v = orc.propagate(pop, t, velocity=True)
    a, e = pop["a"], pop["e"]
    rn = np.linalg.norm(r, axis=2)
    v2 = np.sum(v * v, axis=2)
    assert np.max(np.abs(v2 / (MU * (2 / rn - 1 / a)) - 1)) < 1e-12
    h = np.linalg.norm(np.cross(r, v), axis=2)
    assert np.max(np.abs(h / np.sqrt(MU * a * (1 - e * e)) - 1)) < 1e-12
    # periodicity r(t + T) = r(t), T = 2 pi sqrt(a^3 / mu)
    T = 2 * math.pi * np.sqrt(a ** 3 / MU)
    for q in range(3):
        i = rng.integers(0, 300)
        p1 = orc.propagate(popgen.subset(pop, [i]), [100.0, 100.0 + T[i]])[:, 0]
        assert np.linalg.norm(p1[0] - p1[1]) <= 1e-9 * np.linalg.norm(p1[0])


def test_velocity_is_derivative_of_position(orc):
    rng = np.random.default_rng(5)
    pop = popgen.base_mixture(rng, 50)
    t = 3000.0
    h = 1e-3
    r = orc.propagate(pop, [t - h, t + h])
    _, v = orc.propagate(pop, [t], velocity=True)
    fd = (r[1] - r[0]) / (2 * h)
    assert np.max(np.abs(fd - v[0]) / np.linalg.norm(v[0], axis=1)[:, None]) < 1e-7


def test_perigee_position(orc):
    """nu0 = 0 at t = 0 -> r = a (1 - e) P (P from the rotation-matrix formulation)."""
    rng = np.random.default_rng(6)
    for _ in range(20):
        a, e = rng.uniform(6600, 40000), rng.uniform(0, 0.95)
        inc, raan, argp = rng.uniform(0, math.pi), *rng.uniform(0, 2 * math.pi, 2)
        r = orc.propagate(_one(a, e, inc, raan, argp, 0.0), [0.0])[0, 0]
        P = _perifocal_to_eci(raan, inc, argp)[:, 0]
        assert np.linalg.norm(r - a * (1 - e) * P) < 1e-9 * a


# ---------------------------------------------------------------------------------------
# candidate set K (readings R#6, R#7)
# ---------------------------------------------------------------------------------------

def _dense_pop(n, seed):
    # a compact LEO shell so that a small population still yields many candidates
    rng = np.random.default_rng(seed)
    return {"a": rng.uniform(6900, 6920, n), "e": rng.uniform(0, 0.002, n),
            "inc": rng.uniform(0, math.pi, n), "raan": rng.uniform(0, 2 * math.pi, n),
            "argp": rng.uniform(0, 2 * math.pi, n), "nu0": rng.uniform(0, 2 * math.pi, n)}


def test_grid_equals_brute_force(orc):
    pop = _dense_pop(1500, 11)
    for gc in (25.0, 60.0):
        Kb = orc.candidates_brute(pop, 0.0, 40.0, 1.0, gc)
        Kg = orc.candidates_grid(pop, 0.0, 40.0, 1.0, gc)
        assert len(Kb) > 50
        assert np.array_equal(Kb, Kg)
        Kc = orc.candidates_grid(pop, 0.0, 40.0, 1.0, gc, cell=2.5 * gc)
        assert np.array_equal(Kb, Kc)


def test_config1_grid_equals_brute(orc):
    pop, cfg, _ = popgen.make_config(1)
    gc = orc.cell_size(cfg.d, cfg.dt_grid)
    Kb = orc.candidates_brute(pop, cfg.t0, 120.0, cfg.dt_grid, gc)
    Kg = orc.candidates_grid(pop, cfg.t0, 120.0, cfg.dt_grid, gc)
    assert np.array_equal(Kb, Kg)


def test_grid_origin_and_permutation_invariance(orc):
    pop = _dense_pop(800, 12)
    gc = 40.0
    K0 = orc.candidates_grid(pop, 0.0, 20.0, 1.0, gc)
    rng = np.random.default_rng(13)
    for _ in range(3):
        o = rng.uniform(-1e4, 1e4, 3)
        assert np.array_equal(orc.candidates_grid(pop, 0.0, 20.0, 1.0, gc, origin=o), K0)
    perm = rng.permutation(800)
    Kp = orc.candidates_grid(popgen.subset(pop, perm), 0.0, 20.0, 1.0, gc)
    i, j = perm[Kp["i"]], perm[Kp["j"]]
    mapped = np.zeros(len(Kp), dtype=K0.dtype)
    mapped["i"], mapped["j"], mapped["step"] = np.minimum(i, j), np.maximum(i, j), Kp["step"]
    assert np.array_equal(np.sort(mapped, order=["i", "j", "step"]), K0)


def test_best_and_worst_case(orc):
    """P:101 best case (all far apart: no candidates), P:99 worst case (all co-located)."""
    n = 200
    far = {"a": 7000.0 + 100.0 * np.arange(n), "e": np.zeros(n), "inc": np.full(n, 0.7),
           "raan": np.linspace(0, 6, n), "argp": np.zeros(n), "nu0": np.linspace(0, 6, n)}
    assert len(orc.candidates_grid(far, 0.0, 300.0, 1.0, 17.8)) == 0
    co = {"a": np.full(n, 7000.0), "e": np.zeros(n), "inc": np.linspace(0.1, 3.0, n),
          "raan": np.full(n, 1.0), "argp": np.zeros(n), "nu0": np.zeros(n)}
    K = orc.candidates_grid(co, 0.0, 0.0, 1.0, 17.8)
    assert len(K) == n * (n - 1) // 2
    assert np.array_equal(K, orc.candidates_brute(co, 0.0, 0.0, 1.0, 17.8))


def _coorbit_pair(r, chord, inc=0.9, raan=0.3, u=0.4):
    """Two circular co-planar orbits of equal radius with a constant separation `chord`."""
    phi = 2 * math.asin(chord / (2 * r))
    return {"a": np.array([r, r]), "e": np.zeros(2), "inc": np.array([inc, inc]),
            "raan": np.array([raan, raan]), "argp": np.zeros(2), "nu0": np.array([u, u + phi])}


def test_distance_gate_strict_at_gc(orc):
    """A pair at constant D = g_c - 2 mm is a candidate at every step; g_c + 2 mm never is."""
    gc = 17.8
    K_in = orc.candidates_brute(_coorbit_pair(7000.0, gc - 2e-6), 0.0, 50.0, 1.0, gc)
    K_out = orc.candidates_brute(_coorbit_pair(7000.0, gc + 2e-6), 0.0, 50.0, 1.0, gc)
    assert len(K_in) == 51 and len(K_out) == 0
    assert np.array_equal(K_in, orc.candidates_grid(_coorbit_pair(7000.0, gc - 2e-6), 0.0, 50.0, 1.0, gc))


def test_cell_boundary_straddlers(orc):
    """Pairs placed just either side of a cell face (via grid_origin), incl. negative coords."""
    gc = 17.8
    pop = _coorbit_pair(7000.0, 5.0)
    r = orc.propagate(pop, [0.0])[0]
    mid = 0.5 * (r[0] + r[1])
    for axis in range(3):
        o = np.zeros(3)
        o[axis] = mid[axis]  # a cell face exactly between the two objects on this axis
        K = orc.candidates_grid(pop, 0.0, 0.0, 1.0, gc, origin=o)
        assert len(K) == 1
        o2 = o.copy()
        o2[axis] -= 1e-3      # 1 m off the midpoint
        assert len(orc.candidates_grid(pop, 0.0, 0.0, 1.0, gc, origin=o2)) == 1
    for sign in (-1.0, 1.0):
        flip = dict(pop)
        flip["raan"] = pop["raan"] + (math.pi if sign < 0 else 0.0)
        assert len(orc.candidates_grid(flip, 0.0, 0.0, 1.0, gc, origin=(0.0, 0.0, 0.0))) == 1


# ---------------------------------------------------------------------------------------
# conjunctions: closed forms and dense sampling
# ---------------------------------------------------------------------------------------

def _cfg1():
    import oracle
    pop, cfg, planted = popgen.make_config(1)
    gc = oracle.cell_size(cfg.d, cfg.dt_grid)
    K, C = oracle.screen_grid(pop, cfg.t0, cfg.t1, cfg.dt_grid, cfg.d)
    return pop, cfg, planted, gc, K, C


@pytest.fixture(scope="module")
def cfg1(orc):
    return _cfg1()


def test_closed_form_case_a(cfg1):
    pop, cfg, planted, gc, K, C = cfg1
    found = 0
    for pa in planted.case_a:
        n = math.sqrt(MU / pa.r ** 3)
        tca = (pa.u0 - pa.phi / 2) / n
        pca = 2 * pa.r * abs(math.cos(pa.delta / 2) * math.sin(pa.phi / 2))
        rows = C[(C["i"] == pa.ia) & (C["j"] == pa.ib)]
        if pca < cfg.d:
            assert len(rows) == 1, (pa, rows)
            assert abs(rows["tca"][0] - tca) < 1e-6
            assert abs(rows["pca"][0] - pca) < 1e-9
            assert rows["step"][0] == int(math.floor(tca + 0.5))
            found += 1
        else:
            assert len(rows) == 0
    assert found >= 5


def test_closed_form_case_b(orc, cfg1):
    """Identical a, e, Omega, M0, omega = 0, different i: PCA = 0 at perigee passage."""
    pop, cfg, planted, gc, K, C = cfg1
    for pb in planted.case_b:
        rows = C[(C["i"] == pb.ia) & (C["j"] == pb.ib)]
        assert len(rows) == 1
        t = rows["tca"][0]
        assert rows["pca"][0] < 1e-8
        a, e = pop["a"][pb.ia], pop["e"][pb.ia]
        r = orc.propagate(popgen.subset(pop, [pb.ia]), [t])[0, 0]
        assert abs(np.linalg.norm(r) - a * (1 - e)) < 1e-6   # at perigee
        # D(t) = 2 |r| |sin f| sin(|di|/2): check the shape at +-5 s around TCA
        di = abs(pop["inc"][pb.ib] - pop["inc"][pb.ia])
        for dt_ in (-5.0, 5.0):
            D, _ = orc.pair_distance(pop, pb.ia, pb.ib, [t + dt_])
            rr = orc.propagate(popgen.subset(pop, [pb.ia]), [t + dt_])[0, 0]
            R = _perifocal_to_eci(pop["raan"][pb.ia], pop["inc"][pb.ia], 0.0)
            f = math.atan2((R.T @ rr)[1], (R.T @ rr)[0])
            assert abs(D[0] - 2 * np.linalg.norm(rr) * abs(math.sin(f)) * math.sin(di / 2)) < 1e-8


def test_degenerate_twins(cfg1):
    pop, cfg, planted, gc, K, C = cfg1
    (ia, ib), = planted.twins
    rows = C[(C["i"] == ia) & (C["j"] == ib)]
    assert len(rows) == orc_steps(cfg)
    assert np.all(rows["flags"] & 2) and np.all(rows["pca"] == 0.0)
    assert np.array_equal(rows["step"], np.arange(orc_steps(cfg)))


def orc_steps(cfg):
    return int(math.floor((cfg.t1 - cfg.t0) / cfg.dt_grid)) + 1


def test_dense_sampling_brute_force(orc, cfg1):
    """Every local minimum of D below d found by 1 ms dense sampling of every candidate pair
    appears exactly once in the oracle's output (owner rule: the nearest step), and nothing
    else does."""
    pop, cfg, planted, gc, K, C = cfg1
    pairs = sorted(set(zip(K["i"].tolist(), K["j"].tolist())))
    twins = set(planted.twins)
    t = np.arange(cfg.t0, cfg.t1 + 1e-9, 1e-3)
    expect = []
    for (i, j) in pairs:
        if (i, j) in twins:
            continue
        D, _ = orc.pair_distance(pop, i, j, t)
        m = np.where((D[1:-1] < D[:-2]) & (D[1:-1] <= D[2:]) & (D[1:-1] < cfg.d))[0] + 1
        for q in m:
            k = int(math.floor((t[q] - cfg.t0) / cfg.dt_grid + 0.5))
            steps = K["step"][(K["i"] == i) & (K["j"] == j)]
            if k in steps:   # the method only sees minima whose nearest sample is a candidate
                expect.append((i, j, k, t[q], D[q]))
    got = [r for r in C if (int(r["i"]), int(r["j"])) not in twins]
    assert len(got) == len(expect)
    for (i, j, k, tq, Dq), r in zip(sorted(expect), got):
        assert (i, j, k) == (int(r["i"]), int(r["j"]), int(r["step"]))
        assert abs(r["tca"] - tq) < 1e-3
        assert r["pca"] <= Dq + 1e-12 and Dq - r["pca"] < 1e-3


def test_eq1_guarantee(orc, cfg1):
    """Eq. 1: with g_c = d + 7.8 dt, the nearest sample of every approach below d
    (relative speed <= 15.6 km/s) is within g_c -- i.e. its (i, j, k) is a candidate."""
    pop, cfg, planted, gc, K, C = cfg1
    for r in C:
        if r["flags"] & 2:
            continue
        assert r["step"] == int(math.floor((r["tca"] - cfg.t0) / cfg.dt_grid + 0.5))
    # a fine-step screen (dt = 0.05 s) finds no minimum below d that the 1 s screen missed,
    # except encounters faster than 2 x 7.8 km/s (SURVEY R#18)
    Kf, Cf = orc.screen_grid(pop, cfg.t0, 120.0, 0.05, cfg.d)
    coarse = {(int(r["i"]), int(r["j"]), round(float(r["tca"]), 2)) for r in C if r["tca"] <= 119.0}
    for r in Cf:
        if r["tca"] > 119.0 or r["tca"] < 1.0 or r["flags"] & 2:
            continue
        key = (int(r["i"]), int(r["j"]), round(float(r["tca"]), 2))
        if key not in coarse:
            _, v = orc.propagate(popgen.subset(pop, [r["i"], r["j"]]), [r["tca"]], velocity=True)
            assert np.linalg.norm(v[0, 0] - v[0, 1]) > 15.6


def test_time_slices_partition(orc):
    """Owner rule: screening [k0, k1) and [k1, K) separately gives the disjoint union."""
    pop = _dense_pop(1500, 21)
    d, dt = 10.0, 1.0
    gc = orc.cell_size(d, dt)
    K = orc.candidates_grid(pop, 0.0, 60.0, dt, gc)
    C = orc.conjunctions(pop, 0.0, 60.0, dt, d, gc, K)
    Ka = orc.candidates_grid(pop, 0.0, 60.0, dt, gc, k_end=25)
    Kb = orc.candidates_grid(pop, 0.0, 60.0, dt, gc, k_begin=25)
    Ca = orc.conjunctions(pop, 0.0, 60.0, dt, d, gc, Ka)
    Cb = orc.conjunctions(pop, 0.0, 60.0, dt, d, gc, Kb)
    assert np.array_equal(np.sort(np.concatenate([Ka, Kb]), order=["i", "j", "step"]), K)
    assert np.array_equal(np.sort(np.concatenate([Ca, Cb]), order=["i", "j", "step"]), C)
    assert len(C) > 5
