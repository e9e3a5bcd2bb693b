"""Seeded synthetic satellite populations (input generator shared by the oracle tests, the
CUDA-path tests and bench.py).

This module holds NONE of the screening method's arithmetic: no propagation, no Kepler solve,
no cell keys, no distances.  It only draws Kepler element sets (a, e, i, Omega, omega, nu0)
with the shape of the paper's workloads:

* PAPER.md:193, 221, 223-233 (Sec. V-A, Fig. 9, Table II): (a, e) concentrated near
  a ~ 7000 km, e ~ 0.0025; i ~ U(0, pi); Omega, omega, M ~ U(0, 2pi); true anomaly derived
  from the uniformly drawn mean anomaly.  The KDE itself needs the Celestrak data set, which is
  not available, so a seeded mixture shaped like it is used (SURVEY.md 8(d) "Base mixture").
* Starlink-like Walker shells and planted closed-form encounter pairs (SURVEY.md 8(d),
  Appendix A.4) for the catalog / parity configurations.

Mean anomaly -> true anomaly is done WITHOUT solving Kepler's equation: nu is drawn by
rejection sampling from the density that a uniform M induces on nu,
    p(nu) = (1-e^2)^{3/2} / (2 pi (1 + e cos nu)^2),
accepting nu ~ U(0, 2pi) with probability ((1-e)/(1+e cos nu))^2 (the density divided by its
maximum at nu = 0).  The result is distributed exactly as nu(M) for M ~ U(0, 2pi).

All units: km, rad.  Elements are osculating at epoch t = 0.
"""
from __future__ import annotations

import math
from dataclasses import dataclass, field

import numpy as np

R_EARTH = 6378.137  # km (WGS-84 equatorial radius), used only to turn altitudes into a
TWO_PI = 2.0 * math.pi
FIELDS = ("a", "e", "inc", "raan", "argp", "nu0")


# --------------------------------------------------------------------------------------
# helpers
# --------------------------------------------------------------------------------------

def _nu_from_uniform_mean_anomaly(rng: np.random.Generator, e: np.ndarray) -> np.ndarray:
    """Draw true anomalies distributed as nu(M), M ~ U(0, 2pi), by rejection sampling."""
    e = np.asarray(e, dtype=np.float64)
    nu = np.empty_like(e)
    todo = np.arange(e.size)
    while todo.size:
        cand = rng.uniform(0.0, TWO_PI, todo.size)
        u = rng.uniform(0.0, 1.0, todo.size)
        ee = e[todo]
        acc = u <= ((1.0 - ee) / (1.0 + ee * np.cos(cand))) ** 2
        nu[todo[acc]] = cand[acc]
        todo = todo[~acc]
    return nu


def _empty(n: int) -> dict:
    return {k: np.zeros(n, dtype=np.float64) for k in FIELDS}


def concat(*pops: dict) -> dict:
    return {k: np.ascontiguousarray(np.concatenate([p[k] for p in pops])) for k in FIELDS}


def subset(pop: dict, idx) -> dict:
    return {k: np.ascontiguousarray(pop[k][idx]) for k in FIELDS}


def size(pop: dict) -> int:
    return int(pop["a"].shape[0])


# --------------------------------------------------------------------------------------
# base mixture
# --------------------------------------------------------------------------------------

def base_mixture(rng: np.random.Generator, n: int, incl: str = "paper") -> dict:
    """75 % LEO / 10 % MEO / 10 % GEO / 5 % GTO-HEO mixture shaped like PAPER.md Fig. 9.

    incl = "paper": i ~ U(0, pi) (Table II).  incl = "catalog": a realistic inclination mix
    (SSO 97-99 deg, 53 deg, 70-87 deg, low-inclination GEO).
    """
    cls = rng.choice(4, size=n, p=[0.75, 0.10, 0.10, 0.05])
    a = np.empty(n)
    e = np.empty(n)
    # LEO: altitude mixture, log-normal eccentricity, perigee >= 150 km
    m = cls == 0
    k = int(m.sum())
    comp = rng.choice(3, size=k, p=[0.30, 0.35, 0.35])
    alt = np.where(comp == 0, rng.normal(550.0, 25.0, k),
                   np.where(comp == 1, rng.normal(800.0, 80.0, k), rng.uniform(350.0, 1400.0, k)))
    alt = np.clip(alt, 300.0, 2000.0)
    aa = R_EARTH + alt
    ee = np.clip(np.exp(rng.normal(math.log(0.0025), 1.0, k)), 1e-5, 0.05)
    ee = np.minimum(ee, 1.0 - (R_EARTH + 150.0) / aa)
    a[m], e[m] = aa, ee
    # MEO
    m = cls == 1
    k = int(m.sum())
    a[m] = rng.uniform(20000.0, 30000.0, k)
    e[m] = rng.uniform(0.0, 0.02, k)
    # GEO
    m = cls == 2
    k = int(m.sum())
    a[m] = rng.normal(42164.0, 30.0, k)
    e[m] = rng.uniform(0.0, 1e-3, k)
    # GTO / HEO
    m = cls == 3
    k = int(m.sum())
    rp = R_EARTH + rng.uniform(200.0, 1000.0, k)
    ra = R_EARTH + rng.uniform(20000.0, 40000.0, k)
    a[m] = 0.5 * (rp + ra)
    e[m] = (ra - rp) / (ra + rp)

    if incl == "paper":
        inc = rng.uniform(0.0, math.pi, n)
    elif incl == "catalog":
        inc = np.empty(n)
        deg = math.pi / 180.0
        for c in range(4):
            m = cls == c
            k = int(m.sum())
            if c == 0:
                sel = rng.choice(4, size=k, p=[0.35, 0.15, 0.25, 0.25])
                v = np.where(sel == 0, rng.uniform(97.0, 99.0, k),
                             np.where(sel == 1, rng.normal(53.0, 0.5, k),
                                      np.where(sel == 2, rng.uniform(70.0, 87.0, k),
                                               rng.uniform(0.0, 180.0, k))))
            elif c == 1:
                v = rng.normal(55.0, 3.0, k)
            elif c == 2:
                v = rng.uniform(0.0, 15.0, k)
            else:
                v = rng.uniform(0.0, 30.0, k)
            inc[m] = np.clip(v, 0.0, 180.0) * deg
    else:
        raise ValueError(incl)
    raan = rng.uniform(0.0, TWO_PI, n)
    argp = rng.uniform(0.0, TWO_PI, n)
    nu0 = _nu_from_uniform_mean_anomaly(rng, e)
    return {"a": a, "e": e, "inc": inc, "raan": raan, "argp": argp, "nu0": nu0}


# --------------------------------------------------------------------------------------
# Starlink-like Walker-delta shells
# --------------------------------------------------------------------------------------

# (altitude km, inclination deg, planes, nominal count)
SHELLS = [
    (550.0, 53.0, 72, 1584),
    (540.0, 53.2, 72, 1584),
    (570.0, 70.0, 36, 720),
    (560.0, 97.6, 10, 520),
    (350.0, 38.0, 48, 2500),
    (360.0, 97.0, 30, 1500),
    (530.0, 43.0, 28, 1000),
    (525.0, 33.0, 28, 1000),
]


def walker_shells(rng: np.random.Generator, n: int) -> dict:
    """n objects in Walker-delta shells (e = 1e-4), with small jitter so no two coincide."""
    if n <= 0:
        return _empty(0)
    w = np.array([s[3] for s in SHELLS], dtype=np.float64)
    counts = np.floor(n * w / w.sum()).astype(np.int64)
    counts[0] += n - counts.sum()
    deg = math.pi / 180.0
    parts = []
    for (alt, inc_deg, planes, _), cnt in zip(SHELLS, counts):
        cnt = int(cnt)
        if cnt == 0:
            continue
        per = int(math.ceil(cnt / planes))
        idx = np.arange(cnt)
        p = idx // per
        s = idx % per
        raan = (TWO_PI * p / planes + rng.normal(0.0, 1e-4, cnt)) % TWO_PI
        u = (TWO_PI * s / per + TWO_PI * p / (planes * per) + rng.normal(0.0, 1e-4, cnt)) % TWO_PI
        argp = rng.uniform(0.0, TWO_PI, cnt)
        parts.append({
            "a": R_EARTH + alt + rng.uniform(-0.5, 0.5, cnt),
            "e": np.full(cnt, 1e-4),
            "inc": (inc_deg + rng.normal(0.0, 0.01, cnt)) * deg,
            "raan": raan,
            "argp": argp,
            "nu0": (u - argp) % TWO_PI,
        })
    return concat(*parts)


# --------------------------------------------------------------------------------------
# planted closed-form pairs -- geometry of the FIXTURE only
# --------------------------------------------------------------------------------------

@dataclass
class PlantedCaseA:
    """Two circular orbits of radius r, common node (Omega), inclinations i and i + delta,
    omega = 0; arguments of latitude at epoch u_A(0) = -u0, u_B(0) = -u0 + phi.
    Closed form: TCA = (u0 - phi/2)/n, PCA = 2 r |cos(delta/2) sin(phi/2)|,
    n = sqrt(mu / r^3) -- evaluated by the tests, not here."""
    ia: int
    ib: int
    r: float
    delta: float
    phi: float
    u0: float


@dataclass
class PlantedCaseB:
    """Identical a, e, Omega, M0 with omega = 0 and inclinations i1 != i2:
    D(t) = 2 |r(t)| |sin f(t)| sin(|i1 - i2|/2), zero at perigee and apogee."""
    ia: int
    ib: int


@dataclass
class Planted:
    pop: dict
    case_a: list = field(default_factory=list)
    case_b: list = field(default_factory=list)
    colocated: list = field(default_factory=list)   # groups of indices sharing r(0)
    twins: list = field(default_factory=list)       # identical elements (degenerate D == 0)


def planted_pairs(rng: np.random.Generator, d: float, base_index: int = 0,
                  n_case_a: int = 12, n_case_b: int = 3, n_colocated: int = 5) -> Planted:
    """Closed-form encounter fixtures for the 10-minute config 1 window (t in [0, 600] s).

    Case-A PCAs are spread over [0, 2d]; u0 in [0.08, 0.5] rad puts the node passage of a
    ~7000 km orbit (n ~ 1.08e-3 rad/s) inside the window."""
    rows = []
    case_a, case_b, coloc, twins = [], [], [], []
    idx = base_index
    for q in range(n_case_a):
        r = float(rng.uniform(6800.0, 7300.0))
        delta = float(rng.uniform(0.3, 2.6))
        pca = 2.0 * d * (q + 0.5) / n_case_a
        phi = 2.0 * math.asin(pca / (2.0 * r * abs(math.cos(0.5 * delta))))
        if q % 2:
            phi = -phi
        u0 = float(rng.uniform(0.08, 0.5))
        inc = float(rng.uniform(0.05, math.pi - delta - 0.05))
        raan = float(rng.uniform(0.0, TWO_PI))
        rows.append((r, 0.0, inc, raan, 0.0, (-u0) % TWO_PI))
        rows.append((r, 0.0, inc + delta, raan, 0.0, (-u0 + phi) % TWO_PI))
        case_a.append(PlantedCaseA(idx, idx + 1, r, delta, phi, u0))
        idx += 2
    for q in range(n_case_b):
        a = float(rng.uniform(6900.0, 7400.0))
        e = float(rng.uniform(0.002, 0.02))
        i1 = float(rng.uniform(0.2, 1.4))
        i2 = i1 + float(rng.uniform(0.01, 0.5))
        raan = float(rng.uniform(0.0, TWO_PI))
        # both start shortly before perigee (nu0 slightly negative) so perigee falls in-window
        nu0 = (-float(rng.uniform(0.05, 0.4))) % TWO_PI
        rows.append((a, e, i1, raan, 0.0, nu0))
        rows.append((a, e, i2, raan, 0.0, nu0))
        case_b.append(PlantedCaseB(idx, idx + 1))
        idx += 2
    # co-located group: same point at t = 0 (circular, common node, nu0 = 0), different planes
    r = float(rng.uniform(6900.0, 7200.0))
    raan = float(rng.uniform(0.0, TWO_PI))
    grp = []
    for q in range(n_colocated):
        rows.append((r, 0.0, 0.3 + 0.4 * q, raan, 0.0, 0.0))
        grp.append(idx)
        idx += 1
    coloc.append(grp)
    # one identical twin pair (degenerate: D(t) == 0 for all t)
    el = (float(rng.uniform(6900.0, 7200.0)), 0.001, 1.0, 2.0, 0.5, 0.25)
    rows.append(el)
    rows.append(el)
    twins.append((idx, idx + 1))
    idx += 2
    arr = np.array(rows, dtype=np.float64)
    pop = {k: np.ascontiguousarray(arr[:, c]) for c, k in enumerate(FIELDS)}
    return Planted(pop, case_a, case_b, coloc, twins)


# --------------------------------------------------------------------------------------
# configurations (BASELINE.json "configs")
# --------------------------------------------------------------------------------------

@dataclass
class Config:
    name: str
    n: int
    d: float               # screening threshold [km]
    t0: float
    t1: float
    dt_grid: float | None  # grid-variant sampling step [s]
    dt_hybrid: float | None
    seed: int
    incl: str = "paper"
    shells: int = 0
    planted: bool = False


CONFIGS = {
    1: Config("cfg1_1k_leo_10km_10min", 1000, 10.0, 0.0, 600.0, 1.0, None, 20230501, "paper", 0, True),
    2: Config("cfg2_30k_catalog_24h", 30000, 2.0, 0.0, 86400.0, 1.0, 9.0, 20230502, "catalog"),
    3: Config("cfg3_100k_shells_24h", 100000, 2.0, 0.0, 86400.0, None, 9.0, 20230503, "catalog", 30000),
    4: Config("cfg4_1M_future_catalog_24h", 1000000, 2.0, 0.0, 86400.0, 1.0, 9.0, 20230504, "paper", 60000),
    5: Config("cfg5_8M_stress_7d", 8000000, 2.0, 0.0, 7 * 86400.0, 1.0, 9.0, 20230505, "paper", 60000),
}


def leo_only(rng: np.random.Generator, n: int) -> dict:
    """LEO-only population (config 1: '1,000 synthetic LEO objects')."""
    alt = rng.uniform(400.0, 1200.0, n)
    a = R_EARTH + alt
    e = np.clip(np.exp(rng.normal(math.log(0.0025), 1.0, n)), 1e-5, 0.02)
    inc = rng.uniform(0.0, math.pi, n)
    raan = rng.uniform(0.0, TWO_PI, n)
    argp = rng.uniform(0.0, TWO_PI, n)
    nu0 = _nu_from_uniform_mean_anomaly(rng, e)
    return {"a": a, "e": e, "inc": inc, "raan": raan, "argp": argp, "nu0": nu0}


def make_config(k: int, n: int | None = None):
    """Population for BASELINE.json config k (optionally resized to n objects, same recipe).

    Returns (pop, cfg, planted_or_None)."""
    cfg = CONFIGS[k]
    n = cfg.n if n is None else int(n)
    rng = np.random.default_rng(cfg.seed)
    planted = None
    if k == 1:
        planted = planted_pairs(rng, cfg.d, base_index=0)
        base = leo_only(rng, max(0, n))
        pop = concat(planted.pop, base)
    else:
        n_sh = min(cfg.shells, n) if cfg.shells else 0
        if cfg.shells and n < cfg.n:
            n_sh = int(round(n * cfg.shells / cfg.n))
        pop = concat(walker_shells(rng, n_sh), base_mixture(rng, n - n_sh, cfg.incl))
    return pop, cfg, planted


def random_population(n: int, seed: int, incl: str = "paper", shells: int = 0) -> dict:
    rng = np.random.default_rng(seed)
    return concat(walker_shells(rng, shells), base_mixture(rng, n - shells, incl))


def counter_rotating(m: int, seed: int) -> dict:
    """Near-coplanar counter-rotating population: one orbital plane flown both ways (mutual
    inclinations within ~0.2 deg of 180 deg), a ~ 7000 +- 3 km, e < 4e-4, random omega and M.
    Head-on encounters at ~15 km/s with very wide hybrid node windows (a stress case for the
    time filter)."""
    rng = np.random.default_rng(seed)
    rows = []
    for k in range(m):
        inc, raan = 0.9, 0.4
        if k % 2:
            inc = math.pi - inc + rng.uniform(-2e-3, 2e-3)
            raan = raan + math.pi + rng.uniform(-2e-3, 2e-3)
        rows.append((7000.0 + rng.uniform(-3.0, 3.0), rng.uniform(0.0, 4e-4), inc, raan,
                     rng.uniform(0, 2 * math.pi), rng.uniform(0, 2 * math.pi)))
    arr = np.array(rows, dtype=np.float64)
    return {k: np.ascontiguousarray(arr[:, c]) for c, k in enumerate(FIELDS)}
