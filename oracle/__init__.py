"""CPU oracle -- TEST INFRASTRUCTURE ONLY.

Plain, slow, obviously-correct CPU implementation (plain C, fp64, OpenMP over steps) of the
screening path of Hellwig et al., IPDPS 2023.  Only ``tests/``, ``__graft_entry__.smoke()`` and
``bench.py``'s ``cpu_baseline`` / ``--impl reference`` legs may import this package.  The product
path (``paper_conf_ipps_hellwigcmbw23_b200``) never imports it and shares no code with it.

Functions and the passages they follow are documented in ``oracle/cd_oracle.c``.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess
from pathlib import Path

import numpy as np

HERE = Path(__file__).resolve().parent
LIB = HERE / "liborc.so"
SOURCES = sorted(HERE.glob("*.c"))

MULTI = 1
DEGENERATE = 2
COPLANAR = 4
H_AP, H_COPLANAR, H_PATH, H_TIME = 1, 2, 4, 8

CAND_DTYPE = np.dtype([("i", "<u4"), ("j", "<u4"), ("step", "<u4")])
CONJ_DTYPE = np.dtype([("i", "<u4"), ("j", "<u4"), ("step", "<u4"), ("flags", "<u4"),
                       ("tca", "<f8"), ("pca", "<f8")])


def build(force: bool = False) -> Path:
    """Compile the oracle with gcc (plain C11, -ffp-contract=off: no fused multiply-adds)."""
    newest = max(p.stat().st_mtime for p in SOURCES + [HERE / "cd_oracle.h"])
    if LIB.exists() and not force and LIB.stat().st_mtime >= newest:
        return LIB
    tmp = LIB.with_suffix(f".so.tmp{os.getpid()}")
    cmd = ["gcc", "-std=c11", "-O2", "-fopenmp", "-ffp-contract=off", "-fno-fast-math",
           "-fPIC", "-shared", "-o", str(tmp)] + [str(s) for s in SOURCES] + ["-lm"]
    subprocess.run(cmd, check=True)
    os.replace(tmp, LIB)
    return LIB


PROPAGATORS = {"kepler": 0, "j2": 1}


class _Elements(C.Structure):
    _fields_ = [(k, C.POINTER(C.c_double)) for k in ("a", "e", "inc", "raan", "argp", "nu0")] + \
        [("model", C.c_int)]


_lib = None


def lib():
    global _lib
    if _lib is None:
        build()
        L = C.CDLL(str(LIB))
        P = C.POINTER
        L.orc_mu.restype = C.c_double
        L.orc_j2.restype = C.c_double
        L.orc_earth_radius.restype = C.c_double
        L.orc_num_threads.restype = C.c_int
        L.orc_kepler_newton.restype = C.c_double
        L.orc_kepler_newton.argtypes = [C.c_double, C.c_double]
        L.orc_num_steps.restype = C.c_int64
        L.orc_num_steps.argtypes = [C.c_double, C.c_double, C.c_double]
        L.orc_propagate.restype = None
        L.orc_propagate.argtypes = [P(_Elements), C.c_int64, P(C.c_double), C.c_int64,
                                    P(C.c_double), P(C.c_double)]
        L.orc_candidates_brute.restype = C.c_int64
        L.orc_candidates_brute.argtypes = [P(_Elements), C.c_int64, C.c_double, C.c_double,
                                           C.c_double, C.c_double, C.c_int64, C.c_int64,
                                           P(C.c_void_p)]
        L.orc_candidates_grid.restype = C.c_int64
        L.orc_candidates_grid.argtypes = [P(_Elements), C.c_int64, C.c_double, C.c_double,
                                          C.c_double, C.c_double, C.c_double, P(C.c_double),
                                          C.c_int64, C.c_int64, P(C.c_void_p)]
        L.orc_conjunctions.restype = C.c_int64
        L.orc_conjunctions.argtypes = [P(_Elements), C.c_int64, C.c_double, C.c_double,
                                       C.c_double, C.c_double, C.c_double, C.c_void_p,
                                       C.c_int64, P(C.c_void_p)]
        L.orc_pair_distance.restype = None
        L.orc_pair_distance.argtypes = [P(_Elements), C.c_int64, C.c_int64, P(C.c_double),
                                        C.c_int64, P(C.c_double), P(C.c_double)]
        L.orc_candidate_flags.restype = None
        L.orc_candidate_flags.argtypes = [P(_Elements), C.c_int64, C.c_double, C.c_double,
                                          C.c_double, C.c_void_p, C.c_int64, C.c_void_p]
        L.orc_free.restype = None
        L.orc_free.argtypes = [C.c_void_p]
        if hasattr(L, "orc_hybrid"):
            _bind_hybrid(L)
        _lib = L
    return _lib


def _bind_hybrid(L):
    P = C.POINTER
    L.orc_hybrid.restype = C.c_int64
    L.orc_hybrid.argtypes = [P(_Elements), C.c_int64, C.c_double, C.c_double, C.c_double,
                             C.c_double, C.c_double, C.c_int64, C.c_int64, P(C.c_void_p),
                             P(C.c_int64)]
    L.orc_legacy.restype = C.c_int64
    L.orc_legacy.argtypes = [P(_Elements), C.c_int64, C.c_double, C.c_double, C.c_double,
                             C.c_double, P(C.c_void_p), P(C.c_int64)]
    L.orc_pair_filter.restype = C.c_int
    L.orc_pair_filter.argtypes = [P(_Elements), C.c_int64, C.c_int64, C.c_double, C.c_double,
                                  C.c_double, P(C.c_double), C.c_int, P(C.c_int)]


def _f64(x):
    return np.ascontiguousarray(np.asarray(x, dtype=np.float64))


def _dp(x):
    return x.ctypes.data_as(C.POINTER(C.c_double))


class _Pop:
    """Keeps the contiguous arrays alive while C holds pointers to them."""

    def __init__(self, pop):
        self.arrs = [_f64(pop[k]) for k in ("a", "e", "inc", "raan", "argp", "nu0")]
        self.n = int(self.arrs[0].shape[0])
        # the force model travels with the population: pop["propagator"] in PROPAGATORS
        self.model = PROPAGATORS[pop.get("propagator", "kepler")] if hasattr(pop, "get") else 0
        self.s = _Elements(*[_dp(a) for a in self.arrs], self.model)

    @property
    def ref(self):
        return C.byref(self.s)


def mu() -> float:
    return lib().orc_mu()


def j2() -> float:
    return lib().orc_j2()


def earth_radius() -> float:
    return lib().orc_earth_radius()


def with_propagator(pop, name):
    """The population with its force model set ("kepler" or "j2")."""
    assert name in PROPAGATORS, name
    return dict(pop, propagator=name)


def num_threads() -> int:
    return lib().orc_num_threads()


def num_steps(t0, t1, dt) -> int:
    return int(lib().orc_num_steps(t0, t1, dt))


def kepler(M, e) -> float:
    return lib().orc_kepler_newton(float(M), float(e))


def propagate(pop, times, velocity=False):
    """Positions (and velocities) at `times`: arrays of shape (nt, n, 3), km and km/s."""
    P = _Pop(pop)
    t = _f64(np.atleast_1d(times))
    xyz = np.zeros((t.size, P.n, 3))
    v = np.zeros((t.size, P.n, 3)) if velocity else None
    lib().orc_propagate(P.ref, P.n, _dp(t), t.size, _dp(xyz), _dp(v) if velocity else None)
    return (xyz, v) if velocity else xyz


def _take(ptr, count, dtype):
    if count == 0:
        lib().orc_free(ptr)
        return np.zeros(0, dtype=dtype)
    buf = (C.c_char * (count * dtype.itemsize)).from_address(ptr.value)
    arr = np.frombuffer(bytes(buf), dtype=dtype).copy()
    lib().orc_free(ptr)
    return arr


def candidates_brute(pop, t0, t1, dt, gc, k_begin=0, k_end=-1):
    """O(n^2) candidate set K as a structured array (i, j, step), sorted."""
    P = _Pop(pop)
    out = C.c_void_p()
    c = lib().orc_candidates_brute(P.ref, P.n, t0, t1, dt, gc, k_begin, k_end, C.byref(out))
    return _take(out, c, CAND_DTYPE)


def candidates_grid(pop, t0, t1, dt, gc, cell=0.0, origin=(0.0, 0.0, 0.0), k_begin=0, k_end=-1):
    """Candidate set K through the plain CPU grid (27 cells)."""
    P = _Pop(pop)
    o = _f64(origin)
    out = C.c_void_p()
    c = lib().orc_candidates_grid(P.ref, P.n, t0, t1, dt, gc, cell, _dp(o), k_begin, k_end,
                                  C.byref(out))
    return _take(out, c, CAND_DTYPE)


def conjunctions(pop, t0, t1, dt, d, gc, cands):
    """Local minima below d in each candidate's owner cell (structured CONJ_DTYPE, sorted)."""
    P = _Pop(pop)
    cands = np.ascontiguousarray(cands, dtype=CAND_DTYPE)
    out = C.c_void_p()
    c = lib().orc_conjunctions(P.ref, P.n, t0, t1, dt, d, gc, cands.ctypes.data_as(C.c_void_p),
                               cands.shape[0], C.byref(out))
    return _take(out, c, CONJ_DTYPE)


def candidate_flags(pop, t0, dt, gc, cands):
    """MULTI / DEGENERATE flags of arbitrary candidates (parity exclusions)."""
    P = _Pop(pop)
    cands = np.ascontiguousarray(cands, dtype=CAND_DTYPE)
    f = np.zeros(cands.shape[0], dtype=np.uint32)
    lib().orc_candidate_flags(P.ref, P.n, t0, dt, gc, cands.ctypes.data_as(C.c_void_p),
                              cands.shape[0], f.ctypes.data_as(C.c_void_p))
    return f


def pair_distance(pop, i, j, times):
    P = _Pop(pop)
    t = _f64(np.atleast_1d(times))
    D = np.zeros(t.size)
    g = np.zeros(t.size)
    lib().orc_pair_distance(P.ref, int(i), int(j), _dp(t), t.size, _dp(D), _dp(g))
    return D, g


def pair_filter(pop, i, j, d, tlo, thi):
    """Hybrid filter chain for one pair over [tlo, thi]: (flags, [(lo, hi), ...])."""
    P = _Pop(pop)
    if P.model:
        raise ValueError("hybrid filters assume fixed orbit planes: Kepler propagator only")
    iv = np.zeros(64)
    niv = C.c_int()
    f = lib().orc_pair_filter(P.ref, int(i), int(j), float(d), float(tlo), float(thi), _dp(iv), 32,
                              C.byref(niv))
    return int(f), [(iv[2 * q], iv[2 * q + 1]) for q in range(niv.value)]


def hybrid(pop, t0, t1, dt, d, v_margin=7.8, k_begin=0, k_end=-1):
    """Hybrid variant end to end (O4): conjunctions and the filter-stage counts
    (candidates, ap_rejected, coplanar, path_rejected, time_rejected, time_window_work)."""
    P = _Pop(pop)
    if P.model:
        raise ValueError("hybrid filters assume fixed orbit planes: Kepler propagator only")
    gc = cell_size(d, dt, v_margin)
    out = C.c_void_p()
    counts = (C.c_int64 * 6)()
    c = lib().orc_hybrid(P.ref, P.n, t0, t1, dt, d, gc, k_begin, k_end, C.byref(out), counts)
    keys = ("candidates", "ap_rejected", "coplanar", "path_rejected", "time_rejected", "window_work")
    return _take(out, c, CONJ_DTYPE), dict(zip(keys, list(counts)))


def legacy(pop, t0, t1, dt, d):
    """Legacy full-window filter chain (O5): every pair through AP ->
    coplanar -> orbit path -> time filter over [t0, t1], every local minimum of D below d in the
    surviving intervals.  Returns (conjunctions, counts) with counts = pairs, ap_rejected,
    coplanar, path_rejected, time_rejected, intervals."""
    P = _Pop(pop)
    if P.model:
        raise ValueError("the orbital filters assume fixed orbit planes: Kepler propagator only")
    out = C.c_void_p()
    counts = (C.c_int64 * 6)()
    c = lib().orc_legacy(P.ref, P.n, float(t0), float(t1), float(dt), float(d), C.byref(out), counts)
    keys = ("pairs", "ap_rejected", "coplanar", "path_rejected", "time_rejected", "intervals")
    return _take(out, c, CONJ_DTYPE), dict(zip(keys, list(counts)))


def cell_size(d, dt, v_margin=7.8):
    """Eq. 1: g_c = d + 7.8 * s_ps."""
    return d + v_margin * dt


def screen_grid(pop, t0, t1, dt, d, v_margin=7.8, k_begin=0, k_end=-1, brute=False,
                origin=(0.0, 0.0, 0.0)):
    """Grid variant end to end: candidates (O2) then conjunctions (O3)."""
    gc = cell_size(d, dt, v_margin)
    if brute:
        K = candidates_brute(pop, t0, t1, dt, gc, k_begin, k_end)
    else:
        K = candidates_grid(pop, t0, t1, dt, gc, 0.0, origin, k_begin, k_end)
    return K, conjunctions(pop, t0, t1, dt, d, gc, K)
