"""B200-native conjunction screening (Hellwig et al., IPDPS 2023) -- Python binding.

Thin ctypes binding of ``libcdscreen.so`` (C ABI declared in ``include/cdscreen.h``).  This
module only marshals arguments: every step of the screening path runs in the library's CUDA
kernels.  There is no CPU fallback: if the extension is missing or no B200 is present, calls
raise.

The same names as the C ABI are exported (``cd_screen``, ``cd_screen_ex``, ``cd_candidates``,
``cd_propagate``, ...) plus numpy-friendly wrappers ``screen``, ``candidates``, ``propagate``.
"""
from __future__ import annotations

import ctypes as C
import os
from pathlib import Path

import numpy as np

PKG = Path(__file__).resolve().parent
# CDSCREEN_LIB: load an alternative build of the same library (A/B timing of kernel variants)
LIB_PATH = Path(os.environ.get("CDSCREEN_LIB", str(PKG / "libcdscreen.so")))

CD_OK, CD_EINVAL, CD_ENOMEM, CD_ECUDA, CD_ENCCL, CD_ERANGE, CD_EINTERNAL, CD_ENODEV = range(8)
CD_GRID, CD_HYBRID, CD_LEGACY = 0, 1, 2
CD_PROP_KEPLER, CD_PROP_J2 = 0, 1
PROPAGATORS = {"kepler": CD_PROP_KEPLER, "j2": CD_PROP_J2}
CD_FLAG_DEGENERATE = 2
CD_FLAG_COPLANAR = 4
FIELDS = ("a", "e", "inc", "raan", "argp", "nu0")

CONJ_DTYPE = np.dtype([("i", "<u4"), ("j", "<u4"), ("step", "<u4"), ("flags", "<u4"),
                       ("tca", "<f8"), ("pca", "<f8")])
CAND_DTYPE = np.dtype([("i", "<u4"), ("j", "<u4"), ("step", "<u4")])

# C ABI symbols declared in include/cdscreen.h
ABI_SYMBOLS = ("cd_options_init", "cd_screen", "cd_screen_ex", "cd_candidates", "cd_propagate",
               "cd_conjunctions_sort_device", "cd_conjunctions_free", "cd_candidates_free", "cd_status_str", "cd_last_error",
               "cd_abi_version", "cd_kernel_launches", "cd_plan", "cd_shell_members",
               "cd_release_caches")
ABI_VERSION = 3


class CdError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(f"{status_str(status)}: {msg}")
        self.status = status


class cd_elements(C.Structure):
    _fields_ = [(k, C.c_void_p) for k in FIELDS]


class cd_conjunction(C.Structure):
    _fields_ = [("i", C.c_uint32), ("j", C.c_uint32), ("step", C.c_uint32), ("flags", C.c_uint32),
                ("tca", C.c_double), ("pca", C.c_double)]


class cd_candidate(C.Structure):
    _fields_ = [("i", C.c_uint32), ("j", C.c_uint32), ("step", C.c_uint32)]


class cd_conjunctions(C.Structure):
    _fields_ = [("data", C.c_void_p), ("count", C.c_size_t), ("_owner", C.c_void_p)]


class cd_stats(C.Structure):
    _fields_ = [("steps", C.c_uint64), ("object_steps", C.c_uint64), ("candidates", C.c_uint64),
                ("refined", C.c_uint64), ("conjunctions", C.c_uint64),
                ("hybrid_ap_rejected", C.c_uint64), ("hybrid_coplanar", C.c_uint64),
                ("hybrid_path_rejected", C.c_uint64), ("hybrid_time_rejected", C.c_uint64),
                ("kernel_launches", C.c_uint64), ("retries", C.c_uint64),
                ("ms_total", C.c_double), ("ms_clear", C.c_double),
                ("ms_propagate", C.c_double), ("ms_insert", C.c_double),
                ("ms_scan", C.c_double), ("ms_refine", C.c_double), ("ms_finalize", C.c_double),
                ("ms_precompute", C.c_double), ("launches_clear", C.c_uint64),
                ("launches_propagate", C.c_uint64), ("launches_insert", C.c_uint64),
                ("launches_scan", C.c_uint64), ("launches_refine", C.c_uint64),
                ("step_launches", C.c_uint64), ("cell_factor", C.c_double), ("grid_table", C.c_int),
                ("grids_in_flight", C.c_uint64), ("raw_pairs", C.c_uint64), ("digest", C.c_uint64),
                ("digest_conjunctions", C.c_uint64), ("min_pca", C.c_double)]

    def as_dict(self):
        return {k: getattr(self, k) for k, _ in self._fields_}


ALLOC_FN = C.CFUNCTYPE(C.c_void_p, C.c_size_t, C.c_void_p)
FREE_FN = C.CFUNCTYPE(None, C.c_void_p, C.c_void_p)


class cd_options(C.Structure):
    _fields_ = [("v_margin", C.c_double), ("grid_origin", C.c_double * 3), ("device", C.c_int),
                ("stream", C.c_void_p), ("rank", C.c_int), ("n_ranks", C.c_int),
                ("inputs_on_device", C.c_int), ("outputs_on_device", C.c_int),
                ("kepler_points", C.c_int), ("cell_factor", C.c_double),
                ("batch_object_steps", C.c_size_t), ("round_steps", C.c_size_t),
                ("profile_phases", C.c_int), ("l2_persist", C.c_int), ("grid_table", C.c_int),
                ("stats", C.POINTER(cd_stats)), ("propagator", C.c_int),
                ("shell_lo", C.c_double), ("shell_hi", C.c_double),
                ("alloc", ALLOC_FN), ("free", FREE_FN), ("alloc_ctx", C.c_void_p),
                ("shards", C.c_int), ("resort_steps", C.c_int), ("emit_raw_counts", C.c_int),
                ("digest_only", C.c_int)]


class cd_plan_info(C.Structure):
    _fields_ = [(k, C.c_double) for k in (
        "samples", "est_candidates", "est_candidates_per_step", "capacity", "capacity_bytes",
        "fixed_bytes", "bytes_per_grid", "grids_in_memory", "rounds", "cell_factor")]

    def as_dict(self):
        return {k: getattr(self, k) for k, _ in self._fields_}


_lib = None


def lib():
    """Load libcdscreen.so (built in-tree by __graft_entry__.build()).  Fails loudly."""
    global _lib
    if _lib is None:
        if not LIB_PATH.exists():
            raise ImportError(f"{LIB_PATH} is missing: run `python -c 'import __graft_entry__ as g; "
                              f"g.build()'` (nvcc, sm_100a) -- there is no CPU fallback")
        L = C.CDLL(str(LIB_PATH))
        P = C.POINTER
        L.cd_options_init.restype = None
        L.cd_options_init.argtypes = [P(cd_options)]
        L.cd_screen.restype = C.c_int
        L.cd_screen.argtypes = [P(cd_elements), C.c_size_t, C.c_double, C.c_double, C.c_double,
                                C.c_double, C.c_int, P(cd_conjunctions)]
        L.cd_screen_ex.restype = C.c_int
        L.cd_screen_ex.argtypes = [P(cd_elements), C.c_size_t, C.c_double, C.c_double, C.c_double,
                                   C.c_double, C.c_int, P(cd_options), P(cd_conjunctions)]
        L.cd_candidates.restype = C.c_int
        L.cd_candidates.argtypes = [P(cd_elements), C.c_size_t, C.c_double, C.c_double, C.c_double,
                                    C.c_double, C.c_int, P(cd_options), P(C.c_void_p),
                                    P(C.c_size_t)]
        L.cd_propagate.restype = C.c_int
        L.cd_propagate.argtypes = [P(cd_elements), C.c_size_t, C.c_void_p, C.c_size_t, C.c_void_p,
                                   C.c_void_p, P(cd_options)]
        L.cd_conjunctions_sort_device.restype = C.c_int
        L.cd_conjunctions_sort_device.argtypes = [C.c_void_p, C.c_size_t, C.c_void_p]
        L.cd_conjunctions_free.restype = None
        L.cd_conjunctions_free.argtypes = [P(cd_conjunctions)]
        L.cd_candidates_free.restype = None
        L.cd_candidates_free.argtypes = [C.c_void_p]
        L.cd_status_str.restype = C.c_char_p
        L.cd_status_str.argtypes = [C.c_int]
        L.cd_last_error.restype = C.c_char_p
        L.cd_abi_version.restype = C.c_int
        L.cd_kernel_launches.restype = C.c_uint64
        L.cd_shell_members.restype = C.c_int
        L.cd_shell_members.argtypes = [P(cd_elements), C.c_size_t, C.c_double, C.c_double, C.c_double,
                                       C.c_void_p, P(C.c_size_t)]
        L.cd_plan.restype = C.c_int
        L.cd_plan.argtypes = [C.c_size_t, C.c_double, C.c_double, C.c_double, C.c_double, C.c_int,
                              C.c_size_t, P(cd_plan_info)]
        L.cd_release_caches.restype = C.c_int
        L.cd_release_caches.argtypes = [C.c_int]
        if L.cd_abi_version() != ABI_VERSION:
            raise ImportError(f"{LIB_PATH}: ABI {L.cd_abi_version()} != {ABI_VERSION}: rebuild it")
        _lib = L
    return _lib


def status_str(s: int) -> str:
    return lib().cd_status_str(s).decode()


def last_error() -> str:
    return lib().cd_last_error().decode()


def _check(s):
    if s != CD_OK:
        raise CdError(s, last_error())


# raw C-ABI names -------------------------------------------------------------------------
def cd_options_init(opt):
    lib().cd_options_init(C.byref(opt))


def cd_screen(el, n, t0, t1, dt, d, mode, out):
    return lib().cd_screen(C.byref(el), n, t0, t1, dt, d, mode, C.byref(out))


def cd_screen_ex(el, n, t0, t1, dt, d, mode, opt, out):
    return lib().cd_screen_ex(C.byref(el), n, t0, t1, dt, d, mode,
                              C.byref(opt) if opt is not None else None, C.byref(out))


def cd_candidates(el, n, t0, t1, dt, d, mode, opt, out, count):
    return lib().cd_candidates(C.byref(el), n, t0, t1, dt, d, mode,
                               C.byref(opt) if opt is not None else None, C.byref(out),
                               C.byref(count))


def cd_propagate(el, n, t, nt, xyz, vxyz, opt):
    return lib().cd_propagate(C.byref(el), n, t, nt, xyz, vxyz,
                              C.byref(opt) if opt is not None else None)


def cd_conjunctions_sort_device(ptr, n, stream):
    return lib().cd_conjunctions_sort_device(ptr, n, stream)


def cd_conjunctions_free(c):
    lib().cd_conjunctions_free(C.byref(c))


def cd_candidates_free(p):
    lib().cd_candidates_free(p)


def cd_abi_version() -> int:
    return lib().cd_abi_version()


def cd_kernel_launches() -> int:
    return int(lib().cd_kernel_launches())


def cd_shell_members(el, n, lo, hi, gc, idx, count):
    return lib().cd_shell_members(C.byref(el), n, lo, hi, gc, idx, C.byref(count))


def cd_plan(n, t0, t1, dt, d, mode, mem_bytes, out):
    return lib().cd_plan(n, t0, t1, dt, d, mode, mem_bytes, C.byref(out))


def cd_release_caches(device=-1):
    return lib().cd_release_caches(int(device))


# numpy / torch wrappers --------------------------------------------------------------------
class _Elements:
    """Holds the arrays alive while the C call runs.  numpy -> host pointers; torch CUDA
    tensors -> device pointers (inputs_on_device).  Validates the layout the C ABI assumes
    (cdscreen.h cd_elements: six 1-D fp64 arrays of one length, all on one device) and raises
    ValueError before any pointer reaches C."""

    def __init__(self, pop):
        # optional force model carried by the population dict ("kepler" / "j2")
        self.propagator = pop.get("propagator") if hasattr(pop, "get") else None
        vals = [pop[k] for k in FIELDS]
        cuda = [hasattr(v, "is_cuda") and bool(v.is_cuda) for v in vals]
        if any(cuda) and not all(cuda):
            raise ValueError("elements: mix of CUDA tensors and host arrays")
        self.on_device = all(cuda)
        self.device = None
        if self.on_device:
            import torch
            for k, v in zip(FIELDS, vals):
                if v.dtype != torch.float64:
                    raise ValueError(f"elements[{k!r}]: dtype {v.dtype}, need torch.float64")
                if v.dim() != 1:
                    raise ValueError(f"elements[{k!r}]: need a 1-D tensor, got shape {tuple(v.shape)}")
            devs = {v.device.index for v in vals}
            if len(devs) != 1:
                raise ValueError(f"elements on several devices: {sorted(devs)}")
            self.device = devs.pop()
            self.keep = [v.contiguous() for v in vals]
            ptrs = [t.data_ptr() for t in self.keep]
            lens = [int(t.numel()) for t in self.keep]
        else:
            self.keep = []
            for k, v in zip(FIELDS, vals):
                a = np.asarray(v)
                if a.ndim != 1:
                    raise ValueError(f"elements[{k!r}]: need a 1-D array, got shape {a.shape}")
                self.keep.append(np.ascontiguousarray(a, dtype=np.float64))
            ptrs = [a.ctypes.data for a in self.keep]
            lens = [int(a.shape[0]) for a in self.keep]
        if len(set(lens)) != 1:
            raise ValueError(f"elements: arrays of different lengths {dict(zip(FIELDS, lens))}")
        self.n = lens[0]
        self.s = cd_elements(*ptrs)


class TorchAllocator:
    """cd_options.alloc / free backed by PyTorch's CUDA caching allocator on one device and
    stream (the call's stream: all of the library's use of a block is ordered on it).  Keep the
    object alive while the call runs and while device results from it exist."""

    def __init__(self, device, stream):
        import torch
        self.device = int(device)
        self.stream = stream
        self.live = 0
        self.peak = 0
        self.calls = 0

        def _alloc(nbytes, ctx):
            try:
                p = torch.cuda.caching_allocator_alloc(int(nbytes), self.device, self.stream)
            except Exception:
                return None
            self.live += 1
            self.calls += 1
            self.peak = max(self.peak, self.live)
            return p

        def _free(p, ctx):
            torch.cuda.caching_allocator_delete(p)
            self.live -= 1

        self.c_alloc = ALLOC_FN(_alloc)
        self.c_free = FREE_FN(_free)

    def install(self, opt):
        opt.alloc = self.c_alloc
        opt.free = self.c_free
        opt.alloc_ctx = None


def make_options(rank=0, n_ranks=1, v_margin=None, grid_origin=None, device=None, stream=None,
                 cell_factor=None, batch_object_steps=None, round_steps=None,
                 outputs_on_device=False, inputs_on_device=False, profile_phases=False,
                 l2_persist=None, grid_table=None, propagator=None, shell=None, allocator=None,
                 shards=None, kepler_points=None, resort_steps=None, emit_raw_counts=False,
                 digest_only=False):
    o = cd_options()
    cd_options_init(o)
    o.rank, o.n_ranks = rank, n_ranks
    if v_margin is not None:
        o.v_margin = v_margin
    if grid_origin is not None:
        for c in range(3):
            o.grid_origin[c] = float(grid_origin[c])
    if device is not None:
        o.device = int(device)
    if stream is not None:
        o.stream = stream
    if cell_factor is not None:
        o.cell_factor = float(cell_factor)
    if batch_object_steps is not None:
        o.batch_object_steps = int(batch_object_steps)
    if round_steps is not None:
        o.round_steps = int(round_steps)
    o.outputs_on_device = int(bool(outputs_on_device))
    o.inputs_on_device = int(bool(inputs_on_device))
    o.profile_phases = int(profile_phases)
    if l2_persist is not None:
        o.l2_persist = int(bool(l2_persist))
    if grid_table is not None:
        o.grid_table = int(grid_table)
    if propagator is not None:
        o.propagator = PROPAGATORS[propagator] if isinstance(propagator, str) else int(propagator)
    if shell is not None:
        o.shell_lo, o.shell_hi = float(shell[0]), float(shell[1])
    if allocator is not None:
        # the allocator's blocks are stream-ordered on its stream: the call must run there
        if stream is not None and int(stream or 0) != int(allocator.stream or 0):
            raise ValueError("allocator and stream disagree: the call must run on the allocator's stream")
        o.stream = allocator.stream
        if device is not None and int(device) != allocator.device:
            raise ValueError("allocator and device disagree")
        o.device = allocator.device
        allocator.install(o)
    if shards is not None:
        o.shards = int(shards)
    if kepler_points is not None:
        o.kepler_points = int(kepler_points)
    if resort_steps is not None:
        o.resort_steps = int(resort_steps)
    o.emit_raw_counts = int(bool(emit_raw_counts))
    o.digest_only = int(bool(digest_only))
    return o


def _mode(mode):
    if isinstance(mode, str):
        return {"grid": CD_GRID, "hybrid": CD_HYBRID, "legacy": CD_LEGACY}[mode]
    return int(mode)


def _torch_stream(device=None):
    try:
        import torch
        if torch.cuda.is_available():
            return torch.cuda.current_stream(device).cuda_stream
    except Exception:
        pass
    return None


def _resolve_allocator(kw):
    """allocator="torch": PyTorch's caching allocator on the current device and stream (the call
    then runs on that stream)."""
    if kw.get("allocator") == "torch":
        import torch
        dev = torch.cuda.current_device() if kw.get("device") is None else int(kw["device"])
        stream = kw.get("stream") or torch.cuda.current_stream(dev).cuda_stream
        kw["stream"] = stream
        kw["allocator"] = TorchAllocator(dev, stream)
    return kw.get("allocator")


def _device_options(E, kw):
    """Device inputs (CUDA tensors): run on their device and, unless a stream is given, on torch's
    current stream there -- the stream that wrote them (cdscreen.h "Streams")."""
    if not E.on_device:
        return
    if kw.get("device") is not None and int(kw["device"]) != E.device:
        raise ValueError(f"device={kw['device']} but the elements live on cuda:{E.device}")
    kw["device"] = E.device
    if kw.get("stream") is None and kw.get("allocator") is None:
        kw["stream"] = _torch_stream(E.device)


def screen(pop, t0, t1, dt, d, mode="grid", return_stats=False, **kw):
    """Conjunctions as a structured numpy array (CONJ_DTYPE), sorted by (i, j, step)."""
    E = _Elements(pop)
    st = cd_stats()
    kw.setdefault("propagator", E.propagator)
    keep_alloc = _resolve_allocator(kw)   # noqa: F841 (alive for the call)
    _device_options(E, kw)
    opt = make_options(inputs_on_device=E.on_device, **kw)
    opt.stats = C.pointer(st)
    out = cd_conjunctions()
    _check(cd_screen_ex(E.s, E.n, float(t0), float(t1), float(dt), float(d), _mode(mode), opt, out))
    if opt.outputs_on_device:
        cd_conjunctions_free(out)
        raise ValueError("use cd_screen_ex with a device result for outputs_on_device")
    if out.count:
        # zero-copy view of the library-owned host result; released when the array is
        buf = (C.c_char * (out.count * CONJ_DTYPE.itemsize)).from_address(out.data)
        buf._owner = _ResultOwner(out)
        res = np.frombuffer(buf, dtype=CONJ_DTYPE)
    else:
        cd_conjunctions_free(out)
        res = np.zeros(0, dtype=CONJ_DTYPE)
    return (res, st.as_dict()) if return_stats else res


class _ResultOwner:
    """Frees a library-owned host result (cd_conjunctions_free) when the last view goes."""

    def __init__(self, out):
        self.out = out

    def __del__(self):
        try:
            cd_conjunctions_free(self.out)
        except Exception:
            pass


def candidates(pop, t0, t1, dt, d, mode="grid", return_stats=False, **kw):
    """The level-1 candidate set K as a structured numpy array (CAND_DTYPE), sorted."""
    E = _Elements(pop)
    st = cd_stats()
    kw.setdefault("propagator", E.propagator)
    keep_alloc = _resolve_allocator(kw)   # noqa: F841
    _device_options(E, kw)
    opt = make_options(inputs_on_device=E.on_device, **kw)
    opt.stats = C.pointer(st)
    p = C.c_void_p()
    cnt = C.c_size_t()
    _check(cd_candidates(E.s, E.n, float(t0), float(t1), float(dt), float(d), _mode(mode), opt, p,
                         cnt))
    try:
        if cnt.value:
            buf = (C.c_char * (cnt.value * CAND_DTYPE.itemsize)).from_address(p.value)
            res = np.frombuffer(buf, dtype=CAND_DTYPE).copy()
        else:
            res = np.zeros(0, dtype=CAND_DTYPE)
    finally:
        cd_candidates_free(p)
    return (res, st.as_dict()) if return_stats else res


def propagate(pop, times, velocity=False, **kw):
    """Positions (nt, n, 3) [km] (and velocities [km/s]) at `times` [s from epoch]."""
    E = _Elements(pop)
    t = np.ascontiguousarray(np.atleast_1d(np.asarray(times, dtype=np.float64)))
    xyz = np.zeros((t.size, E.n, 3))
    v = np.zeros((t.size, E.n, 3)) if velocity else None
    kw.setdefault("propagator", E.propagator)
    _device_options(E, kw)
    opt = make_options(inputs_on_device=E.on_device, **kw)
    _check(cd_propagate(E.s, E.n, t.ctypes.data, t.size, xyz.ctypes.data,
                        v.ctypes.data if velocity else None, opt))
    return (xyz, v) if velocity else xyz



def conjunction_digest(conj):
    """The digest of a conjunction array as cd_stats.digest defines it (cdscreen.h): sum mod 2^64
    of i * 0x9E3779B1 + j * 0x85EBCA77 + step * 0xC2B2AE3D."""
    if len(conj) == 0:
        return 0
    h = (conj["i"].astype(np.uint64) * np.uint64(0x9E3779B1) + conj["j"].astype(np.uint64) * np.uint64(0x85EBCA77)
         + conj["step"].astype(np.uint64) * np.uint64(0xC2B2AE3D))
    return int(np.sum(h, dtype=np.uint64))


def release_caches(device=-1):
    """Return the library's cached device memory (private pool, result buffer cache)."""
    _check(cd_release_caches(device))


def plan(n, t0, t1, dt, d, mode="grid", mem_bytes=0):
    """A-priori sizing (Extra-P candidate model, grids in memory, rounds) as a dict."""
    out = cd_plan_info()
    _check(cd_plan(int(n), float(t0), float(t1), float(dt), float(d), _mode(mode), int(mem_bytes), out))
    return out.as_dict()


def shell_members(pop, lo, hi, gc):
    """Indices (uint32, increasing) of the objects a radial shard [lo, hi) must hold."""
    E = _Elements(pop)
    if E.on_device:
        raise ValueError("shell_members takes host arrays")
    idx = np.zeros(max(E.n, 1), dtype=np.uint32)
    cnt = C.c_size_t()
    _check(cd_shell_members(E.s, E.n, float(lo), float(hi), float(gc), idx.ctypes.data, cnt))
    return idx[:cnt.value].copy()
