"""Multi-GPU time slicing, radial object-space shards, and the conjunction-list merge
(SURVEY.md 8(e), 8(f) row 2).

One process per GPU.  The window's K sampling steps are split into contiguous slices; a call
with ``rank=q, n_ranks=S`` screens steps [floor(q K / S), floor((q + 1) K / S)) and reports only
the minima it owns (owner rule), so slices partition the result set with no halo and no
data-path collective.  The one real exchange is the final merge: an all-gather of the per-rank
record counts, then of the (padded) 32-byte records, over NCCL / NVLink (``torch.distributed``
is the plumbing), followed by the library's device sort by (i, j, step).

Radial shards (for populations whose per-step grid would not fit one GPU;
the paper names multiple GPUs for memory as future work): shard s of S keeps the
candidates whose nearer-to-Earth partner is at radius |r| in [b_s, b_{s+1}) at t_k.  It holds
only its members -- objects whose radius range [a(1-e), a(1+e)] meets [b_s, b_{s+1} + g_c): its
own objects plus a g_c halo above the band -- so its grid and entries scale with n/S plus the
halo and the eccentric objects that cross the band.  Positions are recomputed from the
replicated elements on every shard (bit-identical), so the halo needs no exchange: a shard
never reads another shard's grid.  Shards and time slices combine (rank = (shard, slice)).
"""
from __future__ import annotations

import numpy as np

REC_BYTES = 32


def slice_range(K: int, q: int, S: int):
    """Steps owned by slice q of S (same arithmetic as the C library's rank/n_ranks)."""
    return (K * q) // S, (K * (q + 1)) // S


def gather_records(local, group=None):
    """All-gather variable-length record blocks.

    `local` is a uint8 tensor of shape (m, 32) on this rank's device (cuda for NCCL, cpu for
    gloo).  Returns the concatenation over ranks (rank order), shape (sum m, 32)."""
    import torch
    import torch.distributed as dist
    world = dist.get_world_size(group)
    dev = local.device
    cnt = torch.tensor([local.shape[0]], dtype=torch.int64, device=dev)
    counts = [torch.zeros_like(cnt) for _ in range(world)]
    dist.all_gather(counts, cnt, group=group)
    counts = [int(c.item()) for c in counts]
    mx = max(counts) if counts else 0
    if mx == 0:
        return torch.zeros((0, REC_BYTES), dtype=torch.uint8, device=dev)
    pad = torch.zeros((mx, REC_BYTES), dtype=torch.uint8, device=dev)
    pad[: local.shape[0]] = local
    bufs = [torch.empty_like(pad) for _ in range(world)]
    dist.all_gather(bufs, pad, group=group)
    return torch.cat([b[:c] for b, c in zip(bufs, counts)], dim=0)


def merge_conjunctions(local, group=None, stream=None):
    """Gather every rank's records and sort them by (i, j, step) on the device with the library
    (cd_conjunctions_sort_device).  `local`: uint8 cuda tensor (m, 32)."""
    import torch

    from . import _check, cd_conjunctions_sort_device
    allrec = gather_records(local, group)
    if allrec.shape[0] and allrec.is_cuda:
        st = stream if stream is not None else torch.cuda.current_stream().cuda_stream
        _check(cd_conjunctions_sort_device(allrec.data_ptr(), allrec.shape[0], st))
    return allrec


def count_duplicates(recs):
    """Rows of a merged, sorted record tensor (m, 32) whose (i, j, step) equals the previous
    row's.  Under the owner rule every minimum belongs to exactly one slice, so a correct merge
    has none (the north star's dedupe step is this check)."""
    import torch
    if recs is None or recs.shape[0] < 2:
        return 0
    key = recs[:, :12].contiguous().view(torch.int32).view(-1, 3)
    return int((key[1:] == key[:-1]).all(dim=1).sum().item())


def device_records_to_tensor(out, device):
    """Copy a library-owned device result (cd_conjunctions with outputs_on_device) into a torch
    uint8 tensor (m, 32) on `device`."""
    import torch
    from cuda.bindings import runtime as rt
    m = int(out.count)
    t = torch.empty((m, REC_BYTES), dtype=torch.uint8, device=device)
    if m:
        err, = rt.cudaMemcpyAsync(t.data_ptr(), out.data, m * REC_BYTES,
                                  rt.cudaMemcpyKind.cudaMemcpyDeviceToDevice,
                                  torch.cuda.current_stream(device).cuda_stream)
        assert int(err) == 0, err
    return t


def records_to_numpy(t):
    """Host copy of a record tensor (m, 32) as a CONJ_DTYPE array (one D2H copy into pinned
    memory, then a view -- no further copies)."""
    import torch
    from . import CONJ_DTYPE
    if t.is_cuda:
        h = torch.empty(t.shape, dtype=torch.uint8, pin_memory=True)
        h.copy_(t)
        a = h.numpy()
    else:
        a = t.contiguous().numpy()
    return a.reshape(-1).view(CONJ_DTYPE)


FAR_KM = 1.0e9   # upper bound of the outermost shard (cd_options.shell_hi must be finite)


def shell_bounds(pop, S: int):
    """At most S radial bands [b_s, b_{s+1}) with b_0 = 0, b_last = FAR_KM, balanced by the
    objects' mean radius a (quantiles): each shard owns ~n/S objects.  The edges are strictly
    increasing: quantiles that coincide (many objects with one a) merge their bands, as the
    library's own band split does, so there may be fewer than S bands -- iterate over
    len(bounds) - 1."""
    a = np.sort(np.asarray(pop["a"], dtype=np.float64))
    edges = [0.0]
    for s in range(1, S):
        q = float(a[min(len(a) - 1, (len(a) * s) // S)])
        if q > edges[-1]:
            edges.append(q)
    return edges + [FAR_KM]


def screen_shard(pop, t0, t1, dt, d, bounds, s, mode="grid", v_margin=7.8, **kw):
    """Conjunctions of radial shard s (global object ids, sorted by (i, j, step)).  The member
    subset keeps the global order, so the id map is monotonic and i < j survives it."""
    from . import screen, shell_members, FIELDS
    gc = d + v_margin * dt
    lo, hi = bounds[s], bounds[s + 1]
    idx = shell_members(pop, lo, hi, gc)
    sub = {k: np.ascontiguousarray(np.asarray(pop[k])[idx]) for k in FIELDS}
    if "propagator" in pop:
        sub["propagator"] = pop["propagator"]
    res = screen(sub, t0, t1, dt, d, mode=mode, v_margin=v_margin, shell=(lo, hi), **kw)
    res["i"] = idx[res["i"]]
    res["j"] = idx[res["j"]]
    return res, len(idx)


def candidates_shard(pop, t0, t1, dt, d, bounds, s, v_margin=7.8, **kw):
    """The level-1 candidate set of radial shard s (global ids)."""
    from . import candidates, shell_members, FIELDS
    gc = d + v_margin * dt
    lo, hi = bounds[s], bounds[s + 1]
    idx = shell_members(pop, lo, hi, gc)
    sub = {k: np.ascontiguousarray(np.asarray(pop[k])[idx]) for k in FIELDS}
    if "propagator" in pop:
        sub["propagator"] = pop["propagator"]
    res = candidates(sub, t0, t1, dt, d, v_margin=v_margin, shell=(lo, hi), **kw)
    res["i"] = idx[res["i"]]
    res["j"] = idx[res["j"]]
    return res
