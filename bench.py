#!/usr/bin/env python
"""Benchmark of the B200-native screening path (BASELINE.json metric: object-steps/s and wall
time for the 1M-object x 24 h screen at 1/2/4/8 B200).

Workload: BASELINE.json config 4 (1,000,000 objects, d = 2 km, 24 h window, grid variant at
dt = 1 s -> 86,401 sampling steps; the hybrid variant at dt = 9 s is reported alongside).
A bench "step" is one pass of the whole hot path (precompute, propagate + insert, neighbour scan,
refinement, finalize) over one time slice of that window: the timed steps x N ranks slices
partition the 24 h window exactly (owner rule, no overlap), so the timed region screens the
whole day once at every N (strong scaling) and ``value`` = 1e6 x 86,401 / max-over-ranks time.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time
from pathlib import Path

import numpy as np

ROOT = Path(__file__).resolve().parent
sys.path.insert(0, str(ROOT))

PROFILE_EVERY = 16   # time every 16th k_step launch inside the timed region
ALG_BYTES = {"scan": 296.0}   # insert 48 + detect 248 B per object-step (k_step fuses both)
FP64_PEAK_TFLOPS = 148 * 64 * 2 * 1.965e9 / 1e12                        # 37.2 TFLOP/s


def log(*a):
    print(*a, file=sys.stderr, flush=True)


def load_peaks():
    p = ROOT / "MEASURED_PEAKS.json"
    if p.exists():
        d = json.loads(p.read_text())
        return float(d["hbm_gbs"]), "measured"
    return 6650.0, "fallback"


class ClockSampler:
    """nvidia-smi clocks + throttle reasons during the timed region (B200_PROFILING.md)."""

    def __init__(self, index):
        self.index = index
        self.rows = []
        self.proc = None

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), "--query-gpu=clocks.sm,clocks.max.sm,"
                 "clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,"
                 "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
                 "clocks_event_reasons.sw_power_cap", "--format=csv,noheader,nounits", "-lms", "200"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.rows.append([x.strip() for x in line.split(",")])

    def mark(self):
        self.i0 = len(self.rows)

    def mark_end(self):
        self.i1 = len(self.rows)

    def __exit__(self, *a):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except Exception:
                self.proc.kill()

    def summary(self):
        sm = []
        mx = None
        reasons = set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for r in self.rows[getattr(self, "i0", 0):getattr(self, "i1", None)]:
            try:
                sm.append(float(r[0]))
                mx = float(r[1])
                for nm, v in zip(names, r[3:7]):
                    if v.lower().startswith("active"):
                        reasons.add(nm)
            except Exception:
                continue
        load = [x for x in sm if x > 500] or sm
        return {"sm_mhz": float(np.median(load)) if load else None, "sm_max_mhz": mx,
                "reasons": sorted(reasons), "samples": len(sm)}


def cpu_model():
    """The host CPU (lscpu "Model name"), for the cpu_baseline record."""
    try:
        out = subprocess.run(["lscpu"], capture_output=True, text=True, timeout=10).stdout
        for line in out.splitlines():
            if line.startswith("Model name:"):
                return line.split(":", 1)[1].strip()
    except Exception:
        pass
    try:
        for line in Path("/proc/cpuinfo").read_text().splitlines():
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except Exception:
        pass
    return None


def population(args):
    from tools import popgen
    pop, cfg, _ = popgen.make_config(args.config, n=args.n)
    return pop, cfg


def cpu_oracle_sample(pop, cfg, dt, d, k0, nsteps):
    """The oracle as it stands on the host cores: candidates (CPU grid) + conjunctions for
    steps [k0, k0 + nsteps) of the window; returns (seconds, threads)."""
    import oracle
    gc = oracle.cell_size(d, dt)
    t = time.perf_counter()
    K = oracle.candidates_grid(pop, cfg.t0, cfg.t1, dt, gc, k_begin=k0, k_end=k0 + nsteps)
    oracle.conjunctions(pop, cfg.t0, cfg.t1, dt, d, gc, K)
    return time.perf_counter() - t, oracle.num_threads()


def run_reference(args):
    """--impl reference: the oracle (plain C, OpenMP) timed as it stands on the host cores, on a
    bounded sample of the same workload per step.  Rank 0 only."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    import oracle
    pop, cfg = population(args)
    n = len(pop["a"])
    dt = cfg.dt_grid if args.variant == "grid" else cfg.dt_hybrid
    threads = oracle.num_threads()
    per = max(1, min(args.ref_steps or threads, 64))
    K = oracle.num_steps(cfg.t0, cfg.t1, dt)
    total = 0.0
    for s in range(args.warmup + args.steps):
        k0 = ((s * 997) * per) % max(1, K - per)
        sec, _ = cpu_oracle_sample(pop, cfg, dt, cfg.d, k0, per)
        if s >= args.warmup:
            total += sec
    units = n * per * args.steps
    value = units / total
    line = {"impl": "reference", "metric": "object-steps/s (1M objects x 24 h screen)",
            "value": value, "unit": "object-steps/s", "n_gpus": args.gpus, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": 1e3 * total / args.steps,
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f64",
            "data": "synthetic", "config": workload_config(args, cfg, n, dt, K),
            "cpu_baseline": {"value": value, "unit": "object-steps/s", "cores": threads,
                             "kind": "oracle", "cpu_model": cpu_model(),
                             "sample": f"{per} consecutive {dt:g}-s steps of the 24 h window per "
                                       f"bench step (CPU grid + conjunctions), {n} objects"},
            "e2e": {"value": value, "unit": "object-steps/s", "h2d_bytes_per_step": 0,
                    "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


def workload_config(args, cfg, n, dt, K):
    return {"workload": f"BASELINE config {args.config}: {n} objects, d = {cfg.d:g} km, "
                        f"{(cfg.t1 - cfg.t0) / 3600:g} h window, {args.variant} variant, "
                        f"dt = {dt:g} s ({K} steps)",
            "n_objects": n, "threshold_km": cfg.d, "dt_s": dt, "window_s": cfg.t1 - cfg.t0,
            "steps_in_window": K, "variant": args.variant,
            "population": "seeded synthetic (tools/popgen.py), paper-shaped LEO-heavy mixture "
                          "+ Starlink-like shells",
            "l2": "flushed between timed steps (256 MB write); working set > L2"}


def run_ours(args):
    import torch
    import torch.distributed as dist

    import paper_conf_ipps_hellwigcmbw23_b200 as cds
    from paper_conf_ipps_hellwigcmbw23_b200 import dist as cdist

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    # the distributed data plane (NCCL process group, per-slice all-gather merge, max-over-ranks
    # timing) runs whenever there are several ranks, and also at one rank with --dist (torchrun
    # --nproc-per-node 1), so a one-GPU box exercises the same code path
    distributed = world > 1 or args.dist
    # CD_BENCH_BACKEND=gloo (testing only): several ranks sharing one GPU, to exercise the
    # multi-rank logic of this file on a one-GPU box; the product path is NCCL, one rank per GPU
    backend = os.environ.get("CD_BENCH_BACKEND", "nccl")
    if distributed:
        gpu = local if backend == "nccl" else local % max(1, torch.cuda.device_count())
        torch.cuda.set_device(gpu)
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", gpu))
        else:
            dist.init_process_group(backend)
    else:
        torch.cuda.set_device(0)
    dev = torch.device("cuda", torch.cuda.current_device())
    pop, cfg = population(args)
    n = len(pop["a"])
    dt = cfg.dt_grid if args.variant == "grid" else cfg.dt_hybrid
    mode = cds.CD_GRID if args.variant == "grid" else cds.CD_HYBRID
    K = int(np.floor((cfg.t1 - cfg.t0) / dt)) + 1
    S = args.steps * world                                   # slices of the window, timed
    dpop = {k: torch.from_numpy(v).to(dev) for k, v in pop.items()}   # inputs resident in HBM
    flush = torch.empty(64 * 1024 * 1024, dtype=torch.float32, device=dev)   # 256 MB > L2
    stream = torch.cuda.current_stream(dev)

    def barrier():
        if distributed:
            dist.barrier()

    # device scratch memory from PyTorch's caching allocator on the bench stream (cd_options.alloc)
    talloc = cds.TorchAllocator(dev.index, stream.cuda_stream) if args.torch_alloc else None

    # the cell edge the first call settles on is passed to the next calls (cd_stats.cell_factor
    # -> cd_options.cell_factor): later slices skip the density-probe round
    cell = {"grid": None}
    last_merged = {}

    def one_step(s, profile, host_inputs=False):
        q = (s * world + rank) % S
        E = cds._Elements(pop if host_inputs else dpop)
        st = cds.cd_stats()
        opt = cds.make_options(rank=q, n_ranks=S, device=dev.index, stream=stream.cuda_stream,
                               inputs_on_device=not host_inputs,
                               outputs_on_device=not host_inputs, profile_phases=profile,
                               allocator=talloc, cell_factor=cell["grid"])
        import ctypes as C
        opt.stats = C.pointer(st)
        out = cds.cd_conjunctions()
        cds._check(cds.cd_screen_ex(E.s, E.n, cfg.t0, cfg.t1, dt, cfg.d, mode, opt, out))
        try:
            if host_inputs:
                nrec = int(out.count)
                merged = nrec
            else:
                recs = cdist.device_records_to_tensor(out, dev)
                if distributed:   # the slices of all ranks, merged and sorted on every rank
                    recs = cdist.merge_conjunctions(recs, stream=stream.cuda_stream)
                    last_merged["recs"] = recs
                merged = recs.shape[0]
                nrec = int(out.count)
        finally:
            cds.cd_conjunctions_free(out)
        if st.cell_factor > 0 and cell["grid"] is None:
            cell["grid"] = float(st.cell_factor)
        return st.as_dict(), nrec, merged

    # the clock sampler starts before the warm-up so its NVML start-up does not land in the
    # timed region; only samples taken during the timed steps are summarised
    clk = ClockSampler(dev.index).__enter__()
    # warm-up (untimed)
    for w in range(args.warmup):
        one_step(w % args.steps, profile=False)
    torch.cuda.synchronize()

    # timed region: device time with CUDA events on the library's stream, max over ranks
    launches0 = cds.cd_kernel_launches()
    times, stats = [], []
    nconj = 0
    clk.mark()
    if True:
        for s in range(args.steps):
            flush.zero_()                      # L2 flush between timed steps (outside the timing)
            torch.cuda.synchronize()
            barrier()
            e0 = torch.cuda.Event(enable_timing=True)
            e1 = torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            st, nrec, merged = one_step(s, profile=PROFILE_EVERY if args.profile else 0)
            e1.record(stream)
            torch.cuda.synchronize()
            barrier()
            times.append(e0.elapsed_time(e1))
            stats.append(st)
            nconj += nrec
            if os.environ.get("BENCH_VERBOSE"):
                log(f"step {s}: {times[-1]:.1f} ms, lib {st['ms_total']:.1f} ms, cand {st['candidates']}, "
                    f"refined {st['refined']}, retries {st['retries']}, launches {st['kernel_launches']}")
    clk.mark_end()
    clk.__exit__(None, None, None)
    launches = cds.cd_kernel_launches() - launches0
    tot_ms = float(np.sum(times))
    merge_info = None
    if distributed:
        recs = last_merged.get("recs")
        dups = cdist.count_duplicates(recs) if recs is not None else 0
        merge_info = {"backend": dist.get_backend(), "ranks": world,
                      "records_last_step": int(recs.shape[0]) if recs is not None else 0,
                      "duplicates_last_step": int(dups)}
    if distributed:
        t = torch.tensor([tot_ms], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        tot_ms = float(t.item())
        c = torch.tensor([nconj], dtype=torch.int64, device=dev)
        dist.all_reduce(c)
        nconj = int(c.item())
    units = float(n) * sum(st["steps"] for st in stats) * 1.0
    if distributed:
        u = torch.tensor([units], dtype=torch.float64, device=dev)
        dist.all_reduce(u)
        units = float(u.item())
    value = units / (tot_ms / 1e3)

    # the hybrid variant (coarse grid at dt_h + filter chain) over the same window, same slicing
    hyb = None
    if args.variant == "grid" and not args.no_hybrid and cfg.dt_hybrid:
        Kh = int(np.floor((cfg.t1 - cfg.t0) / cfg.dt_hybrid)) + 1
        hms, hst = [], []
        for s in range(args.warmup + args.steps):
            q = (s * world + rank) % S
            E = cds._Elements(dpop)
            st = cds.cd_stats()
            opt = cds.make_options(rank=q, n_ranks=S, device=dev.index, stream=stream.cuda_stream,
                                   inputs_on_device=True, outputs_on_device=True, allocator=talloc,
                                   cell_factor=cell.get("hybrid"))
            import ctypes as C
            opt.stats = C.pointer(st)
            out = cds.cd_conjunctions()
            flush.zero_()
            torch.cuda.synchronize()
            barrier()
            e0 = torch.cuda.Event(enable_timing=True)
            e1 = torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            cds._check(cds.cd_screen_ex(E.s, E.n, cfg.t0, cfg.t1, cfg.dt_hybrid, cfg.d, cds.CD_HYBRID,
                                        opt, out))
            recs = cdist.device_records_to_tensor(out, dev)
            if distributed:
                recs = cdist.merge_conjunctions(recs, stream=stream.cuda_stream)
            cds.cd_conjunctions_free(out)
            if st.cell_factor > 0 and cell.get("hybrid") is None:
                cell["hybrid"] = float(st.cell_factor)
            e1.record(stream)
            torch.cuda.synchronize()
            if s >= args.warmup:
                hms.append(e0.elapsed_time(e1))
                hst.append(st.as_dict())
        htot = float(np.sum(hms))
        keys = ("candidates", "conjunctions", "hybrid_ap_rejected", "hybrid_coplanar",
                "hybrid_path_rejected", "hybrid_time_rejected", "refined", "steps")
        hsum = {k: int(sum(h[k] for h in hst)) for k in keys}
        if distributed:
            t = torch.tensor([htot], dtype=torch.float64, device=dev)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            htot = float(t.item())
            c = torch.tensor([hsum[k] for k in keys], dtype=torch.int64, device=dev)
            dist.all_reduce(c)   # every rank's slices: the whole window
            hsum = dict(zip(keys, (int(x) for x in c.tolist())))
        hunits = float(n) * hsum["steps"]
        hyb = {"variant": "hybrid", "dt_s": cfg.dt_hybrid, "steps_in_window": Kh,
               "value": hunits / (htot / 1e3), "unit": "object-steps/s (coarse steps)",
               "wall_s_window": htot / 1e3,
               "coarse_candidates": hsum["candidates"], "conjunctions": hsum["conjunctions"],
               "filter": {k: hsum[k] for k in ("hybrid_ap_rejected", "hybrid_coplanar",
                                               "hybrid_path_rejected", "hybrid_time_rejected",
                                               "refined")}}

    # end to end through the public API with HOST buffers: pinned host inputs (H2D inside the
    # call), results back in host memory.  One rank: cd_screen with host results.  Distributed:
    # each rank's slice stays on the device for the NCCL merge (all-gather + device sort), and
    # the merged, sorted result is copied to the host (D2H inside the timed region).
    e2e_ms = []
    pin = {k: torch.from_numpy(v).pin_memory() for k, v in pop.items()}
    pin_np = {k: v.numpy() for k, v in pin.items()}
    d2h = 0
    for s in range(args.e2e_steps if args.e2e_steps is not None else args.steps):
        flush.zero_()
        torch.cuda.synchronize()
        barrier()
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        q = (s * world + rank) % S
        if distributed:
            E = cds._Elements(pin_np)
            opt = cds.make_options(rank=q, n_ranks=S, device=dev.index, stream=stream.cuda_stream,
                                   outputs_on_device=True, allocator=talloc, cell_factor=cell["grid"])
            out = cds.cd_conjunctions()
            cds._check(cds.cd_screen_ex(E.s, E.n, cfg.t0, cfg.t1, dt, cfg.d, mode, opt, out))
            recs = cdist.merge_conjunctions(cdist.device_records_to_tensor(out, dev),
                                            stream=stream.cuda_stream)
            cds.cd_conjunctions_free(out)
            host = cdist.records_to_numpy(recs)
            d2h += host.nbytes
        else:
            recs = cds.screen(pin_np, cfg.t0, cfg.t1, dt, cfg.d, mode=args.variant, rank=q, n_ranks=S,
                              device=dev.index, stream=stream.cuda_stream, allocator=talloc,
                              cell_factor=cell["grid"])
            d2h += recs.nbytes
        e1.record(stream)
        torch.cuda.synchronize()
        e2e_ms.append(e0.elapsed_time(e1))
    ne2e = len(e2e_ms)
    e2e_tot = max(float(np.sum(e2e_ms)), 1e-9)
    if distributed:
        t = torch.tensor([e2e_tot], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        e2e_tot = float(t.item())
    e2e_units = float(n) * (K / S) * ne2e * world
    e2e = {"value": e2e_units / (e2e_tot / 1e3), "unit": "object-steps/s",
           "h2d_bytes_per_step": 48 * n, "d2h_bytes_per_step": int(d2h / max(1, ne2e)),
           "steps": ne2e} if ne2e else None

    if rank != 0:
        if distributed:
            dist.destroy_process_group()
        return 0

    # roofline of the dominant kernel (live CUDA-event phase times inside the timed region)
    hbm_peak, peak_kind = load_peaks()
    roof = None
    if args.profile:
        # k_step (fused build + scan) runs as the "propagate" phase (first, build-only launch of
        # each round) and the "scan" phase (all other launches); its algorithmic bytes are
        # SURVEY 8(d)'s 296 B per object-step (insert 48 + detect 248)
        # the step loop of every round is one event span (the launches overlap under
        # programmatic dependent launch): average launch = span time / launches in the spans
        ms_smp = sum(s_["ms_scan"] + s_["ms_propagate"] for s_ in stats)
        nl_smp = sum(s_["launches_scan"] + s_["launches_propagate"] for s_ in stats)
        nl = sum(s_["step_launches"] for s_ in stats)
        avg_s = ms_smp / 1e3 / max(1, nl_smp)
        ms_step = 1e3 * avg_s * nl                         # estimated total k_step time
        objsteps = sum(s_["object_steps"] for s_ in stats)
        tot = max(1e-9, tot_ms)
        alg = ALG_BYTES["scan"] * objsteps
        achieved = alg / max(1, nl) / avg_s / 1e9
        roof = {"kernel": "k_step (fused propagate + insert + neighbour scan)",
                "bound": "hbm", "achieved": achieved, "peak": hbm_peak, "unit": "GB/s",
                "frac": achieved / hbm_peak, "traffic": traffic_from_profiles("k_step"),
                "peak_source": peak_kind, "alg_bytes_per_object_step": ALG_BYTES["scan"],
                "alg_bytes_per_launch": alg / max(1, nl), "avg_launch_ms": 1e3 * avg_s,
                "launches": nl,
                "launches_timed": nl_smp,
                "share_of_step_time": ms_step / tot}

    cpu = None
    if world == 1 and not args.no_cpu_baseline:
        k0 = 43200
        per = args.cpu_steps
        sec, threads = cpu_oracle_sample(pop, cfg, dt, cfg.d, k0, per)
        cpu = {"value": n * per / sec, "unit": "object-steps/s", "cores": threads, "kind": "oracle",
               "cpu_model": cpu_model(),
               "sample": f"steps [{k0}, {k0 + per}) of the same 24 h window ({per} x {n} "
                         f"object-steps: CPU grid candidates + conjunctions), {sec:.1f} s"}

    line = {"metric": "object-steps/s (1M objects x 24 h screen)", "value": value,
            "unit": "object-steps/s", "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": tot_ms / args.steps, "higher_is_better": True, "scaling": "strong",
            "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": dict(workload_config(args, cfg, n, dt, K),
                           slices=S, wall_s_window=tot_ms / 1e3 * (S / (args.steps * world)),
                           device_memory="PyTorch caching allocator (cd_options.alloc)" if args.torch_alloc
                           else "library stream-ordered pool",
                           conjunctions=nconj, parallelism=f"time-slice x{world}"),
            "step_ms": {"min": float(np.min(times)), "median": float(np.median(times)),
                        "max": float(np.max(times))},
            "clocks": clk.summary(), "e2e": e2e, "gpu_launches": launches,
            "roofline": roof, "cpu_baseline": cpu, "hybrid": hyb, "merge": merge_info}
    print(json.dumps(line), flush=True)
    if distributed:
        dist.destroy_process_group()
    return 0


def traffic_from_profiles(phase):
    """dram bytes per launch of the dominant kernel from the committed ncu summary, or None."""
    p = ROOT / "profiles" / "ncu_summary.json"
    if not p.exists():
        return None
    try:
        d = json.loads(p.read_text())
        return d.get(phase, {}).get("dram_bytes_per_launch")
    except Exception:
        return None


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=24)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--variant", default="grid", choices=["grid", "hybrid"])
    ap.add_argument("--config", type=int, default=4)
    ap.add_argument("--n", type=int, default=None, help="override object count (testing)")
    ap.add_argument("--no-profile", dest="profile", action="store_false")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-hybrid", action="store_true")
    ap.add_argument("--cpu-steps", type=int, default=128)
    ap.add_argument("--ref-steps", type=int, default=None)
    ap.add_argument("--e2e-steps", type=int, default=None)
    ap.add_argument("--dist", action="store_true",
                    help="NCCL process group + merge even at one rank (torchrun --nproc-per-node 1)")
    ap.add_argument("--no-torch-alloc", dest="torch_alloc", action="store_false",
                    help="library's own stream-ordered pool instead of PyTorch's caching allocator")
    args = ap.parse_args()
    if args.warmup < 3:
        log("note: --warmup < 3 violates the timing rules; using 3")
        args.warmup = 3
    if args.impl == "reference":
        return run_reference(args)
    return run_ours(args)


if __name__ == "__main__":
    sys.exit(main())
