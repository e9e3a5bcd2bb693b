import sys, time, ctypes as C
sys.path.insert(0, '/root/repo')
import torch, numpy as np
import paper_conf_ipps_hellwigcmbw23_b200 as cds
from paper_conf_ipps_hellwigcmbw23_b200 import dist as cdist
from tools import popgen
pop, cfg, _ = popgen.make_config(4)
dev = torch.device("cuda", 0)
dpop = {k: torch.from_numpy(v).to(dev) for k, v in pop.items()}
stream = torch.cuda.current_stream(dev)
print("stream handle", stream.cuda_stream)
flush = torch.empty(64 * 1024 * 1024, dtype=torch.float32, device=dev)
for variant in ("full", "prof16", "prof1", "flush", "flush_prof16"):
    for s in range(3):
        E = cds._Elements(dpop)
        st = cds.cd_stats()
        opt = cds.make_options(rank=s, n_ranks=24, device=0, stream=stream.cuda_stream, inputs_on_device=True,
                               outputs_on_device=True, profile_phases=16 if "prof16" in variant else (1 if variant == "prof1" else 0))
        opt.stats = C.pointer(st)
        out = cds.cd_conjunctions()
        if "flush" in variant:
            flush.zero_()
        torch.cuda.synchronize()
        e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        t = time.perf_counter(); e0.record(stream)
        cds._check(cds.cd_screen_ex(E.s, E.n, cfg.t0, cfg.t1, 1.0, cfg.d, 0, opt, out))
        t1 = time.perf_counter()
        recs = cdist.device_records_to_tensor(out, dev)
        t2 = time.perf_counter()
        cds.cd_conjunctions_free(out)
        t3 = time.perf_counter()
        e1.record(stream); torch.cuda.synchronize(); t4 = time.perf_counter()
        print(variant, f"events {e0.elapsed_time(e1):.1f} ms, lib ms_total {st.ms_total:.1f}, host call {1e3*(t1-t):.1f} copy {1e3*(t2-t1):.1f} free {1e3*(t3-t2):.1f} tail {1e3*(t4-t3):.1f}")
