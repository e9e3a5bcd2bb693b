#!/usr/bin/env python
"""Write the oracle's full-window results for BASELINE configs 2 and 3 to tests/golden/ (the
full-window parity tests, tests/test_gpu_fullwindow.py, compare the CUDA path against them).

TEST INFRASTRUCTURE: this script calls only oracle/ (and the seeded generator tools/popgen.py);
no value in the files comes from the CUDA path.  A full 24 h oracle screen of config 2 at 1 s
takes ~8 min on 8 host cores, which is why it is stored rather than recomputed in every GPU run.

Per (config, variant) one compressed .npz:
  conj          the oracle's conjunction rows (O3 grid / O4 hybrid), CONJ_DTYPE, sorted
  steps         number of sampling steps K of the window
  cand_count    per-step size of the candidate set (grid: K at dt; hybrid: the coarse set at dt_h)
  cand_digest   per-step BLAKE2b-64 of the step's sorted (i, j) pairs (uint32 little endian)
  meta          json: config, variant, t0, t1, dt, d, g_c, seed, numpy version, oracle threads

    python tools/make_golden.py [--only cfg2_grid,cfg2_hybrid,cfg3_hybrid]
"""
from __future__ import annotations

import argparse
import hashlib
import json
import sys
import time
from pathlib import Path

import numpy as np

ROOT = Path(__file__).resolve().parent.parent
sys.path.insert(0, str(ROOT))

GOLDEN = ROOT / "tests" / "golden"
JOBS = {"cfg2_grid": (2, "grid"), "cfg2_hybrid": (2, "hybrid"), "cfg3_hybrid": (3, "hybrid")}


def _sorted_by_ij(c):
    if len(c) < 2:
        return True
    i, j = c["i"].astype(np.int64), c["j"].astype(np.int64)
    di = np.diff(i)
    return bool(np.all((di > 0) | ((di == 0) & (np.diff(j) >= 0))))


def step_digests(cands, K):
    """(count, digest) per step of a candidate array (any order; an array already sorted by
    (i, j) -- both sides' native order -- takes one stable sort by step)."""
    if _sorted_by_ij(cands):
        order = np.argsort(cands["step"], kind="stable")
    else:
        order = np.lexsort((cands["j"], cands["i"], cands["step"]))
    c = cands[order]
    bounds = np.searchsorted(c["step"], np.arange(K + 1))
    count = np.diff(bounds).astype(np.int64)
    dig = np.zeros(K, dtype=np.uint64)
    ij = np.ascontiguousarray(np.stack([c["i"], c["j"]], 1).astype("<u4"))
    for k in np.nonzero(count)[0]:
        h = hashlib.blake2b(ij[bounds[k]:bounds[k + 1]].tobytes(), digest_size=8)
        dig[k] = np.frombuffer(h.digest(), dtype="<u8")[0]
    return count, dig


def make(name):
    import oracle
    from tools import popgen
    cfgno, variant = JOBS[name]
    pop, cfg, _ = popgen.make_config(cfgno)
    dt = cfg.dt_grid if variant == "grid" else cfg.dt_hybrid
    gc = oracle.cell_size(cfg.d, dt)
    K = oracle.num_steps(cfg.t0, cfg.t1, dt)
    t = time.time()
    cand = oracle.candidates_grid(pop, cfg.t0, cfg.t1, dt, gc)
    if variant == "grid":
        conj = oracle.conjunctions(pop, cfg.t0, cfg.t1, dt, cfg.d, gc, cand)
        counts = {}
    else:
        conj, counts = oracle.hybrid(pop, cfg.t0, cfg.t1, dt, cfg.d)
    sec = time.time() - t
    cnt, dig = step_digests(cand, K)
    meta = {"config": cfgno, "variant": variant, "t0": cfg.t0, "t1": cfg.t1, "dt": dt, "d": cfg.d,
            "gc": gc, "seed": cfg.seed, "n": int(len(pop["a"])), "numpy": np.__version__,
            "oracle_threads": oracle.num_threads(), "oracle_seconds": round(sec, 1),
            "candidates": int(len(cand)), "conjunctions": int(len(conj)), "filter_counts": counts,
            "script": "tools/make_golden.py (oracle/ only)"}
    out = GOLDEN / f"fullwindow_{name}.npz"
    np.savez_compressed(out, conj=conj, steps=np.int64(K), cand_count=cnt, cand_digest=dig,
                        meta=np.array(json.dumps(meta)))
    print(json.dumps(meta), flush=True)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--only", default=",".join(JOBS))
    args = ap.parse_args()
    for name in args.only.split(","):
        make(name)


if __name__ == "__main__":
    main()
