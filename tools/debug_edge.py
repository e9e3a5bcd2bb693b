"""Debug helper: one-sided hybrid rows of the short-window edge test, with D(t) around the TCA."""
import numpy as np
import oracle
from tools import popgen
import paper_conf_ipps_hellwigcmbw23_b200 as cds

pop, cfg, _ = popgen.make_config(1)
dt = 9.0
for t0, t1 in ((300.0, 300.0), (300.0, 300.0 + 0.4 * dt)):
    g = cds.screen(pop, t0, t1, dt, cfg.d, mode="hybrid")
    o, _ = oracle.hybrid(pop, t0, t1, dt, cfg.d)
    G = {(int(r["i"]), int(r["j"]), int(r["step"])): r for r in g}
    O = {(int(r["i"]), int(r["j"]), int(r["step"])): r for r in o}
    print("window", t0, t1, "gpu", len(G), "oracle", len(O))
    for k in sorted(set(G) ^ set(O)):
        r = G.get(k, O.get(k))
        side = "gpu" if k in G else "oracle"
        tca = float(r["tca"])
        ts = np.array([tca - 1e-3, tca - 1e-5, tca, tca + 1e-5, tca + 1e-3])
        D, _ = oracle.pair_distance(pop, k[0], k[1], ts)
        print(side, k, "tca", repr(tca), "pca", float(r["pca"]), "flags", int(r["flags"]), "D", D.tolist())
