"""Oracle parameter study at C3 (n=2^24, k=1000): which (L, L_loc, T, delta)
keep exact recovery and L1 <= 1e-6?  Writes JSON lines.  CPU only (oracle)."""
import json, sys, os, time, itertools
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import numpy as np
import oracle as O
from paper_conf_ipps_wangcc16_b200.workload import planted_signal
n, k = int(sys.argv[1]) if len(sys.argv) > 1 else 2**24, int(sys.argv[2]) if len(sys.argv) > 2 else 1000
seeds = int(sys.argv[3]) if len(sys.argv) > 3 else 4
B = O.default_B(n, k)
sigs = [planted_signal(n, k, 1000 + s) for s in range(seeds)]
grid = []
for delta in (1e-8, 1e-6, 1e-5):
    for L, Lloc in ((16, 8), (12, 8), (12, 6), (10, 6), (8, 8), (8, 6), (16, 6)):
        if Lloc > L: continue
        grid.append((delta, L, Lloc))
for delta, L, Lloc in grid:
    T = Lloc // 2 + 1
    p = O.make_params(n, k, B=B, L=L, loc_loops=Lloc, vote_threshold=T, tolerance=delta, seed=7)
    g = O.filter_taps(p); G = O.filter_response(g, n, n // B)
    res = []
    for s, (x, S, X) in enumerate(sigs):
        p.seed = 7 + s
        r = O.sfft(x, p, taps=g, Ghat=G)
        ok = set(r.locs.tolist()) == set(S.tolist())
        res.append((ok, O.l1_error(r.locs, r.vals, S, X, k), len(r.hits)))
    print(json.dumps({"n": n, "k": k, "B": B, "delta": delta, "L": L, "Lloc": Lloc, "T": T, "w": len(g),
                      "Lw": L * len(g), "exact": sum(o for o, _, _ in res), "seeds": seeds,
                      "l1_max": max(e for _, e, _ in res), "hits_mean": float(np.mean([h for _, _, h in res]))}), flush=True)
