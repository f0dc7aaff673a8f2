"""Oracle parameter study, many seeds, candidate defaults at C3.  CPU only."""
import json, sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import numpy as np
import oracle as O
from paper_conf_ipps_wangcc16_b200.workload import planted_signal
n, k = int(sys.argv[1]), int(sys.argv[2])
seeds = int(sys.argv[3])
cands = [(float(a), int(b), int(c), int(d)) for a, b, c, d in (t.split(",") for t in sys.argv[4].split(";"))] if len(sys.argv) > 4 else [(1e-8, 16, 8, 5), (1e-8, 12, 8, 5), (1e-8, 10, 6, 4), (1e-8, 10, 8, 5), (1e-7, 10, 6, 4), (1e-7, 12, 8, 5), (1e-8, 9, 6, 4)]
B = O.default_B(n, k)
sigs = [planted_signal(n, k, int(os.environ.get("SEED0", "5000")) + s) for s in range(seeds)]
for delta, L, Lloc, T in cands:
    p = O.make_params(n, k, B=B, L=L, loc_loops=Lloc, vote_threshold=T, tolerance=delta, seed=1)
    g = O.filter_taps(p); G = O.filter_response(g, n, n // B)
    ok, l1s, hits = 0, [], []
    for s, (x, S, X) in enumerate(sigs):
        p.seed = 100 + s
        r = O.sfft(x, p, taps=g, Ghat=G)
        ok += set(r.locs.tolist()) == set(S.tolist())
        l1s.append(O.l1_error(r.locs, r.vals, S, X, k)); hits.append(len(r.hits))
    print(json.dumps({"n": n, "k": k, "B": B, "delta": delta, "L": L, "Lloc": Lloc, "T": T, "w": len(g),
                      "Lw": L * len(g), "exact": ok, "seeds": seeds, "l1_max": max(l1s),
                      "l1_median": float(np.median(l1s)), "hits_mean": float(np.mean(hits))}), flush=True)
