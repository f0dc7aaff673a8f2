"""Oracle study at C3 (n=2^24, k=1000): a smaller bucket count B = 8192
(Bcst = 1/2, half the taps per loop) -- does it keep exact recovery and
L1 <= 1e-6?  JSON lines; CPU only (oracle).  Usage: b_study.py B delta seed0 nseeds"""
import json, sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import numpy as np
import oracle as O
from paper_conf_ipps_wangcc16_b200.workload import planted_signal
n, k = 2 ** 24, 1000
B, delta, s0, ns = int(sys.argv[1]), float(sys.argv[2]), int(sys.argv[3]), int(sys.argv[4])
p = O.make_params(n, k, B=B, L=16, tolerance=delta, seed=7)
g = O.filter_taps(p); G = O.filter_response(g, n, n // B)
for s in range(s0, s0 + ns):
    x, S, X = planted_signal(n, k, 1000 + s)
    p.seed = 7 + s
    r = O.sfft(x, p, taps=g, Ghat=G)
    ok = set(r.locs.tolist()) == set(S.tolist())
    print(json.dumps({"B": B, "delta": delta, "seed": s, "w": len(g), "exact": ok,
                      "l1": O.l1_error(r.locs, r.vals, S, X, k), "hits": len(r.hits)}), flush=True)
