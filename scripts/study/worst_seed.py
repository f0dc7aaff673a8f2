"""Per-seed L1 at C3 for given L (oracle); prints the worst seeds and why."""
import json, sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import numpy as np
import oracle as O
from paper_conf_ipps_wangcc16_b200.workload import planted_signal
n, k, L, s0, ns = 2**24, 1000, int(sys.argv[1]), int(sys.argv[2]), int(sys.argv[3])
B = O.default_B(n, k)
p = O.make_params(n, k, B=B, L=L, seed=1)
g = O.filter_taps(p); G = O.filter_response(g, n, n // B)
for s in range(ns):
    x, S, X = planted_signal(n, k, s0 + s)
    p.seed = 100 + s
    r = O.sfft(x, p, taps=g, Ghat=G)
    l1 = O.l1_error(r.locs, r.vals, S, X, k)
    got = dict(zip(r.locs.tolist(), r.vals.tolist())); tru = dict(zip(S.tolist(), X.tolist()))
    errs = sorted(((abs(got.get(f, 0) - tru[f]), f) for f in tru), reverse=True)[:2]
    print(json.dumps({"L": L, "seed": s0 + s, "plan_seed": 100 + s, "l1": l1, "exact": set(r.locs.tolist()) == set(S.tolist()),
                      "worst": [(e, f, f % (n // B)) for e, f in errs]}), flush=True)
