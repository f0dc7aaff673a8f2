"""One transform per configuration for compute-sanitizer runs (no CUDA graph:
CUSFFT_NO_GRAPH=1 is set by the caller).  Usage: sanitize_run.py n k [B] [extra...]"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_wangcc16_b200 import Plan
from paper_conf_ipps_wangcc16_b200.workload import planted_signal
n, k = int(sys.argv[1]), int(sys.argv[2])
B = int(sys.argv[3]) if len(sys.argv) > 3 and sys.argv[3] != "0" else None
kw = {}
for a in sys.argv[4:]:
    key, val = a.split("=")
    kw[key] = float(val) if "." in val or "e" in val else int(val)
L = kw.pop("L", 16)
zero = kw.pop("zero", 0)  # zero=1: x = 0 (every key ties: the crowded-cutoff fallbacks)
x, S, X = planted_signal(n, k, 3)
if zero:
    x[:] = 0
plan = Plan(n, k, B=B, L=L, seed=5, **kw)
locs, vals = plan.execute(torch.from_numpy(x).cuda())
torch.cuda.synchronize()
ok = zero or set(locs.cpu().tolist()) == set(S.tolist())
print("status", plan.status(), "exact", ok, "staged", plan.info()["staged"], "tail", plan.info()["tail"])
