"""Run the C3 transform a few times (target for ncu captures)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import bench
from paper_conf_ipps_wangcc16_b200 import Plan
from paper_conf_ipps_wangcc16_b200.workload import planted_signal
cfg = sys.argv[1] if len(sys.argv) > 1 else "C3"
n, k = {"C1": (2**14, 8), "C2": (2**20, 100), "C3": (2**24, 1000), "C4": (2**27, 1000)}[cfg]
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 4
LL = int(sys.argv[3]) if len(sys.argv) > 3 else 16
x, S, X = planted_signal(n, k, 1)
xd = torch.from_numpy(x).cuda()
plan = Plan(n, k, L=LL, seed=3, **bench.plan_params(cfg))  # the bench's filter parameters
fl = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
fr = torch.ones(64 << 20, dtype=torch.int32, device="cuda")
for _ in range(reps):
    fl.zero_(); fr.sum()  # L2 flush as in bench.py: x cold, nothing of the last execution resident
    locs, vals = plan.execute(xd)
torch.cuda.synchronize()
print("ok", plan.status(), set(locs.cpu().tolist()) == set(S.tolist()))
