"""Fold-stage time with phase 1 skipped (staging warm from the previous call) vs normal."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_wangcc16_b200 import Plan
from paper_conf_ipps_wangcc16_b200.workload import planted_signal
n, k = 2**24, 1000
x, S, X = planted_signal(n, k, 1)
xd = torch.from_numpy(x).cuda()
fl = torch.empty(256 << 20, dtype=torch.uint8, device="cuda"); fr = torch.ones(64 << 20, dtype=torch.int32, device="cuda")
def t(plan, flush, reps=20):
    ts = []
    for _ in range(reps):
        if flush: fl.zero_(); fr.sum()
        a = torch.cuda.Event(enable_timing=True); b = torch.cuda.Event(enable_timing=True)
        a.record(); plan.execute(xd); b.record(); torch.cuda.synchronize(); ts.append(a.elapsed_time(b))
    return sum(ts[3:]) / len(ts[3:]) * 1e3
base = Plan(n, k, L=16, seed=3, tolerance=1e-7); base.set_stage_limit(1)
print("fold stage, flushed:", t(base, True), "us;  warm (no flush):", t(base, False), "us")
os.environ["CUSFFT_SKIP_STAGE"] = "1"
skip = Plan(n, k, L=16, seed=3, tolerance=1e-7); skip.set_stage_limit(1)
base.execute(xd); torch.cuda.synchronize()
print("phase 2 only, staging warm:", t(skip, False), "us; phase 2 only after flush:", t(skip, True), "us")
