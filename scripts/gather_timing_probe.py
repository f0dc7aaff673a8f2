"""Phase-1 (k_stage_packed) duration at C3 measured three ways, bench conditions (L2 flushed
before each execution, staging warm): CUDA events around a direct launch (timing mode 1),
event-record nodes inside the graph (mode 2), and the CUPTI kernel duration (torch.profiler)."""
import os, sys, statistics
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import bench
from paper_conf_ipps_wangcc16_b200 import Plan, default_B
n, k, L = bench.CONFIGS["C3"][:3]
B = default_B(n, k)
x_np, S, X = bench.make_signal(n, k, 1)
dev = torch.device("cuda", 0)
x = torch.from_numpy(x_np).to(dev)
plan = Plan(n, k, B=B, L=L, seed=3, device=0, **bench.plan_params("C3", B))
locs = torch.empty(k, dtype=torch.int64, device=dev)
vals = torch.empty(k, dtype=torch.complex128, device=dev)
flush = bench.L2Flush(dev)
for mode in (1, 2, 1, 2):
    plan.set_timing(mode)
    g = []
    for _ in range(23):
        flush()
        plan.execute(x, locs, vals)
        g.append(plan.stage_times()["gather"])
    plan.set_timing(0)
    print(f"mode {mode}: gather {1e3 * statistics.mean(g[3:]):.2f} us (median {1e3 * statistics.median(g[3:]):.2f})")
