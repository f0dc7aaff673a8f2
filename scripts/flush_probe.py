"""Where do phase 1's DRAM writes come from?  Run the C3 transform after one of
three L2 flushes (for an ncu capture of k_stage_packed):
  wr: 256 MiB write + 256 MiB read (bench.py's flush)
  rd: two 256 MiB reads of different buffers (no dirty lines left by the flush)
  none: no flush (previous execution's lines resident)
Usage: flush_probe.py MODE REPS"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_wangcc16_b200 import Plan
from paper_conf_ipps_wangcc16_b200.workload import planted_signal
mode = sys.argv[1]
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 3
n, k = 2 ** 24, 1000
x, S, X = planted_signal(n, k, 1)
xd = torch.from_numpy(x).cuda()
plan = Plan(n, k, L=16, seed=3, tolerance=1e-7)
fl = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
fr = torch.ones(64 << 20, dtype=torch.int32, device="cuda")
fr2 = torch.ones(64 << 20, dtype=torch.int32, device="cuda")
for _ in range(reps):
    if mode == "wr":
        fl.zero_(); fr.sum()
    elif mode == "rd":
        fr.sum(); fr2.sum()
    locs, vals = plan.execute(xd)
torch.cuda.synchronize()
print("ok", plan.status(), set(locs.cpu().tolist()) == set(S.tolist()))
