"""Probe: DRAM bytes / time of the fold vs cudaLimitMaxL2FetchGranularity."""
import ctypes, sys, os, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_wangcc16_b200 import Plan
from paper_conf_ipps_wangcc16_b200.workload import planted_signal
gran = int(sys.argv[1]) if len(sys.argv) > 1 else -1
torch.cuda.init()
rt = ctypes.CDLL("libcudart.so.12")
val = ctypes.c_size_t()
rt.cudaDeviceGetLimit(ctypes.byref(val), 0x05)
before = val.value
if gran >= 0:
    print("set rc", rt.cudaDeviceSetLimit(0x05, ctypes.c_size_t(gran)))
rt.cudaDeviceGetLimit(ctypes.byref(val), 0x05)
n, k = 2**24, 1000
x, S, X = planted_signal(n, k, 1)
xd = torch.from_numpy(x).cuda()
plan = Plan(n, k, L=16, seed=3)
plan.set_timing(True)
fl = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
ts = []
for i in range(12):
    fl.sum()  # read-flush (clean L2)
    plan.execute(xd)
    ts.append(plan.stage_times()["fold"])
print(json.dumps({"gran_before": before, "gran_now": val.value, "fold_ms": ts[2:]}))
