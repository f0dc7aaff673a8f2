"""Phase trace of the C3 pipeline (needs the -DCUSFFT_TRACE build, CUSFFT_LIB=libcusfft_trace.so)."""
import ctypes, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from paper_conf_ipps_wangcc16_b200 import Plan, load_library
from paper_conf_ipps_wangcc16_b200.workload import planted_signal
n, k = 2**24, 1000
L = int(sys.argv[1]) if len(sys.argv) > 1 else 16
x, S, X = planted_signal(n, k, 1)
xd = torch.from_numpy(x).cuda()
plan = Plan(n, k, L=L, seed=3)
lib = load_library()
fl = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
fr = torch.ones(64 << 20, dtype=torch.int32, device="cuda")
os.environ.get("X")
for rep in range(4):
    fl.zero_(); fr.sum()
    plan.execute(xd)
    torch.cuda.synchronize()
buf = (ctypes.c_ulonglong * 256)()
# one more run on a zeroed trace buffer
zero = (ctypes.c_ulonglong * 256)()
lib.cusfft_debug_trace(buf, 256)
t = np.array(list(buf), dtype=np.float64)
nz = {i: t[i] for i in range(256) if t[i] > 0}
t0 = min(nz.values())
for i, v in sorted(nz.items(), key=lambda kv: kv[1]):
    print(f"slot {i:3d}  +{(v - t0) / 1e3:8.2f} us")
