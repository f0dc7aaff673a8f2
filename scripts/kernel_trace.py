"""Per-kernel device durations of the bench's C3 step from a CUPTI activity
trace (torch.profiler; no kernel replay, no serialisation), the same
conditions as bench.py's timed loop: L2 flushed (and, with --cold, the
persisting lines reset) before every execution, the plan's CUDA graph
launched on the current stream.  Writes a JSON summary (and optionally the
Chrome trace) so bench.py's event-timed kernel numbers can be checked
against it.  Usage: kernel_trace.py OUT.json [--config C3] [--reps 20] [--cold] [--chrome OUT.trace.json] [--plan-kw JSON]
"""
import argparse
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import bench  # noqa: E402
from paper_conf_ipps_wangcc16_b200 import Plan, default_B  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("out")
ap.add_argument("--config", default="C3")
ap.add_argument("--reps", type=int, default=20)
ap.add_argument("--cold", action="store_true")
ap.add_argument("--chrome", default="")
ap.add_argument("--plan-kw", default="{}", help="extra plan parameters as JSON, e.g. '{\"shard_mode\": 2}'")
args = ap.parse_args()

n, k, L = bench.CONFIGS[args.config][:3]
B = default_B(n, k)
x_np, S, X = bench.make_signal(n, k, 1)
dev = torch.device("cuda", 0)
x = torch.from_numpy(x_np).to(dev)
plan = Plan(n, k, B=B, L=L, seed=3, device=0, **{**bench.plan_params(args.config), **json.loads(args.plan_kw)})
locs = torch.empty(k, dtype=torch.int64, device=dev)
vals = torch.empty(k, dtype=torch.complex128, device=dev)
flush = bench.L2Flush(dev)
for _ in range(5):
    flush(cold=args.cold)
    plan.execute(x, locs, vals)
torch.cuda.synchronize()
acts = [torch.profiler.ProfilerActivity.CUDA, torch.profiler.ProfilerActivity.CPU]
with torch.profiler.profile(activities=acts) as prof:
    for _ in range(args.reps):
        flush(cold=args.cold)
        plan.execute(x, locs, vals)
    torch.cuda.synchronize()
if args.chrome:
    prof.export_chrome_trace(args.chrome)
# kernel events in launch order
evs = [e for e in prof.events() if e.device_type == torch.autograd.DeviceType.CUDA]
per = {}
mine = [e for e in evs if "cusfft::" in e.name]
for e in mine:
    short = e.name.split("(")[0].replace("void ", "").replace("cusfft::", "")
    per.setdefault(short, []).append(e.device_time if hasattr(e, "device_time") else e.cuda_time)
# execution spans: first cusfft kernel start to last cusfft kernel end per execution
starts = sorted((e.time_range.start, e.time_range.end, e.name) for e in mine)
spans, cur = [], None
for s0, e0, nm in starts:
    if "k_stage_packed" in nm or (cur is None):
        if cur:
            spans.append(cur[1] - cur[0])
        cur = [s0, e0]
    else:
        cur[1] = max(cur[1], e0)
if cur:
    spans.append(cur[1] - cur[0])
out = {"config": args.config, "plan_kw": json.loads(args.plan_kw), "reps": args.reps, "cold": args.cold,
       "how": "torch.profiler (CUPTI kernel activity), L2 flushed before every execution"
              + (" + cudaCtxResetPersistingL2Cache" if args.cold else ""),
       "kernels_us": {k_: {"launches": len(v), "mean": statistics.mean(v), "median": statistics.median(v),
                           "min": min(v), "max": max(v)} for k_, v in sorted(per.items())},
       "execution_span_us": {"mean": statistics.mean(spans), "median": statistics.median(spans)} if spans else None}
with open(args.out, "w") as f:
    json.dump(out, f, indent=1)
print(json.dumps(out, indent=1))
