"""Per-rank time model of loop-sharded C3 (or C4: SCALE_CONFIG=C4) on G = 1, 2, 4, 8 GPUs, with the
per-rank compute MEASURED on one B200, for both loop-sharded
designs: one all-gather of the per-loop records (shard_mode 0) and two
all-gathers, candidates then per-loop estimates (shard_mode 2), and signal sharding
(shard_mode 1: rank 0 folds only x[0, n/G), one all-reduce of the spectra, modelled as a ring).

For each G the script builds rank 0's plan of a G-rank loop-sharded run
(cusfft_plan_dist without a communicator), and times on the bench's terms
(L2 flushed before every step, CUDA events, graphs):
  local  = cusfft_execute_local  (Steps 1-4 of this rank's L/G loops, one serial chain)
  finish = (local + cusfft_execute_finish) - local (vote + estimation + output over all L loops)
  mode 2: mid = (local + cusfft_execute_mid) - local (vote, hit sort, this rank's estimates),
          finish = (local + mid + finish) - (local + mid) (medians + output)
The exchange buffer is filled with the records of a world = 1 plan of the same
draws (the all-gather's result), so finish does the real work.  The
all-gather itself cannot be timed on one GPU: it is modelled as
alpha + (G-1)/G * bytes / bw with the bytes of the plan and stated alpha / bw.
Usage: scale_model.py OUT.json
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import bench  # noqa: E402
from paper_conf_ipps_wangcc16_b200 import Plan, default_B  # noqa: E402
from paper_conf_ipps_wangcc16_b200.dist import slot_of_loop  # noqa: E402

ALPHA_US = 10.0   # assumed NCCL all-gather latency inside one NVSwitch domain (small messages)
BW_GBS = 700.0    # assumed achieved all-gather bus bandwidth per GPU (NVLink 5, 900 GB/s per direction)

CFG = os.environ.get("SCALE_CONFIG", "C3")
n, k, L = bench.CONFIGS[CFG][:3]
B = default_B(n, k)
prm = bench.plan_params(CFG, B)
x_np, S, X = bench.make_signal(n, k, 1)
dev = torch.device("cuda", 0)
x = torch.from_numpy(x_np).to(dev)
flush = bench.L2Flush(dev)
stream = torch.cuda.current_stream()


def timed(fn, reps=20):
    for _ in range(3):
        flush()
        fn()
    ts = []
    for _ in range(reps):
        flush()
        a = torch.cuda.Event(enable_timing=True)
        b = torch.cuda.Event(enable_timing=True)
        a.record(stream)
        fn()
        b.record(stream)
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b) * 1e3)
    return sum(ts) / len(ts)


ref = Plan(n, k, B=B, L=L, seed=3, device=0, **prm)
locs = torch.empty(k, dtype=torch.int64, device=dev)
vals = torch.empty(k, dtype=torch.complex128, device=dev)
full_us = timed(lambda: ref.execute(x, locs, vals))
ref.execute(x, locs, vals)
torch.cuda.synchronize()
ref_ptr, ref_per = ref.exchange_buffer()
rec_bytes = ref_per // L
ref_buf = torch.as_tensor(__import__("paper_conf_ipps_wangcc16_b200.dist", fromlist=["_CudaBuffer"])._CudaBuffer(
    ref_ptr, ref_per), device=dev)
out = {"config": CFG, "filter": bench.filter_desc(CFG), "single_gpu_us": full_us,
       "allgather_model": {"alpha_us": ALPHA_US, "bw_gbs": BW_GBS,
                           "note": "assumed, not measured (one GPU in this environment)"},
       "ranks": {}}
for G in (1, 2, 4, 8):
    p = Plan(n, k, B=B, L=L, seed=3, device=0, rank=0, world=G, **prm)
    ptr, per = p.exchange_buffer()
    buf = torch.as_tensor(__import__("paper_conf_ipps_wangcc16_b200.dist", fromlist=["_CudaBuffer"])._CudaBuffer(
        ptr, per * G), device=dev)
    local_us = timed(lambda: p.execute_local(x))
    # the all-gather's result: every loop's record at its loop-sharded slot (the local steps
    # rewrite only this rank's slice, so the other slices stay in place across repetitions)
    for r in range(L):
        s = slot_of_loop(r, L, G)
        buf[s * rec_bytes:(s + 1) * rec_bytes].copy_(ref_buf[r * rec_bytes:(r + 1) * rec_bytes])
    torch.cuda.synchronize()
    l2 = torch.empty_like(locs)
    v2 = torch.empty_like(vals)

    def both():  # the per-execution counters are reset by the local steps' first kernel
        p.execute_local(x)
        p.execute_finish(l2, v2)
    finish_us = timed(both) - local_us
    both()
    torch.cuda.synchronize()
    same = torch.equal(l2, locs) and torch.equal(v2, vals)
    ag_bytes = per * G
    ag_us = 0.0 if G == 1 else ALPHA_US + (G - 1) / G * ag_bytes / (BW_GBS * 1e3)
    out["ranks"][G] = {"local_us": local_us, "finish_us": finish_us, "allgather_bytes": ag_bytes,
                       "allgather_model_us": ag_us, "model_total_us": local_us + ag_us + finish_us,
                       "finish_equals_single_gpu_output": same}
    p.close()
# ---- shard_mode 2: the same, with the two exchange buffers filled from a world = 1 mode-2 plan
from paper_conf_ipps_wangcc16_b200.dist import _CudaBuffer  # noqa: E402
from paper_conf_ipps_wangcc16_b200 import DEBUG_PER_LOOP, DEBUG_NUM_HITS  # noqa: E402
import numpy as np  # noqa: E402
MH = 8192
ref2 = Plan(n, k, B=B, L=L, seed=3, device=0, shard_mode=2, max_hits=MH, debug=1, **prm)
l0, v0 = torch.empty_like(locs), torch.empty_like(vals)
full2_us = timed(lambda: ref2.execute(x, l0, v0))
ref2.execute(x, l0, v0)
torch.cuda.synchronize()
assert torch.equal(l0, locs) and torch.equal(v0, vals)
c_ptr, c_per = ref2.exchange_buffer()
Lloc = ref2.info()["loc_loops"]
crec = c_per // Lloc
ref_cand = torch.as_tensor(_CudaBuffer(c_ptr, c_per), device=dev).clone()
H = int(ref2.debug(DEBUG_NUM_HITS)[0])
per_loop = torch.from_numpy(np.ascontiguousarray(ref2.debug(DEBUG_PER_LOOP).reshape(H, L))).to(dev)
out["mode2"] = {"single_gpu_us": full2_us, "hits": H, "max_hits": MH, "ranks": {}}
for G in (1, 2, 4, 8):
    p = Plan(n, k, B=B, L=L, seed=3, device=0, rank=0, world=G, shard_mode=2, max_hits=MH, **prm)
    ptr, per = p.exchange_buffer()
    ptr2, per2 = p.exchange_buffer2()
    cand = torch.as_tensor(_CudaBuffer(ptr, per * G), device=dev)
    x2 = torch.as_tensor(_CudaBuffer(ptr2, per2 * G, "<c16", 16), device=dev).view(G, MH, L // G)
    cmax = per // crec
    for r in range(Lloc):  # loop r: rank r % G, its location slot r // G
        d = ((r % G) * cmax + r // G) * crec
        cand[d:d + crec].copy_(ref_cand[r * crec:(r + 1) * crec])
    for g in range(G):  # per-loop estimates of the sorted hits: rank g's local slot i = loop i G + g
        x2[g, :H, :] = per_loop[:, g::G]
    torch.cuda.synchronize()
    l2 = torch.empty_like(locs)
    v2 = torch.empty_like(vals)
    local_us = timed(lambda: p.execute_local(x))

    def lm():
        p.execute_local(x)
        p.execute_mid()

    def lmf():
        lm()
        p.execute_finish(l2, v2)
    lm_us = timed(lm)
    lmf_us = timed(lmf)
    lmf()
    torch.cuda.synchronize()
    same = torch.equal(l2, locs) and torch.equal(v2, vals)
    b1, b2 = per * G, per2 * G
    ag1 = 0.0 if G == 1 else ALPHA_US + (G - 1) / G * b1 / (BW_GBS * 1e3)
    ag2 = 0.0 if G == 1 else ALPHA_US + (G - 1) / G * b2 / (BW_GBS * 1e3)
    out["mode2"]["ranks"][G] = {"local_us": local_us, "mid_us": lm_us - local_us, "finish_us": lmf_us - lm_us,
                                "allgather1_bytes": b1, "allgather2_bytes": b2, "allgather_model_us": ag1 + ag2,
                                "model_total_us": lmf_us + ag1 + ag2, "finish_equals_single_gpu_output": same}
    p.close()
# ---- signal sharding (shard_mode 1): rank 0 holds x[0, n/G); its exchange buffer then gets the
# summed spectra of the world = 1 plan (the all-reduce's result), so finish does the real work
ref_ptr1, ref_per1 = ref.exchange_buffer()
ref_rec = torch.as_tensor(_CudaBuffer(ref_ptr1, ref_per1), device=dev).clone()
out["signal"] = {"ranks": {}}
for G in (2, 4, 8):
    p = Plan(n, k, B=B, L=L, seed=3, device=0, rank=0, world=G, shard_mode=1, **prm)
    ptr, per = p.exchange_buffer()
    buf = torch.as_tensor(_CudaBuffer(ptr, per), device=dev)
    xs = x[: n // G].clone()
    local_us = timed(lambda: p.execute_local(xs))
    l2 = torch.empty_like(locs)
    v2 = torch.empty_like(vals)

    def both():
        p.execute_local(xs)
        buf.copy_(ref_rec)
        p.execute_finish(l2, v2)
    copy_us = timed(lambda: buf.copy_(ref_rec))
    finish_us = timed(both) - local_us - copy_us
    both()
    torch.cuda.synchronize()
    same = torch.equal(l2, locs)
    ar_us = ALPHA_US + 2 * (G - 1) / G * per / (BW_GBS * 1e3)
    out["signal"]["ranks"][G] = {"local_us": local_us, "finish_us": finish_us, "allreduce_bytes": per,
                                 "allreduce_model_us": ar_us, "model_total_us": local_us + ar_us + finish_us,
                                 "staged": int(p.info()["staged"]), "finish_locs_equal_single_gpu": same}
    p.close()
print(json.dumps(out, indent=1))
with open(sys.argv[1], "w") as f:
    json.dump(out, f, indent=1)
