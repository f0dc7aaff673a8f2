#!/usr/bin/env python
"""Benchmark of the sparse FFT hot path (BASELINE.json metric:
"ms per sparse FFT at n=2^24,k=1000 (1/2/4/8 B200); x vs dense cuFFT; HBM GB/s").

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config C3] [--impl reference]

One step = one whole transform (fold, B-point FFT, cutoff, vote, estimate,
output; for N > 1 plus the all-gather) of a planted k-sparse fp64 signal that
is already resident in HBM.  L2 is flushed (256 MiB write + 256 MiB read) between timed
steps, outside the per-step CUDA events.  Prints ONE JSON line on rank 0.
See DESIGN.md §8 for every field.
"""
from __future__ import annotations

import argparse
import json
import math
import os
import statistics
import subprocess
import sys
import threading
import time

for _v in ("OMP_NUM_THREADS", "OPENBLAS_NUM_THREADS", "MKL_NUM_THREADS"):
    os.environ.setdefault(_v, "1")

import numpy as np  # noqa: E402

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

CONFIGS = {
    # name: (n, k, L, description)   BASELINE.json configs
    "C1": (2 ** 14, 8, 16, "n=2^14, k=8, noiseless fp64 planted spectrum"),
    "C2": (2 ** 20, 100, 16, "n=2^20, k=100, noiseless fp64 planted spectrum"),
    "C3": (2 ** 24, 1000, 16, "n=2^24, k=1000, noiseless fp64 planted spectrum"),
    "C4": (2 ** 27, 1000, 16, "n=2^27, k=1000, noiseless fp64 planted spectrum"),
    "C5": (2 ** 22, 1000, 16, "n=2^22, k=1000, batch of 64 independent noiseless fp64 signals, signals sharded over GPUs"),
    "C5k": (2 ** 22, 1000, 16, "n=2^22, one noiseless fp64 signal, k from --k (the k sweep 50..4096)"),
}
BATCH = {"C5": 64}
# Filter and cutoff parameters per config (the paper leaves them open, DESIGN.md
# §3 [Z1], [Z17], [Z21]): tolerance delta, main-lobe half width lambda = lam_B / B,
# optionally the location loops' own (loc_tol, loc_lam_B), and num_select = num_k * k.
# C3: delta = 1e-7 with lambda = 0.75 / B (2/3 of the taps of lambda = 0.5 / B):
# exact recovery and L1 <= 2.1e-7 on 48 + 192 oracle seeds (scripts/study/n3_study*.jsonl).
FILTERS = {
    "C1": dict(tol=1e-8, lam_B=0.5),
    "C2": dict(tol=1e-8, lam_B=0.5),
    "C3": dict(tol=1e-7, lam_B=0.75),
    "C4": dict(tol=1e-8, lam_B=0.5),
    "C5": dict(tol=1e-8, lam_B=0.5),
    "C5k": dict(tol=1e-8, lam_B=0.5),
}
# the library defaults (cusfft_params_default), reported beside the tuned line
DEFAULT_FILTER = dict(tol=1e-8, lam_B=0.5)


def plan_params(config: str, B: int | None = None, filt: dict | None = None) -> dict:
    """Plan keyword arguments (cusfft_params fields) of a config's filter / cutoff."""
    n, k = CONFIGS[config][:2]
    if B is None:  # the paper's formula B = floor_pow2(sqrt(n k / log2 n))
        B = 1 << int(math.floor(math.log2(math.sqrt(n * k / math.log2(n)))))
    f = dict(FILTERS[config] if filt is None else filt)
    out = dict(tolerance=f["tol"], lobefrac=f["lam_B"] / B)
    if "loc_tol" in f:
        out["loc_tolerance"] = f["loc_tol"]
    if "loc_lam_B" in f:
        out["loc_lobefrac"] = f["loc_lam_B"] / B
    if "num_k" in f:
        out["num_select"] = int(round(f["num_k"] * k))
    return out


def filter_desc(config: str, filt: dict | None = None) -> str:
    f = FILTERS[config] if filt is None else filt
    d = f"Dolph-Chebyshev delta={f['tol']:g}, lambda={f['lam_B']:g}/B"
    if "loc_tol" in f or "loc_lam_B" in f:
        d += f"; location loops delta={f.get('loc_tol', f['tol']):g}, lambda={f.get('loc_lam_B', f['lam_B']):g}/B"
    if "num_k" in f:
        d += f"; num={f['num_k']:g}k"
    return d


METRIC = "ms per sparse FFT at n=2^24,k=1000 (1/2/4/8 B200); x vs dense cuFFT; HBM GB/s"
PEAKS_FILE = os.path.join(ROOT, "MEASURED_PEAKS.json")
FALLBACK_HBM = 6650.0


def hbm_peak():
    try:
        with open(PEAKS_FILE) as f:
            return float(json.load(f)["hbm_gbs"]), "measured (MEASURED_PEAKS.json copy bandwidth)"
    except Exception:
        return FALLBACK_HBM, "fallback (B200_PROFILING.md)"


class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled while the timed loop runs."""

    FIELDS = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index = index
        self.lines = []
        self.proc = None

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", f"--query-gpu={self.FIELDS}", "--format=csv,noheader,nounits", "-lms", "50",
                 "-i", str(self.index)], stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def __exit__(self, *exc):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except Exception:
                self.proc.kill()

    def summary(self):
        sm, mx, reasons = [], None, set()
        names = ("hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap")
        for ln in self.lines:
            parts = [p.strip() for p in ln.split(",")]
            if len(parts) < 9:
                continue
            try:
                sm.append(float(parts[1]))
                mx = float(parts[2])
            except ValueError:
                continue
            for nm, v in zip(names, parts[5:9]):
                if v.lower() == "active":
                    reasons.add(nm)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": mx,
                "reasons": sorted(reasons), "samples": len(sm)}


SNR_DB = None  # --snr: additive complex white Gaussian noise (workload.planted_signal)


def make_signal(n, k, seed):
    from paper_conf_ipps_wangcc16_b200.workload import planted_signal
    return planted_signal(n, k, seed, snr_db=SNR_DB)


# ---------------------------------------------------------------------------
# CPU oracle legs (the oracle is test infrastructure; bench may time it here)
# ---------------------------------------------------------------------------
def host_cores() -> int:
    return len(os.sched_getaffinity(0)) if hasattr(os, "sched_getaffinity") else (os.cpu_count() or 1)


def oracle_time(config, n, k, L, B, x, seed, budget_s=20.0, min_runs=1, max_runs=None):
    """The oracle transform as it stands (plan-time filter excluded), pinned to
    one host core (sched_setaffinity, like taskset -c) with one BLAS thread."""
    import oracle
    prm = plan_params(config, B)
    okw = {kk: prm[kk] for kk in ("tolerance", "lobefrac", "loc_tolerance", "loc_lobefrac", "num_select") if kk in prm}
    p = oracle.make_params(n, k, B=B, L=L, seed=seed, **okw)
    g = oracle.filter_taps(p)
    Ghat = oracle.filter_response(g, n, n // B)
    gl = oracle.filter_taps(oracle.loc_filter_params(p)) if oracle.separate_filters(p) else None
    cores = host_cores()
    pinned = None
    if hasattr(os, "sched_setaffinity"):
        before = os.sched_getaffinity(0)
        core = min(before)
        os.sched_setaffinity(0, {core})
        pinned = core
    times = []
    try:
        t_start = time.perf_counter()
        while True:
            t0 = time.perf_counter()
            res = oracle.sfft(x, p, taps=g, Ghat=Ghat, taps_loc=gl)
            times.append(time.perf_counter() - t0)
            if max_runs is not None and len(times) >= max_runs:
                break
            if len(times) >= min_runs and time.perf_counter() - t_start >= budget_s:
                break
    finally:
        if pinned is not None:
            os.sched_setaffinity(0, before)
    return times, res, cores, pinned


def run_reference(args):
    """--impl reference: the CPU oracle on this arm's workload, on the host cores."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    n, k, L, desc = CONFIGS[args.config]
    from oracle import default_B
    B = args.B or default_B(n, k)
    x, S, X = make_signal(n, k, args.signal_seed)
    times, _, cores, core = oracle_time(args.config, n, k, L, B, x, args.plan_seed, budget_s=0,
                                        min_runs=args.warmup + args.steps, max_runs=args.warmup + args.steps)
    t = times[args.warmup:]
    ms = 1e3 * sum(t) / len(t)
    line = {
        "impl": "reference", "metric": METRIC, "value": ms, "unit": "ms", "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": False,
        "scaling": "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": {"workload": f"{args.config}: {desc}, L={L}, B={B}, {filter_desc(args.config)}",
                   "n": n, "k": k, "B": B, "L": L, **plan_params(args.config, B)},
        "cpu_baseline": {"value": ms, "unit": "ms", "cores": 1, "kind": "oracle",
                         "sample": f"{len(t)} full oracle transforms of the {args.config} workload "
                                   f"(plan-time filter construction excluded), numpy, pinned to core {core}: "
                                   f"1 of {cores} host cores"},
        "e2e": {"value": ms, "unit": "ms", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)
    return 0


# ---------------------------------------------------------------------------
# GPU arm
# ---------------------------------------------------------------------------
class L2Flush:
    """L2 flush between timed steps: write 256 MiB (evicts every normal line),
    then read another 256 MiB so the write-backs happen here, not in the step.
    cold=True first returns every persisting line to normal
    (cudaCtxResetPersistingL2Cache), so a staged plan's staging buffer is
    flushed too (the persisting set-aside otherwise keeps it resident)."""

    def __init__(self, dev):
        import torch
        self.w = torch.empty(256 * 1024 * 1024, dtype=torch.uint8, device=dev)
        self.r = torch.ones(64 * 1024 * 1024, dtype=torch.int32, device=dev)
        self._reset = None

    def __call__(self, cold: bool = False):
        if cold:
            if self._reset is None:
                from cuda.bindings import runtime as rt
                self._reset = rt.cudaCtxResetPersistingL2Cache
            self._reset()
        self.w.zero_()
        self.r.sum()


PAPER_CONTEXT = ("cusFFT (PAPER.md, fp64, Tesla K20x: Kepler GK110, 14 SMs, 250 GB/s, CUDA 5.5; Table I L412-L414): "
                 "15x over cuFFT at n=2^27 (>9x baseline, L406), faster than cuFFT for n > 2^22 (L402); "
                 "0.5x-29x over parallel FFTW 3.3 on a 6-core Xeon E5-2640 Sandy Bridge (Table II L418-L420, L426); "
                 "up to 6.6x over PsFFT (OpenMP sFFT) at n=2^24, transfers included (L426)")


def run_gpu(args):
    import torch
    import torch.distributed as dist

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    if args.gpus != world:
        if world == 1 and args.gpus > 1:
            print(json.dumps({"error": "launch N>1 with torchrun (one process per GPU)"}))
            return 2
    torch.cuda.set_device(local_rank)
    dev = torch.device("cuda", local_rank)
    if world > 1:
        dist.init_process_group("nccl", device_id=dev)

    from paper_conf_ipps_wangcc16_b200 import Plan, default_B, nccl_unique_id

    n, k, L, desc = CONFIGS[args.config]
    B = args.B or default_B(n, k)
    prm = plan_params(args.config, B)
    if args.l2_persist is not None:
        prm["l2_persist"] = args.l2_persist
    x_np, S, X = make_signal(n, k, args.signal_seed)
    x_pin = torch.from_numpy(x_np).pin_memory()
    x = x_pin.to(dev)
    flush = L2Flush(dev)
    stream = torch.cuda.current_stream()

    def time_steps(fn, reps, cold=False):
        ts = []
        for _ in range(reps):
            flush(cold)
            a = torch.cuda.Event(enable_timing=True)
            b = torch.cuda.Event(enable_timing=True)
            a.record(stream)
            fn()
            b.record(stream)
            torch.cuda.synchronize()
            ts.append(a.elapsed_time(b))
        return ts

    # ---- dense cuFFT of the same n (context), complex128, L2 flushed; timed
    # before any plan exists, so cuFFT has the whole L2 (a staged plan holds a
    # persisting-L2 set-aside while it lives, include/cusfft.h)
    dense_ms = statistics.median(time_steps(lambda: torch.fft.fft(x), args.warmup + 10)[args.warmup:])

    t_plan0 = time.perf_counter()
    if world == 1:
        plan = Plan(n, k, B=B, L=L, seed=args.plan_seed, device=local_rank, **prm)
    else:  # the plan owns the exchange: rank 0's ncclUniqueId broadcast once over the process group
        uid = [nccl_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(uid, src=0)
        shard = {"loops": 0, "signal": 1, "loops2": 2}[args.shard]
        extra = dict(max_hits=8192) if shard == 2 else {}  # exchange #2 moves max_hits x L x 16 B
        plan = Plan(n, k, B=B, L=L, seed=args.plan_seed, device=local_rank, rank=rank, world=world,
                    nccl_id=uid[0], shard_mode=shard, **prm, **extra)
        if shard == 1:  # this rank holds only its slice of x
            span = n // world
            x = x[rank * span:(rank + 1) * span].clone()
    plan_ms = 1e3 * (time.perf_counter() - t_plan0)
    locs = torch.empty(k, dtype=torch.int64, device=dev)
    vals = torch.empty(k, dtype=torch.complex128, device=dev)

    def step():
        plan.execute(x, locs, vals)
        return locs, vals
    launches = plan.launches_per_execute()
    info = plan.info()

    # correctness of the benchmarked configuration (untimed)
    l_out, v_out = step()
    torch.cuda.synchronize()
    status = plan.status()
    l_np, v_np = l_out.cpu().numpy(), v_out.cpu().numpy()
    exact = set(l_np.tolist()) == set(S.tolist())
    truth = dict(zip(S.tolist(), X.tolist()))
    got = {int(f): complex(v) for f, v in zip(l_np, v_np) if f >= 0}
    l1 = sum(abs(got.get(f, 0) - truth.get(f, 0)) for f in set(truth) | set(got)) / k

    def barrier():
        if world > 1:
            dist.barrier()

    # warm-up (at least W steps and ~0.3 s so the clock sampler sees load)
    with ClockSampler(local_rank) as clocks:
        t0 = time.perf_counter()
        i = 0
        while i < args.warmup or time.perf_counter() - t0 < 0.3:
            flush()
            step()
            i += 1
        torch.cuda.synchronize()
        # ---- timed region: exactly K steps
        ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
        barrier()
        torch.cuda.synchronize()
        reg0 = torch.cuda.Event(enable_timing=True)
        reg1 = torch.cuda.Event(enable_timing=True)
        reg0.record(stream)
        for s in range(args.steps):
            flush()                             # L2 flush, outside the step's events
            ev[s][0].record(stream)
            step()
            ev[s][1].record(stream)
        reg1.record(stream)
        torch.cuda.synchronize()
        barrier()
        # the cold arm: the same steps with the persisting lines reset before each flush
        cold_ms = time_steps(step, args.steps, cold=True)
        torch.cuda.synchronize()
    step_ms = [a.elapsed_time(b) for a, b in ev]
    ms = sum(step_ms) / len(step_ms)
    cold = sum(cold_ms) / len(cold_ms)
    region_ms = reg0.elapsed_time(reg1)
    if world > 1:
        t = torch.tensor([ms, cold], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms, cold = float(t[0].item()), float(t[1].item())

    # ---- the roofline kernel (phase 1 of the staged fold, the permute gather)
    # timed INSIDE the bench's CUDA graph: event-record nodes before and after it
    # (cusfft_set_timing mode 2), same flush, warm and cold
    gather = {}
    if info["staged"]:
        for nm, cold_flag in (("warm", False), ("cold", True)):
            plan.set_timing(2)
            g, tot = [], []
            for _ in range(max(10, args.steps)):
                flush(cold_flag)
                step()
                st = plan.stage_times()
                g.append(st["gather"])
                tot.append(st["fold"])
            plan.set_timing(0)
            if all(v > 0 for v in g):
                gather[nm] = {"ms": sum(g) / len(g), "graph_ms": sum(tot) / len(tot)}

    # ---- per-stage times inside the CUDA graph: T_s = time of the graph that
    # runs stages 1..s (cusfft_set_stage_limit), stage s = T_s - T_{s-1}
    names = ("fold", "fft", "cutoff", "vote", "estimate", "output")
    stage_ms = {}
    if world == 1:
        prev = 0.0
        reps = max(10, args.steps)
        for si, nm in enumerate(names, start=1):
            if info["tail"] and si == 5:
                continue  # k_tail runs vote and estimation: stage 4 covers both
            plan.set_stage_limit(si)
            step()
            tsi = sum(time_steps(step, reps)) / reps
            stage_ms["vote + estimate (k_tail)" if (info["tail"] and si == 4) else nm] = tsi - prev
            prev = tsi
        plan.set_stage_limit(6)
        # where the location slots' FFT pass 2 is fused with the cutoff (k_fft2_select),
        # "fft" is the estimation slots' FFT and "cutoff" includes the location pass 2

    # ---- CUPTI cross-check of the kernel durations (torch.profiler: no replay)
    cupti = None
    if world == 1 and not args.no_cupti:
        try:
            acts = [torch.profiler.ProfilerActivity.CUDA]
            with torch.profiler.profile(activities=acts) as prof:
                for _ in range(10):
                    flush()
                    step()
                torch.cuda.synchronize()
            per = {}
            for e in prof.events():
                if e.device_type == torch.autograd.DeviceType.CUDA and "cusfft::" in e.name:
                    short = e.name.split("(")[0].replace("void ", "").replace("cusfft::", "")
                    per.setdefault(short, []).append(e.device_time)
            cupti = {kk: {"launches": len(v), "mean_us": sum(v) / len(v)} for kk, v in sorted(per.items())}
        except Exception as exc:  # pragma: no cover
            cupti = {"error": str(exc)[:200]}

    # ---- e2e through the C ABI with host buffers (world == 1 path)
    e2e = None
    if world == 1:
        h_locs = torch.empty(k, dtype=torch.int64).pin_memory()
        h_vals = torch.empty(k, dtype=torch.complex128).pin_memory()
        for _ in range(2):
            plan.execute_host(x_pin, h_locs, h_vals)
        e_ms = []
        for _ in range(args.steps):
            flush()
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            plan.execute_host(x_pin, h_locs, h_vals)
            e_ms.append(1e3 * (time.perf_counter() - t0))
        # pinned x is gathered in place over PCIe (include/cusfft.h): what crosses the bus is the
        # gathered samples, at least the distinct 32-B sectors they occupy
        zc = os.environ.get("CUSFFT_HOST_ZEROCOPY", "1") != "0"
        e2e = {"value": sum(e_ms) / len(e_ms), "unit": "ms",
               "h2d_bytes_per_step": int(info["sectors"]) * 32 if zc else n * 16,
               "d2h_bytes_per_step": k * (8 + 16),
               "note": ("cusfft_execute_host from pinned host memory: x read in place over PCIe by the "
                        "gather (h2d_bytes = the distinct 32-B sectors of x the plan's taps touch, of "
                        f"{n * 16} B)" if zc else "cusfft_execute_host: pinned H2D copy of the whole x")
                       + ", transform, D2H of locs/vals, host wall clock; L2 flushed before each step"}

    # ---- the library-default filter (delta = 1e-8, lambda = 0.5/B) on the same signal
    default_line = None
    if world == 1 and args.config == "C3" and not args.no_default_line:
        pd = Plan(n, k, B=B, L=L, seed=args.plan_seed, device=local_rank, **plan_params(args.config, B, DEFAULT_FILTER))
        l2_, v2_ = torch.empty_like(locs), torch.empty_like(vals)
        for _ in range(3):
            flush()
            pd.execute(x, l2_, v2_)
        ts = time_steps(lambda: pd.execute(x, l2_, v2_), args.steps)
        default_line = {"filter": filter_desc(args.config, DEFAULT_FILTER), "taps": pd.w,
                        "ms": sum(ts) / len(ts), "exact_recovery": set(l2_.cpu().tolist()) == set(S.tolist()),
                        "status": pd.status()}
        pd.close()

    ablations = None
    if world == 1 and args.ablations:
        ablations = {}
        variants = [("separate_filters_n3_loc_d1e-6", dict(loc_tolerance=1e-6, loc_lobefrac=prm["lobefrac"])),
                    ("cutoff_sort_alg3", dict(cutoff_mode=1)),
                    ("cutoff_threshold_alg6", dict(cutoff_mode=2, cutoff_threshold=1e-3)),
                    ("direct_gather_no_stage", dict(gather=1)),
                    ("remap_execute_paper_sec5a", dict(gather=2)),
                    ("no_l2_persist", dict(l2_persist=0))]
        for name, kw in variants:
            p2 = Plan(n, k, B=B, L=L, seed=args.plan_seed, device=local_rank, **{**prm, **kw})
            l2_, v2_ = torch.empty_like(locs), torch.empty_like(vals)
            for _ in range(3):
                p2.execute(x, l2_, v2_)
            ts = time_steps(lambda: p2.execute(x, l2_, v2_), max(10, args.steps))
            ok = set(l2_.cpu().tolist()) == set(S.tolist())
            ablations[name] = {"ms": sum(ts) / len(ts), "exact_recovery": ok, "status": p2.status()}
            p2.close()

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:  # N = 1 only (bench contract)
        times, _, cores, core = oracle_time(args.config, n, k, L, B, x_np, args.plan_seed,
                                            budget_s=args.cpu_budget_s, min_runs=1)
        cpu = {"value": 1e3 * sum(times) / len(times), "unit": "ms", "cores": 1, "kind": "oracle",
               "sample": f"{len(times)} full oracle transform(s) of the same {args.config} signal "
                         f"(plan-time filter construction excluded), numpy, pinned to core {core}: "
                         f"1 of {cores} host cores"}

    peak, peak_src = hbm_peak()
    # roofline kernel: the address-ordered permute gather (fold phase 1) -- it
    # carries all of the transform's HBM traffic.  Algorithmic bytes: 32 B per
    # distinct sector of x the plan's gathers touch.
    sum_w = int(info["w_loc"]) * plan.loc_loops + int(info["w"]) * (L - plan.loc_loops) if info["filters"] == 2 else L * plan.w
    lw_local = sum_w // world if world > 1 and args.shard in ("loops", "loops2") else sum_w
    gather_bytes = lw_local * 32  # one 32-B sector per gathered 16-B sample (L w 32 B)
    rk_ms = gather["warm"]["ms"] if "warm" in gather else stage_ms.get("fold", 0.0)
    achieved = gather_bytes / (rk_ms * 1e-3) / 1e9
    cupti_gather_us = None
    if isinstance(cupti, dict):
        for kk, vv in cupti.items():
            if kk.startswith("k_stage_packed") and isinstance(vv, dict):
                cupti_gather_us = vv.get("mean_us")
    traffic = None
    tf = os.path.join(ROOT, "profiles", f"fold_traffic_{args.config}.json")
    if os.path.exists(tf):
        try:
            with open(tf) as f:
                tj = json.load(f)
            if tj.get("sum_w") == sum_w:  # only a capture of this very plan counts
                traffic = tj.get("k_stage_packed_dram_bytes_per_launch")
        except Exception:
            traffic = None
    line = {
        "metric": METRIC, "value": ms, "unit": "ms", "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": False,
        "scaling": "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": {"workload": f"{args.config}: {desc}, L={L}, B={B}, {filter_desc(args.config)}, "
                               f"{sum_w} gathers (taps x loops)",
                   "n": n, "k": k, "B": B, "L": L, "taps": plan.w, "taps_loc": int(info["w_loc"]),
                   **prm, "loc_loops": plan.loc_loops, "vote_threshold": plan.T,
                   "parallelism": f"{args.shard}-sharded x{world} (NCCL in the plan's graph)" if world > 1 else "single GPU",
                   "l2": "flushed between timed steps (256 MiB write + 256 MiB read), outside the step events; "
                         "the staging buffer's persisting lines survive it (warm); value_cold resets them too",
                   "signal_seed": args.signal_seed, "plan_seed": args.plan_seed,
                   "snr_db": SNR_DB},
        "value_cold": cold,
        "plan_ms": plan_ms,
        "gpu_launches": launches * args.steps,
        "timed_region_ms_incl_flush": region_ms,
        "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                     "frac": achieved / peak, "traffic": traffic,
                     "kernel": ("k_stage_packed (fold phase 1: address-ordered permute gather of x)" if "warm" in gather
                                else f"the whole fold stage ({int(info['staged'])} stage groups: phase 1 + phase 2 each)"
                                if info["staged"] else "the whole fold stage (direct gather k_fold_fft1)"),
                     "algorithmic_bytes_per_launch": gather_bytes, "kernel_ms": rk_ms,
                     "algorithmic_bytes_note": f"L*w*32 B: {lw_local} gathers x one 32-B sector (SURVEY 8(d)); "
                                               f"{int(info['sectors'])} distinct sectors = {int(info['sectors']) * 32} B",
                     "kernel_ms_how": "CUDA event-record nodes around the kernel inside the bench's graph "
                                      "(adds the event latency), L2 flushed before each execution",
                     "kernel_ms_cupti": cupti_gather_us * 1e-3 if cupti_gather_us else None,
                     "frac_cupti": (gather_bytes / (cupti_gather_us * 1e-6) / 1e9 / peak) if cupti_gather_us else None,
                     "kernel_ms_cold": gather.get("cold", {}).get("ms"),
                     "frac_cold": (gather_bytes / (gather["cold"]["ms"] * 1e-3) / 1e9 / peak) if "cold" in gather else None,
                     "peak_source": peak_src},
        "stage_ms": stage_ms,
        "kernels_cupti_us": cupti,
        "default_filter": default_line,
        "ablations": ablations,
        "dense_cufft_ms": dense_ms, "speedup_vs_dense_cufft": dense_ms / ms,
        "accuracy": {"exact_recovery": exact, "l1_per_coefficient": l1, "status": status},
        "clocks": clocks.summary(),
        "e2e": e2e,
        "cpu_baseline": cpu,
        "paper_context": PAPER_CONTEXT,
    }
    if rank == 0:
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()
    return 0


def run_gpu_batch(args):
    """C5: a batch of independent signals, sharded over ranks with no collective
    (dist.BatchShardedSfft); each rank runs cusfft_execute_batch on its share
    with --pipeline clone plans in flight.  value = ms per transform, amortised
    over the whole batch (max over ranks of the batch time / batch size)."""
    import torch
    import torch.distributed as dist

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local_rank)
    dev = torch.device("cuda", local_rank)
    if world > 1:
        dist.init_process_group("nccl", device_id=dev)
    from paper_conf_ipps_wangcc16_b200 import Plan, default_B
    from paper_conf_ipps_wangcc16_b200.dist import BatchShardedSfft
    n, k, L, desc = CONFIGS[args.config]
    count = BATCH[args.config]
    B = default_B(n, k)
    plan = Plan(n, k, B=B, L=L, seed=args.plan_seed, device=local_rank, **plan_params(args.config, B))
    plan.set_pipeline(args.pipeline)

    class _Eng:
        execute_batch = staticmethod(plan.execute_batch)
    drv = BatchShardedSfft(_Eng, count)
    mine = list(range(drv.lo, drv.hi))
    sigs = [make_signal(n, k, args.signal_seed + b) for b in mine]
    xb_pin = torch.from_numpy(np.stack([s_[0] for s_ in sigs])).pin_memory()
    xb = xb_pin.to(dev)
    locs = torch.empty(len(mine), k, dtype=torch.int64, device=dev)
    vals = torch.empty(len(mine), k, dtype=torch.complex128, device=dev)
    plan.execute_batch(xb, locs, vals)
    torch.cuda.synchronize()
    status = plan.status()
    exact = all(set(locs[i].cpu().tolist()) == set(sigs[i][1].tolist()) for i in range(len(mine)))
    flush = L2Flush(dev)
    stream = torch.cuda.current_stream()

    def barrier():
        if world > 1:
            dist.barrier()
    with ClockSampler(local_rank) as clocks:
        for _ in range(args.warmup):
            flush()
            plan.execute_batch(xb, locs, vals)
        torch.cuda.synchronize()
        ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
        barrier()
        torch.cuda.synchronize()
        for s_ in range(args.steps):
            flush()
            ev[s_][0].record(stream)
            plan.execute_batch(xb, locs, vals)
            ev[s_][1].record(stream)
        torch.cuda.synchronize()
        barrier()
    batch_ms = sum(a.elapsed_time(b) for a, b in ev) / args.steps
    if world > 1:
        t = torch.tensor([batch_ms], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        batch_ms = float(t.item())
        ok = torch.tensor([1 if exact else 0], device=dev)
        dist.all_reduce(ok, op=dist.ReduceOp.MIN)
        exact = bool(ok.item())
    ms = batch_ms / count
    # e2e: pinned host batch -> device, transform, results -> host, every step
    h_locs = torch.empty(len(mine), k, dtype=torch.int64).pin_memory()
    h_vals = torch.empty(len(mine), k, dtype=torch.complex128).pin_memory()
    e_ms = []
    for _ in range(max(3, args.steps // 4)):
        barrier()
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        xb.copy_(xb_pin, non_blocking=True)
        plan.execute_batch(xb, locs, vals)
        h_locs.copy_(locs, non_blocking=True)
        h_vals.copy_(vals, non_blocking=True)
        torch.cuda.synchronize()
        e_ms.append(1e3 * (time.perf_counter() - t0))
    e2e_ms = sum(e_ms) / len(e_ms)
    if world > 1:
        t = torch.tensor([e2e_ms], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        e2e_ms = float(t.item())
    line = {
        "metric": METRIC, "value": ms, "unit": "ms", "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": batch_ms, "higher_is_better": False,
        "scaling": "weak" if world > 1 else "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": {"workload": f"{args.config}: {desc}, L={L}, B={B}, w={plan.w}, pipeline depth {args.pipeline}",
                   "n": n, "k": k, "B": B, "L": L, "batch": count, "per_rank": len(mine),
                   "parallelism": f"signal-batch sharded x{world} (no collective)",
                   "l2": "flushed between timed steps (one step = the rank's whole batch)"},
        "gpu_launches": plan.launches_per_execute() * len(mine) * args.steps,
        "accuracy": {"exact_recovery": exact, "status": status},
        "clocks": clocks.summary(),
        "e2e": {"value": e2e_ms / count, "unit": "ms", "h2d_bytes_per_step": len(mine) * n * 16,
                "d2h_bytes_per_step": len(mine) * k * 24,
                "note": "per transform: pinned H2D of the rank's batch, execute_batch, D2H of results"},
    }
    if rank == 0:
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()
    return 0


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="cusfft", choices=["cusfft", "reference"])
    ap.add_argument("--config", default="C3", choices=sorted(CONFIGS))
    ap.add_argument("--signal-seed", type=int, default=1)
    ap.add_argument("--plan-seed", type=int, default=3)
    ap.add_argument("--shard", default="loops", choices=["loops", "signal", "loops2"],
                    help="N>1: loop sharding (one all-gather of the per-loop records), signal sharding "
                         "(SURVEY N1, all-reduce) or loop sharding with two all-gathers (candidates, then "
                         "per-loop estimates: SURVEY 8(e) steps 1-5)")
    ap.add_argument("--B", type=int, default=0, help="bucket count (default: the paper's formula, DESIGN.md Z3)")
    ap.add_argument("--pipeline", type=int, default=3,
                    help="C5 batch: clone plans in flight per GPU (3 measured best: 38.3 / 36.9 / 38.0 us per transform at 2 / 3 / 4)")
    ap.add_argument("--cpu-budget-s", type=float, default=15.0)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-cupti", action="store_true")
    ap.add_argument("--no-default-line", action="store_true")
    ap.add_argument("--ablations", action="store_true",
                    help="also time the cutoff variants (Alg. 3 sort, Alg. 6 threshold), the direct gather, no L2 set-aside")
    ap.add_argument("--k", type=int, default=0, help="C5k: sparsity k (the k sweep)")
    ap.add_argument("--bcst", type=float, default=1.0, help="B = floor_pow2(bcst sqrt(n k / log2 n)) (k sweep: 2 for k >= 2000)")
    ap.add_argument("--l2-persist", type=int, default=None, choices=[0, 1],
                    help="plan parameter l2_persist (default: the library default)")
    ap.add_argument("--snr", type=float, default=None, help="additive noise SNR in dB (C4 sweep); default noiseless")
    args = ap.parse_args()
    if args.warmup < 3:
        args.warmup = 3
    global SNR_DB
    SNR_DB = args.snr
    if args.k:
        n_, _, L_, d_ = CONFIGS[args.config]
        CONFIGS[args.config] = (n_, args.k, L_, d_.replace("k from --k", f"k={args.k}"))
    if args.bcst != 1.0 and not args.B:
        n_, k_ = CONFIGS[args.config][:2]
        args.B = 1 << int(math.floor(math.log2(args.bcst * math.sqrt(n_ * k_ / math.log2(n_)))))
    if args.impl == "reference":
        return run_reference(args)
    if args.config in BATCH:
        return run_gpu_batch(args)
    return run_gpu(args)


if __name__ == "__main__":
    sys.exit(main())
