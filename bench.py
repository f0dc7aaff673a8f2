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
}
BATCH = {"C5": 64}
# Filter tolerance delta per config (the paper leaves it open).  C3: 1e-7 keeps
# exact recovery and L1 <= 1.75e-7 on 48/48 oracle seeds (DESIGN.md §3 study)
# with 12% fewer taps than the library default 1e-8.
TOLERANCE = {"C1": 1e-8, "C2": 1e-8, "C3": 1e-7, "C4": 1e-8, "C5": 1e-8}
METRIC = "ms per sparse FFT at n=2^24,k=1000 (1/2/4/8 B200); x vs dense cuFFT; HBM GB/s"
PEAKS_FILE = os.path.join(ROOT, "MEASURED_PEAKS.json")
FALLBACK_HBM = 6650.0


def hbm_peak():
    try:
        with open(PEAKS_FILE) as f:
            return float(json.load(f)["hbm_gbs"]), "measured (MEASURED_PEAKS.json copy bandwidth)"
    except Exception:
        return FALLBACK_HBM, "fallback (B200_PROFILING.md)"


def fold_bytes(L: int, w: int, B: int, sectors: int):
    """Algorithmic bytes of the fold stage: the distinct
    32-B DRAM sectors of x that the plan's L*w gather positions touch (exact,
    counted at plan time; a random 16-B sample cannot cost less than its
    sector, and a sector shared by several loops need be read once), the w fp64
    taps, and the L*B complex fp64 buckets written (u, plus v when the first
    FFT pass is fused, B > 2048).  `useful` counts 16 B per sample instead."""
    out = L * B * 16 * (2 if 2048 < B <= 65536 else 1)
    return sectors * 32 + w * 8 + out, L * w * 16 + w * 8 + out


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


def make_signal(n, k, seed):
    from paper_conf_ipps_wangcc16_b200.workload import planted_signal
    return planted_signal(n, k, seed)


# ---------------------------------------------------------------------------
# CPU oracle legs (the oracle is test infrastructure; bench may time it here)
# ---------------------------------------------------------------------------
def oracle_time(n, k, L, B, x, seed, budget_s=20.0, min_runs=1, max_runs=None, tolerance=1e-8):
    import oracle
    p = oracle.make_params(n, k, B=B, L=L, seed=seed, tolerance=tolerance)
    g = oracle.filter_taps(p)
    Ghat = oracle.filter_response(g, n, n // B)
    times = []
    t_start = time.perf_counter()
    while True:
        t0 = time.perf_counter()
        res = oracle.sfft(x, p, taps=g, Ghat=Ghat)
        times.append(time.perf_counter() - t0)
        if max_runs is not None and len(times) >= max_runs:
            break
        if len(times) >= min_runs and time.perf_counter() - t_start >= budget_s:
            break
    return times, res


def run_reference(args):
    """--impl reference: the CPU oracle on this arm's workload, on the host cores."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    n, k, L, desc = CONFIGS[args.config]
    from oracle import default_B
    B = default_B(n, k)
    x, S, X = make_signal(n, k, args.signal_seed)
    times, _ = oracle_time(n, k, L, B, x, args.plan_seed, budget_s=0, min_runs=args.warmup + args.steps,
                           max_runs=args.warmup + args.steps, tolerance=TOLERANCE[args.config])
    t = times[args.warmup:]
    ms = 1e3 * sum(t) / len(t)
    line = {
        "impl": "reference", "metric": METRIC, "value": ms, "unit": "ms", "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": False,
        "scaling": "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": {"workload": f"{args.config}: {desc}, L={L}, B={B}, delta={TOLERANCE[args.config]:g}",
                   "n": n, "k": k, "B": B, "L": L, "tolerance": TOLERANCE[args.config]},
        "cpu_baseline": {"value": ms, "unit": "ms", "cores": 1, "kind": "oracle",
                         "sample": f"{len(t)} full oracle transforms of the {args.config} workload "
                                   "(plan-time filter construction excluded), numpy single thread"},
        "e2e": {"value": ms, "unit": "ms", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)
    return 0


# ---------------------------------------------------------------------------
# GPU arm
# ---------------------------------------------------------------------------
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

    from paper_conf_ipps_wangcc16_b200 import Plan, default_B
    from paper_conf_ipps_wangcc16_b200.dist import CudaEngine, LoopShardedSfft, signal_range

    n, k, L, desc = CONFIGS[args.config]
    B = args.B or default_B(n, k)
    x_np, S, X = make_signal(n, k, args.signal_seed)
    x_pin = torch.from_numpy(x_np).pin_memory()
    x = x_pin.to(dev)

    flush_w = torch.empty(256 * 1024 * 1024, dtype=torch.uint8, device=dev)
    flush_r = torch.ones(64 * 1024 * 1024, dtype=torch.int32, device=dev)

    class _Flush:
        """L2 flush between timed steps: write 256 MiB (evicts everything), then
        read another 256 MiB so the write-backs happen here, not in the step."""

        @staticmethod
        def zero_():
            flush_w.zero_()
            flush_r.sum()

    flush = _Flush()

    # ---- dense cuFFT of the same n (context), complex128, L2 flushed; timed
    # before any plan exists, so cuFFT has the whole L2 (a staged plan holds a
    # persisting-L2 set-aside while it lives)
    dense = []
    for i in range(args.warmup + 10):
        flush.zero_()
        a = torch.cuda.Event(enable_timing=True)
        b = torch.cuda.Event(enable_timing=True)
        a.record(torch.cuda.current_stream())
        torch.fft.fft(x)
        b.record(torch.cuda.current_stream())
        torch.cuda.synchronize()
        if i >= args.warmup:
            dense.append(a.elapsed_time(b))
    dense_ms = statistics.median(dense)

    if world == 1:
        plan = Plan(n, k, B=B, L=L, seed=args.plan_seed, device=local_rank, tolerance=TOLERANCE[args.config])
        locs = torch.empty(k, dtype=torch.int64, device=dev)
        vals = torch.empty(k, dtype=torch.complex128, device=dev)

        def step():
            plan.execute(x, locs, vals)
            return locs, vals
        launches = plan.launches_per_execute()
    else:
        shard = 1 if args.shard == "signal" else 0
        eng = CudaEngine(n, k, B=B, L=L, rank=rank, world=world, device=local_rank, seed=args.plan_seed,
                         tolerance=TOLERANCE[args.config], shard_mode=shard)
        runner = LoopShardedSfft(eng)
        plan = eng.plan
        if shard:  # this rank holds only its slice of x
            lo, hi = signal_range(rank, n, world)
            x = x[lo:hi].clone()

        def step():
            return runner.execute(x)
        launches = eng.launches_per_execute()

    # correctness of the benchmarked configuration (untimed)
    l_out, v_out = step()
    torch.cuda.synchronize()
    status = plan.status()
    l_np, v_np = l_out.cpu().numpy(), v_out.cpu().numpy()
    exact = set(l_np.tolist()) == set(S.tolist())
    truth = dict(zip(S.tolist(), X.tolist()))
    got = {int(f): complex(v) for f, v in zip(l_np, v_np) if f >= 0}
    l1 = sum(abs(got.get(f, 0) - truth.get(f, 0)) for f in set(truth) | set(got)) / k

    stream = torch.cuda.current_stream()

    def barrier():
        if world > 1:
            dist.barrier()

    # warm-up (at least W steps and ~0.3 s so the clock sampler sees load)
    with ClockSampler(local_rank) as clocks:
        t0 = time.perf_counter()
        i = 0
        while i < args.warmup or time.perf_counter() - t0 < 0.3:
            flush.zero_()
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
            flush.zero_()                       # L2 flush, outside the step's events
            ev[s][0].record(stream)
            step()
            ev[s][1].record(stream)
        reg1.record(stream)
        torch.cuda.synchronize()
        barrier()
        # keep load on for the sampler a little longer
        t1 = time.perf_counter()
        while time.perf_counter() - t1 < 0.2:
            step()
        torch.cuda.synchronize()
    step_ms = [a.elapsed_time(b) for a, b in ev]
    ms = sum(step_ms) / len(step_ms)
    region_ms = reg0.elapsed_time(reg1)
    if world > 1:
        t = torch.tensor([ms], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = float(t.item())

    # ---- per-stage times inside the CUDA graph: T_s = time of the graph that
    # runs stages 1..s (cusfft_set_stage_limit), stage s = T_s - T_{s-1}.
    # T_1 is the fold kernel alone (+ an 8-int memset node): the roofline's
    # kernel time, measured with CUDA events on the plan's (current) stream.
    def timed_mean(reps):
        ts = []
        for _ in range(reps):
            flush.zero_()
            a = torch.cuda.Event(enable_timing=True)
            b = torch.cuda.Event(enable_timing=True)
            a.record(stream)
            step()
            b.record(stream)
            torch.cuda.synchronize()
            ts.append(a.elapsed_time(b))
        return sum(ts) / len(ts)

    names = ("fold", "fft", "cutoff", "vote", "estimate", "output")
    stage_ms = {}
    if world == 1:
        prev = 0.0
        reps = max(10, args.steps)
        for si, nm in enumerate(names, start=1):
            plan.set_stage_limit(si)
            step()
            tsi = timed_mean(reps)
            stage_ms[nm] = tsi - prev
            prev = tsi
        plan.set_stage_limit(6)
        fold_ms = stage_ms["fold"]
    else:
        plan.set_timing(True)
        acc = {nm: [] for nm in names}
        for _ in range(max(5, args.steps)):
            flush.zero_()
            step()
            st = plan.stage_times()
            for nm in names:
                acc[nm].append(st[nm])
        plan.set_timing(False)
        stage_ms = {nm: sum(v) / len(v) for nm, v in acc.items()}
        fold_ms = stage_ms["fold"]

    # ---- the gather kernel alone (phase 1 of the staged fold, k_stage*): events
    # recorded on the plan's stream right before and after its launch (timing
    # mode: direct launches, no graph), L2 flushed before every execution
    gather_ms = None
    if plan.info()["staged"]:
        plan.set_timing(True)
        g = []
        for _ in range(max(10, args.steps)):
            flush.zero_()
            step()
            g.append(plan.stage_times()["gather"])
        plan.set_timing(False)
        if all(v > 0 for v in g):
            gather_ms = sum(g) / len(g)


    # ---- e2e through the C ABI with host buffers (world == 1 path)
    e2e = None
    if world == 1:
        h_locs = torch.empty(k, dtype=torch.int64).pin_memory()
        h_vals = torch.empty(k, dtype=torch.complex128).pin_memory()
        for _ in range(2):
            plan.execute_host(x_pin, h_locs, h_vals)
        e_ms = []
        for _ in range(args.steps):
            flush.zero_()
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            plan.execute_host(x_pin, h_locs, h_vals)
            e_ms.append(1e3 * (time.perf_counter() - t0))
        e2e = {"value": sum(e_ms) / len(e_ms), "unit": "ms", "h2d_bytes_per_step": n * 16,
               "d2h_bytes_per_step": k * (8 + 16),
               "note": "cusfft_execute_host: pinned H2D of x, transform, D2H of locs/vals, host wall clock"}

    ablations = None
    if world == 1 and args.ablations:
        ablations = {}
        variants = [("cutoff_sort_alg3", dict(cutoff_mode=1), {}),
                    ("cutoff_threshold_alg6", dict(cutoff_mode=2, cutoff_threshold=1e-3), {}),
                    ("direct_gather_no_stage", {}, {"CUSFFT_NO_STAGE": "1"})]
        for name, kw, env in variants:
            old = {e: os.environ.get(e) for e in env}
            os.environ.update(env)
            try:
                p2 = Plan(n, k, B=B, L=L, seed=args.plan_seed, device=local_rank, tolerance=TOLERANCE[args.config], **kw)
            finally:
                for e, v in old.items():
                    if v is None:
                        os.environ.pop(e, None)
                    else:
                        os.environ[e] = v
            l2_, v2_ = torch.empty_like(locs), torch.empty_like(vals)

            def step2():
                p2.execute(x, l2_, v2_)
            for _ in range(3):
                step2()
            ts = []
            for _ in range(max(10, args.steps)):
                flush.zero_()
                a = torch.cuda.Event(enable_timing=True)
                b = torch.cuda.Event(enable_timing=True)
                a.record(stream)
                step2()
                b.record(stream)
                torch.cuda.synchronize()
                ts.append(a.elapsed_time(b))
            ok = set(l2_.cpu().tolist()) == set(S.tolist())
            ablations[name] = {"ms": sum(ts) / len(ts), "exact_recovery": ok, "status": p2.status()}
            p2.close()

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:  # N = 1 only (bench contract)
        times, _ = oracle_time(n, k, L, B, x_np, args.plan_seed, budget_s=args.cpu_budget_s, min_runs=1,
                               tolerance=TOLERANCE[args.config])
        cpu = {"value": 1e3 * sum(times) / len(times), "unit": "ms", "cores": 1, "kind": "oracle",
               "sample": f"{len(times)} full oracle transform(s) of the same {args.config} signal "
                         "(plan-time filter construction excluded), numpy single thread"}

    peak, peak_src = hbm_peak()
    info = plan.info()
    sector, useful = fold_bytes(plan.L // world if world > 1 else L, plan.w, B, int(info["sectors"]))
    # roofline kernel: the address-ordered permute gather (fold phase 1) when
    # the plan is staged -- it carries all of the fold's HBM traffic; phase 2
    # streams the staging buffer from L2 (reported as fold_stage below)
    gather_bytes = int(info["sectors"]) * 32
    rk_ms = gather_ms if gather_ms else fold_ms
    rk_bytes = gather_bytes if gather_ms else sector
    achieved = rk_bytes / (rk_ms * 1e-3) / 1e9
    traffic = None
    tf = os.path.join(ROOT, "profiles", f"fold_traffic_{args.config}.json")
    if os.path.exists(tf):
        try:
            with open(tf) as f:
                tj = json.load(f)
            parts = {kk.split("<")[0]: vv for kk, vv in tj.get("parts", {}).items()}
            traffic = (parts.get("k_stage_packed", {}).get("dram_bytes_per_launch")
                       if gather_ms else tj.get("dram_bytes_per_launch"))
        except Exception:
            traffic = None
    line = {
        "metric": METRIC, "value": ms, "unit": "ms", "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": False,
        "scaling": "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": {"workload": f"{args.config}: {desc}, L={L}, B={B}, w={plan.w} taps "
                               f"(Dolph-Chebyshev, delta={TOLERANCE[args.config]:g})",
                   "n": n, "k": k, "B": B, "L": L, "taps": plan.w, "tolerance": TOLERANCE[args.config],
                   "loc_loops": plan.loc_loops,
                   "vote_threshold": plan.T, "parallelism": f"{args.shard}-sharded x{world}" if world > 1 else "single GPU",
                   "l2": "flushed between timed steps (256 MiB write + 256 MiB read), outside the step events",
                   "signal_seed": args.signal_seed, "plan_seed": args.plan_seed},
        "gpu_launches": launches * args.steps,
        "timed_region_ms_incl_flush": region_ms,
        "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                     "frac": achieved / peak, "traffic": traffic,
                     "kernel": ("k_stage_packed (fold phase 1: address-ordered permute gather of x)" if gather_ms
                                else "fold stage (k_fold_fft1)"),
                     "algorithmic_bytes_per_launch": rk_bytes, "kernel_ms": rk_ms,
                     "algorithmic_bytes_note": "distinct 32-B sectors of x the plan's L*w gather positions touch x 32 B",
                     "peak_source": peak_src,
                     "fold_stage": {"kernels": "k_stage_packed + k_fold_fft1_tma" if info["staged"] else "k_fold_fft1",
                                    "ms": fold_ms, "algorithmic_bytes": sector, "useful_bytes": useful,
                                    "gbs": sector / (fold_ms * 1e-3) / 1e9,
                                    "frac": sector / (fold_ms * 1e-3) / 1e9 / peak,
                                    "note": "graph-prefix time (includes the graph launch)"}},
        "stage_ms": stage_ms,
        "ablations": ablations,
        "dense_cufft_ms": dense_ms, "speedup_vs_dense_cufft": dense_ms / ms,
        "accuracy": {"exact_recovery": exact, "l1_per_coefficient": l1, "status": status},
        "clocks": clocks.summary(),
        "e2e": e2e,
        "cpu_baseline": cpu,
        "paper_context": "cusFFT (K20x, fp64): 15x over cuFFT at n=2^27, >9x baseline (PAPER.md:L406)",
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
    plan = Plan(n, k, B=B, L=L, seed=args.plan_seed, device=local_rank, tolerance=TOLERANCE[args.config])
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

    def step():
        return drv.execute(xb) if len(mine) else (locs, vals)
    plan.execute_batch(xb, locs, vals)
    torch.cuda.synchronize()
    status = plan.status()
    exact = all(set(locs[i].cpu().tolist()) == set(sigs[i][1].tolist()) for i in range(len(mine)))
    flush_w = torch.empty(256 * 1024 * 1024, dtype=torch.uint8, device=dev)
    flush_r = torch.ones(64 * 1024 * 1024, dtype=torch.int32, device=dev)
    stream = torch.cuda.current_stream()

    def barrier():
        if world > 1:
            dist.barrier()
    with ClockSampler(local_rank) as clocks:
        for _ in range(args.warmup):
            flush_w.zero_(); flush_r.sum()
            plan.execute_batch(xb, locs, vals)
        torch.cuda.synchronize()
        ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
        barrier()
        torch.cuda.synchronize()
        for s_ in range(args.steps):
            flush_w.zero_(); flush_r.sum()
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
        "scaling": "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
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
    ap.add_argument("--shard", default="loops", choices=["loops", "signal"],
                    help="N>1: loop sharding (all-gather) or signal sharding (SURVEY N1, all-reduce)")
    ap.add_argument("--B", type=int, default=0, help="bucket count (default: the paper's formula, DESIGN.md Z3)")
    ap.add_argument("--pipeline", type=int, default=2, help="C5 batch: clone plans in flight per GPU")
    ap.add_argument("--cpu-budget-s", type=float, default=15.0)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--ablations", action="store_true",
                    help="also time the cutoff variants (Alg. 3 sort, Alg. 6 threshold) and the direct gather")
    args = ap.parse_args()
    if args.warmup < 3:
        args.warmup = 3
    if args.impl == "reference":
        return run_reference(args)
    if args.config in BATCH:
        return run_gpu_batch(args)
    return run_gpu(args)


if __name__ == "__main__":
    sys.exit(main())
