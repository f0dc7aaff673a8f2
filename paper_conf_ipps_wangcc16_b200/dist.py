"""Multi-GPU execution (one process per GPU, torch.distributed).

Two shardings:

* loops (default) --
The L loops of the sFFT are independent until the vote and all
share B and the filter (one batched B-point FFT, L232), so rank g of G runs
Steps 1-4 for the loops r with r mod G == g on a replicated signal.  The only
exchange is ONE all-gather of the per-loop records (u^_r, the cutoff bitmap
and winner list of location loops) over NCCL / NVLink; then every rank runs
the vote, the estimation and the output selection redundantly, so outputs are
identical on all ranks and identical to the single-GPU plan (the loop draws
depend only on (seed, r)).

* loops, two collectives (``shard_mode=2``, the
north_star's design) -- the same loop ownership; exchange #1 all-gathers
only the location loops' candidate records (cutoff bitmap, count, winner
list J); every rank votes (identical hit set) and estimates ITS loops for
every hit; exchange #2 all-gathers those per-loop estimates; every rank takes
the medians and selects the output.  Bit-identical to the single-GPU plan.

* signal (``shard_mode=1``) -- rank g holds only the slice
x[g n/G, (g+1) n/G) and folds the samples it owns for ALL L loops (Step 1-2
restricted to its range; PAPER.md:L92 -- the fold is a sum over samples, and the
B-point FFT of Step 3 is linear, so the partial bucket spectra add).  The
exchange is ONE sum all-reduce (fp64) of the per-loop spectra; every rank then
runs the cutoff, vote, estimation and output.  x never has to be replicated
(n up to G x the single-GPU memory); outputs equal the single-GPU plan up to
fp64 rounding of the sum order.

The engine interface keeps the exchange logic independent of the compute
engine, so the gloo CPU tests drive this exact code with a test engine:
  engine.local(x)            Steps 1-4 for this rank's loops
  engine.exchange_tensor()   the exchange buffer (uint8 [world * per_rank] for
                             the all-gather; float64 [...] for the all-reduce)
  engine.exchange_kind       0 = all-gather (loops), 1 = sum all-reduce (signal),
                             2 = two all-gathers (loops, shard_mode 2)
  engine.mid()               kind 2 only: vote + this rank's per-loop estimates
  engine.exchange_tensor2()  kind 2 only: the per-loop estimate buffer
  engine.finish()            Steps 4-6 + output (kind 2: medians + output), returns (locs, vals)
"""
from __future__ import annotations


import torch
import torch.distributed as dist


def loops_of_rank(rank: int, L: int, world: int):
    """Loops rank `rank` computes: r = i * world + rank, i < L / world."""
    if L % world:
        raise ValueError("world must divide L")
    return [i * world + rank for i in range(L // world)]


def slot_of_loop(r: int, L: int, world: int) -> int:
    """Position of loop r in the rank-major exchange buffer."""
    return (r % world) * (L // world) + r // world


def signal_range(rank: int, n: int, world: int):
    """Samples [lo, hi) of x rank `rank` holds under signal sharding."""
    if n % world:
        raise ValueError("world must divide n")
    span = n // world
    return rank * span, (rank + 1) * span


class _CudaBuffer:
    """__cuda_array_interface__ view of a device allocation owned by the plan."""

    def __init__(self, ptr: int, nbytes: int, typestr: str = "|u1", itemsize: int = 1):
        self.__cuda_array_interface__ = {
            "shape": (nbytes // itemsize,), "typestr": typestr, "data": (ptr, False), "version": 3, "strides": None,
        }


class CudaEngine:
    """The CUDA library behind the engine interface (a cusfft_plan_dist plan)."""

    def __init__(self, n, k, B=None, L=16, rank=0, world=1, device=None, **params):
        from ._binding import Plan
        if device is None:
            device = torch.cuda.current_device()
        self.device = torch.device("cuda", device)
        self.plan = Plan(n, k, B=B, L=L, rank=rank, world=world, device=device, **params)
        ptr, per = self.plan.exchange_buffer()
        self.per_rank = per
        self.exchange_kind = self.plan.exchange_kind()
        if self.exchange_kind == 1:  # the whole buffer, summed as float64
            self._buf = torch.as_tensor(_CudaBuffer(ptr, per, "<f8", 8), device=self.device)
        else:
            self._buf = torch.as_tensor(_CudaBuffer(ptr, per * world), device=self.device)
        self._buf2 = None
        if self.exchange_kind == 2:
            ptr2, per2 = self.plan.exchange_buffer2()
            self.per_rank2 = per2
            self._buf2 = torch.as_tensor(_CudaBuffer(ptr2, per2 * world), device=self.device)
        self.locs = torch.empty(k, dtype=torch.int64, device=self.device)
        self.vals = torch.empty(k, dtype=torch.complex128, device=self.device)

    def local(self, x):
        """x: the whole signal (loop sharding) or this rank's slice (signal sharding)."""
        self.plan.execute_local(x)

    def exchange_tensor(self):
        return self._buf

    def mid(self):
        self.plan.execute_mid()

    def exchange_tensor2(self):
        return self._buf2

    def finish(self):
        self.plan.execute_finish(self.locs, self.vals)
        return self.locs, self.vals

    def launches_per_execute(self) -> int:
        return self.plan.launches_per_execute()


def _host_staged(buf, group) -> bool:
    """gloo exchanges host tensors: a device buffer goes through host memory
    (multi-process tests on one GPU; NCCL exchanges device memory directly)."""
    return buf.is_cuda and dist.get_backend(group) == "gloo"


def _all_gather_inplace(buf, rank, world, group):
    per = buf.numel() // world
    if _host_staged(buf, group):
        h = buf.cpu()
        dist.all_gather_into_tensor(h, h[rank * per:(rank + 1) * per].clone(), group=group)
        buf.copy_(h)
        return
    # in place: input is this rank's slice of the output (NCCL in-place all-gather)
    dist.all_gather_into_tensor(buf, buf[rank * per:(rank + 1) * per], group=group)


def _all_reduce_sum(buf, group):
    if _host_staged(buf, group):
        h = buf.cpu()
        dist.all_reduce(h, op=dist.ReduceOp.SUM, group=group)
        buf.copy_(h)
        return
    dist.all_reduce(buf, op=dist.ReduceOp.SUM, group=group)


class LoopShardedSfft:
    """execute(x) = local steps, the engine's exchange (kind 0: one all-gather
    of the per-loop records; 1: one sum all-reduce of the partial spectra;
    2: all-gather of the candidate records, the vote and this rank's per-loop
    estimates, all-gather of those), then the remaining steps on every rank.
    x is the whole signal or this rank's slice, as the engine expects."""

    def __init__(self, engine, group=None):
        self.engine = engine
        self.group = group
        self.world = dist.get_world_size(group) if dist.is_initialized() else 1
        self.rank = dist.get_rank(group) if dist.is_initialized() else 0

    def execute(self, x):
        self.engine.local(x)
        kind = getattr(self.engine, "exchange_kind", 0)
        if kind == 2:
            if self.world > 1:
                _all_gather_inplace(self.engine.exchange_tensor(), self.rank, self.world, self.group)
            self.engine.mid()
            if self.world > 1:
                _all_gather_inplace(self.engine.exchange_tensor2(), self.rank, self.world, self.group)
            return self.engine.finish()
        if self.world > 1:
            buf = self.engine.exchange_tensor()
            if kind == 1:
                _all_reduce_sum(buf, self.group)
                return self.engine.finish()
            _all_gather_inplace(buf, self.rank, self.world, self.group)
        return self.engine.finish()


def batch_range(rank: int, count: int, world: int):
    """Signals [lo, hi) of a batch of `count` independent signals owned by
    `rank` (batched configuration): contiguous, sizes differ by
    at most one, every signal owned once."""
    if world < 1 or not 0 <= rank < world or count < 0:
        raise ValueError("bad rank / world / count")
    base, extra = divmod(count, world)
    lo = rank * base + min(rank, extra)
    return lo, lo + base + (1 if rank < extra else 0)


class BatchShardedSfft:
    """Independent signals sharded across ranks with NO collective on the data
    path: rank g transforms signals batch_range(g, count, world) with its own
    single-GPU plan (engine.execute_batch).  gather_outputs() is optional output
    plumbing (an all-gather of the k-sparse results), outside the transform."""

    def __init__(self, engine, count: int, group=None):
        self.engine = engine
        self.count = int(count)
        self.group = group
        self.world = dist.get_world_size(group) if dist.is_initialized() else 1
        self.rank = dist.get_rank(group) if dist.is_initialized() else 0
        self.lo, self.hi = batch_range(self.rank, self.count, self.world)

    def execute(self, xb_local):
        """xb_local: this rank's signals [hi - lo, n].  Returns its (locs, vals)."""
        if xb_local.shape[0] != self.hi - self.lo:
            raise ValueError("xb_local must hold exactly this rank's signals")
        return self.engine.execute_batch(xb_local)

    def gather_outputs(self, locs, vals):
        """All ranks' (locs, vals) in batch order (pads ranks to the largest share)."""
        if self.world == 1:
            return locs, vals
        share = -(-self.count // self.world)
        k = locs.shape[1]
        pl = locs.new_full((share, k), -1)
        pv = vals.new_zeros((share, k))
        pl[:locs.shape[0]] = locs
        pv[:vals.shape[0]] = vals
        al = [torch.empty_like(pl) for _ in range(self.world)]
        av = [torch.empty_like(pv) for _ in range(self.world)]
        dist.all_gather(al, pl, group=self.group)
        dist.all_gather(av, pv, group=self.group)
        out_l, out_v = [], []
        for g in range(self.world):
            lo, hi = batch_range(g, self.count, self.world)
            out_l.append(al[g][:hi - lo])
            out_v.append(av[g][:hi - lo])
        return torch.cat(out_l), torch.cat(out_v)


__all__ = ["loops_of_rank", "slot_of_loop", "signal_range", "batch_range", "CudaEngine", "LoopShardedSfft",
           "BatchShardedSfft"]
