"""Loop-sharded multi-GPU execution (one process per GPU, torch.distributed).

The L loops of the sFFT are independent until the vote and all
share B and the filter (one batched B-point FFT, L232), so rank g of G runs
Steps 1-4 for the loops r with r mod G == g on a replicated signal.  The only
exchange is ONE all-gather of the per-loop records (u^_r, the cutoff bitmap
and winner list of location loops) over NCCL / NVLink; then every rank runs
the vote, the estimation and the output selection redundantly, so outputs are
identical on all ranks and identical to the single-GPU plan (the loop draws
depend only on (seed, r)).  See DESIGN.md §7.

The engine interface keeps the exchange logic independent of the compute
engine, so the gloo CPU tests drive this exact code with a test engine:
  engine.local(x)            Steps 1-4 for this rank's loops
  engine.exchange_tensor()   the all-gather buffer (uint8 [world * per_rank])
  engine.finish()            Steps 5-6 + output, returns (locs, vals)
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


class _CudaBuffer:
    """__cuda_array_interface__ view of a device allocation owned by the plan."""

    def __init__(self, ptr: int, nbytes: int):
        self.__cuda_array_interface__ = {
            "shape": (nbytes,), "typestr": "|u1", "data": (ptr, False), "version": 3, "strides": None,
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
        self._buf = torch.as_tensor(_CudaBuffer(ptr, per * world), device=self.device)
        self.locs = torch.empty(k, dtype=torch.int64, device=self.device)
        self.vals = torch.empty(k, dtype=torch.complex128, device=self.device)

    def local(self, x):
        self.plan.execute_local(x)

    def exchange_tensor(self):
        return self._buf

    def finish(self):
        self.plan.execute_finish(self.locs, self.vals)
        return self.locs, self.vals

    def launches_per_execute(self) -> int:
        return self.plan.launches_per_execute()


class LoopShardedSfft:
    """execute(x) = local Steps 1-4, one all-gather, then Steps 5-6 everywhere."""

    def __init__(self, engine, group=None):
        self.engine = engine
        self.group = group
        self.world = dist.get_world_size(group) if dist.is_initialized() else 1
        self.rank = dist.get_rank(group) if dist.is_initialized() else 0

    def execute(self, x):
        self.engine.local(x)
        if self.world > 1:
            buf = self.engine.exchange_tensor()
            per = buf.numel() // self.world
            mine = buf[self.rank * per:(self.rank + 1) * per]
            # in place: input is this rank's slice of the output (NCCL in-place all-gather)
            dist.all_gather_into_tensor(buf, mine, group=self.group)
        return self.engine.finish()


__all__ = ["loops_of_rank", "slot_of_loop", "CudaEngine", "LoopShardedSfft"]
