"""Multi-GPU execution (paper_conf_ipps_wangcc16_b200.dist): loop sharding
(all-gather) and signal sharding (sum all-reduce).

CPU (gloo, world_size 2): the exchange logic of LoopShardedSfft — loop
ownership, rank-major slot layout, one all-gather, rank-identical outputs —
driven with a test engine whose per-loop arithmetic is the oracle's (tests may
use the oracle; the product path never does).  GPU: two cusfft_plan_dist plans
(rank 0 and 1 of 2) on one device with the all-gather emulated by copies must
reproduce the single-GPU plan bit for bit.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle as O
from paper_conf_ipps_wangcc16_b200._binding import DEBUG_HITS as DEBUG_HITS_ID, DEBUG_WINNERS as DEBUG_WINNERS_ID
from paper_conf_ipps_wangcc16_b200.dist import LoopShardedSfft, loops_of_rank, signal_range, slot_of_loop
from paper_conf_ipps_wangcc16_b200.workload import planted_signal


def test_slot_mapping_is_a_rank_major_permutation():
    for L, world in [(16, 1), (16, 2), (16, 4), (16, 8), (12, 3)]:
        slots = [slot_of_loop(r, L, world) for r in range(L)]
        assert sorted(slots) == list(range(L))
        for g in range(world):
            mine = loops_of_rank(g, L, world)
            assert sorted(slot_of_loop(r, L, world) for r in mine) == list(range(g * L // world, (g + 1) * L // world))
            assert all(r % world == g for r in mine)
    with pytest.raises(ValueError):
        loops_of_rank(0, 10, 4)


class OracleEngine:
    """Test engine with the engine interface of dist.CudaEngine: per-loop
    records (u^_r as fp64 pairs, then the cutoff list J_r for location loops)
    in the rank-major exchange buffer; the oracle does the arithmetic."""

    def __init__(self, x, p: O.SfftParams, rank: int, world: int):
        self.x, self.p, self.rank, self.world = x, p, rank, world
        self.a, self.sigma, self.tau = O.draw_permutations(p.seed, p.n, p.L, p.tau_mode)
        self.g = O.filter_taps(p)
        self.Lg = p.L // world
        self.rec = p.B * 16 + p.num_select * 8
        self.buf = torch.zeros(world * self.Lg * self.rec, dtype=torch.uint8)

    def _slot_view(self, s):
        return self.buf[s * self.rec:(s + 1) * self.rec]

    def local(self, x):
        for r in loops_of_rank(self.rank, self.p.L, self.world):
            uh = O.bucket_fft(O.perm_filter(x, self.g, int(self.sigma[r]), int(self.tau[r]), self.p.B))
            J = O.cutoff(uh, self.p.num_select) if r < self.p.loc_loops else np.zeros(self.p.num_select, np.int64)
            rec = np.concatenate([uh.view(np.float64).view(np.uint8), J.astype(np.int64).view(np.uint8)])
            self._slot_view(slot_of_loop(r, self.p.L, self.world)).copy_(torch.from_numpy(rec))

    def exchange_tensor(self):
        return self.buf

    def finish(self):
        p = self.p
        uhat, J = [], []
        for r in range(p.L):
            rec = self._slot_view(slot_of_loop(r, p.L, self.world)).numpy()
            uhat.append(rec[:p.B * 16].view(np.complex128).copy())
            if r < p.loc_loops:
                J.append(rec[p.B * 16:].view(np.int64).copy())
        hits = np.sort(O.location_recovery(J, self.a[:p.loc_loops], p.n, p.B, p.vote_threshold))
        G = O.filter_response(self.g, p.n, p.n // p.B)
        vals, _ = O.estimate(hits, np.stack(uhat), self.sigma, self.tau, G, p.n, p.B)
        return O.select_output(hits, vals, p.k)


class OracleSignalEngine:
    """Signal-sharded test engine: this rank holds x[lo, hi) and folds only
    those samples for every loop (the oracle's Step 1-2 on the slice
    zero-extended to n), Step 3 on the partial buckets; the exchange buffer
    is the L x B partial spectra as float64, summed by the all-reduce."""

    exchange_kind = 1

    def __init__(self, p: O.SfftParams, rank: int, world: int):
        self.p, self.rank, self.world = p, rank, world
        self.a, self.sigma, self.tau = O.draw_permutations(p.seed, p.n, p.L, p.tau_mode)
        self.g = O.filter_taps(p)
        self.lo, self.hi = signal_range(rank, p.n, world)
        self.buf = torch.zeros(p.L * p.B * 2, dtype=torch.float64)

    def local(self, xs):
        assert len(xs) == self.hi - self.lo
        xz = np.zeros(self.p.n, np.complex128)
        xz[self.lo:self.hi] = xs
        for r in range(self.p.L):
            uh = O.bucket_fft(O.perm_filter(xz, self.g, int(self.sigma[r]), int(self.tau[r]), self.p.B))
            self.buf[r * 2 * self.p.B:(r + 1) * 2 * self.p.B] = torch.from_numpy(uh.view(np.float64))

    def exchange_tensor(self):
        return self.buf

    def finish(self):
        p = self.p
        uhat = self.buf.numpy().view(np.complex128).reshape(p.L, p.B)
        J = [O.cutoff(uhat[r], p.num_select) for r in range(p.loc_loops)]
        hits = np.sort(O.location_recovery(J, self.a[:p.loc_loops], p.n, p.B, p.vote_threshold))
        G = O.filter_response(self.g, p.n, p.n // p.B)
        vals, _ = O.estimate(hits, uhat, self.sigma, self.tau, G, p.n, p.B)
        return O.select_output(hits, vals, p.k)


class OracleTwoExchangeEngine:
    """Test engine for exchange kind 2 (shard_mode 2): local() writes this
    rank's location loops' winner lists J into its slice of buffer 1
    (int64 [world][cmax][num]); mid() votes over every gathered list (the
    hit set is identical on every rank; sorted), estimates this rank's loops
    for every hit into its slice of buffer 2 (complex128 as fp64 pairs,
    [world][HCAP][Lg]); finish() takes the medians over all loops and selects
    the output.  The arithmetic is the oracle's."""

    exchange_kind = 2
    HCAP = 256

    def __init__(self, x, p: O.SfftParams, rank: int, world: int):
        self.x, self.p, self.rank, self.world = x, p, rank, world
        self.a, self.sigma, self.tau = O.draw_permutations(p.seed, p.n, p.L, p.tau_mode)
        self.g = O.filter_taps(p)
        self.Lg = p.L // world
        self.cmax = -(-p.loc_loops // world)
        self.buf = torch.zeros(world * self.cmax * p.num_select, dtype=torch.int64)
        self.buf2 = torch.zeros(world * self.HCAP * self.Lg * 2, dtype=torch.float64)
        self.uhat = {}

    def local(self, x):
        p = self.p
        for i, r in enumerate(loops_of_rank(self.rank, p.L, self.world)):
            self.uhat[r] = O.bucket_fft(O.perm_filter(x, self.g, int(self.sigma[r]), int(self.tau[r]), p.B))
            if r < p.loc_loops:  # location loops are a prefix of the rank's loops
                c = (self.rank * self.cmax + i) * p.num_select
                self.buf[c:c + p.num_select] = torch.from_numpy(O.cutoff(self.uhat[r], p.num_select))

    def exchange_tensor(self):
        return self.buf

    def mid(self):
        p = self.p
        J = []
        for r in range(p.loc_loops):
            c = ((r % self.world) * self.cmax + r // self.world) * p.num_select
            J.append(self.buf[c:c + p.num_select].numpy().copy())
        self.hits = np.sort(O.location_recovery(J, self.a[:p.loc_loops], p.n, p.B, p.vote_threshold))
        assert len(self.hits) <= self.HCAP
        mine = loops_of_rank(self.rank, p.L, self.world)
        G = O.filter_response(self.g, p.n, p.n // p.B)
        _, per = O.estimate(self.hits, np.stack([self.uhat[r] for r in mine]), self.sigma[mine], self.tau[mine],
                            G, p.n, p.B)
        v = self.buf2.numpy().reshape(self.world, self.HCAP, self.Lg, 2)
        v[self.rank, :len(self.hits), :, 0] = per.real
        v[self.rank, :len(self.hits), :, 1] = per.imag

    def exchange_tensor2(self):
        return self.buf2

    def finish(self):
        p, H = self.p, len(self.hits)
        v = self.buf2.numpy().reshape(self.world, self.HCAP, self.Lg, 2)[:, :H]
        per = (v[..., 0] + 1j * v[..., 1]).transpose(1, 0, 2).reshape(H, p.L)  # loops in rank-major order
        med = (p.L - 1) // 2
        vals = np.sort(per.real, axis=1)[:, med] + 1j * np.sort(per.imag, axis=1)[:, med]
        return O.select_output(self.hits, vals, p.k)


def _two_worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        n, k = 2 ** 12, 6
        x, S, X = planted_signal(n, k, seed=4)
        p = O.make_params(n, k, L=8, loc_loops=5, vote_threshold=3, seed=9)
        locs, vals = LoopShardedSfft(OracleTwoExchangeEngine(x, p, rank, world)).execute(x)
        q.put((rank, locs.tolist(), vals.tolist()))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [1, 2, 4])
def test_loop_sharded_two_exchanges_gloo(world):
    """Exchange kind 2 (candidate records, then per-loop estimates): every
    rank's output equals the single-process oracle exactly."""
    n, k = 2 ** 12, 6
    x, S, X = planted_signal(n, k, seed=4)
    ref = O.sfft(x, O.make_params(n, k, L=8, loc_loops=5, vote_threshold=3, seed=9))
    if world == 1:
        p = O.make_params(n, k, L=8, loc_loops=5, vote_threshold=3, seed=9)
        locs, vals = LoopShardedSfft(OracleTwoExchangeEngine(x, p, 0, 1)).execute(x)
        assert np.array_equal(locs, ref.locs)
        np.testing.assert_array_equal(vals, ref.vals)
        return
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_two_worker, args=(r, world, port, q)) for r in range(world)]
    for pr in procs:
        pr.start()
    out = [q.get(timeout=300) for _ in range(world)]
    for pr in procs:
        pr.join(timeout=60)
        assert pr.exitcode == 0
    for rank, locs, vals in out:
        assert locs == ref.locs.tolist(), rank
        np.testing.assert_array_equal(np.array(vals), ref.vals)


def test_signal_range_partitions_x():
    for n, world in [(2 ** 12, 1), (2 ** 12, 2), (2 ** 12, 8)]:
        rs = [signal_range(g, n, world) for g in range(world)]
        assert rs[0][0] == 0 and rs[-1][1] == n
        assert all(rs[i][1] == rs[i + 1][0] for i in range(world - 1))
    with pytest.raises(ValueError):
        signal_range(0, 2 ** 12, 3)


def test_partial_folds_sum_to_full_fold():
    """The property signal sharding rests on: Steps 1-3 are linear in x, so
    the spectra of the range-restricted folds sum to the full one."""
    n, k = 2 ** 12, 6
    x, S, X = planted_signal(n, k, seed=6)
    p = O.make_params(n, k, L=3, seed=1)
    a, sigma, tau = O.draw_permutations(p.seed, n, p.L, p.tau_mode)
    g = O.filter_taps(p)
    for r in range(p.L):
        full = O.bucket_fft(O.perm_filter(x, g, int(sigma[r]), int(tau[r]), p.B))
        part = np.zeros_like(full)
        for rank in range(4):
            lo, hi = signal_range(rank, n, 4)
            xz = np.zeros_like(x)
            xz[lo:hi] = x[lo:hi]
            part += O.bucket_fft(O.perm_filter(xz, g, int(sigma[r]), int(tau[r]), p.B))
        np.testing.assert_allclose(part, full, rtol=0, atol=1e-12 * np.abs(full).max())


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        n, k = 2 ** 12, 6
        x, S, X = planted_signal(n, k, seed=4)
        p = O.make_params(n, k, L=8, loc_loops=5, vote_threshold=3, seed=9)
        eng = OracleEngine(x, p, rank, world)
        locs, vals = LoopShardedSfft(eng).execute(x)
        q.put((rank, locs.tolist(), vals.tolist()))
    finally:
        dist.destroy_process_group()


def _signal_worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        n, k = 2 ** 12, 6
        x, S, X = planted_signal(n, k, seed=4)
        p = O.make_params(n, k, L=7, loc_loops=5, vote_threshold=3, seed=9)  # world need not divide L
        lo, hi = signal_range(rank, n, world)
        locs, vals = LoopShardedSfft(OracleSignalEngine(p, rank, world)).execute(x[lo:hi])
        q.put((rank, locs.tolist(), vals.tolist()))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 4])
def test_signal_sharded_allreduce_gloo(world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_signal_worker, args=(r, world, port, q)) for r in range(world)]
    for pr in procs:
        pr.start()
    out = [q.get(timeout=300) for _ in range(world)]
    for pr in procs:
        pr.join(timeout=60)
        assert pr.exitcode == 0
    n, k = 2 ** 12, 6
    x, S, X = planted_signal(n, k, seed=4)
    ref = O.sfft(x, O.make_params(n, k, L=7, loc_loops=5, vote_threshold=3, seed=9))
    assert sorted(ref.locs.tolist()) == sorted(S.tolist())
    for rank, locs, vals in out:
        assert locs == ref.locs.tolist(), rank
        # the all-reduce sums partial spectra in another order: fp64 rounding only
        np.testing.assert_allclose(np.array(vals), ref.vals, rtol=1e-9, atol=1e-12)
        assert vals == out[0][2]  # every rank finishes from the same summed buffer


@pytest.mark.parametrize("world", [2, 4])
def test_loop_sharded_exchange_gloo(world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for pr in procs:
        pr.start()
    out = [q.get(timeout=300) for _ in range(world)]
    for pr in procs:
        pr.join(timeout=60)
        assert pr.exitcode == 0
    n, k = 2 ** 12, 6
    x, S, X = planted_signal(n, k, seed=4)
    ref = O.sfft(x, O.make_params(n, k, L=8, loc_loops=5, vote_threshold=3, seed=9))
    for rank, locs, vals in out:
        assert locs == ref.locs.tolist(), rank
        np.testing.assert_array_equal(np.array(vals), ref.vals)


def test_loop_sharded_world1_no_collective():
    n, k = 2 ** 12, 6
    x, S, X = planted_signal(n, k, seed=5)
    p = O.make_params(n, k, L=6, loc_loops=5, vote_threshold=3, seed=2)
    locs, vals = LoopShardedSfft(OracleEngine(x, p, 0, 1)).execute(x)
    ref = O.sfft(x, p)
    assert np.array_equal(locs, ref.locs)
    np.testing.assert_array_equal(vals, ref.vals)


@pytest.mark.gpu
@pytest.mark.parametrize("world", [2, 4])
def test_dist_plans_emulated_allgather_match_single_gpu(world):
    """cusfft_plan_dist ranks on one GPU; the all-gather is emulated by device
    copies between the ranks' exchange buffers."""
    from paper_conf_ipps_wangcc16_b200 import Plan
    from paper_conf_ipps_wangcc16_b200.dist import CudaEngine
    n, k, L = 2 ** 20, 100, 16
    x, S, X = planted_signal(n, k, seed=8)
    xd = torch.from_numpy(x).cuda()
    ref_l, ref_v = Plan(n, k, L=L, seed=5).execute(xd)
    engines = [CudaEngine(n, k, L=L, rank=r, world=world, seed=5) for r in range(world)]
    for e in engines:
        e.local(xd)
    torch.cuda.synchronize()
    per = engines[0].per_rank
    for dst in engines:
        for r, src in enumerate(engines):
            if src is not dst:
                dst.exchange_tensor()[r * per:(r + 1) * per].copy_(src.exchange_tensor()[r * per:(r + 1) * per])
    torch.cuda.synchronize()
    for e in engines:
        locs, vals = e.finish()
        torch.cuda.synchronize()
        assert e.plan.status() == 0
        assert torch.equal(locs, ref_l)
        assert torch.equal(vals, ref_v)


@pytest.mark.gpu
@pytest.mark.parametrize("world,n,k,L,Lloc", [(1, 2 ** 20, 100, 16, 8), (2, 2 ** 20, 100, 16, 8),
                                              (4, 2 ** 22, 1000, 16, 8), (8, 2 ** 18, 50, 16, 5)])
def test_two_exchange_plans_emulated_match_single_gpu(world, n, k, L, Lloc):
    """shard_mode 2 ranks on one GPU (candidate all-gather and estimate
    all-gather emulated by device copies) reproduce the single-GPU plan bit
    for bit, at world 1 through the whole-transform call as well."""
    from paper_conf_ipps_wangcc16_b200 import Plan
    from paper_conf_ipps_wangcc16_b200.dist import CudaEngine
    x, S, X = planted_signal(n, k, seed=8)
    xd = torch.from_numpy(x).cuda()
    kw = dict(seed=5, loc_loops=Lloc, vote_threshold=Lloc // 2 + 1, max_hits=8192)
    ref = Plan(n, k, L=L, debug=1, **kw)
    ref_l, ref_v = ref.execute(xd)
    if world == 1:
        one = Plan(n, k, L=L, shard_mode=2, debug=1, **kw)
        assert one.exchange_kind() == 2
        l1, v1 = one.execute(xd)
        torch.cuda.synchronize()
        assert one.status() == 0
        assert torch.equal(l1, ref_l) and torch.equal(v1, ref_v)
        h_ref = ref.debug(DEBUG_HITS_ID)
        assert np.array_equal(np.sort(h_ref), one.debug(DEBUG_HITS_ID))  # sorted hit list
        assert np.array_equal(ref.debug(DEBUG_WINNERS_ID), one.debug(DEBUG_WINNERS_ID))
    engines = [CudaEngine(n, k, L=L, rank=r, world=world, shard_mode=2, **kw) for r in range(world)]
    assert all(e.exchange_kind == 2 for e in engines)
    for rep in range(2):  # the second execution replays the captured graphs
        for e in engines:
            e.local(xd)
        torch.cuda.synchronize()
        for name, per in (("exchange_tensor", engines[0].per_rank), ("exchange_tensor2", engines[0].per_rank2)):
            if name == "exchange_tensor2":
                for e in engines:
                    e.mid()
                torch.cuda.synchronize()
            for dst in engines:
                for r, src in enumerate(engines):
                    if src is not dst:
                        getattr(dst, name)()[r * per:(r + 1) * per].copy_(getattr(src, name)()[r * per:(r + 1) * per])
            torch.cuda.synchronize()
        for e in engines:
            locs, vals = e.finish()
            torch.cuda.synchronize()
            assert e.plan.status() == 0
            assert torch.equal(locs, ref_l)
            assert torch.equal(vals, ref_v)


@pytest.mark.gpu
@pytest.mark.parametrize("world,n,k,L", [(2, 2 ** 20, 100, 16), (4, 2 ** 20, 100, 16), (8, 2 ** 18, 50, 12)])
def test_signal_sharded_plans_emulated_allreduce(world, n, k, L):
    """Signal-sharded cusfft_plan_dist ranks on one GPU, each given only its
    slice of x; the all-reduce is emulated by summing the ranks' exchange
    buffers (fp64).  Equal to the single-GPU plan: locations and winners
    exactly, values within fp64 rounding of the reordered sum."""
    from paper_conf_ipps_wangcc16_b200 import Plan
    from paper_conf_ipps_wangcc16_b200.dist import CudaEngine
    x, S, X = planted_signal(n, k, seed=11)
    xd = torch.from_numpy(x).cuda()
    ref = Plan(n, k, L=L, seed=3)
    ref_l, ref_v = ref.execute(xd)
    engines = [CudaEngine(n, k, L=L, rank=r, world=world, seed=3, shard_mode=1) for r in range(world)]
    assert all(e.exchange_kind == 1 for e in engines)
    if n == 2 ** 20:  # B = 2048: each rank stages (only) its own samples
        assert all(e.plan.info()["staged"] == 1 for e in engines)
    for r, e in enumerate(engines):
        lo, hi = signal_range(r, n, world)
        e.local(xd[lo:hi].clone())  # the rank holds only its slice
    torch.cuda.synchronize()
    total = sum(e.exchange_tensor().clone() for e in engines)
    for e in engines:
        e.exchange_tensor().copy_(total)
    torch.cuda.synchronize()
    for e in engines:
        locs, vals = e.finish()
        torch.cuda.synchronize()
        assert e.plan.status() == 0
        assert torch.equal(locs, ref_l)
        torch.testing.assert_close(vals, ref_v, rtol=1e-9, atol=1e-12 * float(ref_v.abs().max()))
        assert sorted(locs.tolist()) == sorted(S.tolist())
    # a second execution reuses the captured graphs
    for r, e in enumerate(engines):
        lo, hi = signal_range(r, n, world)
        e.local(xd[lo:hi].clone())
    torch.cuda.synchronize()
    total = sum(e.exchange_tensor().clone() for e in engines)
    for e in engines:
        e.exchange_tensor().copy_(total)
        locs, vals = e.finish()
        torch.cuda.synchronize()
        assert torch.equal(locs, ref_l)


# ---------------------------------------------------------------------------
# Batched independent signals (SURVEY.md §8(e) batched config): no collective
# on the data path; each rank transforms its contiguous share.
# ---------------------------------------------------------------------------
def test_batch_range_partitions_signals():
    from paper_conf_ipps_wangcc16_b200.dist import batch_range
    for count, world in [(64, 8), (64, 3), (5, 8), (0, 2), (7, 1)]:
        spans = [batch_range(g, count, world) for g in range(world)]
        assert spans[0][0] == 0 and spans[-1][1] == count
        for (a, b), (c, d) in zip(spans, spans[1:]):
            assert b == c
        sizes = [b - a for a, b in spans]
        assert max(sizes) - min(sizes) <= 1
    with pytest.raises(ValueError):
        batch_range(2, 4, 2)


class OracleBatchEngine:
    """execute_batch with the oracle's arithmetic (test infrastructure)."""

    def __init__(self, p):
        self.p = p

    def execute_batch(self, xb):
        outs = [O.sfft(np.asarray(x), self.p) for x in xb]
        return (torch.from_numpy(np.stack([o.locs for o in outs])),
                torch.from_numpy(np.stack([o.vals for o in outs])))


def _batch_worker(rank, world, port, q):
    from paper_conf_ipps_wangcc16_b200.dist import BatchShardedSfft
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        n, k, count = 2 ** 12, 6, 5
        xs = np.stack([planted_signal(n, k, seed=40 + b)[0] for b in range(count)])
        p = O.make_params(n, k, L=8, loc_loops=5, vote_threshold=3, seed=9)
        drv = BatchShardedSfft(OracleBatchEngine(p), count)
        locs, vals = drv.execute(xs[drv.lo:drv.hi])
        gl, gv = drv.gather_outputs(locs, vals)
        q.put((rank, drv.lo, drv.hi, gl.tolist(), gv.tolist()))
    finally:
        dist.destroy_process_group()


def test_batch_sharded_gloo():
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_batch_worker, args=(r, world, port, q)) for r in range(world)]
    for pr in procs:
        pr.start()
    out = sorted(q.get(timeout=300) for _ in range(world))
    for pr in procs:
        pr.join(timeout=60)
        assert pr.exitcode == 0
    n, k, count = 2 ** 12, 6, 5
    p = O.make_params(n, k, L=8, loc_loops=5, vote_threshold=3, seed=9)
    assert [(lo, hi) for _, lo, hi, _, _ in out] == [(0, 3), (3, 5)]
    for b in range(count):
        x, S, X = planted_signal(n, k, seed=40 + b)
        ref = O.sfft(x, p)
        for _, _, _, gl, gv in out:  # every rank holds every result after the (optional) gather
            assert gl[b] == ref.locs.tolist()
            np.testing.assert_array_equal(np.array(gv[b]), ref.vals)


# ---------------------------------------------------------------------------
# The CUDA engine through a real collective: world-size processes on the one
# test GPU, each with its own cusfft_plan_dist plan, exchanging over gloo
# (host-staged: no kernel waits on another process).  Every rank's output must
# equal the single-GPU plan's bit for bit (loop sharding, both kinds) or to
# fp64 rounding of the reordered sum (signal sharding).
# ---------------------------------------------------------------------------
def _cuda_worker(rank, world, port, q, mode):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_ipps_wangcc16_b200.dist import CudaEngine
        n, k, L = 2 ** 20, 100, 16
        x, S, X = planted_signal(n, k, seed=8)
        xd = torch.from_numpy(x).cuda()
        kw = dict(max_hits=4096) if mode == 2 else {}
        eng = CudaEngine(n, k, L=L, rank=rank, world=world, seed=5, shard_mode=mode, **kw)
        if mode == 1:
            lo, hi = signal_range(rank, n, world)
            xd = xd[lo:hi].clone()
        outs = []
        for _ in range(2):  # capture, then replay
            locs, vals = LoopShardedSfft(eng).execute(xd)
            torch.cuda.synchronize()
            outs.append((locs.cpu().tolist(), torch.view_as_real(vals).cpu().numpy().tolist(), eng.plan.status()))
        q.put((rank, outs))
    finally:
        dist.destroy_process_group()


@pytest.mark.gpu
@pytest.mark.parametrize("mode,world", [(0, 2), (2, 2), (1, 2), (0, 4), (2, 4)])
def test_cuda_engine_real_collective_gloo(mode, world):
    from paper_conf_ipps_wangcc16_b200 import Plan
    n, k, L = 2 ** 20, 100, 16
    x, S, X = planted_signal(n, k, seed=8)
    ref_l, ref_v = Plan(n, k, L=L, seed=5).execute(torch.from_numpy(x).cuda())
    torch.cuda.synchronize()
    ref_l, ref_v = ref_l.cpu().numpy(), ref_v.cpu().numpy()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_cuda_worker, args=(r, world, port, q, mode)) for r in range(world)]
    for pr in procs:
        pr.start()
    out = [q.get(timeout=600) for _ in range(world)]
    for pr in procs:
        pr.join(timeout=120)
        assert pr.exitcode == 0
    for rank, runs in out:
        for locs, vals, status in runs:
            assert status == 0
            v = np.array(vals)[:, 0] + 1j * np.array(vals)[:, 1]
            assert locs == ref_l.tolist(), (rank, mode)
            if mode == 1:  # the all-reduce sums partial spectra in another order
                np.testing.assert_allclose(v, ref_v, rtol=1e-9, atol=1e-12 * np.abs(ref_v).max())
            else:
                np.testing.assert_array_equal(v, ref_v)
