"""CUDA path vs the CPU oracle, through the C ABI (-m gpu).

Bars: integer/index results (draws, cutoff winners, hits,
output locations) bit-exact; the fold bit-exact when both sides use the same
taps (same per-bucket addition order, no FMA); floating-point values within
1e-9 relative (north_star).  Near-ties in the cutoff (relative gap < 1e-12
between the num-th and (num+1)-th |u^|^2) are reported, not failed.
"""
import os

import numpy as np
import pytest

torch = pytest.importorskip("torch")

import oracle as O  # noqa: E402
from paper_conf_ipps_wangcc16_b200 import (  # noqa: E402
    DEBUG_GHAT, DEBUG_HIT_VALS, DEBUG_HITS, DEBUG_NUM_HITS, DEBUG_PER_LOOP, DEBUG_TAPS, DEBUG_U,
    DEBUG_UHAT, DEBUG_WINNERS, Plan)
from paper_conf_ipps_wangcc16_b200 import _binding as b  # noqa: E402
from paper_conf_ipps_wangcc16_b200.workload import dense_signal, planted_signal  # noqa: E402

pytestmark = pytest.mark.gpu
DEV = "cuda:0"
REL = 1e-9


def _oracle_params(n, k, B, L, **kw):
    okw = {key: kw[key] for key in ("loc_loops", "vote_threshold", "num_select", "filter", "tolerance",
                                    "lobefrac", "loc_tolerance", "loc_lobefrac", "tau_mode", "seed",
                                    "cutoff_mode", "cutoff_threshold") if key in kw}
    return O.make_params(n, k, B=B, L=L, **okw)


def run_pair(x, n, k, B=None, L=16, shared_taps=False, **kw):
    B = B or O.default_B(n, k)
    p = _oracle_params(n, k, B, L, **kw)
    taps = O.filter_taps(p) if shared_taps else None
    ref = O.sfft(x, p, taps=taps)
    plan = Plan(n, k, B=B, L=L, debug=1, taps=taps, **kw)
    xd = torch.from_numpy(np.ascontiguousarray(x)).to(DEV)
    locs, vals = plan.execute(xd)
    torch.cuda.synchronize()
    return plan, ref, locs.cpu().numpy(), vals.cpu().numpy()


def _near_tie(uhat_r, num):
    m2 = np.sort(uhat_r.real * uhat_r.real + uhat_r.imag * uhat_r.imag)[::-1]
    if num >= m2.shape[0]:
        return False
    a, c = m2[num - 1], m2[num]
    return a == 0 or (a - c) / a < 1e-12


def check_all(plan, ref, locs, vals, fold_bit_exact):
    assert plan.status() == 0
    info = plan.info()
    assert np.array_equal(info["a"], ref.a) and np.array_equal(info["sigma"], ref.sigma)
    assert np.array_equal(info["tau"], ref.tau)
    u = plan.debug(DEBUG_U)
    if fold_bit_exact:
        assert np.array_equal(u, ref.u), "fold not bit-exact"
    else:
        scale = np.abs(ref.u).max()
        assert np.abs(u - ref.u).max() <= 1e-12 * scale + 1e-300
    uh = plan.debug(DEBUG_UHAT)
    scale = np.maximum(np.abs(ref.uhat).max(axis=1, keepdims=True), 1e-300)
    assert (np.abs(uh - ref.uhat) / scale).max() <= 1e-12
    win = plan.debug(DEBUG_WINNERS)
    ties = 0
    thr = plan.params.cutoff_threshold if plan.params.cutoff_mode == 2 else None
    for r in range(plan.loc_loops):
        got = win[r][win[r] >= 0]
        if not np.array_equal(got, ref.J[r]):
            if thr is None:
                assert _near_tie(ref.uhat[r], plan.num), f"winners differ in loop {r}"
            else:  # Alg. 6: only buckets within rounding of the threshold may differ
                diff = np.setxor1d(got, ref.J[r])
                m2 = np.abs(ref.uhat[r][diff]) ** 2
                assert np.all(np.abs(m2 - thr) <= 1e-12 * thr), f"winners differ in loop {r}"
            ties += 1
    if ties:
        pytest.skip(f"{ties} near-tied cutoff(s); downstream comparison not meaningful")
    hits = plan.debug(DEBUG_HITS)
    assert plan.debug(DEBUG_NUM_HITS)[0] == len(ref.hits)
    order = np.argsort(hits)
    assert np.array_equal(hits[order], ref.hits)
    hv = plan.debug(DEBUG_HIT_VALS)[order]
    assert_close(hv, ref.hit_vals)
    pl = plan.debug(DEBUG_PER_LOOP)
    if pl.size:
        assert_close(pl[order], ref.per_loop)
    assert np.array_equal(locs, ref.locs)
    assert_close(vals, ref.vals)


def assert_close(got, want):
    """|got - want| <= 1e-9 |want| + 1e-12 max|want|: 1e-9 relative on every
    coefficient (north_star) plus an absolute floor for values at the rounding
    noise of the B-point FFT, whose error is normwise (~1e-15 max|u^|)."""
    scale = np.abs(want).max() if want.size else 0.0
    err = np.abs(got - want)
    bound = REL * np.abs(want) + 1e-12 * scale
    assert np.all(err <= bound), float((err / np.maximum(bound, 1e-300)).max())


CASES = [
    # (n, k, B, L, extra)
    (2 ** 14, 8, None, 16, {}),                       # C1
    (2 ** 16, 32, None, 16, {}),
    (2 ** 16, 32, 512, 8, dict(loc_loops=8, vote_threshold=5)),
    (2 ** 18, 100, 4096, 16, {}),                     # two-pass FFT, B1 = B2 = 64
    (2 ** 20, 100, None, 16, {}),                     # C2
    (2 ** 16, 20, None, 5, dict(loc_loops=5, vote_threshold=3)),   # odd L
    (2 ** 16, 20, None, 12, dict(filter=1)),          # Gaussian filter
    (2 ** 16, 20, None, 16, dict(tau_mode=0)),        # Alg. 2 literal tau = 0
    (2 ** 15, 1, None, 16, {}),                       # k = 1
    (2 ** 16, 32, None, 16, dict(loc_loops=8, vote_threshold=4)),   # vote: no pair enumeration (T <= L_loc/2)
    (2 ** 16, 32, None, 14, dict(loc_loops=7, vote_threshold=5)),   # vote: pairs + odd singleton loop
    (2 ** 16, 32, None, 16, dict(loc_loops=12, vote_threshold=7)),  # tail: 16-bit vote table (L_loc > 8)
    (2 ** 16, 32, None, 24, dict(loc_loops=20, vote_threshold=11)),  # tail: 32-bit table, warp-per-hit estimate (L > 16)
    (2 ** 21, 60, 32768, 8, dict(loc_loops=6, vote_threshold=4)),   # B > 16384, q0 enumeration (T <= L_loc/2)
    (2 ** 18, 100, 4096, 16, dict(gather=2)),         # the paper's remap + execute
    (2 ** 16, 20, None, 5, dict(loc_loops=5, vote_threshold=3, gather=2)),  # remap, odd L, one-pass FFT
]


@pytest.mark.parametrize("n,k,B,L,extra", CASES)
def test_parity_shared_taps(n, k, B, L, extra):
    x, S, X = planted_signal(n, k, seed=n % 97 + k)
    plan, ref, locs, vals = run_pair(x, n, k, B, L, shared_taps=True, seed=11, **extra)
    check_all(plan, ref, locs, vals, fold_bit_exact=True)


@pytest.mark.parametrize("gs", [1, 3, 8])
def test_parity_stage_groups_shared_taps(gs, monkeypatch):
    """Stage groups (the staged gather of C4-sized plans, forced here at n =
    2^18): every group's fold stays bit-exact with the oracle's Alg. 1 order."""
    monkeypatch.setenv("CUSFFT_STAGE_GROUP", str(gs))
    n, k, B, L = 2 ** 18, 100, 4096, 16
    x, S, X = planted_signal(n, k, seed=77)
    plan, ref, locs, vals = run_pair(x, n, k, B, L, shared_taps=True, seed=11)
    assert plan.info()["staged"] == {1: 16, 3: 6, 8: 2}[gs]
    check_all(plan, ref, locs, vals, fold_bit_exact=True)


@pytest.mark.parametrize("n,k,B,L,extra", CASES[:6])
def test_parity_own_filter(n, k, B, L, extra):
    """The plan builds its own filter on the GPU; the oracle builds its own."""
    x, S, X = planted_signal(n, k, seed=3 + k)
    plan, ref, locs, vals = run_pair(x, n, k, B, L, shared_taps=False, seed=5, **extra)
    check_all(plan, ref, locs, vals, fold_bit_exact=False)


@pytest.mark.parametrize("mode,extra", [(1, {}), (2, dict(cutoff_threshold=1e-3)), (2, dict(cutoff_threshold=0.05))])
@pytest.mark.parametrize("n,k,B", [(2 ** 14, 8, None), (2 ** 16, 32, None), (2 ** 20, 100, None), (2 ** 18, 100, 4096)])
def test_parity_cutoff_modes(mode, extra, n, k, B):
    """Alg. 3 sort & select and Alg. 6 threshold cutoffs vs the oracle's."""
    x, S, X = planted_signal(n, k, seed=17 + k)
    plan, ref, locs, vals = run_pair(x, n, k, B, 16, shared_taps=True, seed=13, cutoff_mode=mode, **extra)
    check_all(plan, ref, locs, vals, fold_bit_exact=True)
    assert set(locs.tolist()) == set(S.tolist())


@pytest.mark.parametrize("filt", [0, 1])
@pytest.mark.parametrize("n,k", [(2 ** 14, 8), (2 ** 20, 100), (2 ** 24, 1000)])
def test_filter_construction(filt, n, k):
    p = O.make_params(n, k, filter=filt)
    g = O.filter_taps(p)
    G = O.filter_response(g, n, n // p.B)
    plan = Plan(n, k, B=p.B, L=2, filter=filt)
    gg = plan.debug(DEBUG_TAPS)
    assert gg.shape == g.shape
    assert np.abs(gg - g).max() <= 1e-12 * np.abs(g).max()
    GG = plan.debug(DEBUG_GHAT)
    assert np.abs(GG - G).max() <= 1e-12


def test_parity_noisy():
    n, k = 2 ** 20, 100
    x, S, X = planted_signal(n, k, seed=4, snr_db=20.0)
    plan, ref, locs, vals = run_pair(x, n, k, None, 16, shared_taps=True, seed=2)
    check_all(plan, ref, locs, vals, fold_bit_exact=True)


def test_parity_dense_signal_all_ties_free():
    """A dense random signal (no sparsity): many hits, exercises vote/estimate/output at scale."""
    n, k = 2 ** 16, 64
    x = dense_signal(n, 9)
    plan, ref, locs, vals = run_pair(x, n, k, 256, 16, shared_taps=True, seed=3)
    check_all(plan, ref, locs, vals, fold_bit_exact=True)


def test_zero_signal_ties():
    """x = 0: every |u^|^2 ties, so the cutoff keeps buckets 0..num-1 and the
    output keeps the k smallest hits (ties to the smaller f) — both sides."""
    n, k = 2 ** 12, 4
    x = np.zeros(n, dtype=np.complex128)
    plan, ref, locs, vals = run_pair(x, n, k, 64, 8, shared_taps=True, seed=1)
    win = plan.debug(DEBUG_WINNERS)
    assert all(np.array_equal(w, np.arange(plan.num)) for w in win)
    check_all(plan, ref, locs, vals, fold_bit_exact=True)
    assert np.all(vals == 0)


@pytest.mark.parametrize("B", [8192, 16384])
def test_fft2_select_crowded_fallback(B):
    """Shapes of the fused FFT-pass-2 + cutoff cluster kernel (k_fft2_select):
    x = 0 puts every key of a slot in the boundary bin (the fallback to the
    single-CTA selection inside the cluster kernel), a dense signal puts
    hundreds of keys there (more than the per-CTA candidate cap); both match
    the oracle's winners (ties to the smaller bucket) and outputs."""
    n, k = 2 ** 18, 64
    x = np.zeros(n, dtype=np.complex128)
    plan, ref, locs, vals = run_pair(x, n, k, B, 8, shared_taps=True, seed=1)
    win = plan.debug(DEBUG_WINNERS)
    assert all(np.array_equal(w, np.arange(plan.num)) for w in win)
    check_all(plan, ref, locs, vals, fold_bit_exact=True)
    x = dense_signal(n, 12)
    plan, ref, locs, vals = run_pair(x, n, k, B, 8, shared_taps=True, seed=2)
    check_all(plan, ref, locs, vals, fold_bit_exact=True)


def test_num_select_equals_B():
    n, k = 2 ** 10, 4
    x, S, X = planted_signal(n, k, seed=1)
    plan, ref, locs, vals = run_pair(x, n, k, 16, 6, shared_taps=True, seed=1, num_select=16,
                                     loc_loops=3, vote_threshold=2)
    check_all(plan, ref, locs, vals, fold_bit_exact=True)


@pytest.mark.parametrize("tol,B", [(1e-8, None), (1e-7, None), (1e-7, 8192)])
def test_C3_full_size_parity_and_recovery(tol, B):
    """BASELINE.json configs[2]: n = 2^24, k = 1000, L = 16, in the bench's launch
    config (delta = 1e-7, staged fold), at the library default delta, and with
    half the formula's buckets (B = 8192, DESIGN.md §3 study)."""
    n, k = 2 ** 24, 1000
    x, S, X = planted_signal(n, k, seed=1)
    plan, ref, locs, vals = run_pair(x, n, k, B, 16, shared_taps=False, seed=3, tolerance=tol)
    assert plan.info()["staged"] == 1
    check_all(plan, ref, locs, vals, fold_bit_exact=False)
    assert set(locs.tolist()) == set(S.tolist())
    assert O.l1_error(locs, vals, S, X, k) <= 1e-6


@pytest.mark.parametrize("n,k", [(2 ** 14, 8), (2 ** 20, 100), (2 ** 22, 500)])
def test_planted_recovery_many_seeds(n, k):
    plan = Plan(n, k, L=16, seed=21, num_select=2 * k if n == 2 ** 14 else k)
    worst = 0.0
    for s in range(6):
        x, S, X = planted_signal(n, k, seed=100 + s)
        locs, vals = plan.execute(torch.from_numpy(x).to(DEV))
        locs, vals = locs.cpu().numpy(), vals.cpu().numpy()
        assert set(locs.tolist()) == set(S.tolist())
        worst = max(worst, O.l1_error(locs, vals, S, X, k))
    assert worst <= 1e-6


def test_execute_host_matches_device():
    n, k = 2 ** 16, 16
    x, S, X = planted_signal(n, k, seed=5)
    plan = Plan(n, k, L=16, seed=4)
    l1, v1 = plan.execute(torch.from_numpy(x).to(DEV))
    xh = torch.from_numpy(x).pin_memory()
    l2, v2 = plan.execute_host(xh)
    assert np.array_equal(l1.cpu().numpy(), l2)
    assert np.array_equal(v1.cpu().numpy(), v2)
    l3, v3 = plan.execute_host(x)          # pageable numpy
    assert np.array_equal(l2, l3) and np.array_equal(v2, v3)


def test_execute_host_zero_copy_staged():
    """A staged plan reads a pinned host signal in place over PCIe
    (include/cusfft.h): the outputs equal the device-input path, and a second
    signal written into the same pinned buffer is the one transformed next."""
    n, k = 2 ** 22, 1000
    x1, S1, _ = planted_signal(n, k, seed=41)
    x2, S2, _ = planted_signal(n, k, seed=42)
    plan = Plan(n, k, L=16, seed=4)
    assert plan.info()["staged"]
    xh = torch.from_numpy(x1).pin_memory()
    for x, S in ((x1, S1), (x2, S2)):
        xh.copy_(torch.from_numpy(x))
        lh, vh = plan.execute_host(xh)
        ld, vd = plan.execute(torch.from_numpy(x).to(DEV))
        torch.cuda.synchronize()
        assert np.array_equal(ld.cpu().numpy(), lh) and np.array_equal(vd.cpu().numpy(), vh)
        assert sorted(lh.tolist()) == sorted(S.tolist())


def test_repeat_and_stream_semantics():
    n, k = 2 ** 16, 16
    x, S, X = planted_signal(n, k, seed=6)
    plan = Plan(n, k, L=16, seed=4)
    xd = torch.from_numpy(x).to(DEV)
    l1, v1 = plan.execute(xd)
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        l2, v2 = plan.execute(xd)
    s.synchronize()
    assert torch.equal(l1, l2) and torch.equal(v1, v2)


def test_hit_overflow_status():
    n, k = 2 ** 14, 8
    x = dense_signal(n, 1)
    plan = Plan(n, k, L=16, seed=4, max_hits=4)
    plan.execute(torch.from_numpy(x).to(DEV))
    assert plan.status() == b.HIT_OVERFLOW
    assert plan.debug(DEBUG_NUM_HITS)[0] > 4


def test_stage_timing_and_launch_count():
    n, k = 2 ** 20, 100
    x, S, X = planted_signal(n, k, seed=6)
    plan = Plan(n, k, L=16, seed=4)
    plan.set_timing(True)
    plan.execute(torch.from_numpy(x).to(DEV))
    t = plan.stage_times()
    assert all(v >= 0 for nm, v in t.items() if nm != "gather") and t["fold"] > 0
    assert (t["gather"] > 0) == bool(plan.info()["staged"])
    # C2 (B = 2048 = 64 x 32: staged fold with FFT pass 1 inside): phase 1, phase 2 x 2 slot ranges,
    # FFT pass 2, cutoff, vote + estimation, output (timing mode: no graph branches)
    assert plan.info()["tail"] == 1 and plan.launches_per_execute() == 7


def test_C4_full_size_parity():
    """BASELINE.json configs[3] size: n = 2^27, k = 1000 (B = 65536, two-pass
    FFT with B1 = B2 = 256; the staging of all 16 loops (218 MB) would not fit
    L2, so the staged gather runs in 4 stage groups of 4 loops)."""
    n, k = 2 ** 27, 1000
    x, S, X = planted_signal(n, k, seed=2)
    plan, ref, locs, vals = run_pair(x, n, k, None, 16, shared_taps=False, seed=4)
    assert plan.info()["staged"] == 4
    check_all(plan, ref, locs, vals, fold_bit_exact=False)
    assert set(locs.tolist()) == set(S.tolist())
    assert O.l1_error(locs, vals, S, X, k) <= 1e-6


@pytest.mark.parametrize("snr_db", [40.0, 20.0, 10.0])
def test_parity_snr_sweep(snr_db):
    """configs[3]'s additive-noise sweep at n = 2^20 (k = 100): outputs match
    the oracle whatever the noise does to recovery."""
    n, k = 2 ** 20, 100
    x, S, X = planted_signal(n, k, seed=11, snr_db=snr_db)
    plan, ref, locs, vals = run_pair(x, n, k, None, 16, shared_taps=True, seed=6)
    check_all(plan, ref, locs, vals, fold_bit_exact=True)


@pytest.mark.gpu
@pytest.mark.parametrize("env,kw", [({"CUSFFT_NO_GRAPH": "1"}, {}), ({"CUSFFT_TAIL": "0"}, {}),
                                    ({"CUSFFT_FFT2SEL": "0"}, {}),
                                    ({}, dict(gather=1)), ({}, dict(l2_persist=0)),
                                    ({"CUSFFT_TAIL": "0", "CUSFFT_NO_GRAPH": "1"}, dict(gather=1)),
                                    ({}, dict(gather=2)), ({"CUSFFT_NO_GRAPH": "1"}, dict(gather=2)),
                                    ({"CUSFFT_STAGE_GROUP": "4"}, {}), ({"CUSFFT_STAGE_GROUP": "3"}, {}),
                                    ({"CUSFFT_STAGE_GROUP": "8"}, {})])
def test_kernel_paths_agree(env, kw, monkeypatch):
    """Every alternative path (no CUDA graph, the k_vote / k_estimate /
    k_output chain instead of the fused tail, the direct gather or the
    paper's remap + execute kernels instead of the staged gather, the staged
    gather in stage groups of 4 / 3 slots or split over the two graph branches,
    no persisting-L2 set-aside) gives the default path's hits
    and output exactly (same fold order, same selection rules)."""
    import torch
    from paper_conf_ipps_wangcc16_b200 import Plan
    # n = 2^22, k = 1000: B = 8192, two FFT passes, staged fold, two-branch graph
    n, k = 2 ** 22, 1000
    x, S, X = planted_signal(n, k, seed=21)
    xd = torch.from_numpy(x).cuda()
    base = Plan(n, k, L=16, seed=4, debug=1)
    assert base.info()["staged"] and base.info()["tail"]
    l0, v0 = base.execute(xd)
    h0 = np.sort(base.debug(DEBUG_HITS))
    for key, val in env.items():
        monkeypatch.setenv(key, val)
    alt = Plan(n, k, L=16, seed=4, debug=1, **kw)
    l1, v1 = alt.execute(xd)
    torch.cuda.synchronize()
    assert alt.status() == 0
    assert alt.info()["tail"] == (0 if env.get("CUSFFT_TAIL") == "0" else 1)
    # groups never straddle slot 8; 8-loop groups = phase 1 split over the two graph branches
    groups = {"4": 4, "3": 6, "8": 2}.get(env.get("CUSFFT_STAGE_GROUP"), 1)
    assert alt.info()["staged"] == (0 if kw.get("gather") in (1, 2) else groups)
    assert np.array_equal(np.sort(alt.debug(DEBUG_HITS)), h0)
    assert torch.equal(l1, l0)
    assert torch.equal(v1, v0)


@pytest.mark.gpu
@pytest.mark.parametrize("depth", [1, 2, 3])
def test_execute_batch_matches_single(depth):
    """cusfft_execute_batch: signal b's outputs equal cusfft_execute on it, for
    any pipeline depth (clone plans on their own streams), with a row stride
    larger than n; status covers the clones."""
    import torch
    from paper_conf_ipps_wangcc16_b200 import Plan
    n, k, count = 2 ** 18, 50, 5
    xs = np.stack([planted_signal(n, k, seed=60 + b)[0] for b in range(count)])
    xpad = torch.zeros(count, n + 64, dtype=torch.complex128, device="cuda")
    xpad[:, :n] = torch.from_numpy(xs).cuda()
    xb = xpad[:, :n]
    with Plan(n, k, L=16, seed=5) as plan:
        ref = [plan.execute(xb[b].contiguous()) for b in range(count)]
        ref = [(l.clone(), v.clone()) for l, v in ref]
        plan.set_pipeline(depth)
        for _ in range(2):  # second call replays the cached graphs
            locs, vals = plan.execute_batch(xb)
            torch.cuda.synchronize()
            assert plan.status() == 0
            for b in range(count):
                assert torch.equal(locs[b], ref[b][0])
                assert torch.equal(vals[b], ref[b][1])
    for b in range(count):
        x, S, X = planted_signal(n, k, seed=60 + b)
        assert set(ref[b][0].cpu().tolist()) == set(S.tolist())


@pytest.mark.gpu
@pytest.mark.parametrize("k,bcst", [(50, 1.0), (200, 1.0), (1000, 1.0), (2000, 2.0), (4096, 2.0)])
def test_C5_k_sweep_parity(k, bcst):
    """C5 (BASELINE.json configs[4]): n = 2^22, k = 50 ... 4096 (B from the
    formula; Bcst = 2 for k >= 2000).  GPU = oracle on the
    recovered set (exact) and values (1e-9), planted support recovered."""
    import torch
    import oracle as O
    from paper_conf_ipps_wangcc16_b200 import Plan, default_B
    n = 2 ** 22
    B = default_B(n, k, bcst)
    x, S, X = planted_signal(n, k, seed=70 + k)
    with Plan(n, k, B=B, L=16, seed=8) as plan:
        locs, vals = plan.execute(torch.from_numpy(x).cuda())
        torch.cuda.synchronize()
        assert plan.status() == 0
        locs, vals = locs.cpu().numpy(), vals.cpu().numpy()
    ref = O.sfft(x, O.make_params(n, k, B=B, L=16, seed=8))
    assert np.array_equal(locs, ref.locs)
    np.testing.assert_allclose(vals, ref.vals, rtol=1e-9, atol=1e-12)
    assert set(locs.tolist()) == set(S.tolist())
    assert O.l1_error(locs, vals, S, X, k) <= 1e-6


@pytest.mark.gpu
def test_debug_and_plain_plans_agree():
    """A plan without debug buffers (the fold output u is then not written by
    the bulk-copy fold; the FFT reads v) returns exactly the debug plan's
    output, and refuses the U artefact instead of returning stale data."""
    from paper_conf_ipps_wangcc16_b200 import Plan
    n, k = 2 ** 22, 1000
    x, S, X = planted_signal(n, k, seed=33)
    xd = torch.from_numpy(x).to(DEV)
    dbg = Plan(n, k, L=16, seed=9, debug=1)
    plain = Plan(n, k, L=16, seed=9)
    assert plain.info()["staged"]
    l0, v0 = dbg.execute(xd)
    l1, v1 = plain.execute(xd)
    torch.cuda.synchronize()
    assert torch.equal(l0, l1) and torch.equal(v0, v1)
    assert set(l1.cpu().tolist()) == set(S.tolist())
    with pytest.raises(Exception):
        plain.debug(DEBUG_U)


@pytest.mark.gpu
def test_l2_setaside_held_and_released():
    """A staged plan holds the device's persisting-L2 set-aside (the staging
    buffer is stored evict_last) and the last plan to go restores the value it
    found, so other work gets the whole L2 back."""
    import gc
    from cuda.bindings import runtime as rt
    from paper_conf_ipps_wangcc16_b200 import Plan
    lim = rt.cudaLimit.cudaLimitPersistingL2CacheSize
    gc.collect()
    torch.cuda.synchronize()
    before = rt.cudaDeviceGetLimit(lim)[1]
    maxp = rt.cudaDeviceGetAttribute(rt.cudaDeviceAttr.cudaDevAttrMaxPersistingL2CacheSize, 0)[1]
    plan = Plan(2 ** 22, 1000, L=16, seed=1)
    assert plan.info()["staged"]
    during = rt.cudaDeviceGetLimit(lim)[1]
    if maxp > 0:
        assert during > 0
    plan.close()
    after = rt.cudaDeviceGetLimit(lim)[1]
    assert after == before or after == during  # == during only if another live plan still holds it
    if before == 0:
        assert after == 0


@pytest.mark.gpu
def test_C3_bench_plan_elementwise():
    """The bench's own plan (bench.py C3 configuration, debug = 0, default
    launch path) against the oracle element by element: locations exact,
    values within 1e-9 relative (north_star), planted truth recovered."""
    import bench
    n, k, L = bench.CONFIGS["C3"][:3]
    prm = bench.plan_params("C3")
    x, S, X = planted_signal(n, k, seed=1)
    B = O.default_B(n, k)
    plan = Plan(n, k, B=B, L=L, seed=3, **prm)
    assert plan.info()["staged"] == 1 and plan.info()["tail"] == 1
    locs, vals = plan.execute(torch.from_numpy(x).to(DEV))
    torch.cuda.synchronize()
    assert plan.status() == 0
    locs, vals = locs.cpu().numpy(), vals.cpu().numpy()
    ref = O.sfft(x, _oracle_params(n, k, B, L, seed=3, **prm))
    assert np.array_equal(locs, ref.locs)
    assert_close(vals, ref.vals)
    assert set(locs.tolist()) == set(S.tolist())
    assert O.l1_error(locs, vals, S, X, k) <= 1e-6


@pytest.mark.gpu
def test_C4_noisy_parity():
    """BASELINE.json configs[3]: n = 2^27, k = 1000 with additive Gaussian
    noise (SNR 20 dB), full size: GPU = oracle (debug artefacts, hits,
    outputs) whatever the noise does to recovery."""
    n, k = 2 ** 27, 1000
    x, S, X = planted_signal(n, k, seed=12, snr_db=20.0)
    plan, ref, locs, vals = run_pair(x, n, k, None, 16, shared_taps=False, seed=7)
    check_all(plan, ref, locs, vals, fold_bit_exact=False)


@pytest.mark.gpu
def test_C1_gpu_values_equal_direct_dft():
    """BASELINE.json configs[0] (C1): the GPU's recovered values
    equal (1/n) x^_f by direct summation, at fixed seeds."""
    n, k = 2 ** 14, 8
    t = np.arange(n)
    for seed in range(4):
        x, S, X = planted_signal(n, k, seed)
        with Plan(n, k, L=16, seed=200 + seed, num_select=2 * k) as plan:
            locs, vals = plan.execute(torch.from_numpy(x).to(DEV))
            locs, vals = locs.cpu().numpy(), vals.cpu().numpy()
        assert set(locs.tolist()) == set(S.tolist())
        ref = np.array([np.sum(x * np.exp(-2j * np.pi * ((int(f) * t) % n) / n)) for f in locs]) / n
        np.testing.assert_allclose(vals, ref, rtol=0, atol=1e-9)


@pytest.mark.gpu
@pytest.mark.parametrize("n,k,extra", [
    (2 ** 16, 32, dict(loc_tolerance=1e-6, loc_lobefrac=1.0 / 512, tolerance=1e-8, num_select=64)),
    (2 ** 22, 1000, dict(loc_tolerance=1e-6, loc_lobefrac=1.0 / 8192, tolerance=1e-7, lobefrac=0.75 / 8192)),
])
def test_parity_separate_filters(n, k, extra):
    """location loops with their own (delta, lambda) filter; GPU-built
    filters against the oracle's, staged or direct fold, the fused tail with
    two G^ tables.  The 2^22 case is staged (two filter groups in one
    address-sorted schedule)."""
    x, S, X = planted_signal(n, k, seed=5)
    plan, ref, locs, vals = run_pair(x, n, k, None, 16, shared_taps=False, seed=8, **extra)
    info = plan.info()
    assert info["filters"] == 2 and info["w_loc"] < info["w"]
    gl = plan.debug(b.DEBUG_LOC_TAPS)
    assert np.abs(gl - ref.extra["taps_loc"]).max() <= 1e-12 * np.abs(gl).max()
    check_all(plan, ref, locs, vals, fold_bit_exact=False)
    assert set(locs.tolist()) == set(S.tolist())


@pytest.mark.parametrize("env,kw", [({"CUSFFT_STAGE_GROUP": "3"}, {}), ({}, dict(shard_mode=2, max_hits=8192)),
                                    ({"CUSFFT_STAGE_GROUP": "4"}, dict(shard_mode=2, max_hits=8192))])
def test_separate_filters_with_groups_and_two_exchanges(env, kw, monkeypatch):
    """Combinations: separate location / estimation filters (N3) with stage
    groups (each group one filter) and / or the two-collective finish (world
    1): the output equals the plain separate-filter plan's bit for bit."""
    n, k = 2 ** 22, 1000
    x, S, X = planted_signal(n, k, seed=9)
    xd = torch.from_numpy(x).to(DEV)
    filt = dict(loc_tolerance=1e-6, loc_lobefrac=1.0 / 8192, tolerance=1e-7, lobefrac=0.75 / 8192)
    base = Plan(n, k, L=16, seed=8, **filt)
    l0, v0 = base.execute(xd)
    for key, val in env.items():
        monkeypatch.setenv(key, val)
    alt = Plan(n, k, L=16, seed=8, **filt, **kw)
    l1, v1 = alt.execute(xd)
    torch.cuda.synchronize()
    assert alt.status() == 0 and alt.info()["filters"] == 2
    if env:
        assert alt.info()["staged"] > 1
    assert torch.equal(l0, l1) and torch.equal(v0, v1)
    assert sorted(l1.tolist()) == sorted(S.tolist())


def test_execute_host_zero_copy_stage_groups(monkeypatch):
    """The in-place PCIe gather of a pinned host signal through stage groups
    (several phase-1 launches read the host buffer)."""
    monkeypatch.setenv("CUSFFT_STAGE_GROUP", "4")
    n, k = 2 ** 22, 1000
    x, S, X = planted_signal(n, k, seed=43)
    plan = Plan(n, k, L=16, seed=4)
    assert plan.info()["staged"] == 4
    lh, vh = plan.execute_host(torch.from_numpy(x).pin_memory())
    ld, vd = plan.execute(torch.from_numpy(x).to(DEV))
    torch.cuda.synchronize()
    assert np.array_equal(ld.cpu().numpy(), lh) and np.array_equal(vd.cpu().numpy(), vh)
    assert sorted(lh.tolist()) == sorted(S.tolist())


@pytest.mark.gpu
@pytest.mark.parametrize("shard_mode", [0, 2])
def test_library_owned_nccl_exchange_world1(shard_mode):
    """cusfft_plan_dist with an ncclUniqueId: the plan owns a communicator and
    cusfft_execute runs the whole transform with the collective(s) inside the
    plan's CUDA graph (a one-rank communicator on the single test GPU; shard
    mode 2: both all-gathers); the output equals the plain plan's bit for bit."""
    from paper_conf_ipps_wangcc16_b200 import nccl_unique_id
    n, k = 2 ** 22, 1000
    x, S, X = planted_signal(n, k, seed=27)
    xd = torch.from_numpy(x).to(DEV)
    plain = Plan(n, k, L=16, seed=6)
    l0, v0 = plain.execute(xd)
    extra = dict(shard_mode=2, max_hits=8192) if shard_mode == 2 else {}
    owned = Plan(n, k, L=16, seed=6, rank=0, world=1, nccl_id=nccl_unique_id(), **extra)
    assert owned.info()["owns_comm"] == 1
    for _ in range(2):  # capture, then replay
        l1, v1 = owned.execute(xd)
        torch.cuda.synchronize()
        assert owned.status() == 0
        assert torch.equal(l0, l1) and torch.equal(v0, v1)


@pytest.mark.gpu
def test_k8192_output_smem():
    """k up to 8192 (include/cusfft.h limit): the output selection's shared
    memory (205 KB at kp2 = 8192) fits; the plan runs and recovers a planted signal."""
    n, k = 2 ** 22, 8192
    B = 65536
    x, S, X = planted_signal(n, k, seed=31)
    with Plan(n, k, B=B, L=16, seed=2) as plan:
        locs, vals = plan.execute(torch.from_numpy(x).to(DEV))
        torch.cuda.synchronize()
        assert plan.status() == 0
        got = set(locs.cpu().tolist())
    assert len(got & set(S.tolist())) >= int(0.99 * k)


@pytest.mark.gpu
def test_l2_persist_opt_out():
    """params.l2_persist = 0: a staged plan leaves the device's persisting-L2 limit alone."""
    import gc
    from cuda.bindings import runtime as rt
    lim = rt.cudaLimit.cudaLimitPersistingL2CacheSize
    gc.collect()
    torch.cuda.synchronize()
    before = rt.cudaDeviceGetLimit(lim)[1]
    plan = Plan(2 ** 22, 1000, L=16, seed=1, l2_persist=0)
    assert plan.info()["staged"]
    assert rt.cudaDeviceGetLimit(lim)[1] == before
    plan.close()


@pytest.mark.gpu
def test_plans_of_different_shapes_coexist():
    """Kernels are shared by every plan of the process: creating a plan of a
    small shape must not lower a per-function launch limit (dynamic shared
    memory) another live plan needs — e.g. the fused tail's vote table at B =
    32768 after a B = 512 plan, or the two-collective ranking's hit list."""
    n1, k1 = 2 ** 21, 60
    x1, S1, _ = planted_signal(n1, k1, seed=31)
    n2, k2 = 2 ** 16, 20
    x2, S2, _ = planted_signal(n2, k2, seed=32)
    xd1, xd2 = torch.from_numpy(x1).to(DEV), torch.from_numpy(x2).to(DEV)
    with Plan(n1, k1, B=32768, L=16, seed=3) as alone:  # before any other shape exists
        l0, v0 = alone.execute(xd1)
        torch.cuda.synchronize()
    big = Plan(n1, k1, B=32768, L=16, seed=3)
    big2 = Plan(n1, k1, B=32768, L=16, seed=3, shard_mode=2, max_hits=32768)
    small = Plan(n2, k2, L=16, seed=4)
    small2 = Plan(n2, k2, L=16, seed=4, shard_mode=2, max_hits=1024)
    ls, vs = small.execute(xd2)
    lb, vb = big.execute(xd1)
    lb2, vb2 = big2.execute(xd1)
    ls2, vs2 = small2.execute(xd2)
    torch.cuda.synchronize()
    for p in (big, big2, small, small2):
        assert p.status() == 0
    assert torch.equal(lb, lb2) and torch.equal(vb, vb2)
    assert torch.equal(ls, ls2) and torch.equal(vs, vs2)
    assert torch.equal(lb, l0) and torch.equal(vb, v0)
    assert sorted(ls.tolist()) == sorted(S2.tolist())


def test_concurrent_plans_on_separate_streams():
    """Distinct plans are independent (include/cusfft.h, Conventions): two
    staged plans (each holding a
    persisting-L2 window and its own branch streams) and a small plan enqueued
    on three streams, interleaved several times without host synchronisation,
    give the outputs of the same plans run one at a time."""
    cases = [(2 ** 22, 1000, 51), (2 ** 22, 300, 52), (2 ** 16, 20, 53)]
    plans, xs, ref = [], [], []
    for n, k, seed in cases:
        x, S, _ = planted_signal(n, k, seed=seed)
        p = Plan(n, k, L=16, seed=seed)
        xd = torch.from_numpy(x).to(DEV)
        l0, v0 = p.execute(xd)
        torch.cuda.synchronize()
        assert sorted(l0.tolist()) == sorted(S.tolist())
        plans.append(p)
        xs.append(xd)
        ref.append((l0.clone(), v0.clone()))
    assert plans[0].info()["staged"] and plans[1].info()["staged"]
    streams = [torch.cuda.Stream() for _ in plans]
    outs = []
    for rep in range(4):
        for p, xd, s in zip(plans, xs, streams):
            with torch.cuda.stream(s):
                outs.append(p.execute(xd))
    torch.cuda.synchronize()
    for j, (l, v) in enumerate(outs):
        i = j % len(plans)
        assert plans[i].status() == 0
        assert torch.equal(l, ref[i][0]) and torch.equal(v, ref[i][1]), (j, i)


def _random_config(i):
    """A seeded random small configuration (n, k, B, L, extra) covering the
    parameter space the fixed CASES sample: B single- and two-pass, L_loc, T
    with and without pair enumeration, both filters, tau modes, noise."""
    rng = np.random.default_rng(1000 + i)
    m = int(rng.integers(12, 19))
    n = 2 ** m
    k = int(rng.integers(1, 48))
    L = int(rng.integers(5, 21))
    Lloc = int(rng.integers(3, min(L, 12) + 1))
    T = int(rng.integers(Lloc // 2 + 1, Lloc + 1)) if rng.random() < 0.7 else int(rng.integers(2, Lloc // 2 + 2))
    T = max(1, min(T, Lloc))
    B = None if rng.random() < 0.5 else 2 ** int(rng.integers(max(5, m - 10), min(m - 5, 14) + 1))
    if B is not None and B <= 2 * k:
        B = None
    extra = dict(loc_loops=Lloc, vote_threshold=T, filter=int(rng.random() < 0.25), tau_mode=int(rng.random() < 0.85))
    snr = None if rng.random() < 0.7 else float(rng.choice([10.0, 20.0, 40.0]))
    return n, k, B, L, extra, snr


@pytest.mark.parametrize("i", range(48))
def test_parity_random_configs(i):
    """Property sweep: 48 seeded random configurations, the GPU against the
    oracle with shared taps (fold bit-exact, cutoff winners / hits / output
    locations exact, values to 1e-9)."""
    n, k, B, L, extra, snr = _random_config(i)
    x, S, X = planted_signal(n, k, seed=77 + i, snr_db=snr)
    plan, ref, locs, vals = run_pair(x, n, k, B, L, shared_taps=True, seed=100 + i, **extra)
    check_all(plan, ref, locs, vals, fold_bit_exact=True)


def test_filter_longer_than_signal_rejected():
    """A filter of more taps than samples (n = 8192, B = 1024: w ~ 12,400 at
    the default delta / lambda) would wrap around x: CUSFFT_INVALID_PARAM."""
    with pytest.raises(b.CusfftError) as ei:
        Plan(2 ** 13, 4, B=1024, L=8, seed=1)
    assert ei.value.code == b.INVALID_PARAM


@pytest.mark.parametrize("i", range(16))
def test_parity_random_staged_configs(i):
    """Property sweep of the staged path (n = 2^20 ... 2^22, B >= 2048: address-
    sorted phase 1, the fused FFT-pass-2 + cutoff cluster kernel where it
    applies), randomly with the two-collective finish at world 1 and forced
    stage groups; the GPU against the oracle with shared taps."""
    rng = np.random.default_rng(5000 + i)
    n = 2 ** int(rng.integers(20, 23))
    k = int(rng.integers(20, 600))
    L = int(rng.integers(8, 17))
    Lloc = int(rng.integers(4, min(L, 10) + 1))
    T = int(rng.integers(Lloc // 2 + 1, Lloc + 1))
    B = int(O.default_B(n, k)) * int(rng.choice([1, 2]))
    extra = dict(loc_loops=Lloc, vote_threshold=T)
    if rng.random() < 0.3:
        extra.update(shard_mode=2, max_hits=16384)
    x, S, X = planted_signal(n, k, seed=300 + i)
    env = {}
    if rng.random() < 0.3:
        env["CUSFFT_STAGE_GROUP"] = str(int(rng.integers(2, 5)))
    old = {key: os.environ.get(key) for key in env}
    os.environ.update(env)
    try:
        plan, ref, locs, vals = run_pair(x, n, k, max(B, 2048), L, shared_taps=True, seed=400 + i, **extra)
    finally:
        for key, v in old.items():
            if v is None:
                os.environ.pop(key, None)
            else:
                os.environ[key] = v
    assert plan.info()["staged"] >= 1
    check_all(plan, ref, locs, vals, fold_bit_exact=True)
