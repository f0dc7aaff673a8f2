"""The C-ABI library loads, exports every symbol include/cusfft.h declares, and
its host-only entry points behave as documented (no GPU needed)."""
import ctypes
import math
import os
import re
import subprocess

import pytest

import paper_conf_ipps_wangcc16_b200 as pkg
from paper_conf_ipps_wangcc16_b200 import _binding as b

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "cusfft.h")


def _header_functions():
    src = open(HEADER).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(cusfft_[A-Za-z0-9_]+)\s*\(", src)))


def test_header_and_binding_agree():
    assert _header_functions() == sorted(b.EXPORTED)


def test_library_exports_every_header_symbol():
    lib = pkg.load_library()
    for name in _header_functions():
        assert hasattr(lib, name), name
    out = subprocess.run(["nm", "-D", "--defined-only", b.LIB_PATH], capture_output=True, text=True).stdout
    for name in _header_functions():
        assert re.search(rf"\bT {name}$", out, flags=re.M), name


def test_library_is_sm100a():
    out = subprocess.run(["cuobjdump", "--list-elf", b.LIB_PATH], capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_params_struct_layout():
    # include/cusfft.h cusfft_params (x86-64 SysV layout): 17 v1 fields (104 B) +
    # loc_tolerance, loc_lobefrac, l2_persist, gather
    assert ctypes.sizeof(b.CusfftParams) == 128
    assert b.CusfftParams.loc_tolerance.offset == 104 and b.CusfftParams.gather.offset == 124


def test_abi_version_and_strerror():
    lib = pkg.load_library()
    assert lib.cusfft_abi_version() == 2
    for code in range(0, -13, -1):
        assert lib.cusfft_strerror(code)
    assert b"unknown" in lib.cusfft_strerror(-99)


def test_default_B_matches_paper_rule():
    # B = floor_pow2(sqrt(n k / log2 n))
    for n, k in [(2 ** 14, 8), (2 ** 18, 1000), (2 ** 20, 100), (2 ** 24, 1000), (2 ** 27, 1000)]:
        v = math.sqrt(n * k / math.log2(n))
        assert pkg.default_B(n, k) == 2 ** int(math.floor(math.log2(v)))
    assert pkg.default_B(2 ** 18, 1000) == 2048
    assert pkg.default_B(2 ** 22, 4096, 2.0) == 32768


def test_params_default_values():
    p = pkg.default_params(2 ** 24, 1000, 16384)
    assert p.filter == 0 and p.tolerance == 1e-8 and p.lobefrac == 0.5 / 16384
    assert p.box_width == 1023 and p.num_select == 1000 and p.tau_mode == 1
    assert p.loc_loops == 0 and p.vote_threshold == 0 and p.device == -1
    assert p.loc_tolerance == 0.0 and p.loc_lobefrac == 0.0 and p.l2_persist == 1 and p.gather == 0


@pytest.mark.parametrize("n,k,B,code", [
    (1000, 8, 64, b.INVALID_N), (8, 2, 4, b.INVALID_N), (2 ** 32, 8, 64, b.INVALID_N),
    (2 ** 14, 8, 48, b.INVALID_B), (2 ** 14, 8, 2 ** 14, b.INVALID_B), (2 ** 14, 0, 64, b.INVALID_K),
])
def test_params_default_rejects(n, k, B, code):
    lib = pkg.load_library()
    p = b.CusfftParams()
    assert lib.cusfft_params_default(ctypes.byref(p), n, k, B) == code


def test_null_pointers_and_invalid_plan():
    lib = pkg.load_library()
    assert lib.cusfft_params_default(None, 2 ** 14, 8, 64) == b.NULL_PTR
    assert lib.cusfft_plan(None, 2 ** 14, 8, 64, 16, None) == b.NULL_PTR
    assert lib.cusfft_destroy(None) == b.INVALID_PLAN
    assert lib.cusfft_execute(None, None, None, None) == b.INVALID_PLAN
    assert lib.cusfft_status(None) == b.INVALID_PLAN
    assert lib.cusfft_launches_per_execute(None) == b.INVALID_PLAN
    assert lib.cusfft_execute_batch(None, None, 0, 0, None, None) == b.INVALID_PLAN
    assert lib.cusfft_set_pipeline(None, 2) == b.INVALID_PLAN


@pytest.mark.parametrize("kw,code", [
    (dict(loc_loops=20), b.INVALID_LOOPS), (dict(vote_threshold=9), b.INVALID_LOOPS),
    (dict(num_select=4), b.INVALID_K), (dict(num_select=65), b.INVALID_K),
    (dict(tolerance=0.0), b.INVALID_PARAM), (dict(box_width=256), b.INVALID_PARAM),
    (dict(tau_mode=2), b.INVALID_PARAM), (dict(cutoff_mode=3), b.INVALID_PARAM),
    (dict(cutoff_mode=2, cutoff_threshold=0.0), b.INVALID_PARAM),
    (dict(loc_tolerance=1.5), b.INVALID_PARAM), (dict(loc_lobefrac=0.6), b.INVALID_PARAM),
    (dict(l2_persist=2), b.INVALID_PARAM), (dict(gather=3), b.INVALID_PARAM),
])
def test_plan_validation_before_device(kw, code):
    """Parameter validation happens before any CUDA call, so it is testable here."""
    lib = pkg.load_library()
    p = pkg.default_params(2 ** 14, 8, 64)
    for key, v in kw.items():
        setattr(p, key, v)
    h = ctypes.c_void_p()
    assert lib.cusfft_plan(ctypes.byref(h), 2 ** 14, 8, 64, 16, ctypes.byref(p)) == code
    assert not h.value


@pytest.mark.parametrize("world,L,shard,code", [
    (3, 16, 0, b.INVALID_LOOPS),   # loop sharding: world must divide L
    (2, 16, 3, b.INVALID_PARAM),   # unknown shard mode
    (3, 16, 2, b.INVALID_LOOPS),   # two-exchange loop sharding: world must divide L
    (3, 16, 1, b.INVALID_PARAM),   # signal sharding: world must divide n
])
def test_dist_plan_validation(world, L, shard, code):
    lib = pkg.load_library()
    p = pkg.default_params(2 ** 14, 8, 64)
    p.shard_mode = shard
    h = ctypes.c_void_p()
    assert lib.cusfft_plan_dist(ctypes.byref(h), 2 ** 14, 8, 64, L, ctypes.byref(p), 0, world, None) == code
    assert not h.value


def test_two_exchange_mode_limits():
    """shard_mode 2 sorts the hit list in shared memory (max_hits <= 32768)
    and takes medians of at most 64 loops per thread (include/cusfft.h)."""
    lib = pkg.load_library()
    p = pkg.default_params(2 ** 14, 8, 64)
    p.shard_mode = 2
    p.max_hits = 40000
    h = ctypes.c_void_p()
    assert lib.cusfft_plan_dist(ctypes.byref(h), 2 ** 14, 8, 64, 16, ctypes.byref(p), 0, 2, None) == b.INVALID_PARAM
    assert not h.value


def test_signal_sharding_accepts_any_L():
    """Signal sharding does not need world | L: validation passes and only the
    device probe fails here (no GPU), i.e. CUSFFT_CUDA, not a parameter code."""
    torch = pytest.importorskip("torch")
    if torch.cuda.is_available():
        pytest.skip("a GPU is present")
    lib = pkg.load_library()
    p = pkg.default_params(2 ** 14, 8, 64)
    p.shard_mode = 1
    h = ctypes.c_void_p()
    assert lib.cusfft_plan_dist(ctypes.byref(h), 2 ** 14, 8, 64, 15, ctypes.byref(p), 1, 4, None) == b.CUDA


def test_no_cpu_fallback_without_device():
    """Without a CUDA device plan creation fails loudly (CUSFFT_CUDA)."""
    torch = pytest.importorskip("torch")
    if torch.cuda.is_available():
        pytest.skip("a GPU is present")
    with pytest.raises(b.CusfftError) as e:
        pkg.Plan(2 ** 14, 8)
    assert e.value.code == b.CUDA


def test_nccl_unique_id_host_only():
    """cusfft_nccl_unique_id loads NCCL at run time (no link dependency) and
    returns 128 bytes; a NULL destination is refused."""
    lib = pkg.load_library()
    assert lib.cusfft_nccl_unique_id(None) == b.NULL_PTR
    try:
        uid = pkg.nccl_unique_id()
    except b.CusfftError as e:  # NCCL not loadable in this environment
        assert e.code == b.NCCL
        return
    assert isinstance(uid, bytes) and len(uid) == 128
