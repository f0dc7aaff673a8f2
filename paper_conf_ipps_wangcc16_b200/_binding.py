"""ctypes binding of ``libcusfft.so`` (the C ABI in ``include/cusfft.h``).

Argument marshalling only: every step of the transform runs in the CUDA
kernels of ``csrc/``.  There is no CPU fallback — if the shared library is
missing or no CUDA device is present, plan creation raises.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
# CUSFFT_LIB selects an alternative in-tree build (e.g. the -DCUSFFT_TRACE one).
LIB_PATH = os.path.join(_HERE, os.environ.get("CUSFFT_LIB", "libcusfft.so"))

SUCCESS = 0
INVALID_N, INVALID_B, INVALID_K, INVALID_LOOPS, INVALID_PARAM = -1, -2, -3, -4, -5
NULL_PTR, ALLOC, CUDA, HIT_OVERFLOW, INVALID_PLAN, INTERNAL, NCCL = -6, -7, -8, -9, -10, -11, -12

FILTER_DOLPH_CHEBYSHEV = 0
FILTER_GAUSSIAN = 1

CUTOFF_EXACT, CUTOFF_SORT, CUTOFF_THRESHOLD = 0, 1, 2

DEBUG_U, DEBUG_UHAT, DEBUG_WINNERS, DEBUG_HITS, DEBUG_HIT_VALS = 0, 1, 2, 3, 4
DEBUG_PER_LOOP, DEBUG_TAPS, DEBUG_GHAT, DEBUG_NUM_HITS = 5, 6, 7, 8
DEBUG_LOC_TAPS, DEBUG_LOC_GHAT = 9, 10

# Every symbol include/cusfft.h declares (checked by tests/test_abi.py).
EXPORTED = (
    "cusfft_params_default", "cusfft_default_B", "cusfft_plan", "cusfft_plan_dist", "cusfft_nccl_unique_id",
    "cusfft_destroy", "cusfft_set_stream", "cusfft_execute", "cusfft_execute_host", "cusfft_execute_batch",
    "cusfft_set_pipeline",
    "cusfft_execute_local", "cusfft_execute_mid", "cusfft_execute_finish", "cusfft_exchange_buffer",
    "cusfft_exchange_buffer2", "cusfft_exchange_kind",
    "cusfft_get_info", "cusfft_get_debug", "cusfft_status", "cusfft_set_timing",
    "cusfft_get_stage_times", "cusfft_set_stage_limit", "cusfft_launches_per_execute", "cusfft_strerror",
    "cusfft_last_cuda_error", "cusfft_last_nccl_error", "cusfft_abi_version",
)


class CusfftParams(ctypes.Structure):
    _fields_ = [
        ("filter", ctypes.c_int32),
        ("tolerance", ctypes.c_double),
        ("lobefrac", ctypes.c_double),
        ("box_width", ctypes.c_int64),
        ("loc_loops", ctypes.c_int32),
        ("vote_threshold", ctypes.c_int32),
        ("num_select", ctypes.c_int32),
        ("tau_mode", ctypes.c_int32),
        ("seed", ctypes.c_uint64),
        ("max_hits", ctypes.c_int64),
        ("device", ctypes.c_int32),
        ("debug", ctypes.c_int32),
        ("taps", ctypes.POINTER(ctypes.c_double)),
        ("num_taps", ctypes.c_int64),
        ("cutoff_mode", ctypes.c_int32),
        ("shard_mode", ctypes.c_int32),
        ("cutoff_threshold", ctypes.c_double),
        ("loc_tolerance", ctypes.c_double),
        ("loc_lobefrac", ctypes.c_double),
        ("l2_persist", ctypes.c_int32),
        ("gather", ctypes.c_int32),
    ]


_lib = None


def load_library():
    """Load libcusfft.so (built in-tree by ``__graft_entry__.build()``)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise RuntimeError(
            f"CUDA extension {LIB_PATH} is missing; build it with "
            "`python -c 'import __graft_entry__ as g; g.build()'` (no CPU fallback exists)")
    lib = ctypes.CDLL(LIB_PATH)
    P = ctypes.c_void_p
    i64, i32 = ctypes.c_int64, ctypes.c_int32
    pp = ctypes.POINTER(CusfftParams)
    sig = {
        "cusfft_params_default": (ctypes.c_int, [pp, i64, i64, i64]),
        "cusfft_default_B": (i64, [i64, i64, ctypes.c_double]),
        "cusfft_plan": (ctypes.c_int, [ctypes.POINTER(P), i64, i64, i64, i32, pp]),
        "cusfft_plan_dist": (ctypes.c_int, [ctypes.POINTER(P), i64, i64, i64, i32, pp, i32, i32, P]),
        "cusfft_nccl_unique_id": (ctypes.c_int, [P]),
        "cusfft_destroy": (ctypes.c_int, [P]),
        "cusfft_set_stream": (ctypes.c_int, [P, P]),
        "cusfft_execute": (ctypes.c_int, [P, P, P, P]),
        "cusfft_execute_host": (ctypes.c_int, [P, P, P, P]),
        "cusfft_execute_batch": (ctypes.c_int, [P, P, i64, i64, P, P]),
        "cusfft_set_pipeline": (ctypes.c_int, [P, i32]),
        "cusfft_execute_local": (ctypes.c_int, [P, P]),
        "cusfft_execute_mid": (ctypes.c_int, [P]),
        "cusfft_execute_finish": (ctypes.c_int, [P, P, P]),
        "cusfft_exchange_buffer": (ctypes.c_int, [P, ctypes.POINTER(P), ctypes.POINTER(i64)]),
        "cusfft_exchange_buffer2": (ctypes.c_int, [P, ctypes.POINTER(P), ctypes.POINTER(i64)]),
        "cusfft_exchange_kind": (i32, [P]),
        "cusfft_get_info": (ctypes.c_int, [P, P, P, P, P]),
        "cusfft_get_debug": (i64, [P, i32, P, i64]),
        "cusfft_status": (ctypes.c_int, [P]),
        "cusfft_set_timing": (ctypes.c_int, [P, i32]),
        "cusfft_get_stage_times": (ctypes.c_int, [P, P, i32]),
        "cusfft_set_stage_limit": (ctypes.c_int, [P, i32]),
        "cusfft_launches_per_execute": (i32, [P]),
        "cusfft_strerror": (ctypes.c_char_p, [ctypes.c_int]),
        "cusfft_last_cuda_error": (i32, []),
        "cusfft_last_nccl_error": (i32, []),
        "cusfft_abi_version": (i32, []),
    }
    for name, (res, args) in sig.items():
        fn = getattr(lib, name)
        fn.restype = res
        fn.argtypes = args
    _lib = lib
    return lib


class CusfftError(RuntimeError):
    def __init__(self, code: int, what: str = ""):
        lib = load_library()
        msg = lib.cusfft_strerror(code).decode()
        if code == CUDA:
            msg += f" (cudaError {lib.cusfft_last_cuda_error()})"
        if code == NCCL:
            msg += f" (ncclResult {lib.cusfft_last_nccl_error()})"
        super().__init__(f"{what}: {msg} [{code}]" if what else f"{msg} [{code}]")
        self.code = code


def check(code: int, what: str = ""):
    if code != SUCCESS:
        raise CusfftError(code, what)
    return code


def default_B(n: int, k: int, bcst: float = 1.0) -> int:
    return int(load_library().cusfft_default_B(n, k, bcst))


def default_params(n: int, k: int, B: int) -> CusfftParams:
    p = CusfftParams()
    check(load_library().cusfft_params_default(ctypes.byref(p), n, k, B), "cusfft_params_default")
    return p


def nccl_unique_id() -> bytes:
    """128 bytes of a fresh ncclUniqueId (cusfft_nccl_unique_id) for cusfft_plan_dist."""
    buf = ctypes.create_string_buffer(128)
    check(load_library().cusfft_nccl_unique_id(buf), "cusfft_nccl_unique_id")
    return buf.raw


def _ptr(t) -> int:
    """Raw data pointer of a torch tensor or numpy array."""
    if hasattr(t, "data_ptr"):
        return t.data_ptr()
    return t.ctypes.data


class Plan:
    """A cusfft plan: ``Plan(n, k, B=None, L=16, **params)``.

    ``params`` are the fields of ``cusfft_params`` (filter, tolerance,
    lobefrac, box_width, loc_loops, vote_threshold, num_select, tau_mode,
    seed, max_hits, device, debug, cutoff_mode, shard_mode, cutoff_threshold,
    loc_tolerance, loc_lobefrac, l2_persist, gather) plus ``taps`` (a float64
    array of user taps).  ``rank`` / ``world`` make a multi-GPU plan
    (cusfft_plan_dist); ``nccl_id`` (128 bytes from ``nccl_unique_id()`` on
    one rank, shared by the caller) lets the plan own the exchange.
    """

    def __init__(self, n: int, k: int, B: int | None = None, L: int = 16, rank: int = 0,
                 world: int = 1, nccl_id: bytes | None = None, **params):
        self._lib = load_library()
        self._h = ctypes.c_void_p()
        if B is None:
            B = default_B(n, k)
        self.n, self.k, self.B, self.L = int(n), int(k), int(B), int(L)
        self.rank, self.world = int(rank), int(world)
        prm = default_params(self.n, self.k, self.B)
        taps = params.pop("taps", None)
        for key, val in params.items():
            if not hasattr(prm, key):
                raise TypeError(f"unknown cusfft parameter {key!r}")
            setattr(prm, key, val)
        if taps is not None:
            self._taps = np.ascontiguousarray(taps, dtype=np.float64)
            prm.taps = self._taps.ctypes.data_as(ctypes.POINTER(ctypes.c_double))
            prm.num_taps = self._taps.shape[0]
        self.params = prm
        if self.world == 1 and nccl_id is None:
            rc = self._lib.cusfft_plan(ctypes.byref(self._h), self.n, self.k, self.B, self.L, ctypes.byref(prm))
        else:
            uid = None
            if nccl_id is not None:
                if len(nccl_id) != 128:
                    raise ValueError("nccl_id must be 128 bytes")
                self._uid = ctypes.create_string_buffer(bytes(nccl_id), 128)
                uid = ctypes.cast(self._uid, ctypes.c_void_p)
            rc = self._lib.cusfft_plan_dist(ctypes.byref(self._h), self.n, self.k, self.B, self.L,
                                            ctypes.byref(prm), self.rank, self.world, uid)
        check(rc, "cusfft_plan")
        info = self.info()
        self.w, self.nb, self.num, self.loc_loops, self.T, self.max_hits = (
            int(info["w"]), int(info["nb"]), int(info["num"]), int(info["loc_loops"]),
            int(info["T"]), int(info["max_hits"]))

    # -- lifetime
    def close(self):
        if getattr(self, "_h", None) is not None and self._h.value:
            self._lib.cusfft_destroy(self._h)
            self._h = ctypes.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.close()

    # -- execution
    def set_stream(self, stream_handle: int):
        check(self._lib.cusfft_set_stream(self._h, ctypes.c_void_p(stream_handle)), "cusfft_set_stream")

    def _use_current_stream(self):
        import torch
        self.set_stream(torch.cuda.current_stream().cuda_stream)

    def execute(self, x, locs=None, vals=None):
        """x: complex128 CUDA tensor [n].  Returns (locs int64[k], vals complex128[k])."""
        import torch
        if x.dtype != torch.complex128 or not x.is_cuda or x.numel() != self.n or not x.is_contiguous():
            raise ValueError("x must be a contiguous complex128 CUDA tensor of length n")
        if locs is None:
            locs = torch.empty(self.k, dtype=torch.int64, device=x.device)
        if vals is None:
            vals = torch.empty(self.k, dtype=torch.complex128, device=x.device)
        self._use_current_stream()
        check(self._lib.cusfft_execute(self._h, ctypes.c_void_p(x.data_ptr()), ctypes.c_void_p(locs.data_ptr()),
                                       ctypes.c_void_p(vals.data_ptr())), "cusfft_execute")
        return locs, vals

    def execute_batch(self, xb, locs=None, vals=None):
        """xb: complex128 CUDA tensor [count, n] (rows may be strided: row stride >= n
        elements, unit element stride).  Returns (locs int64[count, k], vals complex128[count, k]);
        row b equals execute(xb[b]).  See set_pipeline."""
        import torch
        if (xb.dtype != torch.complex128 or not xb.is_cuda or xb.dim() != 2 or xb.shape[1] != self.n
                or xb.stride(1) != 1):
            raise ValueError("xb must be a complex128 CUDA tensor [count, n] with unit element stride")
        count = xb.shape[0]
        if locs is None:
            locs = torch.empty(count, self.k, dtype=torch.int64, device=xb.device)
        if vals is None:
            vals = torch.empty(count, self.k, dtype=torch.complex128, device=xb.device)
        if not (locs.is_contiguous() and vals.is_contiguous() and locs.shape == (count, self.k)
                and vals.shape == (count, self.k)):
            raise ValueError("locs / vals must be contiguous [count, k]")
        self._use_current_stream()
        check(self._lib.cusfft_execute_batch(self._h, ctypes.c_void_p(xb.data_ptr()), count,
                                             max(xb.stride(0), self.n) if count > 1 else self.n,
                                             ctypes.c_void_p(locs.data_ptr()), ctypes.c_void_p(vals.data_ptr())),
              "cusfft_execute_batch")
        return locs, vals

    def set_pipeline(self, depth: int):
        """Pipeline depth of execute_batch (1..8 in-flight signals on internal clone plans)."""
        check(self._lib.cusfft_set_pipeline(self._h, int(depth)), "cusfft_set_pipeline")

    def execute_raw(self, x_ptr: int, locs_ptr: int, vals_ptr: int):
        """Enqueue on the plan's current stream with raw device pointers."""
        return check(self._lib.cusfft_execute(self._h, ctypes.c_void_p(x_ptr), ctypes.c_void_p(locs_ptr),
                                              ctypes.c_void_p(vals_ptr)), "cusfft_execute")

    def execute_host(self, x, locs=None, vals=None):
        """x: host complex128 [n] (numpy or pinned torch).  Synchronous; returns host arrays."""
        if locs is None:
            locs = np.empty(self.k, dtype=np.int64)
        if vals is None:
            vals = np.empty(self.k, dtype=np.complex128)
        if isinstance(x, np.ndarray):
            x = np.ascontiguousarray(x, dtype=np.complex128)
        check(self._lib.cusfft_execute_host(self._h, ctypes.c_void_p(_ptr(x)), ctypes.c_void_p(_ptr(locs)),
                                            ctypes.c_void_p(_ptr(vals))), "cusfft_execute_host")
        return locs, vals

    def execute_local(self, x):
        """x: the whole signal (loop sharding) or this rank's slice (signal sharding)."""
        self._use_current_stream()
        check(self._lib.cusfft_execute_local(self._h, ctypes.c_void_p(x.data_ptr())), "cusfft_execute_local")

    def execute_mid(self):
        """shard_mode 2, between the two exchanges: vote, sorted hit list, this rank's per-loop estimates."""
        self._use_current_stream()
        check(self._lib.cusfft_execute_mid(self._h), "cusfft_execute_mid")

    def execute_finish(self, locs, vals):
        self._use_current_stream()
        check(self._lib.cusfft_execute_finish(self._h, ctypes.c_void_p(locs.data_ptr()),
                                              ctypes.c_void_p(vals.data_ptr())), "cusfft_execute_finish")
        return locs, vals

    def exchange_buffer(self):
        """(device pointer, bytes per rank) of the all-gather buffer."""
        ptr = ctypes.c_void_p()
        per = ctypes.c_int64()
        check(self._lib.cusfft_exchange_buffer(self._h, ctypes.byref(ptr), ctypes.byref(per)),
              "cusfft_exchange_buffer")
        return int(ptr.value), int(per.value)

    def exchange_buffer2(self):
        """shard_mode 2: (device pointer, bytes per rank) of the per-loop estimate all-gather buffer."""
        ptr = ctypes.c_void_p()
        per = ctypes.c_int64()
        check(self._lib.cusfft_exchange_buffer2(self._h, ctypes.byref(ptr), ctypes.byref(per)),
              "cusfft_exchange_buffer2")
        return int(ptr.value), int(per.value)

    def exchange_kind(self) -> int:
        """0: all-gather of rank slices (loop sharding); 1: fp64 sum all-reduce (signal sharding);
        2: two all-gathers (shard_mode 2: candidate records, then per-loop estimates)."""
        k = int(self._lib.cusfft_exchange_kind(self._h))
        if k < 0:
            check(k, "cusfft_exchange_kind")
        return k

    def status(self) -> int:
        return int(self._lib.cusfft_status(self._h))

    # -- introspection
    def info(self):
        info = np.zeros(16, dtype=np.int64)
        a = np.zeros(self.L, dtype=np.int64)
        s = np.zeros(self.L, dtype=np.int64)
        t = np.zeros(self.L, dtype=np.int64)
        check(self._lib.cusfft_get_info(self._h, ctypes.c_void_p(info.ctypes.data), ctypes.c_void_p(a.ctypes.data),
                                        ctypes.c_void_p(s.ctypes.data), ctypes.c_void_p(t.ctypes.data)),
              "cusfft_get_info")
        keys = ("n", "k", "B", "L", "w", "nb", "num", "loc_loops", "T", "max_hits", "sectors", "staged",
                "w_loc", "filters", "tail", "owns_comm")
        d = dict(zip(keys, info.tolist()))
        d.update(a=a, sigma=s, tau=t)
        return d

    def debug(self, what: int):
        dtype = {DEBUG_U: np.complex128, DEBUG_UHAT: np.complex128, DEBUG_WINNERS: np.int32,
                 DEBUG_HITS: np.int32, DEBUG_HIT_VALS: np.complex128, DEBUG_PER_LOOP: np.complex128,
                 DEBUG_TAPS: np.float64, DEBUG_GHAT: np.complex128, DEBUG_NUM_HITS: np.int64,
                 DEBUG_LOC_TAPS: np.float64, DEBUG_LOC_GHAT: np.complex128}[what]
        need = int(self._lib.cusfft_get_debug(self._h, what, None, 0))
        if need < 0:
            check(need, "cusfft_get_debug")
        buf = np.zeros(need // np.dtype(dtype).itemsize, dtype=dtype)
        if need:
            got = int(self._lib.cusfft_get_debug(self._h, what, ctypes.c_void_p(buf.ctypes.data), need))
            if got < 0:
                check(got, "cusfft_get_debug")
        if what in (DEBUG_U,):
            buf = buf.reshape(-1, self.B)
        elif what == DEBUG_UHAT:
            buf = buf.reshape(self.L, self.B)
        elif what == DEBUG_WINNERS:
            buf = buf.reshape(self.loc_loops, -1)
        elif what == DEBUG_PER_LOOP and buf.size:
            buf = buf.reshape(-1, self.L)
        return buf

    def set_timing(self, mode: int = 1):
        """0 off; 1 direct launches with stage events; 2 events around phase 1 inside the CUDA graph."""
        check(self._lib.cusfft_set_timing(self._h, int(mode)), "cusfft_set_timing")

    def stage_times(self):
        """Stage times (ms) of the last timed execution; 'gather' is phase 1 of
        the staged fold alone (-1 when the plan is not staged).  With the fused
        tail (info()['tail'] == 1) 'vote' covers vote + estimate + output."""
        ms = (ctypes.c_float * 7)()
        check(self._lib.cusfft_get_stage_times(self._h, ms, 7), "cusfft_get_stage_times")
        return dict(zip(("fold", "fft", "cutoff", "vote", "estimate", "output", "gather"), list(ms)))

    def set_stage_limit(self, stages: int):
        check(self._lib.cusfft_set_stage_limit(self._h, stages), "cusfft_set_stage_limit")

    def launches_per_execute(self) -> int:
        return int(self._lib.cusfft_launches_per_execute(self._h))
