"""B200-native sparse FFT engine (the sFFT hot path cusFFT parallelises,
Wang/Chandrasekaran/Chapman, IPDPS'16).

The product is the C-ABI library ``libcusfft.so`` (``include/cusfft.h``,
kernels in ``csrc/``).  This package is its thin Python binding plus the
multi-GPU loop-sharding driver (``dist``) and the seeded input generator
(``workload``).  No step of the transform runs in Python and there is no CPU
fallback.
"""
from ._binding import (  # noqa: F401
    DEBUG_GHAT, DEBUG_HIT_VALS, DEBUG_HITS, DEBUG_NUM_HITS, DEBUG_PER_LOOP, DEBUG_TAPS,
    DEBUG_LOC_GHAT, DEBUG_LOC_TAPS, DEBUG_U, DEBUG_UHAT, DEBUG_WINNERS, FILTER_DOLPH_CHEBYSHEV, FILTER_GAUSSIAN,
    CusfftError, CusfftParams, Plan, default_B, default_params, load_library, nccl_unique_id,
)

__all__ = ["Plan", "default_B", "default_params", "load_library", "nccl_unique_id", "CusfftError", "CusfftParams"]
