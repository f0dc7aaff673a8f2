"""Seeded synthetic inputs shaped like the paper's workloads.

Shared by the tests, ``bench.py`` and ``smoke()``; it holds none of the sFFT's
arithmetic (no permutation, filter, bucketing, selection or estimation) — only
the recipe for a planted k-sparse spectrum and its time-domain signal
(DESIGN.md §5 "input recipe", SURVEY.md §8(c) [Z16], §8(d)).

Signal model: k distinct locations drawn uniformly without replacement from
[0, n); coefficients X_f = e^{i theta}, theta ~ U[0, 2 pi) (unit magnitude,
the paper's "exact 1000 non-zero coefficients"); time signal
x_t = sum_f X_f e^{+2 pi i f t / n} so that the forward DFT divided by n
returns X.  Optional complex white Gaussian noise at a given SNR (per-sample
signal power = sum |X_f|^2).
"""
from __future__ import annotations

import numpy as np


def planted_spectrum(n: int, k: int, seed: int, unit_magnitude: bool = True):
    """Return (support int64[k] sorted, X complex128[k])."""
    rng = np.random.default_rng([0x5F5F7, seed])
    support = np.sort(rng.choice(n, size=k, replace=False)).astype(np.int64)
    theta = rng.uniform(0.0, 2.0 * np.pi, size=k)
    mag = np.ones(k) if unit_magnitude else rng.uniform(0.5, 2.0, size=k)
    return support, mag * np.exp(1j * theta)


def planted_signal(n: int, k: int, seed: int, snr_db: float | None = None,
                   unit_magnitude: bool = True):
    """Return (x complex128[n], support, X).  x = n * ifft(spectrum)."""
    support, X = planted_spectrum(n, k, seed, unit_magnitude)
    spec = np.zeros(n, dtype=np.complex128)
    spec[support] = X
    x = np.fft.ifft(spec) * n
    if snr_db is not None:
        rng = np.random.default_rng([0x401CE, seed])
        power = float(np.sum(np.abs(X) ** 2))
        var = power / (10.0 ** (snr_db / 10.0))
        noise = rng.standard_normal(n) + 1j * rng.standard_normal(n)
        x = x + noise * np.sqrt(var / 2.0)
    return np.ascontiguousarray(x), support, X


def dense_signal(n: int, seed: int):
    """Dense complex Gaussian signal (no sparsity) for identity checks."""
    rng = np.random.default_rng([0xDE45E, seed])
    return rng.standard_normal(n) + 1j * rng.standard_normal(n)
