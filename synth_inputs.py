"""Seeded, counter-based synthetic inputs shared by the oracle tests and the CUDA path.

This module holds NONE of the FMM-FFT's arithmetic: it only manufactures input vectors.
It is the one module both sides (``oracle/`` and the GPU tests / bench) may import.

Workload recipe (the paper
uses random inputs, each component uniform on [-1, 1]):

    x[n] = u(seed, 2n) + i * u(seed, 2n+1),   u = 2 * U53(splitmix64(seed*K + c)) - 1

where U53 maps the top 53 bits of a 64-bit word to [0, 1). The generator is counter-based
(the value at global index n depends only on (seed, n)), so every rank of a distributed run
produces its own shard x[g*N/G : (g+1)*N/G] independently, bit-identical to the slice of the
full vector. complex64 runs round the float64 values to float32; the reference DFT is taken of
the rounded values.
"""
from __future__ import annotations

import numpy as np

DEFAULT_SEED = 20171112  # the paper's conference date

_GOLDEN = np.uint64(0x9E3779B97F4A7C15)
_M1 = np.uint64(0xBF58476D1CE4E5B9)
_M2 = np.uint64(0x94D049BB133111EB)


def _splitmix64(z: np.ndarray) -> np.ndarray:
    """splitmix64 finaliser on a uint64 array (wrapping arithmetic)."""
    with np.errstate(over="ignore"):
        z = z + _GOLDEN
        z = (z ^ (z >> np.uint64(30))) * _M1
        z = (z ^ (z >> np.uint64(27))) * _M2
        z = z ^ (z >> np.uint64(31))
    return z


def uniform_pm1(seed: int, counters: np.ndarray) -> np.ndarray:
    """float64 values uniform on [-1, 1), one per uint64 counter."""
    with np.errstate(over="ignore"):
        key = np.uint64(seed & 0xFFFFFFFFFFFFFFFF) * np.uint64(0xD1B54A32D192ED03)
        bits = _splitmix64(counters.astype(np.uint64) ^ key)
    u = (bits >> np.uint64(11)).astype(np.float64) * (1.0 / 9007199254740992.0)
    return 2.0 * u - 1.0


def complex_uniform(n0: int, count: int, seed: int = DEFAULT_SEED,
                    dtype=np.complex128, chunk: int = 1 << 22) -> np.ndarray:
    """x[n0 : n0+count] of the global seeded vector, as ``dtype`` (complex64 or complex128).
    Chunks are filled by a thread pool (numpy releases the GIL); values depend only on n."""
    out = np.empty(count, dtype=dtype)

    def fill(a):
        b = min(count, a + chunk)
        n = np.arange(n0 + a, n0 + b, dtype=np.uint64)
        out[a:b].real = uniform_pm1(seed, np.uint64(2) * n)
        out[a:b].imag = uniform_pm1(seed, np.uint64(2) * n + np.uint64(1))

    starts = range(0, count, chunk)
    if count > 4 * chunk:
        import os
        from concurrent.futures import ThreadPoolExecutor
        with ThreadPoolExecutor(max_workers=min(16, os.cpu_count() or 1)) as ex:
            list(ex.map(fill, starts))
    else:
        for a in starts:
            fill(a)
    return out


def real_uniform(n0: int, count: int, seed: int = DEFAULT_SEED, dtype=np.float64) -> np.ndarray:
    """Real inputs x[n0 : n0+count] (FMMFFT_FLAG_REAL), uniform on [-1, 1), as ``dtype``."""
    n = np.arange(n0, n0 + count, dtype=np.uint64)
    return uniform_pm1(seed, n).astype(dtype)


def shard(N: int, G: int, rank: int, seed: int = DEFAULT_SEED, dtype=np.complex128) -> np.ndarray:
    """Rank ``rank``'s block of the length-N input: x[rank*N/G : (rank+1)*N/G]."""
    assert N % G == 0
    n = N // G
    return complex_uniform(rank * n, n, seed=seed, dtype=dtype)


# ---- structured inputs for closed-form tests only (never the benchmark workload) ----

def delta(N: int, j0: int = 0, dtype=np.complex128) -> np.ndarray:
    x = np.zeros(N, dtype=dtype)
    x[j0] = 1.0
    return x


def tone(N: int, k0: int, dtype=np.complex128) -> np.ndarray:
    """x_j = exp(+2*pi*i*k0*j/N), angle reduced exactly (k0*j mod N)."""
    j = np.arange(N, dtype=np.int64)
    e = (k0 * j) % N
    return np.exp(2j * np.pi * e / N).astype(dtype)
