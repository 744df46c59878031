"""Time cuFFT (through torch.fft.fft, the library comparator of BASELINE.json's metric) on one GPU
for the workloads' N and precision, with the same L2 flush and CUDA-event timing as bench.py.

    python scripts/cufft_baseline.py [--steps K]

Prints one JSON line per (N, precision): GFLOP/s = 5 N log2 N / t. Not part of the product path.
"""
import argparse
import json
import math

import torch


def time_fft(N, dtype, steps):
    x = (torch.rand(N, dtype=dtype, device="cuda") - 0.5) * 2
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    for _ in range(5):
        torch.fft.fft(x)
    torch.cuda.synchronize()
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(steps)]
    for a, b in ev:
        flush.zero_()
        a.record()
        torch.fft.fft(x)
        b.record()
    torch.cuda.synchronize()
    ms = sum(a.elapsed_time(b) for a, b in ev) / steps
    return ms


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--steps", type=int, default=50)
    args = ap.parse_args()
    for lg, dt in ((20, torch.complex64), (24, torch.complex64), (26, torch.complex64), (28, torch.complex64),
                   (20, torch.complex128), (26, torch.complex128), (28, torch.complex128)):
        N = 1 << lg
        ms = time_fft(N, dt, args.steps)
        print(json.dumps({"lib": "cufft (torch.fft.fft)", "N": N, "dtype": str(dt), "ms": ms,
                          "gflops": 5 * N * math.log2(N) / (ms * 1e-3) / 1e9}), flush=True)
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
