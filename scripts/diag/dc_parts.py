"""Diagnostic: where the k1 = 0 (row-DC) error comes from — r_p, the P-FFT output W row sums, and
complex128 for comparison (N = 2^26, P = 16, B = 4, G = 1)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import numpy as np, torch
import synth_inputs as SI
from oracle import fmmfft_oracle as O
from paper_conf_sc_cecka17_b200 import FmmFFT

lN = int(sys.argv[1]) if len(sys.argv) > 1 else 26
N, P, B, Q = 1 << lN, 16, 4, 16
M = N // P
for prec, dt in (("c64", np.complex64), ("c128", np.complex128)):
    x = SI.complex_uniform(0, N, dtype=dt)
    xp = x.astype(np.complex128).reshape(M, P)            # x[p + P m]
    r_exact = xp.sum(axis=0)                              # r_p = sum_m x_p[m]
    pl = FmmFFT(N=N, P=P, B=B, Q=Q, precision=prec, debug=True)
    y = pl(torch.from_numpy(x).cuda())
    torch.cuda.synchronize()
    r = pl.debug_buffer("r").cpu().numpy().astype(np.complex128)
    W = pl.debug_buffer("W").cpu().numpy().astype(np.complex128).reshape(P, M)
    yc = y.cpu().numpy().astype(np.complex128)
    ks = np.arange(P) * M
    ref = O.dft_at(x, ks)
    # exact DC of row k2: sum_p w_P^{p k2} r_p
    p = np.arange(P)
    dc_exact = np.array([np.sum(np.exp(-2j * np.pi * ((p * k2) % P) / P) * r_exact) for k2 in range(P)])
    print(prec, "r rel err per p:", np.array2string(np.abs(r[1:] - r_exact[1:]) / np.abs(r_exact[1:]), precision=2))
    print(prec, "dc_exact vs dft_at:", np.max(np.abs(dc_exact - ref)) / np.max(np.abs(ref)))
    print(prec, "W row sums vs exact DC:", np.linalg.norm(W.sum(axis=1) - dc_exact) / np.linalg.norm(dc_exact))
    print(prec, "y DC bins vs exact:", np.linalg.norm(yc[ks] - dc_exact) / np.linalg.norm(dc_exact))
    pl.close()
    # per-p DC of T' = POST(T): the P-FFT is exact enough to invert: T'_p DC = (1/P) sum_k2 w^{-p k2} DC_k2
    Wsum = W.sum(axis=1)
    tdc = np.array([np.sum(np.exp(2j * np.pi * ((pp * np.arange(P)) % P) / P) * Wsum) / P for pp in range(P)])
    print(prec, "T'_p DC rel err per p:", np.array2string(np.abs(tdc - r_exact) / np.abs(r_exact), precision=2))
