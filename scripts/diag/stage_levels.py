"""Diagnostic: per-level M^l / L^l relative error vs the oracle on a wide tree (per-level kernels)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import numpy as np, torch
import synth_inputs as SI
from oracle import fmmfft_oracle as O
from paper_conf_sc_cecka17_b200 import FmmFFT

for (N, P, B, Q, M_L, prec) in [(1 << 22, 16, 4, 16, 64, "c64"), (1 << 22, 16, 4, 16, 64, "c128"), (1 << 20, 64, 2, 16, 64, "c64")]:
    L = O.tree_levels(N, P, M_L)
    x = SI.complex_uniform(0, N, dtype=np.complex64 if prec == "c64" else np.complex128)
    S = x.astype(np.complex128).reshape(2 ** L, M_L, P)
    st = O.fmm_stages(S, N, P, B, Q)
    pl = FmmFFT(N=N, P=P, B=B, Q=Q, precision=prec, M_L=M_L, debug=True)
    pl(torch.from_numpy(x).cuda())
    torch.cuda.synchronize()
    print(f"N={N} P={P} B={B} {prec} variant={pl.info['variant']}")
    for lev in range(B, L + 1):
        Mg = pl.debug_buffer("M", lev).cpu().numpy().reshape(2 ** lev, Q, P)[:, :, 1:]
        Lg = pl.debug_buffer("L", lev).cpu().numpy().reshape(2 ** lev, Q, P)[:, :, 1:]
        em = np.linalg.norm(Mg - st["M"][lev]) / np.linalg.norm(st["M"][lev])
        el = np.linalg.norm(Lg - st["L"][lev]) / np.linalg.norm(st["L"][lev])
        # sum over boxes (the part that feeds the DC) per p
        sm = np.abs(Lg.sum(axis=(0, 1)) - st["L"][lev].sum(axis=(0, 1))) / np.abs(st["L"][lev]).sum(axis=(0, 1)) * 2 ** lev
        print(f"  l={lev:2d}  M {em:.1e}  L {el:.1e}  L box-sum err / mean|L| (max over p) {sm.max():.1e}")
    pl.close()
