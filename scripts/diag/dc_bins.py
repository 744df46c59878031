"""Diagnostic: error of the k1 = 0 output bins (y[M k2], the DC of every M-point row) vs random
bins, against eq. (1) evaluated at those bins (oracle dft_at)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import numpy as np, torch
import synth_inputs as SI
from oracle import fmmfft_oracle as O
from paper_conf_sc_cecka17_b200 import FmmFFT

def rl(a, b):
    return float(np.linalg.norm(a - b) / np.linalg.norm(b))

cases = [(26, 16, 4, 1, 64), (26, 128, 4, 8, 64), (28, 64, 4, 1, 64), (28, 64, 4, 8, 64), (30, 64, 4, 1, 64), (30, 64, 4, 8, 64)]
xs = {}
for lN, P, B, G, M_L in cases:
    N = 1 << lN
    if lN not in xs:
        xs.clear()
        xs[lN] = SI.complex_uniform(0, N, dtype=np.complex64)
    x = xs[lN]
    M = N // P
    rng = np.random.default_rng(3)
    kdc = np.arange(P) * M
    kr = rng.integers(0, N, 64)
    ks = np.concatenate([kdc, kr])
    ref = O.dft_at(x, ks)
    for s2t in ("tc", "simt"):
        if s2t == "simt":
            os.environ["FMMFFT_S2T"] = "simt"
        pl = FmmFFT(N=N, P=P, G=G, B=B, Q=16, precision="c64", M_L=M_L, virtual=G > 1)
        yd = pl(torch.from_numpy(x).cuda())
        ys = yd[torch.from_numpy(ks).cuda()].cpu().numpy().astype(np.complex128)
        pl.close()
        del yd
        os.environ.pop("FMMFFT_S2T", None)
        print(f"N=2^{lN} P={P} B={B} G={G} s2t={s2t}: dc bins {rl(ys[:P], ref[:P]):.2e}  random bins {rl(ys[P:], ref[P:]):.2e}"
              f"  worst dc bin k2={int(np.argmax(np.abs(ys[:P]-ref[:P])))}", flush=True)
        torch.cuda.empty_cache()
