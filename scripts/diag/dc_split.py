"""Diagnostic: DC (sum over m) of the near field T_near and of the whole FMM output T per FMM p,
GPU complex64 vs the float64 oracle (N = 2^24, P = 16, B = 4, Q = 16, M_L = 64)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import numpy as np, torch
import synth_inputs as SI
from oracle import fmmfft_oracle as O
from paper_conf_sc_cecka17_b200 import FmmFFT

N, P, B, Q, M_L = 1 << 24, 16, 4, 16, 64
M = N // P
L = O.tree_levels(N, P, M_L)
x = SI.complex_uniform(0, N, dtype=np.complex64)
S = x.astype(np.complex128).reshape(2 ** L, M_L, P)
st = O.fmm_stages(S, N, P, B, Q)
r_ex = S.sum(axis=(0, 1))
p = np.arange(P)
dcT_ex = M / np.tan(np.pi * p[1:] / P) * r_ex[1:]                      # M cot(pi p/P) r_p (closed form)
dcT_or = st["T"].sum(axis=(0, 1))[1:]
dcN_or = st["T_near"].sum(axis=(0, 1))[1:]
print("oracle DC(T) vs closed form:", np.array2string(np.abs(dcT_or - dcT_ex) / np.abs(dcT_ex), precision=1))
for env in (None, "simt"):
    if env:
        os.environ["FMMFFT_S2T"] = env
    pl = FmmFFT(N=N, P=P, B=B, Q=Q, precision="c64", debug=True, M_L=M_L)
    pl(torch.from_numpy(x).cuda())
    torch.cuda.synchronize()
    t = pl.debug_buffer("T_near").cpu().numpy()
    f = t.view(np.float32).reshape(P, 2 ** L, 2, M_L).astype(np.float64)
    Tn = f[:, :, 0, :] + 1j * f[:, :, 1, :]                           # [p, b, m]
    dcN = Tn.sum(axis=(1, 2))[1:]
    W = pl.debug_buffer("W").cpu().numpy().astype(np.complex128).reshape(P, M)
    Wsum = W.sum(axis=1)
    tdc = np.array([np.sum(np.exp(2j * np.pi * ((pp * np.arange(P)) % P) / P) * Wsum) / P for pp in range(P)])[1:]
    rho = (np.exp(-1j * np.pi * p / P) * np.sin(np.pi * p / P) / M)[1:]
    r = pl.debug_buffer("r").cpu().numpy().astype(np.complex128)[1:]
    dcT = tdc / rho - 1j * M * r                                      # undo POST: sum_m T = DC(T')/rho - i M r
    print(env or "tc", "DC(T_near) rel err vs oracle:", np.array2string(np.abs(dcN - dcN_or) / np.abs(dcN_or), precision=1))
    print(env or "tc", "DC(T) rel err vs closed form:", np.array2string(np.abs(dcT - dcT_ex) / np.abs(dcT_ex), precision=1))
    print(env or "tc", "|DC(T_near)| / |DC(T)|:", np.array2string(np.abs(dcN_or) / np.abs(dcT_ex), precision=1))
    # far-field DC = DC(T) - DC(T_near); compare with the oracle's
    far_or = dcT_or - dcN_or
    print(env or "tc", "DC(T_far) rel err vs oracle:", np.array2string(np.abs((dcT - dcN) - far_or) / np.abs(far_or), precision=1))
    pl.close()
    os.environ.pop("FMMFFT_S2T", None)
