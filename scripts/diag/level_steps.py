"""Diagnostic: the error each GPU tree step introduces on its own. For every level, recompute the
step in float64 from the GPU's own inputs (M^{l+1} -> M^l; M^l, L^{l-1} -> L^l) and report the
step's relative error and the bias of its errors (|mean over boxes| / rms)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import numpy as np, torch
import synth_inputs as SI
from oracle import fmmfft_oracle as O
from paper_conf_sc_cecka17_b200 import FmmFFT

N, P, B, Q, M_L = [int(v) for v in sys.argv[1:6]] if len(sys.argv) > 5 else (1 << 22, 16, 4, 16, 64)
prec = sys.argv[6] if len(sys.argv) > 6 else "c64"
L = O.tree_levels(N, P, M_L)
x = SI.complex_uniform(0, N, dtype=np.complex64 if prec == "c64" else np.complex128)
pl = FmmFFT(N=N, P=P, B=B, Q=Q, precision=prec, M_L=M_L, debug=True)
pl(torch.from_numpy(x).cuda())
torch.cuda.synchronize()
print(f"N={N} P={P} B={B} Q={Q} M_L={M_L} {prec} variant={pl.info['variant']}")
Mg = {l: pl.debug_buffer("M", l).cpu().numpy().astype(np.complex128).reshape(2 ** l, Q, P)[:, :, 1:] for l in range(B, L + 1)}
Lg = {l: pl.debug_buffer("L", l).cpu().numpy().astype(np.complex128).reshape(2 ** l, Q, P)[:, :, 1:] for l in range(B, L + 1)}
M2M = O.op_M2M(Q)

def report(tag, gpu, ref):
    e = gpu - ref
    rel = np.linalg.norm(e) / np.linalg.norm(ref)
    bias = np.abs(e.mean(axis=0)) / np.sqrt(np.mean(np.abs(e) ** 2, axis=0))     # per (q, p)
    print(f"  {tag:10s} rel {rel:.1e}  bias |mean|/rms: median {np.median(bias):.2f} max {bias.max():.2f}"
          f"  (random ~ {1/np.sqrt(gpu.shape[0]):.2f})")

S = x.astype(np.complex128).reshape(2 ** L, M_L, P)
report(f"S2M L={L}", Mg[L], np.einsum("qm,bmp->bqp", O.op_S2M(Q, M_L), S[:, :, 1:]))
for lev in range(L - 1, B - 1, -1):
    report(f"M2M l={lev}", Mg[lev], np.einsum("qk,bkp->bqp", M2M, Mg[lev + 1].reshape(2 ** lev, 2 * Q, P - 1)))
nb = 2 ** B
ref = np.zeros((nb, Q, P - 1), complex)
for s in O.m2l_shifts(B, B, 0):
    ref += np.einsum("pij,bjp->bip", O.op_M2L(N, P, Q, B, s), Mg[B][(np.arange(nb) + s) % nb])
report(f"M2L-B l={B}", Lg[B], ref)
for lev in range(B + 1, L + 1):
    nb = 2 ** lev
    ref = np.einsum("qk,bkp->bqp", M2M.T, Lg[lev - 1]).reshape(nb, Q, P - 1)
    for parity in (0, 1):
        b = np.arange(parity, nb, 2)
        for s in O.m2l_shifts(lev, B, parity):
            ref[b] += np.einsum("pij,bjp->bip", O.op_M2L(N, P, Q, lev, s), Mg[lev][(b + s) % nb])
    report(f"M2L+L2L {lev}", Lg[lev], ref)
