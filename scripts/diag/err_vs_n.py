"""Diagnostic: relative l2 error vs N of the FMM-FFT (complex64), the in-house four-step FFT and
cuFFT, each against numpy's float64 FFT of the same rounded input."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import numpy as np, torch
import synth_inputs as SI
from paper_conf_sc_cecka17_b200 import FmmFFT

def rel(a, b):
    return float(np.linalg.norm(a.astype(np.complex128) - b) / np.linalg.norm(b))

for lN in [int(v) for v in sys.argv[1:]] or [20, 22, 24, 26, 28]:
    N = 1 << lN
    x = SI.complex_uniform(0, N, dtype=np.complex64)
    ref = np.fft.fft(x.astype(np.complex128))
    xd = torch.from_numpy(x).cuda()
    out = {"N": f"2^{lN}"}
    for P, B in [(16, 4), (64, 2), (256, 2)]:
        try:
            pl = FmmFFT(N=N, P=P, B=B, Q=16, precision="c64")
            out[f"fmm P={P}"] = rel(pl(xd).cpu().numpy(), ref)
            pl.close()
        except Exception as e:
            out[f"fmm P={P}"] = str(e)[:60]
    for P, B, Q in [(16, 4, 24), (16, 4, 12)]:
        pl = FmmFFT(N=N, P=P, B=B, Q=Q, precision="c64")
        out[f"fmm P={P} Q={Q}"] = rel(pl(xd).cpu().numpy(), ref)
        pl.close()
    os.environ["FMMFFT_S2T"] = "simt"
    pl = FmmFFT(N=N, P=16, B=4, Q=16, precision="c64")
    out["fmm P=16 simt-s2t"] = rel(pl(xd).cpu().numpy(), ref)
    pl.close()
    del os.environ["FMMFFT_S2T"]
    d = FmmFFT(N=N, P=1, precision="c64", direct=True)
    out["fourstep"] = rel(d(xd).cpu().numpy(), ref)
    d.close()
    out["cufft"] = rel(torch.fft.fft(xd).cpu().numpy(), ref)
    print(out, flush=True)
