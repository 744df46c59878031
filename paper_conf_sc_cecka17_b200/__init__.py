"""B200-native FMM-FFT (Cecka, SC17): a distributed in-order 1D complex FFT N = M P via the
Edelman factorisation F_N = F_{M,P} H^_{M,P}, with sm_100a CUDA kernels behind the C ABI of
include/fmmfft.h. The CUDA library is required — there is no CPU fallback: touching FmmFFT
(or init_comm / destroy_comm) raises ImportError if libfmmfft.so is missing."""

__all__ = ["FmmFFT", "init_comm", "init_comm_local", "destroy_comm", "autotune"]


def __getattr__(name):  # lazy, so `python -m paper_conf_sc_cecka17_b200.build` works unbuilt
    if name in __all__:
        from . import fmmfft
        return getattr(fmmfft, name)
    raise AttributeError(name)
