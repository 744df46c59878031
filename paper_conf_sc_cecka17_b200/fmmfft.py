"""Python API over the C ABI (include/fmmfft.h). PyTorch provides device memory, streams and the
process group; every FMM-FFT step runs in libfmmfft.so's sm_100a kernels.

    plan = FmmFFT(N=1 << 20, P=64, G=1, B=2, Q=16, precision="c64")
    y = plan(x)                      # x: torch.complex64 CUDA tensor of N/G elements

Multi-GPU (one process per GPU, launched by torchrun): call ``init_comm()`` once after
``torch.distributed.init_process_group``; every rank then builds the same plan and calls it
on its block x[g N/G : (g+1) N/G].
"""
from __future__ import annotations

import ctypes

import torch

from . import _lib
from ._lib import (C64, C128, FLAG_DEBUG, FLAG_DIRECT, FLAG_INVERSE, FLAG_PROFILE, FLAG_REAL, FLAG_VIRTUAL,
                   FLAG_VIRTUAL_NCCL, check, lib)

_DT = {"c64": (C64, torch.complex64), "c128": (C128, torch.complex128)}


def _stream_ptr(stream) -> ctypes.c_void_p:
    s = stream if stream is not None else torch.cuda.current_stream()
    return ctypes.c_void_p(s.cuda_stream)


def init_comm(group=None) -> None:
    """NCCL communicator for this process's rank (collective). Rank 0 creates the unique id and
    torch.distributed broadcasts it; binds to the current CUDA device."""
    import torch.distributed as dist
    rank, world = dist.get_rank(group), dist.get_world_size(group)
    buf = torch.zeros(128, dtype=torch.uint8)
    if rank == 0:
        raw = ctypes.create_string_buffer(128)
        check(lib.fmmfft_get_unique_id(raw))
        buf = torch.frombuffer(bytearray(raw.raw), dtype=torch.uint8).clone()
    if dist.get_backend(group) == "nccl":
        buf = buf.cuda()
    dist.broadcast(buf, src=0, group=group)
    check(lib.fmmfft_comm_init(rank, world, bytes(buf.cpu().numpy().tobytes())))


def init_comm_local() -> None:
    """A 1-rank NCCL communicator on the current device, no process group needed: the transport
    of virtual plans created with transport="nccl" (FMMFFT_FLAG_VIRTUAL_NCCL)."""
    raw = ctypes.create_string_buffer(128)
    check(lib.fmmfft_get_unique_id(raw))
    check(lib.fmmfft_comm_init(0, 1, raw.raw))


def autotune(N: int, G: int = 1, precision: str = "c64", tol: float = 1e-5, measure: bool = True) -> dict:
    """(P, B, Q, M_L) for an FMM-FFT of length N on G GPUs meeting relative-l2 error `tol`
    (fmmfft_autotune: Q from the error model, (P, B) timed on the current device when measure,
    else ranked by the roofline model). Returns the plan arguments plus ms / error / candidates."""
    t = _lib.Tune()
    check(lib.fmmfft_autotune(N, G, _DT[precision][0], float(tol), 1 if measure else 0, ctypes.byref(t)))
    return {f: getattr(t, f) for f, _ in _lib.Tune._fields_}


def destroy_comm() -> None:
    check(lib.fmmfft_comm_destroy())


class _DevView:
    """__cuda_array_interface__ wrapper so torch can view a library-owned device buffer."""

    def __init__(self, ptr: int, nbytes: int, dtype: torch.dtype):
        n = nbytes // (8 if dtype == torch.complex64 else 16)
        self.__cuda_array_interface__ = {
            "shape": (2 * n,), "typestr": "<f4" if dtype == torch.complex64 else "<f8",
            "data": (ptr, False), "version": 3, "strides": None,
        }


class FmmFFT:
    def __init__(self, N: int, P: int, G: int = 1, B: int = 2, Q: int = 16, precision: str = "c64",
                 M_L: int = 64, virtual: bool = False, profile: bool = False, debug: bool = False,
                 inverse: bool = False, direct: bool = False, real: bool = False, transport: str = "copy"):
        """direct=True: no FMM — the plain four-step FFT of length N on one GPU with the same M-FFT
        kernels (the in-house Cooley-Tukey comparator; P, B, Q, M_L ignored).
        real=True (FMMFFT_FLAG_REAL): N real inputs -> N/2+1 complex outputs; P, B, Q, M_L
        describe the complex plan of length N/2 (G = 1).
        transport="nccl" (virtual plans): the virtual ranks' exchanges through NCCL on a 1-rank
        communicator (init_comm_local) instead of device copies."""
        self.N, self.P, self.G, self.B, self.Q, self.M_L = N, P, G, B, Q, M_L
        self.precision = precision
        self.virtual = virtual
        self._prec, self.dtype = _DT[precision]
        flags = (FLAG_VIRTUAL if virtual else 0) | (FLAG_PROFILE if profile else 0) | (FLAG_DEBUG if debug else 0) | \
                (FLAG_INVERSE if inverse else 0) | (FLAG_DIRECT if direct else 0) | (FLAG_REAL if real else 0) | \
                (FLAG_VIRTUAL_NCCL if transport == "nccl" else 0)
        self.inverse = inverse
        self.real = real
        rdt = torch.float32 if precision == "c64" else torch.float64
        # real forward: N reals -> N/2+1 complex; real inverse: N/2+1 complex -> N reals
        self.in_dtype = rdt if real and not inverse else self.dtype
        self.out_dtype = rdt if real and inverse else self.dtype
        h = ctypes.c_void_p()
        check(lib.fmmfft_plan_ex(ctypes.byref(h), N, P, G, B, Q, self._prec, M_L, flags))
        self._h = h
        self.n_local = N if virtual else N // G

    # -- execution
    def __call__(self, x: torch.Tensor, out: torch.Tensor | None = None, stream=None) -> torch.Tensor:
        half = self.n_local // 2 + 1              # real plans: this rank's N/(2G) + 1 (virtual: N/2 + 1)
        n_in = half if self.real and self.inverse else self.n_local
        n_out = half if self.real and not self.inverse else self.n_local
        if x.dtype != self.in_dtype or not x.is_cuda or not x.is_contiguous() or x.numel() != n_in:
            raise ValueError(f"expected a contiguous CUDA {self.in_dtype} tensor of {n_in} elements")
        if out is None:
            out = torch.empty(n_out, dtype=self.out_dtype, device=x.device)
        elif out.dtype != self.out_dtype or not out.is_contiguous() or out.numel() != n_out:
            raise ValueError(f"out must be a contiguous {self.out_dtype} tensor of {n_out} elements")
        check(lib.fmmfft_execute(self._h, ctypes.c_void_p(x.data_ptr()), ctypes.c_void_p(out.data_ptr()),
                                 _stream_ptr(stream)))
        return out

    def execute_host(self, x_host: torch.Tensor, out_host: torch.Tensor, stream=None) -> None:
        """End-to-end path through the C ABI with host buffers (pinned for async copies)."""
        check(lib.fmmfft_execute_host(self._h, ctypes.c_void_p(x_host.data_ptr()),
                                      ctypes.c_void_p(out_host.data_ptr()), _stream_ptr(stream)))

    # -- introspection
    @property
    def info(self) -> dict:
        inf = _lib.Info()
        check(lib.fmmfft_get_info(self._h, ctypes.byref(inf)))
        return {f: getattr(inf, f) for f, _ in _lib.Info._fields_}

    def stage_times(self) -> dict:
        arr = (ctypes.c_float * 32)()
        n = ctypes.c_int()
        check(lib.fmmfft_stage_times(self._h, arr, 32, ctypes.byref(n)))
        return {lib.fmmfft_stage_name(i).decode(): float(arr[i]) for i in range(n.value)}

    def debug_buffer(self, which: str, level: int = 0, rank: int = 0) -> torch.Tensor:
        """Copy of an internal buffer after an execute (for stage parity tests)."""
        ids = {"T_near": 0, "M": 1, "L": 2, "W": 3, "r": 4}
        ptr, nbytes = ctypes.c_void_p(), ctypes.c_size_t()
        check(lib.fmmfft_debug_buffer(self._h, rank, ids[which], level, ctypes.byref(ptr), ctypes.byref(nbytes)))
        torch.cuda.synchronize()
        flat = torch.as_tensor(_DevView(ptr.value, nbytes.value, self.dtype), device="cuda")
        return torch.view_as_complex(flat.view(-1, 2)).clone()

    def close(self) -> None:
        if getattr(self, "_h", None):
            check(lib.fmmfft_destroy(self._h))
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass
