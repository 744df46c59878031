"""Worker of tests/test_gpu_parity.py::test_two_rank_nccl (launched by torch.distributed.run):
each rank runs the G = 2 FMM-FFT over NCCL on its own GPU and checks its output block against
the CPU float64 DFT of the whole seeded input."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402
import torch.distributed as dist  # noqa: E402

import synth_inputs as SI  # noqa: E402
from oracle import fmmfft_oracle as O  # noqa: E402


def main():
    rank, world = int(os.environ["RANK"]), int(os.environ["WORLD_SIZE"])
    torch.cuda.set_device(int(os.environ["LOCAL_RANK"]))
    dist.init_process_group("nccl", device_id=torch.device("cuda", int(os.environ["LOCAL_RANK"])))
    from paper_conf_sc_cecka17_b200 import FmmFFT, destroy_comm, init_comm
    init_comm()
    for N, P, B, Q, prec, M_L in [(1 << 18, 32, 2, 16, "c64", 64), (1 << 16, 16, 3, 16, "c128", 16)]:
        npdt = np.complex64 if prec == "c64" else np.complex128
        x = SI.complex_uniform(0, N, dtype=npdt)
        n = N // world
        plan = FmmFFT(N=N, P=P, G=world, B=B, Q=Q, precision=prec, M_L=M_L)
        y = plan(torch.from_numpy(x[rank * n:(rank + 1) * n]).cuda()).cpu().numpy()
        y2 = plan(torch.from_numpy(x[rank * n:(rank + 1) * n]).cuda()).cpu().numpy()
        plan.close()
        ref = O.fft_radix2(x)[rank * n:(rank + 1) * n]
        err = O.rel_l2(y, ref)
        tol = 1e-5 if prec == "c64" else 1e-11
        assert err < tol and np.array_equal(y, y2), (rank, prec, err)
    dist.barrier()
    destroy_comm()
    print("NCCL_WORKER_OK", rank, flush=True)
    dist.destroy_process_group()


if __name__ == "__main__":
    main()
