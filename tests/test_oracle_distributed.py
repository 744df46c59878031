"""Pins for the block-distributed oracle (oracle/distributed.py): G ranks with explicit S halos,
M^l halos, the level-l_g all-gather (reading R16) and the one all-to-all must reproduce the
global oracle to rounding and the DFT within the paper's bound — in threads (G = 1..8) and in
two real processes over torch.distributed gloo (world_size 2, 127.0.0.1)."""
import os
import socket

import numpy as np
import pytest

import synth_inputs as SI
from oracle import distributed as D
from oracle import fmmfft_oracle as O


@pytest.mark.parametrize("N,P,B,Q,M_L,G", [
    (1 << 12, 16, 2, 16, 16, 1),
    (1 << 12, 16, 2, 16, 16, 2),
    (1 << 14, 16, 2, 16, 16, 4),
    (1 << 14, 16, 2, 12, 16, 8),       # l_g = 4 > B = 2: replicated levels 2..4
    (1 << 15, 16, 4, 16, 16, 8),       # l_g = B = 4
    (1 << 16, 32, 3, 16, 32, 8),
    (1 << 14, 16, 2, 16, 64, 8),       # L = 4 = l_g: no distributed level at all
])
def test_virtual_ranks_match_global(N, P, B, Q, M_L, G):
    x = SI.complex_uniform(0, N)
    y = D.fmmfft_virtual(x, P, B, Q, M_L, G)
    assert O.rel_l2(y, O.fmmfft(x, P, B, Q, M_L)) < 1e-14
    assert O.rel_l2(y, np.fft.fft(x)) < (3e-14 if Q >= 16 else 1e-9)   # M_L = 16: see test_oracle_fmm


@pytest.mark.parametrize("N,P,B,Q,M_L,G", [
    (1 << 13, 16, 2, 16, 16, 1),
    (1 << 13, 16, 2, 16, 16, 2),
    (1 << 15, 16, 2, 16, 16, 4),
    (1 << 15, 16, 2, 12, 16, 8),
])
def test_real_input_virtual_ranks(N, P, B, Q, M_L, G):
    # reading R18 at G ranks: the mirror exchange + per-rank even/odd separation equals the
    # definition (eq. 1 for real x, first half: O.rdft, pinned to numpy.fft.rfft) and inverts
    x = SI.real_uniform(0, N)
    X = D.rdft_virtual(x, P, B, Q, M_L, G)
    assert X.shape == (N // 2 + 1,)
    ref = O.rdft(x)
    assert O.rel_l2(X, ref) < (3e-14 if Q >= 16 else 1e-9)
    assert abs(X[0].imag) < 1e-12 * abs(X[0]) + 1e-12 and abs(X[-1].imag) < 1e-12 * np.abs(X).max()
    Xb = ref.copy()
    Xb[0] += 0.7j                       # non-real DC / Nyquist parts are ignored by the inverse
    Xb[-1] += 0.3j
    xr = D.irdft_virtual(Xb, P, B, Q, M_L, G)
    assert np.linalg.norm(xr - x) / np.linalg.norm(x) < (3e-14 if Q >= 16 else 1e-9)


def test_mirror_exchange_pairs():
    # every rank receives rank G-1-g's block and A[(G-g) H/G] (R2C: A[H] = A[0]; C2R: A[H] = X_H)
    for G in (1, 2, 3, 4, 8):
        nl = 5
        A = np.arange(G * nl + 1) * (1 + 1j)                           # global A_0 .. A_H
        for c2r in (False, True):
            res = D._run_threads(G, lambda g, comm: D.mirror_exchange(A[g * nl:(g + 1) * nl], A[G * nl], g, G, comm, c2r))
            for g, (mir, xtra) in enumerate(res):
                assert np.array_equal(mir, A[(G - 1 - g) * nl:(G - g) * nl])
                want = A[(G - g) * nl] if (c2r or g > 0) else A[0]
                assert xtra == want, (G, c2r, g)


def test_shards_are_slices_of_the_global_vector():
    N, G = 1 << 12, 4
    full = SI.complex_uniform(0, N)
    for g in range(G):
        assert np.array_equal(SI.shard(N, G, g), full[g * N // G:(g + 1) * N // G])


class GlooGroup:
    """The oracle's exchange interface over torch.distributed (gloo) — test plumbing only."""

    def __init__(self, torch, dist):
        self.t, self.d = torch, dist
        self.G = dist.get_world_size()

    def _tens(self, a):
        return self.t.from_numpy(np.ascontiguousarray(a))

    def allgather(self, rank, arr):
        out = [self.t.empty_like(self._tens(arr)) for _ in range(self.G)]
        self.d.all_gather(out, self._tens(arr))
        return [o.numpy() for o in out]

    def alltoall(self, rank, chunks):
        got = []
        for s in range(self.G):                       # gather-based all-to-all (gloo lacks all_to_all)
            parts = [self.t.empty_like(self._tens(chunks[0])) for _ in range(self.G)]
            self.d.all_gather(parts, self._tens(chunks[s]))
            if s == rank:
                got = [p.numpy() for p in parts]
        return got

    def ring(self, rank, to_left, to_right):
        G = self.G
        left, right = (rank - 1) % G, (rank + 1) % G
        fl = self.t.empty_like(self._tens(to_right))
        fr = self.t.empty_like(self._tens(to_left))
        # tag 0 = travelling left, tag 1 = travelling right (G = 2: both neighbours are one rank)
        reqs = [self.d.isend(self._tens(to_left), left, tag=0), self.d.isend(self._tens(to_right), right, tag=1),
                self.d.irecv(fl, left, tag=1), self.d.irecv(fr, right, tag=0)]
        for r in reqs:
            r.wait()
        return fl.numpy(), fr.numpy()


def _gloo_worker(rank, world, port, q):
    import torch
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        N, P, B, Q, M_L = 1 << 14, 16, 3, 16, 16
        x = SI.shard(N, world, rank)
        comm = GlooGroup(torch, dist)
        y = D.fmmfft_rank(x, N, P, B, Q, M_L, rank, world, comm)
        xr = SI.real_uniform(0, 2 * N)[rank * N:(rank + 1) * N]       # 2N reals: H = N
        X = D.rdft_rank(xr, 2 * N, P, B, Q, M_L, rank, world, comm)
        q.put((rank, (y, X)))
    finally:
        dist.destroy_process_group()


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def test_gloo_two_processes():
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_gloo_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    got = dict(q.get(timeout=300) for _ in procs)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    N = 1 << 14
    y = np.concatenate([got[0][0], got[1][0]])
    x = SI.complex_uniform(0, N)
    assert O.rel_l2(y, O.fmmfft(x, 16, 3, 16, 16)) < 1e-14
    assert O.rel_l2(y, O.fft_radix2(x)) < 3e-14
    # real input over the two processes: the mirror exchange through gloo (R18)
    X = np.concatenate([got[0][1], got[1][1]])
    assert O.rel_l2(X, O.rdft(SI.real_uniform(0, 2 * N))) < 3e-14
