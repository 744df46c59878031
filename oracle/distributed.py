"""Block-distributed ("virtual-G") CPU oracle of the FMM-FFT — TEST INFRASTRUCTURE ONLY.

Same rules as fmmfft_oracle.py: only tests/, __graft_entry__.smoke() and bench.py's CPU legs
import it; it shares nothing with the CUDA path (it has its own exchange schedule).

Rank g of G holds the contiguous input block x[g N/G, (g+1) N/G), i.e. the leaf boxes
[g 2^L/G, (g+1) 2^L/G) with all p, and ends with the output block
y[g N/G, (g+1) N/G). Communication follows Algorithm 1 and §5.2:

  line 2   S halo: one leaf box from each cyclic neighbour
  line 7   M^l halo: two boxes from each neighbour, levels l > l_g
  line 9   all-gather of the multipoles at level l_g = max(B, log2 G + 1)   (R16)
  line 16  the one all-to-all transpose of the 2D FFT

Reading R16: the paper all-gathers M^B; when 2^l / G < 2 at some level l > B a
rank no longer owns the two boxes per side its neighbours need, so this oracle (and the CUDA
path) gathers level l_g instead and computes the few levels l_g..B on the gathered data
redundantly on every rank. Results equal the global oracle up to rounding (pinned in tests).
"""
from __future__ import annotations

import math
import threading

import numpy as np

from . import fmmfft_oracle as O


class ThreadGroup:
    """In-process exchange for G ranks running in G Python threads (lockstep collectives)."""

    def __init__(self, G: int):
        self.G = G
        self._bar = threading.Barrier(G)
        self._slots = [None] * G

    def _exchange(self, rank, item):
        self._slots[rank] = item
        self._bar.wait()
        got = list(self._slots)
        self._bar.wait()
        return got

    def allgather(self, rank, arr):
        return self._exchange(rank, arr)

    def alltoall(self, rank, chunks):
        got = self._exchange(rank, chunks)
        return [got[s][rank] for s in range(self.G)]

    def ring(self, rank, to_left, to_right):
        """Send to_left to rank-1 and to_right to rank+1 (cyclic); return (from_left, from_right)."""
        got = self._exchange(rank, (to_left, to_right))
        G = self.G
        return got[(rank - 1) % G][1], got[(rank + 1) % G][0]


def top_level(L: int, B: int, G: int) -> int:
    """l_g: the finest level handled by the all-gather (reading R16)."""
    lg = max(B, int(round(math.log2(G))) + 1)
    return min(lg, L)


def fmmfft_rank(x_local: np.ndarray, N: int, P: int, B: int, Q: int, M_L: int,
                rank: int, G: int, comm) -> np.ndarray:
    """One rank's part of the distributed FMM-FFT (Algorithm 1 + the distributed 2D FFT).
    Returns this rank's output block y[rank N/G, (rank+1) N/G)."""
    M = N // P
    L = O.tree_levels(N, P, M_L)
    lg = top_level(L, B, G)
    nb = 2 ** L // G
    assert nb * G == 2 ** L and nb >= 1
    S = np.asarray(x_local, dtype=np.complex128).reshape(nb, M_L, P)
    S2M, M2M = O.op_S2M(Q, M_L), O.op_M2M(Q)
    L2L, L2T = M2M.T, S2M.T

    # line 1: S2M on own leaf boxes
    Mexp = {L: np.einsum("qm,bmp->bqp", S2M, S[:, :, 1:])}
    # line 2: S halo — box -1 from the left neighbour, box nb from the right neighbour
    halo_l, halo_r = comm.ring(rank, S[0], S[-1])
    # line 3: S2T over the window [box b-1, b, b+1]
    Sx = np.concatenate([halo_l[None], S, halo_r[None]], axis=0)     # boxes -1..nb
    A = O.op_S2T(N, P, M_L)
    j = np.arange(-M_L, 2 * M_L)
    Swin = np.concatenate([Sx[:-2], Sx[1:-1], Sx[2:]], axis=1)       # [b, j+M_L, p]
    T = np.empty(S.shape, dtype=np.complex128)
    for i in range(M_L):
        T[:, i, :] = np.einsum("pj,bjp->bp", A[:, j - i + 2 * M_L - 1], Swin)

    # lines 4-5: M2M on own boxes down to l_g (every rank owns >= 2 boxes there)
    for lev in range(L - 1, lg - 1, -1):
        nbl = 2 ** lev // G
        Mexp[lev] = np.einsum("qk,bkp->bqp", M2M, Mexp[lev + 1].reshape(nbl, 2 * Q, P - 1))

    # line 7: M^l halos, two boxes per side, for the distributed levels l > l_g
    Mhalo = {}
    for lev in range(L, lg, -1):
        hl, hr = comm.ring(rank, Mexp[lev][:2], Mexp[lev][-2:])
        Mhalo[lev] = np.concatenate([hl, Mexp[lev], hr], axis=0)       # boxes -2 .. nb_l+1
    # line 9: all-gather level l_g, then the replicated top of the tree (l_g .. B)
    Mfull = {lg: np.concatenate(comm.allgather(rank, Mexp[lg]), axis=0)}
    for lev in range(lg - 1, B - 1, -1):
        Mfull[lev] = np.einsum("qk,bkp->bqp", M2M, Mfull[lev + 1].reshape(2 ** lev, 2 * Q, P - 1))

    # lines 8, 10, 11 on the replicated levels: M2L for l in (B, l_g], M2L-B, REDUCE
    Lfull = {}
    for lev in range(lg, B, -1):
        nbf = 2 ** lev
        out = np.zeros((nbf, Q, P - 1), dtype=np.complex128)
        for parity in (0, 1):
            b = np.arange(parity, nbf, 2)
            for s in O.m2l_shifts(lev, B, parity):
                out[b] += np.einsum("pij,bjp->bip", O.op_M2L(N, P, Q, lev, s), Mfull[lev][(b + s) % nbf])
        Lfull[lev] = out
    nbB = 2 ** B
    b = np.arange(nbB)
    out = np.zeros((nbB, Q, P - 1), dtype=np.complex128)
    for s in O.m2l_shifts(B, B, 0):
        out += np.einsum("pij,bjp->bip", O.op_M2L(N, P, Q, B, s), Mfull[B][(b + s) % nbB])
    Lfull[B] = out
    r = Mfull[B].sum(axis=(0, 1))
    # line 13 on the replicated levels
    for lev in range(B, lg):
        Lfull[lev + 1] = Lfull[lev + 1] + np.einsum("qk,bkp->bqp", L2L, Lfull[lev]).reshape(
            2 ** (lev + 1), Q, P - 1)

    # line 8 (distributed levels) interleaved with line 13 going down from l_g to L
    Lloc = Lfull[lg][rank * (2 ** lg // G):(rank + 1) * (2 ** lg // G)]
    for lev in range(lg + 1, L + 1):
        nbl = 2 ** lev // G
        out = np.einsum("qk,bkp->bqp", L2L, Lloc).reshape(nbl, Q, P - 1)
        b0 = rank * nbl                                                # global index of box 0
        for parity in (0, 1):
            bl = np.arange(parity, nbl, 2)                              # b0 is even
            for s in O.m2l_shifts(lev, B, parity):
                out[bl] += np.einsum("pij,bjp->bip", O.op_M2L(N, P, Q, lev, s), Mhalo[lev][bl + s + 2])
        Lloc = out
        del b0

    # line 14 L2T, line 15 POST
    T[:, :, 1:] += np.einsum("mq,bqp->bmp", L2T, Lloc)
    T = O.post(T, r, N, P)

    # line 16: distributed 2D FFT. Local P-point FFTs for the M/G local m, then the all-to-all.
    Ml = M // G
    Tm = T.reshape(Ml, P)                                              # [m_local, p]
    W = O.fft_radix2(Tm, axis=1).T                                     # W[k2, m_local]
    Pl = P // G
    got = comm.alltoall(rank, [W[d * Pl:(d + 1) * Pl] for d in range(G)])
    Wl = np.concatenate(got, axis=1)                                   # [k2_local, m_global]
    Y = O.fft_radix2(Wl, axis=1)                                       # [k2_local, k1]
    return Y.reshape(Pl * M)


def _run_threads(G: int, fn):
    """fn(g, comm) on G threads sharing one ThreadGroup; returns the G results in rank order."""
    comm = ThreadGroup(G)
    outs = [None] * G
    errs = []

    def run(g):
        try:
            outs[g] = fn(g, comm)
        except BaseException as e:  # noqa: BLE001 - surface worker errors to the caller
            errs.append(e)
            comm._bar.abort()

    th = [threading.Thread(target=run, args=(g,)) for g in range(G)]
    for t in th:
        t.start()
    for t in th:
        t.join()
    if errs:
        raise errs[0]
    return outs


def fmmfft_virtual(x: np.ndarray, P: int, B: int, Q: int, M_L: int = 64, G: int = 2) -> np.ndarray:
    """Run G ranks in threads on the blocks of x; return the concatenated output blocks."""
    x = np.asarray(x, dtype=np.complex128)
    N = len(x)
    return np.concatenate(_run_threads(G, lambda g, comm: fmmfft_rank(x[g * N // G:(g + 1) * N // G], N, P, B, Q,
                                                                       M_L, g, G, comm)))


# --------------------------------------------------------------------------------------------
# Real input at G ranks (reading R18): N reals block-distributed, packed as
# z_j = x_{2j} + i x_{2j+1} (rank g's z block is its own reals), the distributed complex FMM-FFT
# of length H = N/2, then X_k = E_k + w_N^k O_k with E_k = (Z_k + conj Z_{H-k})/2,
# O_k = -i (Z_k - conj Z_{H-k})/2. Z_{H-k} for rank g's k lives on rank G-1-g (and one element,
# A[(G-g) H/G], on rank (G-g) mod G): the mirror exchange below. Output: rank g holds X_k for
# k in [g H/G, (g+1) H/G); the last rank also X_H.
# --------------------------------------------------------------------------------------------
def mirror_exchange(A_local: np.ndarray, extra_H, rank: int, G: int, comm, c2r: bool):
    """Rank g receives rank G-1-g's block and the element A[(G-g) H/G] (A[H] = Z[0] for the
    forward — rank 0's first element; = X_H for the inverse — rank G-1's extra value extra_H)."""
    nl = len(A_local)
    chunks = [np.zeros(nl + 2, dtype=np.complex128) for _ in range(G)]
    chunks[G - 1 - rank][:nl] = A_local
    if not c2r:
        chunks[(G - rank) % G][nl] = A_local[0]
    else:
        if rank > 0:
            chunks[G - rank][nl] = A_local[0]
        if rank == G - 1:
            chunks[0][nl + 1] = extra_H
    got = comm.alltoall(rank, chunks)
    mir = np.asarray(got[G - 1 - rank][:nl])
    if not c2r:
        xtra = got[(G - rank) % G][nl]
    else:
        xtra = got[G - 1][nl + 1] if rank == 0 else got[G - rank][nl]
    return mir, xtra


def rdft_rank(x_local: np.ndarray, N: int, P: int, B: int, Q: int, M_L: int, rank: int, G: int, comm) -> np.ndarray:
    """Rank g's X_k, k in its block (+ X_{N/2} on the last rank), of N block-distributed reals."""
    H = N // 2
    nl = H // G
    x_local = np.asarray(x_local, dtype=np.float64)
    z = x_local[0::2] + 1j * x_local[1::2]
    Z = fmmfft_rank(z, H, P, B, Q, M_L, rank, G, comm)
    mir, xtra = mirror_exchange(Z, None, rank, G, comm, c2r=False)
    j = np.arange(nl)
    zb = np.concatenate([[xtra], mir[nl - j[1:]]])                     # Z_{H-k}
    k = rank * nl + j
    E = (Z + np.conj(zb)) / 2
    Od = -1j * (Z - np.conj(zb)) / 2
    X = E + np.exp(-2j * np.pi * k / N) * Od
    if rank == G - 1:                                                  # X_H = E_0 - O_0 from Z_0
        X = np.concatenate([X, [mir[0].real - mir[0].imag]])
    return X


def irdft_rank(X_local: np.ndarray, N: int, P: int, B: int, Q: int, M_L: int, rank: int, G: int, comm) -> np.ndarray:
    """The inverse: rank g's N/G reals from its X block (the last rank's block ends with X_{N/2});
    the imaginary parts of X_0 and X_{N/2} are ignored (a real signal's are zero)."""
    H = N // 2
    nl = H // G
    X_local = np.asarray(X_local, dtype=np.complex128)
    a = X_local[:nl].copy()
    mir, xtra = mirror_exchange(a, X_local[nl] if rank == G - 1 else None, rank, G, comm, c2r=True)
    j = np.arange(nl)
    xb = np.concatenate([[xtra], mir[nl - j[1:]]])                     # X_{H-k}
    k = rank * nl + j
    if rank == 0:
        a[0], xb[0] = a[0].real, xb[0].real
    E = (a + np.conj(xb)) / 2
    Od = np.exp(2j * np.pi * k / N) * (a - np.conj(xb)) / 2
    Z = E + 1j * Od                                                    # DFT_H of z_j = x_{2j} + i x_{2j+1}
    z = np.conj(fmmfft_rank(np.conj(Z), H, P, B, Q, M_L, rank, G, comm)) / H
    x = np.empty(2 * nl)
    x[0::2], x[1::2] = z.real, z.imag
    return x


def rdft_virtual(x: np.ndarray, P: int, B: int, Q: int, M_L: int = 64, G: int = 2) -> np.ndarray:
    x = np.asarray(x, dtype=np.float64)
    N = len(x)
    return np.concatenate(_run_threads(G, lambda g, comm: rdft_rank(x[g * N // G:(g + 1) * N // G], N, P, B, Q, M_L,
                                                                    g, G, comm)))


def irdft_virtual(X: np.ndarray, P: int, B: int, Q: int, M_L: int = 64, G: int = 2) -> np.ndarray:
    X = np.asarray(X, dtype=np.complex128)
    N = 2 * (len(X) - 1)
    nl = N // 2 // G
    blk = lambda g: X[g * nl:(g + 1) * nl + (1 if g == G - 1 else 0)]   # noqa: E731
    return np.concatenate(_run_threads(G, lambda g, comm: irdft_rank(blk(g), N, P, B, Q, M_L, g, G, comm)))
