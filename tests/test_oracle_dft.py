"""Pins for oracle O1 (the DFT, eq. 1) and O2 (eq. 2 with dense C_p).

Every check compares the oracle with something other than itself: closed forms of the DFT,
Parseval, linearity, a brute-force sum, an independent library FFT (numpy.fft), and the
independent derivation C_p = F_M^{-1} diag(w_N^{pk}) F_M.
"""
import numpy as np
import pytest

import synth_inputs as SI
from oracle import fmmfft_oracle as O


@pytest.mark.parametrize("N", [1, 2, 8, 64, 1024])
def test_delta_gives_ones(N):
    # x = e_0  ->  y_k = 1 for all k (eq. 1)
    y = O.fft_radix2(SI.delta(N))
    assert np.max(np.abs(y - 1.0)) < 1e-15
    assert np.max(np.abs(O.dft_direct(SI.delta(N)) - 1.0)) < 1e-15


@pytest.mark.parametrize("N,j0", [(16, 3), (256, 17), (1024, 1000)])
def test_shifted_delta(N, j0):
    # x = e_{j0} -> y_k = w_N^{j0 k}, angle reduced exactly
    k = np.arange(N)
    expect = np.exp(-2j * np.pi * ((j0 * k) % N) / N)
    for f in (O.fft_radix2, O.dft_direct):
        assert np.max(np.abs(f(SI.delta(N, j0)) - expect)) < 1e-13


@pytest.mark.parametrize("N", [8, 512])
def test_constant_gives_scaled_delta(N):
    y = O.fft_radix2(np.ones(N, dtype=complex))
    expect = np.zeros(N, dtype=complex)
    expect[0] = N
    assert np.max(np.abs(y - expect)) < 1e-12 * N


@pytest.mark.parametrize("N,k0", [(64, 5), (4096, 1234), (4096, 4095)])
def test_tone_gives_delta(N, k0):
    # x_j = exp(+2 pi i k0 j / N) -> y = N e_{k0}
    y = O.fft_radix2(SI.tone(N, k0))
    expect = np.zeros(N, dtype=complex)
    expect[k0] = N
    assert np.max(np.abs(y - expect)) < 1e-10


def test_parseval_and_linearity():
    N = 2048
    x = SI.complex_uniform(0, N, seed=1)
    z = SI.complex_uniform(0, N, seed=2)
    y = O.fft_radix2(x)
    assert abs(np.sum(np.abs(y) ** 2) - N * np.sum(np.abs(x) ** 2)) < 1e-10 * N * np.sum(np.abs(x) ** 2)
    a, b = 0.3 - 1.1j, 2.0 + 0.5j
    lhs = O.fft_radix2(a * x + b * z)
    rhs = a * y + b * O.fft_radix2(z)
    assert O.rel_l2(lhs, rhs) < 1e-14


def test_real_input_conjugate_symmetry():
    N = 1024
    x = SI.complex_uniform(0, N, seed=3).real.astype(complex)
    y = O.fft_radix2(x)
    k = np.arange(N)
    assert np.max(np.abs(y[(-k) % N] - np.conj(y))) < 1e-11


@pytest.mark.parametrize("N", [2, 16, 256, 4096])
def test_radix2_matches_direct_bruteforce(N):
    x = SI.complex_uniform(0, N)
    assert O.rel_l2(O.fft_radix2(x), O.dft_direct(x)) < 1e-14


@pytest.mark.parametrize("N", [4096, 1 << 16])
def test_radix2_matches_numpy_fft(N):
    x = SI.complex_uniform(0, N)
    assert O.rel_l2(O.fft_radix2(x), np.fft.fft(x)) < 1e-14


def test_radix2_batched_axis():
    X = SI.complex_uniform(0, 64 * 32).reshape(64, 32)
    assert O.rel_l2(O.fft_radix2(X, axis=0), np.fft.fft(X, axis=0)) < 1e-14
    assert O.rel_l2(O.fft_radix2(X, axis=1), np.fft.fft(X, axis=1)) < 1e-14


@pytest.mark.parametrize("M,P", [(64, 8), (16, 4), (32, 2)])
def test_kernel_matrix_closed_form(M, P):
    """[C_p]_{mn} = rho_p[cot(pi(n-m)/M + pi p/N) + i] must equal
    F_M^{-1} diag(w_N^{pk}) F_M, the twiddle step of Cooley-Tukey moved into the p-th block
    (SURVEY.md §8(c) derivation). Dense DFT matrices from exact integer angles."""
    N = M * P
    k = np.arange(M)
    F = np.exp(-2j * np.pi * (np.outer(k, k) % M) / M)
    Finv = np.conj(F) / M
    for p in range(P):
        D = np.diag(np.exp(-2j * np.pi * ((p * k) % N) / N))
        ref = Finv @ D @ F
        assert np.max(np.abs(O.kernel_matrix(M, P, p) - ref)) < 1e-13


@pytest.mark.parametrize("M,P", [(64, 8), (128, 4)])
def test_kernel_matrix_unitary(M, P):
    for p in range(P):
        C = O.kernel_matrix(M, P, p)
        assert np.max(np.abs(C.conj().T @ C - np.eye(M))) < 1e-12


@pytest.mark.parametrize("M,P", [(8, 4), (16, 2), (32, 8), (64, 16)])
def test_dense_factorisation_equals_dft(M, P):
    """eq. (2): F_N = F_{M,P} H^_{M,P} exactly."""
    x = SI.complex_uniform(0, M * P)
    assert O.rel_l2(O.fmmfft_dense(x, P), O.dft_direct(x)) < 5e-15


def test_fft2d_layout_against_library():
    """F_{M,P} of steps (2)-(4): y[k1 + M k2] = sum_m w_M^{m k1} sum_p w_P^{p k2} T[p + P m]
    is a 2D DFT of T viewed as [m, p]; compare with numpy.fft.fft2 (independent library)."""
    M, P = 32, 8
    T = SI.complex_uniform(0, M * P)
    Y = np.fft.fft2(T.reshape(M, P))            # Y[k1, k2]
    expect = Y.T.reshape(M * P)                 # index k1 + M k2
    assert O.rel_l2(O.fft2d_MP(T, M, P), expect) < 1e-14


# ------------------------------------------------------------------ the inverse transform (§8(f) NEXT-1)
def test_inverse_closed_forms():
    N = 64
    # F^{-1} delta_0 = 1/N (constant); F^{-1} delta_k0 = tone w_N^{-j k0} / N
    d = np.zeros(N, complex)
    d[0] = 1
    assert np.allclose(O.dft_direct(d, inverse=True), np.full(N, 1 / N), atol=1e-16)
    d[:] = 0
    d[5] = 1
    j = np.arange(N)
    assert np.allclose(O.dft_direct(d, inverse=True), np.exp(2j * np.pi * 5 * j / N) / N, atol=1e-16)


@pytest.mark.parametrize("N", [2, 16, 256, 4096])
def test_inverse_roundtrip_and_radix2(N):
    x = SI.complex_uniform(0, N)
    y = O.dft_direct(x)
    assert O.rel_l2(O.dft_direct(y, inverse=True), x) < 1e-13
    assert O.rel_l2(O.fft_radix2(y, inverse=True), x) < 1e-13
    assert O.rel_l2(O.fft_radix2(x, inverse=True), O.dft_direct(x, inverse=True)) < 1e-13
    assert O.rel_l2(O.fft_radix2(x, inverse=True), np.fft.ifft(x)) < 1e-13


# ---- real-input transform (SURVEY §8(f) NEXT-1, C = 1)

@pytest.mark.parametrize("N", [2, 16, 1024, 24])
def test_rdft_vs_numpy_and_hermitian(N):
    rng = np.random.default_rng(N)
    x = rng.standard_normal(N)
    y = O.rdft(x)
    assert y.shape == (N // 2 + 1,)
    # independent library routine
    assert np.max(np.abs(y - np.fft.rfft(x))) < 1e-12 * max(1, np.sqrt(N))
    # the full DFT of a real vector is Hermitian: y_{N-k} = conj(y_k); y_0, y_{N/2} real
    full = O.dft_direct(x.astype(complex))
    assert np.max(np.abs(full[1:][::-1] - np.conj(full[1:]))) < 1e-10
    assert abs(y[0].imag) < 1e-12 and abs(y[-1].imag) < 1e-10
    assert abs(y[0] - x.sum()) < 1e-10
    assert abs(y[-1] - (x[0::2].sum() - x[1::2].sum())) < 1e-10


@pytest.mark.parametrize("N,k0", [(64, 5), (4096, 1000)])
def test_rdft_cosine(N, k0):
    # x_j = cos(2 pi k0 j / N) -> y_k0 = N/2, every other k in 0..N/2 zero
    j = np.arange(N)
    y = O.rdft(np.cos(2 * np.pi * ((k0 * j) % N) / N))
    expect = np.zeros(N // 2 + 1, dtype=complex)
    expect[k0] = N / 2
    assert np.max(np.abs(y - expect)) < 1e-10 * N


@pytest.mark.parametrize("N,J", [(1024, 32), (4096, 64), (4096, 4096), (2048, 1)])
def test_dft_at_matches_direct_and_radix2(N, J):
    # dft_at is eq. (1) evaluated at selected k with the exponent split j = j1 + J j2: it must
    # reproduce the brute-force sum and the radix-2 FFT at every k
    x = SI.complex_uniform(0, N, seed=7)
    ks = np.arange(N)
    y = O.dft_at(x, ks, J=J)
    scale = np.sqrt(N)
    assert np.max(np.abs(y - O.dft_direct(x))) < 1e-13 * scale * 10
    assert np.max(np.abs(y - O.fft_radix2(x))) < 1e-13 * scale * 10


def test_dft_at_closed_forms():
    N = 1 << 16
    k = np.array([0, 1, 4321, N - 1])
    assert np.max(np.abs(O.dft_at(SI.delta(N, 777), k) - np.exp(-2j * np.pi * ((777 * k) % N) / N))) < 1e-12
    y = O.dft_at(SI.tone(N, 4321), k)
    assert abs(y[2] - N) < 1e-8 * N and np.max(np.abs(y[[0, 1, 3]])) < 1e-8 * N
