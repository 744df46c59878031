"""GPU parity: the CUDA path (through the C ABI) against the CPU float64 oracle on the same seeded
inputs — stage by stage (T_near, M^l, L^l, r, W) and end to end — plus edge cases.

Tolerances: the north star's relative l2 bounds against the float64
DFT of the same (rounded) input, 1e-5 for complex64 and 1e-11 for complex128; stage buffers
against the oracle's same stage at 1e-5 (fp32 arithmetic over <= 3 M_L-term sums of
cotangents) and 1e-12 (fp64).
"""
import numpy as np
import pytest

import synth_inputs as SI
from oracle import distributed as D
from oracle import fmmfft_oracle as O

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

TOL_E2E = {"c64": 1e-5, "c128": 1e-11}
TOL_STAGE = {"c64": 1e-5, "c128": 1e-12}
NPDT = {"c64": np.complex64, "c128": np.complex128}


@pytest.fixture(scope="module")
def F():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_sc_cecka17_b200 import build
    build.build()
    from paper_conf_sc_cecka17_b200 import FmmFFT
    return FmmFFT


def run(F, N, P, B, Q, prec, M_L=64, G=1, virtual=False, seed=SI.DEFAULT_SEED, debug=False):
    x = SI.complex_uniform(0, N, seed=seed, dtype=NPDT[prec])
    plan = F(N=N, P=P, G=G, B=B, Q=Q, precision=prec, M_L=M_L, virtual=virtual, debug=debug)
    xd = torch.from_numpy(x).cuda()
    y = plan(xd)
    torch.cuda.synchronize()
    return plan, x, y.cpu().numpy()


def t_near(plan, P, L, M_L):
    """T_near debug buffer ([p][b][re/im][m] reals) as complex [b][m][p]."""
    t = plan.debug_buffer("T_near").cpu().numpy()
    f = t.view(np.float32 if t.dtype == np.complex64 else np.float64).reshape(P, 2 ** L, 2, M_L)
    return (f[:, :, 0, :] + 1j * f[:, :, 1, :]).astype(t.dtype).transpose(1, 2, 0)


def rel(a, b):
    return O.rel_l2(np.asarray(a, dtype=np.complex128), b)


# ------------------------------------------------------------------ end to end
@pytest.mark.parametrize("N,P,B,Q,prec,M_L", [
    (1 << 12, 16, 2, 16, "c128", 64),      # cfg1 (L = B = 2)
    (1 << 12, 16, 2, 16, "c64", 64),
    (1 << 12, 16, 2, 16, "c128", 16),      # cfg1 with L = 4
    (1 << 20, 64, 2, 16, "c64", 64),       # cfg2 (the bench workload at N = 1)
    (1 << 20, 64, 2, 16, "c128", 64),
    (1 << 16, 32, 3, 16, "c64", 32),
    (1 << 16, 8, 4, 16, "c128", 16),
    (1 << 18, 128, 2, 24, "c128", 64),     # Q = 24 (cfg4's order)
    (1 << 18, 256, 2, 8, "c64", 16),       # Q = 8 (the paper's single-precision order)
    (1 << 17, 2, 3, 16, "c64", 128),       # P = 2, M_L = 128
    (1 << 19, 512, 2, 16, "c64", 16),      # P = 512 (cfg4's P/G shape)
    (1 << 16, 4, 5, 16, "c64", 32),
    (1 << 20, 16, 4, 16, "c64", 64),       # wide tree (L = 10): per-level k_m2l_lvl for l >= 6
    (1 << 20, 16, 4, 24, "c128", 16),      # L = 12, Q = 24, fp64 k_m2l_lvl
    (1 << 20, 32, 3, 8, "c64", 32),        # L = 10, Q = 8
    (1 << 22, 16, 4, 24, "c64", 64),       # k_s2m_w at Q = 24: 3 symmetric q quads, fused M2M, cluster top
    (1 << 22, 32, 3, 8, "c64", 64),        # k_s2m_w at Q = 8 (one symmetric quad)
])
def test_end_to_end_vs_dft(F, N, P, B, Q, prec, M_L):
    plan, x, y = run(F, N, P, B, Q, prec, M_L)
    ref = O.dft_direct(x) if N <= 1 << 12 else O.fft_radix2(x)
    err = rel(y, ref)
    assert err < TOL_E2E[prec], err          # the north star's bound at every Q (incl. Q = 8)
    if prec == "c128" and Q >= 16:
        # the FMM itself reaches the paper's double-precision accuracy
        assert err < (2e-14 if M_L >= 32 else 3e-14) * 4


def test_cfg1_c128_matches_oracle_and_direct_dft(F):
    plan, x, y = run(F, 1 << 12, 16, 2, 16, "c128")
    assert rel(y, O.fmmfft(x, 16, 2, 16)) < 1e-13
    assert rel(y, O.dft_direct(x)) < 1e-11


# ------------------------------------------------------------------ stage by stage
@pytest.mark.parametrize("prec", ["c64", "c128"])
@pytest.mark.parametrize("N,P,B,Q,M_L", [(1 << 16, 16, 2, 16, 32), (1 << 18, 64, 3, 16, 64),
                                         (1 << 20, 16, 4, 16, 16)])   # L = 12: per-level 12, cluster top 4..11 (c64)
def test_stages_match_oracle(F, prec, N, P, B, Q, M_L):
    plan, x, y = run(F, N, P, B, Q, prec, M_L, debug=True)
    L = O.tree_levels(N, P, M_L)
    S = x.astype(np.complex128).reshape(2 ** L, M_L, P)
    st = O.fmm_stages(S, N, P, B, Q)
    tol = TOL_STAGE[prec]
    Tn = t_near(plan, P, L, M_L)
    assert rel(Tn, st["T_near"]) < tol
    assert np.array_equal(Tn[:, :, 0], S[:, :, 0].astype(Tn.dtype))        # p = 0 copies exactly
    for lev in range(B, L + 1):
        Mg = plan.debug_buffer("M", lev).cpu().numpy().reshape(2 ** lev, Q, P)
        assert rel(Mg[:, :, 1:], st["M"][lev]) < tol, ("M", lev)
        Lg = plan.debug_buffer("L", lev).cpu().numpy().reshape(2 ** lev, Q, P)
        assert rel(Lg[:, :, 1:], st["L"][lev]) < tol, ("L", lev)
    r = plan.debug_buffer("r").cpu().numpy()
    assert rel(r[1:], st["r"]) < tol
    # W = P-point FFTs of POST(T) (before the transpose), stored [k2][m]
    T = O.post(st["T"], st["r"], N, P).reshape(N // P, P)
    W = O.fft_radix2(T, axis=1).T
    Wg = plan.debug_buffer("W").cpu().numpy().reshape(P, N // P)
    assert rel(Wg, W) < tol
    assert rel(y, O.fft2d_MP(O.post(st["T"], st["r"], N, P).reshape(N), N // P, P)) < tol


# ------------------------------------------------------------------ distributed data flow (virtual ranks)
@pytest.mark.parametrize("N,P,B,Q,prec,M_L,G", [
    (1 << 14, 16, 2, 16, "c64", 16, 2),
    (1 << 16, 32, 2, 16, "c128", 16, 4),
    (1 << 16, 32, 2, 16, "c64", 16, 8),      # l_g = 4 > B: replicated top levels
    (1 << 18, 64, 4, 16, "c64", 32, 8),      # l_g = B = 4
    (1 << 16, 16, 2, 16, "c128", 64, 8),     # L = 6, l_g = 4
    (1 << 15, 16, 2, 16, "c64", 64, 8),      # L = 5: one box per rank at level 3
    (1 << 20, 128, 2, 24, "c128", 64, 8),    # cfg4 shape, reduced N
    (1 << 20, 32, 2, 16, "c64", 32, 4),      # 256 leaves per rank: k_m2l_lvl on halo'd levels 8..10
    (1 << 20, 16, 3, 16, "c128", 16, 2),     # fp64 k_m2l_lvl, 2048 leaves per rank
])
def test_virtual_ranks_vs_oracle(F, N, P, B, Q, prec, M_L, G):
    plan, x, y = run(F, N, P, B, Q, prec, M_L, G=G, virtual=True)
    ref = O.fft_radix2(x)
    assert rel(y, ref) < TOL_E2E[prec]
    assert rel(y, D.fmmfft_virtual(x.astype(np.complex128), P, B, Q, M_L, G)) < (TOL_E2E[prec] if prec == "c64" else 1e-12)


def test_virtual_matches_single_rank(F):
    N, P, B, Q, M_L = 1 << 18, 64, 2, 16, 32
    _, x, y1 = run(F, N, P, B, Q, "c128", M_L, G=1)
    _, _, y8 = run(F, N, P, B, Q, "c128", M_L, G=8, virtual=True)
    assert rel(y8, y1) < 1e-13


# ------------------------------------------------------------------ structured inputs, edge cases
def test_delta_and_tone(F):
    N, P = 1 << 16, 32
    plan = F(N=N, P=P, B=2, Q=16, precision="c128")
    k = np.arange(N)
    y = plan(torch.from_numpy(SI.delta(N, 12345)).cuda()).cpu().numpy()
    assert np.max(np.abs(y - np.exp(-2j * np.pi * ((12345 * k) % N) / N))) < 1e-12
    y = plan(torch.from_numpy(SI.tone(N, 999)).cuda()).cpu().numpy()
    e = np.zeros(N, complex)
    e[999] = N
    assert np.max(np.abs(y - e)) < 1e-9 * N
    y = plan(torch.zeros(N, dtype=torch.complex128, device="cuda")).cpu().numpy()
    assert np.all(y == 0)


def test_input_not_modified_and_repeatable(F):
    N, P = 1 << 16, 16
    plan = F(N=N, P=P, B=2, Q=16, precision="c64")
    x = torch.from_numpy(SI.complex_uniform(0, N, dtype=np.complex64)).cuda()
    x0 = x.clone()
    y1 = plan(x)
    y2 = plan(x)
    torch.cuda.synchronize()
    assert torch.equal(x, x0)
    assert torch.equal(y1, y2)                 # deterministic: no atomics on the path


def test_execute_rejects_bad_buffers(F):
    from paper_conf_sc_cecka17_b200._lib import FmmfftError
    N = 1 << 16
    plan = F(N=N, P=16, B=2, Q=16, precision="c64")
    x = torch.zeros(N, dtype=torch.complex64, device="cuda")
    with pytest.raises(FmmfftError):
        plan(x, out=x)                           # in == out overlap
    with pytest.raises(ValueError):
        plan(torch.zeros(N, dtype=torch.complex128, device="cuda"))


def test_execute_host_path(F):
    N, P = 1 << 18, 64
    plan = F(N=N, P=P, B=2, Q=16, precision="c64")
    x = SI.complex_uniform(0, N, dtype=np.complex64)
    xh = torch.from_numpy(x).pin_memory()
    yh = torch.empty_like(xh).pin_memory()
    s = torch.cuda.current_stream()
    plan.execute_host(xh, yh, s)
    s.synchronize()
    assert rel(yh.numpy(), O.fft_radix2(x)) < 1e-5


def test_profile_stage_times(F):
    plan = F(N=1 << 20, P=64, B=2, Q=16, precision="c64", profile=True)
    x = torch.from_numpy(SI.complex_uniform(0, 1 << 20, dtype=np.complex64)).cuda()
    plan(x)
    t = plan.stage_times()
    assert list(t) == ["comm_S", "s2m", "m2m", "comm_M", "top", "down", "post_pfft", "a2a", "mfft", "s2t"]
    assert all(v >= 0 for v in t.values()) and t["s2t"] > 0
    assert plan.info["kernels_per_execute"] >= 4


# ------------------------------------------------------------------ full-size configs, full vector
def blockwise_rel(y, ref, nblk=256):
    """Largest relative l2 error over nblk equal output blocks: an error confined to one rank's
    block, one halo tile or one M-FFT column block cannot hide in the global norm."""
    yb = np.asarray(y, dtype=np.complex128).reshape(nblk, -1)
    rb = np.asarray(ref, dtype=np.complex128).reshape(nblk, -1)
    return float(np.max(np.linalg.norm(yb - rb, axis=1) / np.linalg.norm(rb, axis=1)))


@pytest.fixture(scope="module")
def cfg3_ref():
    """cfg3's input (N = 2^26, complex64 values) and its float64 radix-2 DFT (oracle O1)."""
    x = SI.complex_uniform(0, 1 << 26, dtype=np.complex64)
    return x, O.fft_radix2(x)


@pytest.mark.parametrize("P,G", [(16, 1), (32, 2), (64, 4), (128, 8)])
def test_cfg3_full_vector(F, cfg3_ref, P, G):
    # configs[2]: N = 2^26 complex64, P = 16 G, B = 4, Q = 16 — every output element vs the DFT
    # (G > 1 as G virtual ranks: the per-rank trees with halos, the gathered top, the all-to-all)
    x, ref = cfg3_ref
    plan = F(N=1 << 26, P=P, G=G, B=4, Q=16, precision="c64", M_L=64, virtual=G > 1)
    y = plan(torch.from_numpy(x).cuda()).cpu().numpy()
    plan.close()
    assert rel(y, ref) < 1e-5
    assert blockwise_rel(y, ref) < 2e-5
    # the k1 = 0 bin of every M-point row (y[M k2], reading R19) meets the bound on its own
    ks = np.arange(P) * ((1 << 26) // P)
    assert rel(y[ks], ref[ks]) < 1e-5


def test_cfg4_shape_full_vector(F):
    # configs[3]'s G = 8 shape (P = 512, B = 2, Q = 24, complex128) at N = 2^26 (8 virtual ranks,
    # L = 11: 256 leaves per rank), every element vs the float64 DFT at 1e-11
    N = 1 << 26
    x = SI.complex_uniform(0, N, dtype=np.complex128)
    plan = F(N=N, P=512, G=8, B=2, Q=24, precision="c128", M_L=64, virtual=True)
    y = plan(torch.from_numpy(x).cuda()).cpu().numpy()
    plan.close()
    ref = O.fft_radix2(x)
    assert rel(y, ref) < 1e-11
    assert blockwise_rel(y, ref) < 2e-11


@pytest.mark.parametrize("N,P,prec,M_L", [(1 << 18, 2, "c64", 64), (1 << 18, 4, "c128", 32), (1 << 20, 8, "c64", 64)])
def test_p_equals_g(F, N, P, prec, M_L):
    # P = G: one k2 row per rank after the all-to-all
    plan, x, y = run(F, N, P, 2, 16, prec, M_L, G=P, virtual=True)
    assert rel(y, O.fft_radix2(x)) < TOL_E2E[prec]


def test_cfg5_point_virtual_g8(F):
    # configs[4] sweep point N = 2^30 complex64, P = 64, B = 4, Q = 16 at G = 8 (virtual ranks on
    # one GPU): 16 outputs against eq. (1) evaluated directly, plus Parseval over the whole vector
    N = 1 << 30
    x = SI.complex_uniform(0, N, dtype=np.complex64)
    plan = F(N=N, P=64, G=8, B=4, Q=16, precision="c64", M_L=64, virtual=True)
    xd = torch.from_numpy(x).cuda()
    yd = plan(xd)
    torch.cuda.synchronize()
    plan.close()
    ny = float(torch.sum(torch.abs(yd.to(torch.complex128)) ** 2))
    nx = float(np.sum(np.abs(x.astype(np.complex128)) ** 2))
    assert abs(ny / (N * nx) - 1) < 1e-5
    rng = np.random.default_rng(5)
    ks = np.concatenate([[0, 1, N // 8, N // 2, N - 1], rng.integers(0, N, 11)])
    ys = yd[torch.from_numpy(ks).cuda()].cpu().numpy()
    del xd, yd
    ref = O.dft_at(x, ks)
    assert np.linalg.norm(ys - ref) / np.linalg.norm(ref) < 1e-5


@pytest.mark.parametrize("N,P,B,Q,prec", [
    (1 << 20, 64, 2, 16, "c64"),       # cfg2 — exactly the bench.py N = 1 launch configuration
    (1 << 28, 64, 2, 24, "c128"),      # cfg4 (N = 2^28 complex128, Q = 24) on one GPU
])
def test_full_size_sampled(F, N, P, B, Q, prec):
    plan, x, y = run(F, N, P, B, Q, prec, 64)
    plan.close()
    rng = np.random.default_rng(0)
    ks = np.concatenate([[0, 1, N // 2, N - 1], rng.integers(0, N, 12)])
    ref = O.dft_at(x, ks)
    assert np.linalg.norm(y[ks] - ref) / np.linalg.norm(ref) < TOL_E2E[prec]
    # Parseval holds at any size: ||y||^2 = N ||x||^2
    ny = np.sum(np.abs(y.astype(np.complex128)) ** 2)
    nx = np.sum(np.abs(x.astype(np.complex128)) ** 2)
    assert abs(ny / (N * nx) - 1) < TOL_E2E[prec]


def test_real_full_size_sampled(F):
    # 2^27 reals: the complex plan is cfg3's shape at G = 1 (N/2 = 2^26, P = 16, B = 4, Q = 16)
    N = 1 << 27
    x = SI.real_uniform(0, N, dtype=np.float32)
    plan = F(N=N, P=16, B=4, Q=16, precision="c64", real=True)
    y = plan(torch.from_numpy(x).cuda()).cpu().numpy()
    plan.close()
    rng = np.random.default_rng(1)
    ks = np.concatenate([[0, 1, N // 4, N // 2 - 1, N // 2], rng.integers(0, N // 2 + 1, 7)])
    ref = O.dft_at(x, ks)
    assert np.linalg.norm(y[ks] - ref) / np.linalg.norm(ref) < 1e-5
    # Parseval for a real signal: |X_0|^2 + |X_{N/2}|^2 + 2 sum_{0<k<N/2} |X_k|^2 = N ||x||^2
    a = np.abs(y.astype(np.complex128)) ** 2
    ny = a[0] + a[-1] + 2 * np.sum(a[1:-1])
    assert abs(ny / (N * np.sum(x.astype(np.float64) ** 2)) - 1) < 1e-5


# ------------------------------------------------------------------ alternative kernel paths
@pytest.mark.parametrize("env", [
    {"FMMFFT_S2T": "simt"},      # S2T on the FFMA2 SIMT kernel (k_near_up) instead of tcgen05
    {"FMMFFT_TREE": "w", "FMMFFT_TOP": "w"},   # far field as wide per-level kernels (k_up, k_base, k_tree_down + k_m2l_lvl)
    {"FMMFFT_TREE": "w"},        # per-level kernels below, the top subtree of each FMM on a k_tree_pc cluster
    {"FMMFFT_NO_GRAPH": "1"},    # eager launches instead of a CUDA graph
    {"FMMFFT_MFFT": "pass"},     # multi-pass M-point FFT (k_fft_pass) instead of k_fft_row
    {"FMMFFT_MFFT": "fs"},       # four-step M-point FFT (k_fft_col + k_fft_rowt) instead of k_fft_row
])
@pytest.mark.parametrize("N,P,B,Q,G", [(1 << 20, 64, 2, 16, 1), (1 << 20, 64, 3, 16, 4)])
def test_alternative_paths(F, monkeypatch, env, N, P, B, Q, G):
    for k, v in env.items():
        monkeypatch.setenv(k, v)                   # read at plan creation
    prec = "c64"
    plan, x, y = run(F, N, P, B, Q, prec, 64, G=G, virtual=G > 1)
    assert rel(y, O.fft_radix2(x)) < TOL_E2E[prec]
    if G == 1:
        L = O.tree_levels(N, P, 64)
        st = O.fmm_stages(x.astype(np.complex128).reshape(2 ** L, 64, P), N, P, B, Q)
        Tn = t_near(plan, P, L, 64)
        assert rel(Tn, st["T_near"]) < TOL_STAGE[prec]
        assert np.array_equal(Tn[:, :, 0], x.reshape(2 ** L, 64, P)[:, :, 0])
        LL = plan.debug_buffer("L", L).cpu().numpy()
        if plan.info["variant"] & 64:            # FMMFFT_VARIANT_PMAJ: leaf L^L stored [p][b][q]
            LL = LL.reshape(P, 2 ** L, Q).transpose(1, 2, 0)
        else:
            LL = LL.reshape(2 ** L, Q, P)
        assert rel(LL[:, :, 1:], st["L"][L]) < TOL_STAGE[prec]


# ------------------------------------------------------------------ fast-convolution S2T (§8(f) NEXT-4)
@pytest.mark.parametrize("N,P,B,Q,prec,G", [
    (1 << 18, 64, 3, 16, "c64", 1),          # 64 boxes: 2 chunks of 32, periodic wrap at both ends
    (1 << 18, 64, 3, 16, "c128", 1),
    (1 << 20, 16, 4, 16, "c64", 1),          # 1024 boxes: several chunks per CTA
    (1 << 20, 16, 4, 24, "c128", 1),
    (1 << 20, 16, 3, 16, "c64", 2),          # virtual ranks: halo boxes at the rank edges
    (1 << 20, 32, 3, 16, "c128", 4),
])
def test_s2t_fft(F, monkeypatch, N, P, B, Q, prec, G):
    # T_near by per-box DFT_128, the three kernel spectra and the inverse DFT_128 equals the
    # oracle's direct sum (Alg. 1 line 3) at the stage tolerance; p = 0 (C_0 = I) copies exactly
    monkeypatch.setenv("FMMFFT_S2T", "fft")
    plan, x, y = run(F, N, P, B, Q, prec, 64, G=G, virtual=G > 1, debug=G == 1)
    assert plan.info["variant"] & 128                  # FMMFFT_VARIANT_S2T_FFT
    assert rel(y, O.fft_radix2(x)) < TOL_E2E[prec]
    if G == 1:
        L = O.tree_levels(N, P, 64)
        S = x.astype(np.complex128).reshape(2 ** L, 64, P)
        Tn = t_near(plan, P, L, 64)
        assert rel(Tn, O.stage_s2t(S, N, P)) < TOL_STAGE[prec]
        assert np.array_equal(Tn[:, :, 0], x.reshape(2 ** L, 64, P)[:, :, 0])


@pytest.mark.parametrize("kind", ["dmma", "simt"])
def test_s2t_c128_direct_kernels(F, monkeypatch, kind):
    # the complex128 direct-sum S2T kernels the fast convolution replaced as the default:
    # k_s2t_dmma (FP64 tensor pipe) and k_near_up (DFMA), same stage parity
    monkeypatch.setenv("FMMFFT_S2T", kind)
    N, P, B, Q = 1 << 18, 64, 3, 16
    plan, x, y = run(F, N, P, B, Q, "c128", 64, debug=True)
    assert not plan.info["variant"] & 128
    assert rel(y, O.fft_radix2(x)) < TOL_E2E["c128"]
    L = O.tree_levels(N, P, 64)
    S = x.astype(np.complex128).reshape(2 ** L, 64, P)
    assert rel(t_near(plan, P, L, 64), O.stage_s2t(S, N, P)) < TOL_STAGE["c128"]


# ------------------------------------------------------------------ large-M four-step FFT passes
@pytest.mark.parametrize("N,P,prec,G,env", [
    (1 << 23, 2, "c64", 1, None),        # M = 2^22: column pass 2^11 + transposing row pass 2^11
    (1 << 24, 2, "c64", 1, None),        # M = 2^23: two column passes + row pass
    (1 << 22, 2, "c128", 1, None),       # fp64, M = 2^21: three passes of 2^7
    (1 << 21, 4, "c128", 1, None),       # fp64, M = 2^19: 2^9 + 2^10
    (1 << 23, 4, "c64", 4, None),        # first column pass reads the all-to-all receive layout
    (1 << 21, 4, "c64", 1, {"FMMFFT_MFFT": "pass"}),   # the multi-pass Stockham kernel instead
])
def test_large_m_fft(F, monkeypatch, N, P, prec, G, env):
    for k, v in (env or {}).items():
        monkeypatch.setenv(k, v)
    plan, x, y = run(F, N, P, 2, 16, prec, 64, G=G, virtual=G > 1)
    assert rel(y, O.fft_radix2(x)) < TOL_E2E[prec]


# ------------------------------------------------------------------ inverse transform (§8(f) NEXT-1)
@pytest.mark.parametrize("N,P,B,Q,prec,M_L,G", [
    (1 << 12, 16, 2, 16, "c128", 64, 1),
    (1 << 20, 64, 2, 16, "c64", 64, 1),       # the cfg2 shape
    (1 << 20, 16, 3, 16, "c128", 16, 2),      # distributed (virtual ranks)
    (1 << 23, 2, 2, 16, "c64", 64, 1),        # four-step M-FFT
])
def test_inverse_vs_oracle(F, N, P, B, Q, prec, M_L, G):
    x = SI.complex_uniform(0, N, dtype=NPDT[prec])
    inv = F(N=N, P=P, G=G, B=B, Q=Q, precision=prec, M_L=M_L, virtual=G > 1, inverse=True)
    y = inv(torch.from_numpy(x).cuda()).cpu().numpy()
    ref = O.dft_direct(x, inverse=True) if N <= 1 << 12 else O.fft_radix2(x, inverse=True)
    assert rel(y, ref) < TOL_E2E[prec]
    # round trip forward -> inverse
    fwd = F(N=N, P=P, G=G, B=B, Q=Q, precision=prec, M_L=M_L, virtual=G > 1)
    z = inv(fwd(torch.from_numpy(x).cuda())).cpu().numpy()
    assert rel(z, x) < 2 * TOL_E2E[prec]


# ------------------------------------------------------------------ in-house four-step FFT, no FMM (§8(f) NEXT-3)
@pytest.mark.parametrize("N,prec,inverse", [
    (1 << 13, "c64", False), (1 << 20, "c64", False), (1 << 23, "c64", False),   # 2 / 2 / 3 passes
    (1 << 21, "c128", False), (1 << 16, "c128", True), (1 << 22, "c64", True),
])
def test_direct_fft(F, N, prec, inverse):
    x = SI.complex_uniform(0, N, dtype=NPDT[prec])
    plan = F(N=N, P=1, precision=prec, direct=True, inverse=inverse)
    y = plan(torch.from_numpy(x).cuda()).cpu().numpy()
    ref = O.fft_radix2(x, inverse=inverse)
    assert rel(y, ref) < (1e-6 if prec == "c64" else 1e-13)


@pytest.mark.parametrize("N,G,prec,inverse", [
    (1 << 20, 2, "c64", False), (1 << 22, 4, "c64", False), (1 << 24, 8, "c64", False),
    (1 << 18, 8, "c128", False), (1 << 21, 4, "c128", True), (1 << 16, 2, "c64", True),
])
def test_direct_distributed(F, N, G, prec, inverse):
    """The distributed radix-P Cooley-Tukey FFT with three all-to-alls (NEXT-3) through
    virtual ranks: every element against the float64 DFT."""
    x = SI.complex_uniform(0, N, dtype=NPDT[prec])
    plan = F(N=N, P=1, G=G, precision=prec, direct=True, virtual=True, inverse=inverse)
    y = plan(torch.from_numpy(x).cuda()).cpu().numpy()
    ref = O.fft_radix2(x, inverse=inverse)
    assert rel(y, ref) < (1e-6 if prec == "c64" else 1e-13)


def test_direct_distributed_nccl_transport(F, nccl_local):
    N, G = 1 << 20, 4
    x = torch.from_numpy(SI.complex_uniform(0, N, dtype=np.complex64)).cuda()
    a = F(N=N, P=1, G=G, precision="c64", direct=True, virtual=True, transport="nccl")
    b = F(N=N, P=1, G=G, precision="c64", direct=True, virtual=True)
    ya, yb = a(x), b(x)
    torch.cuda.synchronize()
    assert torch.equal(ya, yb)
    a.close()
    b.close()


# ------------------------------------------------------------------ autotuner, measured (§8(f) NEXT-2)
def test_autotune_measured_meets_tol(F):
    from paper_conf_sc_cecka17_b200 import autotune
    N = 1 << 20
    t = autotune(N, G=1, precision="c64", tol=1e-5, measure=True)
    assert t["candidates"] >= 3 and t["ms"] > 0
    plan, x, y = run(F, N, t["P"], t["B"], t["Q"], "c64", t["M_L"])
    assert rel(y, O.fft_radix2(x)) < 1e-5


@pytest.mark.parametrize("N", [1 << 20, 1 << 22])
def test_autotune_c128_meets_tol(F, N):
    # the complex128 pick (Q from the error model, e.g. Q = 16 instead of cfg4's Q = 24) must still
    # meet the north star's 1e-11 bound against the float64 FFT
    from paper_conf_sc_cecka17_b200 import autotune
    t = autotune(N, G=1, precision="c128", tol=1e-11, measure=False)
    plan, x, y = run(F, N, t["P"], t["B"], t["Q"], "c128", t["M_L"])
    assert rel(y, O.fft_radix2(x)) < 1e-11


@pytest.mark.parametrize("P,Q,prec", [(16, 16, "c64"), (32, 8, "c64"), (8, 24, "c128"), (2, 16, "c64"), (64, 16, "c64"),
                                       (64, 24, "c128"), (128, 16, "c64")])
def test_post_pfft_variants(F, P, Q, prec):
    """k_post_pfft_r (P <= 32, registers) and the shared-memory-tile k_post_pfft (P > 32) agree with the oracle."""
    N = 1 << 18
    plan, x, y = run(F, N, P, 2, Q, prec, 64)
    assert rel(y, O.fft_radix2(x)) < (1e-5 if prec == "c64" else 1e-11)


# ------------------------------------------------------------------ real input, C = 1 (§8(f) NEXT-1)
@pytest.mark.parametrize("N,P,B,Q,prec,direct", [
    (1 << 13, 16, 2, 16, "c128", False),   # complex plan = cfg1 (N/2 = 2^12)
    (1 << 13, 16, 2, 16, "c64", False),
    (1 << 21, 64, 2, 16, "c64", False),    # complex plan = cfg2
    (1 << 21, 64, 2, 16, "c128", False),
    (1 << 16, 1, 2, 16, "c64", True),      # four-step (DIRECT) complex plan
    (1 << 16, 1, 2, 16, "c128", True),
])
def test_real_input_vs_oracle(F, N, P, B, Q, prec, direct):
    rdt = np.float32 if prec == "c64" else np.float64
    x = SI.real_uniform(0, N, dtype=rdt)
    plan = F(N=N, P=P, B=B, Q=Q, precision=prec, direct=direct, real=True)
    assert plan.info["N"] == N
    y = plan(torch.from_numpy(x).cuda()).cpu().numpy()
    assert y.shape == (N // 2 + 1,)
    ref = O.rdft(x.astype(np.float64))
    assert rel(y, ref) < TOL_E2E[prec]
    # X_0 and X_{N/2} of a real input are real (up to rounding)
    scale = np.sqrt(np.mean(np.abs(ref) ** 2))
    assert abs(y[0].imag) < 10 * TOL_E2E[prec] * scale and abs(y[-1].imag) < 10 * TOL_E2E[prec] * scale
    # end-to-end path with host buffers gives the same result
    xh = torch.from_numpy(x).pin_memory()
    oh = torch.empty(N // 2 + 1, dtype=plan.dtype).pin_memory()
    plan.execute_host(xh, oh)
    torch.cuda.synchronize()
    assert rel(oh.numpy(), ref) < TOL_E2E[prec]


def test_real_rejects_unsupported(F):
    from paper_conf_sc_cecka17_b200._lib import FmmfftError
    with pytest.raises(FmmfftError):
        F(N=(1 << 13) + 1, P=16, real=True)                    # odd real length
    with pytest.raises(FmmfftError):
        F(N=3 << 12, P=16, G=2, virtual=True, real=True)       # N/2 not a power of two


@pytest.mark.parametrize("N,P,G,prec,direct,transport", [
    (1 << 17, 16, 2, "c64", False, "copy"),
    (1 << 17, 32, 4, "c128", False, "copy"),
    (1 << 18, 64, 8, "c64", False, "copy"),
    (1 << 17, 16, 4, "c64", True, "copy"),      # the distributed six-step FFT (NEXT-3) underneath
    (1 << 17, 16, 2, "c128", False, "nccl"),    # the mirror exchange through NCCL send / recv
])
def test_real_distributed(F, request, N, P, G, prec, direct, transport):
    # real input at G > 1 (virtual ranks): the complex plan of N/2 block-distributed, then the
    # mirror exchange (rank g <- rank G-1-g's block + one element) and the per-rank separation;
    # the global output X_0..X_{N/2} (rank g's block at g N/(2G), X_{N/2} after the last block)
    if transport == "nccl":
        request.getfixturevalue("nccl_local")
    rdt = np.float32 if prec == "c64" else np.float64
    x = SI.real_uniform(0, N, dtype=rdt)
    ref = O.rdft(x.astype(np.float64))
    fwd = F(N=N, P=P, G=G, B=2, Q=16, precision=prec, direct=direct, real=True, virtual=True, transport=transport)
    y = fwd(torch.from_numpy(x).cuda())
    assert y.shape == (N // 2 + 1,)
    assert rel(y.cpu().numpy(), ref) < TOL_E2E[prec]
    assert blockwise_rel(y.cpu().numpy()[:-1], ref[:-1], G) < 2 * TOL_E2E[prec]
    # complex-to-real inverse of the oracle's spectrum (non-real X_0 / X_{N/2} parts ignored)
    X = ref.copy()
    X[0] += 0.7j
    X[-1] += 0.3j
    inv = F(N=N, P=P, G=G, B=2, Q=16, precision=prec, direct=direct, real=True, inverse=True, virtual=True,
            transport=transport)
    z = inv(torch.from_numpy(X.astype(NPDT[prec])).cuda()).cpu().numpy()
    assert z.shape == (N,)
    assert np.linalg.norm(z - x) / np.linalg.norm(x) < TOL_E2E[prec]
    # device round trip
    w = inv(y).cpu().numpy()
    assert np.linalg.norm(w - x) / np.linalg.norm(x) < 2 * TOL_E2E[prec]


@pytest.mark.parametrize("N,P,B,Q,prec,direct", [
    (1 << 13, 16, 2, 16, "c128", False),
    (1 << 13, 16, 2, 16, "c64", False),
    (1 << 21, 64, 2, 16, "c64", False),
    (1 << 21, 64, 2, 16, "c128", False),
    (1 << 16, 1, 2, 16, "c64", True),
    (1 << 16, 1, 2, 16, "c128", True),
])
def test_real_inverse_vs_oracle(F, N, P, B, Q, prec, direct):
    # the spectrum of a seeded real signal, X_0..X_{N/2} (oracle rdft); the C2R inverse returns
    # the signal: x = (1/N) sum_k X_k w_N^{-jk} with X_{N-k} = conj(X_k) (eq. 1 inverted)
    rdt = np.float32 if prec == "c64" else np.float64
    x = SI.real_uniform(0, N, dtype=np.float64)
    X = O.rdft(x)
    ref = np.real(O.fft_radix2(np.concatenate([X, np.conj(X[-2:0:-1])]), inverse=True))
    assert np.max(np.abs(ref - x)) < 1e-12                      # the oracle round trip itself
    inv = F(N=N, P=P, B=B, Q=Q, precision=prec, direct=direct, real=True, inverse=True)
    y = inv(torch.from_numpy(X.astype(NPDT[prec])).cuda()).cpu().numpy()
    assert y.dtype == rdt and y.shape == (N,)
    assert np.linalg.norm(y - ref) / np.linalg.norm(ref) < TOL_E2E[prec]
    # the imaginary parts of X_0 and X_{N/2} are ignored (fmmfft.h): a spectrum with non-real
    # DC / Nyquist values gives the same signal
    Xb = X.copy()
    Xb[0] += 0.7j
    Xb[-1] += 0.3j
    yb = inv(torch.from_numpy(Xb.astype(NPDT[prec])).cuda()).cpu().numpy()
    assert np.linalg.norm(yb - ref) / np.linalg.norm(ref) < TOL_E2E[prec]
    # forward real plan -> inverse real plan round trip on the device
    fwd = F(N=N, P=P, B=B, Q=Q, precision=prec, direct=direct, real=True)
    z = inv(fwd(torch.from_numpy(x.astype(rdt)).cuda())).cpu().numpy()
    assert np.linalg.norm(z - x) / np.linalg.norm(x) < 2 * TOL_E2E[prec]


# ------------------------------------------------------------------ NCCL transport
@pytest.fixture(scope="module")
def nccl_local(F):
    """A 1-rank NCCL communicator on this GPU: virtual plans with transport="nccl" then run every
    exchange (S halo, M^l halos, all-gather, all-to-all) as ncclSend / ncclRecv / group calls,
    captured in the execute graph — the NCCL branch's calls on one GPU."""
    from paper_conf_sc_cecka17_b200 import destroy_comm, init_comm_local
    init_comm_local()
    yield
    import gc
    gc.collect()
    destroy_comm()


@pytest.mark.parametrize("N,P,B,Q,prec,M_L,G", [
    (1 << 16, 32, 2, 16, "c64", 16, 8),      # l_g = 4 > B: replicated top levels
    (1 << 18, 64, 4, 16, "c64", 32, 8),      # l_g = B
    (1 << 20, 32, 2, 16, "c64", 32, 4),      # halo'd per-level kernels
    (1 << 16, 16, 2, 16, "c128", 64, 2),     # G = 2: both neighbours are the same rank
])
def test_nccl_transport_matches_copies(F, nccl_local, N, P, B, Q, prec, M_L, G):
    x = SI.complex_uniform(0, N, dtype=NPDT[prec])
    xd = torch.from_numpy(x).cuda()
    a = F(N=N, P=P, G=G, B=B, Q=Q, precision=prec, M_L=M_L, virtual=True, transport="nccl")
    b = F(N=N, P=P, G=G, B=B, Q=Q, precision=prec, M_L=M_L, virtual=True)
    ya, yb = a(xd), b(xd)
    ya2 = a(xd)                                  # graph replay of the captured NCCL calls
    torch.cuda.synchronize()
    assert torch.equal(ya, yb) and torch.equal(ya, ya2)
    assert rel(ya.cpu().numpy(), O.fft_radix2(x)) < TOL_E2E[prec]
    a.close()
    b.close()


def test_comm_destroy_refused_while_plans_live(F, nccl_local):
    from paper_conf_sc_cecka17_b200 import destroy_comm
    from paper_conf_sc_cecka17_b200._lib import FmmfftError
    a = F(N=1 << 14, P=16, G=2, B=2, Q=16, precision="c64", M_L=16, virtual=True, transport="nccl")
    with pytest.raises(FmmfftError):
        destroy_comm()
    a.close()


def test_two_rank_nccl(F):
    """The real multi-process path: 2 ranks, one GPU each, NCCL over NVLink (needs >= 2 GPUs)."""
    if torch.cuda.device_count() < 2:
        pytest.skip("needs 2 GPUs")
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    r = subprocess.run([sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node=2",
                        "--master-addr", "127.0.0.1", "--master-port", "29533",
                        os.path.join(root, "tests", "nccl_worker.py")], capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, r.stdout[-2000:] + r.stderr[-2000:]
    assert r.stdout.count("NCCL_WORKER_OK") == 2
