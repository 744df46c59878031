// kernel_s2t_fft.cuh — S2T (Alg. 1 line 3, §4.6) as a fast convolution
// (the paper's "symmetries / fast-convolution" next step).
//
// The near field of leaf box b for FMM p is the "interleaved overlapped convolution"
//     T_b[i] = sum_{j=-64}^{127} f_p(j - i) S_window[j],   f_p(k) = S2T_{pk} = cot(pi (p + P k) / N),
// M_L = 64, the window being boxes b-1, b, b+1. Split by source box (s = -1, 0, 1 <-> box b+s):
//     T_b[i] = sum_s sum_{j'<64} g_s(i - j') x_{b+s}[j'],   g_s(n) = f_p(64 s - n),  |i - j'| <= 63,
// so each term is a CIRCULAR convolution of length 128 of the zero-padded box x (64 -> 128 points)
// with h_s[n mod 128] = g_s(n) (n in [-63, 63]; h_s[64] = 0): the 127 distinct lags fit 128 slots
// without aliasing onto the 64 outputs kept. With X = DFT_128(x) and H_s = DFT_128(h_s) / 128
// (host, float64, per plan):
//     T_b = IDFT_128( sum_s H_s . X_{b+s} )[0 .. 63]
// — one forward FFT per SOURCE box (shared by its three targets), 3 complex products per
// frequency, one inverse FFT per target: ~8 K flop per (box, p) instead of the direct 48 K
// (6 C M_L^2). The result is the same sum up to rounding (no approximation).
//
// FFT_128 = 8 x 16 on a group of 8 threads (16 values each): n = t + 8 n2, f = k2 + 16 k1,
//   forward: DFT_16 over n2 in thread t (n2 >= 8 are the zero padding), twiddle w_128^{t k2},
//            exchange, DFT_8 over t in thread t' for rows k2 = 2t', 2t'+1;
//   inverse: DFT_8^-1 over k1 in thread t' (rows 2t', 2t'+1), twiddle w_128^{-k2 a}, exchange,
//            DFT_16^-1 over k2 in thread a -> u[a + 8 b], b < 8 (the 64 outputs kept).
// CTA = (p, run of 32-box chunks), 256 threads = 32 groups: per chunk, group g transforms source
// box bc + 1 + g into a ring of 34 frequency-domain box slots (the two previous boxes carried),
// then, after one barrier, forms target bc + g from slots bc-1+g .. bc+1+g and inverse-transforms
// it through the slot the same group writes next (no second barrier needed for the exchange).
// Slots are [16 rows k2][8 cols], column XOR-swizzled by (row / 2) mod 8: the row-wise (t') and
// column-wise (t, a) accesses of a group are both bank-conflict-free without padding.
// S is read in its natural [b][m][p] order (cp.async gathers of one p, the P CTAs of a box range
// adjacent in the grid so they share the lines in L2) — no p-major copy. T_near is written
// p-major planar [p][b][re/im][m] (what k_post_pfft reads).
#pragma once
#include "common.cuh"
#include "kernels_fft.cuh"

namespace fmmfft {

constexpr int S2TF_CHUNK = 32;                             // boxes per chunk (= thread groups)
constexpr int S2TF_SLOTS = S2TF_CHUNK + 2;
constexpr int S2TF_THREADS = 256;
template <typename R> __host__ __device__ constexpr size_t s2tf_smem_bytes() {
    // slots [34][128] + S staging [32][64] + H [3][128]
    return ((size_t)S2TF_SLOTS * 128 + (size_t)S2TF_CHUNK * 64 + 3 * 128) * sizeof(C2<R>);
}
// H table per p, ordered [s][cc][k1][t'] for f = (2 t' + cc) + 16 k1: a group's 8 threads read 8
// consecutive entries
constexpr int S2TF_H_PER_P = 3 * 128;

__device__ __forceinline__ int s2tf_idx(int row, int col) { return row * 8 + (col ^ ((row >> 1) & 7)); }

template <typename C> __device__ __forceinline__ C cswap(C a) { C r; r.x = a.y; r.y = a.x; return r; }

#ifndef FMMFFT_S2TF_MINB_D
#define FMMFFT_S2TF_MINB_D 2          // complex128 CTAs per SM (register budget)
#endif
template <typename R>
__global__ void __launch_bounds__(S2TF_THREADS, sizeof(R) == 4 ? 2 : FMMFFT_S2TF_MINB_D)
k_s2t_fft(const C2<R>* __restrict__ S, const C2<R>* __restrict__ haloL, const C2<R>* __restrict__ haloR,
          R* __restrict__ Tn, const C2<R>* __restrict__ Htab, int P, int nb, int chunks_per_cta) {
    pdl_trigger();
    using C = C2<R>;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    C* slots = reinterpret_cast<C*>(smem_raw);                   // [34][128]
    C* Ssm = slots + S2TF_SLOTS * 128;                           // [32][64]
    C* Hsm = Ssm + S2TF_CHUNK * 64;                              // [3][2][8][8]
    const int tid = threadIdx.x, g = tid >> 3, t = tid & 7;
    const int p = blockIdx.x;
    const int b0 = blockIdx.y * chunks_per_cta * S2TF_CHUNK;
    const int nch = min(chunks_per_cta, (nb - b0) / S2TF_CHUNK);
    if (nch <= 0) return;
    if (p == 0) {                                                // S2T_{0k} = delta_{k0}: T = S exactly (R1)
        pdl_wait();
        for (int idx = tid; idx < nch * S2TF_CHUNK * 64; idx += S2TF_THREADS) {
            const int bb = b0 + (idx >> 6), m = idx & 63;
            const C x = S[((size_t)bb * 64 + m) * P];
            Tn[(size_t)bb * 128 + m] = x.x;
            Tn[(size_t)bb * 128 + 64 + m] = x.y;
        }
        return;
    }
    // twiddles as powers of one per-thread root (product tree, registers): table lookups
    // w_128^{t k2} from shared memory were up to 8-way bank conflicts (ncu)
    const C wf = twiddle_pow2(R(0), t, 7);                       // w_128^t
    C wi[2];
#pragma unroll
    for (int cc = 0; cc < 2; ++cc) {                             // conj(w_128^{k2}), k2 = 2t + cc
        const C w = twiddle_pow2(R(0), 2 * t + cc, 7);
        wi[cc].x = w.x; wi[cc].y = -w.y;
    }
    {
        const C* hp = Htab + (size_t)p * S2TF_H_PER_P;
        for (int k = tid; k < S2TF_H_PER_P; k += S2TF_THREADS) cp_async_elem(Hsm + k, hp + k);
    }
    const size_t box = (size_t)64 * P;
    auto src_of = [&](int b) -> const C* {                       // box b of this rank (halo / periodic)
        return (b < 0 ? haloL : (b >= nb ? haloR : S + (size_t)b * box)) + p;
    };
    // S of forward boxes: chunk c = -1 -> boxes b0-1, b0 (rows 0, 1); c >= 0 -> b0+32c+1+r
    auto load_S = [&](int c) {
        const int nbx = c < 0 ? 2 : S2TF_CHUNK;
        const int first = c < 0 ? b0 - 1 : b0 + S2TF_CHUNK * c + 1;
        for (int idx = tid; idx < nbx * 64; idx += S2TF_THREADS) {
            const int r = idx >> 6, m = idx & 63;
            cp_async_elem(Ssm + idx, src_of(first + r) + (size_t)m * P);
        }
    };
    auto slot_of = [&](int b) { return slots + ((b - b0 + 1 + 2 * S2TF_SLOTS) % S2TF_SLOTS) * 128; };
    pdl_wait();
    load_S(-1);
    cp_async_wait_all();
    __syncthreads();

    C v[16];
    for (int c = -1; c < nch; ++c) {
        const int bc = b0 + S2TF_CHUNK * c;
        // ---- forward FFT of source box fb (group g), into its slot
        const bool fwd = c >= 0 || g < 2;
        const int fb = c < 0 ? b0 - 1 + g : bc + 1 + g;
        C* E = slot_of(fb);
        if (fwd) {
            const C* xs = Ssm + g * 64;
#pragma unroll
            for (int n2 = 0; n2 < 8; ++n2) v[n2] = xs[t + 8 * n2];
#pragma unroll
            for (int n2 = 8; n2 < 16; ++n2) v[n2] = zero<C>();
            dft16(v);                                            // Y[t][k2]
            twiddle_powers<16>(v, wf);                           // Y[t][k2] w_128^{t k2}
#pragma unroll
            for (int k2 = 0; k2 < 16; ++k2) E[s2tf_idx(k2, t)] = v[k2];
        }
        __syncthreads();                                         // S staging free, Y rows complete
        if (c + 1 < nch) load_S(c + 1);                          // prefetch the next chunk's S
        if (fwd) {
#pragma unroll
            for (int cc = 0; cc < 2; ++cc) {
                const int row = 2 * t + cc;
#pragma unroll
                for (int tt = 0; tt < 8; ++tt) v[cc * 8 + tt] = E[s2tf_idx(row, tt)];
                dft8(v + cc * 8);                                // X[row + 16 k1], k1 < 8
#pragma unroll
                for (int k1 = 0; k1 < 8; ++k1) E[s2tf_idx(row, k1)] = v[cc * 8 + k1];   // own rows: in place
            }
        }
        __syncthreads();                                         // every slot of the window ready
        if (c < 0) {
            cp_async_wait_all();
            __syncthreads();
            continue;
        }
        // ---- target tb = bc + g: U = sum_s H_s X_{tb+s} (frequencies of rows 2t, 2t+1)
        const int tb = bc + g;
#pragma unroll
        for (int k = 0; k < 16; ++k) v[k] = zero<C>();
#pragma unroll
        for (int s = 0; s < 3; ++s) {
            const C* Xs = slot_of(tb - 1 + s);
            const C* Hs = Hsm + s * 128 + t;
#pragma unroll
            for (int cc = 0; cc < 2; ++cc)
#pragma unroll
                for (int k1 = 0; k1 < 8; ++k1) {
                    const C x = Xs[s2tf_idx(2 * t + cc, k1)], h = Hs[(cc * 8 + k1) * 8];
                    C& a = v[cc * 8 + k1];
                    a.x = fma(h.x, x.x, fma(-h.y, x.y, a.x));
                    a.y = fma(h.x, x.y, fma(h.y, x.x, a.y));
                }
        }
        __syncthreads();                                         // all reads of the window done
        // ---- inverse FFT of target tb through slot(tb - 1) (= the slot this group fills next)
        C* F = slot_of(tb - 1);
#pragma unroll
        for (int cc = 0; cc < 2; ++cc) {
            const int k2 = 2 * t + cc;
            C* u = v + cc * 8;
#pragma unroll
            for (int k1 = 0; k1 < 8; ++k1) u[k1] = cswap(u[k1]);
            dft8(u);                                             // inverse DFT_8 over k1 (swap trick)
#pragma unroll
            for (int a = 0; a < 8; ++a) u[a] = cswap(u[a]);
            twiddle_powers<8>(u, wi[cc]);                        // w_128^{-k2 a}
#pragma unroll
            for (int a = 0; a < 8; ++a) F[s2tf_idx(k2, a)] = u[a];
        }
        __syncwarp();
#pragma unroll
        for (int k2 = 0; k2 < 16; ++k2) v[k2] = cswap(F[s2tf_idx(k2, t)]);
        dft16(v);                                                // inverse DFT_16 over k2 -> u[t + 8 b]
        {
            R* o = Tn + ((size_t)p * nb + tb) * 128 + t;         // [p][b][re/im][m]
#pragma unroll
            for (int b = 0; b < 8; ++b) {
                o[8 * b] = v[b].y;                               // swap back: re = .y, im = .x
                o[64 + 8 * b] = v[b].x;
            }
        }
        __syncwarp();                                            // F is this group's next forward slot
        cp_async_wait_all();
        __syncthreads();                                         // next chunk's S landed
    }
}

}  // namespace fmmfft
