// kernels_fft.cuh — the 2D FFT F_{M,P} of Alg. 1 line 16:
//   * k_post_pfft: L2T (line 14) + POST (line 15) + the M local P-point FFTs (§3 step 2),
//     writing W[k2][m] already transposed into the per-destination all-to-all layout
//     (the paper fuses POST into cuFFTXt's load callback; here the whole chain
//     L2T -> POST -> FFT_P -> transposed store is one kernel);
//   * k_fft_pass: one pass of a multi-pass Stockham FFT over rows of length M (§3 step 4),
//     the first pass reading the all-to-all receive layout directly.
// Both use the same shared-memory Stockham autosort FFT on a tile of `ncols` columns.
#pragma once
#include "common.cuh"

namespace fmmfft {

// X[t] = sum_u v[u] w_E^{ut}, natural order, for E = 2, 4, 8.
template <typename C> __device__ __forceinline__ void dft2(C* v) {
    C a = v[0], b = v[1];
    v[0] = cadd(a, b); v[1] = csub(a, b);
}
template <typename C> __device__ __forceinline__ void dft4(C* v) {
    C t0 = cadd(v[0], v[2]), t1 = csub(v[0], v[2]);
    C t2 = cadd(v[1], v[3]), t3 = mul_mi(csub(v[1], v[3]));
    v[0] = cadd(t0, t2); v[2] = csub(t0, t2);
    v[1] = cadd(t1, t3); v[3] = csub(t1, t3);
}
template <typename C> __device__ __forceinline__ void dft8(C* v) {
    using R = decltype(v[0].x);
    C e[4] = {v[0], v[2], v[4], v[6]};
    C o[4] = {v[1], v[3], v[5], v[7]};
    dft4(e); dft4(o);
    const R h = (R)0.70710678118654752440;
    // w8^1 = (1 - i) h, w8^2 = -i, w8^3 = (-1 - i) h
    C o1; o1.x = (o[1].x + o[1].y) * h; o1.y = (o[1].y - o[1].x) * h;
    C o2 = mul_mi(o[2]);
    C o3; o3.x = (o[3].y - o[3].x) * h; o3.y = -(o[3].x + o[3].y) * h;
    v[0] = cadd(e[0], o[0]); v[4] = csub(e[0], o[0]);
    v[1] = cadd(e[1], o1);   v[5] = csub(e[1], o1);
    v[2] = cadd(e[2], o2);   v[6] = csub(e[2], o2);
    v[3] = cadd(e[3], o3);   v[7] = csub(e[3], o3);
}
template <int E, typename C> __device__ __forceinline__ void dftE(C* v) {
    if constexpr (E == 2) dft2(v);
    else if constexpr (E == 4) dft4(v);
    else dft8(v);
}

// One radix-E Stockham stage on a shared tile: columns col < ncols of length len (power of
// two), column stride ld. For each butterfly j < len/E with k = j mod Ns:
//   v_t = x[j + t len/E] w_{Ns E}^{k t};  v = DFT_E(v);  y[(j - k) E + k + t Ns] = v_t.
// In place: each thread keeps its butterflies' values in registers across a barrier.
// tw[u] = w_len^u for u < len. EPT = elements per thread (ncols * len <= EPT * blockDim).
template <int E, int EPT, typename C>
__device__ __forceinline__ void stockham_stage(C* tile, int ncols, int len, int ld, int Ns, const C* tw) {
    constexpr int NB = EPT / E;
    const int nthr = blockDim.x, tid = threadIdx.x;
    const int per = len / E;
    const int total = ncols * per;
    const int tws = len / (Ns * E);
    C v[NB][E];
#pragma unroll
    for (int k = 0; k < NB; ++k) {
        const int bf = tid + k * nthr;
        if (bf < total) {
            const int col = bf / per, j = bf % per, kk = j % Ns;
            const C* x = tile + col * ld + j;
#pragma unroll
            for (int t = 0; t < E; ++t) v[k][t] = x[t * per];
            if (Ns > 1) {
#pragma unroll
                for (int t = 1; t < E; ++t) v[k][t] = cmul(v[k][t], tw[(kk * t * tws) & (len - 1)]);
            }
            dftE<E>(v[k]);
        }
    }
    __syncthreads();
#pragma unroll
    for (int k = 0; k < NB; ++k) {
        const int bf = tid + k * nthr;
        if (bf < total) {
            const int col = bf / per, j = bf % per, kk = j % Ns;
            C* y = tile + col * ld + (j - kk) * E + kk;
#pragma unroll
            for (int t = 0; t < E; ++t) y[t * Ns] = v[k][t];
        }
    }
    __syncthreads();
}

// Full in-place FFT of every column: radix-8 stages, then one radix-4 or radix-2 stage.
template <int EPT, typename C>
__device__ void fft_columns(C* tile, int ncols, int len, int ld, const C* tw) {
    int Ns = 1;
    while (Ns < len) {
        const int rem = len / Ns;
        if (rem >= 8) { stockham_stage<8, EPT>(tile, ncols, len, ld, Ns, tw); Ns *= 8; }
        else if (rem == 4) { stockham_stage<4, EPT>(tile, ncols, len, ld, Ns, tw); Ns *= 4; }
        else { stockham_stage<2, EPT>(tile, ncols, len, ld, Ns, tw); Ns *= 2; }
    }
}

template <typename R>
__device__ __forceinline__ void fill_twiddles(C2<R>* tw, int len) {
    for (int u = threadIdx.x; u < len; u += blockDim.x) tw[u] = twiddle<R>(u, len);
}

// ---------------------------------------------------------------------------------------------
// L2T + POST + P-point FFT + transposed store (Alg. 1 lines 14-16, §3 step 2).
//   T_{pmb}  = T_near_{pmb} + L2T_{mq} L^L_{pqb}                       p >= 1
//   T_{pmb} <- rho_p (T_{pmb} + i r_p)                                   p >= 1   (R1)
//   W[k2][m] = sum_p w_P^{p k2} T_{pm}
// CTA = (leaf box b, m sub-tile of MS rows). W row k2 has length M/G (this rank's m range):
// element (k2, m_local) at W[k2 * Mg + m_local] — which is the all-to-all send layout
// [destination r][k2 local][m local] with k2 = r P/G + k2 local.
// ---------------------------------------------------------------------------------------------
template <typename R, int EPT>
__global__ void __launch_bounds__(256)
k_post_pfft(const C2<R>* __restrict__ Tn, const C2<R>* __restrict__ LL, const C2<R>* __restrict__ r,
            const C2<R>* __restrict__ rho, const R* __restrict__ s2m, C2<R>* __restrict__ W,
            int P, int M_L, int Q, int MS, long long Mg) {
    using C = C2<R>;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    const int ld = P + 1;
    C* tile = reinterpret_cast<C*>(smem_raw);                    // [MS][P + 1]
    C* tw = tile + MS * ld;                                       // [P]
    R* s2m_sm = reinterpret_cast<R*>(tw + P);                    // [Q][MS]
    const int tid = threadIdx.x, nthr = blockDim.x;
    const int nsub = M_L / MS;
    const int b = blockIdx.x / nsub, m0 = (blockIdx.x % nsub) * MS;

    fill_twiddles<R>(tw, P);
    for (int idx = tid; idx < Q * MS; idx += nthr) s2m_sm[idx] = s2m[(idx / MS) * M_L + m0 + idx % MS];
    const C* src = Tn + ((size_t)b * M_L + m0) * P;
    for (int idx = tid; idx < MS * P; idx += nthr) tile[(idx / P) * ld + idx % P] = ldg_c(src + idx);
    __syncthreads();

    // L2T + POST: thread owns one p and a group of MG consecutive m (L^L loaded once per q).
    constexpr int MG = 8;
    const int ngrp = (MS + MG - 1) / MG;
    const C* Lb = LL + (size_t)b * Q * P;
    for (int idx = tid; idx < P * ngrp; idx += nthr) {
        const int p = idx % P, g = idx / P;
        if (p == 0) continue;                                      // C_0 = I (R1)
        C acc[MG];
#pragma unroll
        for (int u = 0; u < MG; ++u) acc[u] = zero<C>();
        for (int q = 0; q < Q; ++q) {
            const C l = ldg_c(Lb + (size_t)q * P + p);
#pragma unroll
            for (int u = 0; u < MG; ++u)
                if (g * MG + u < MS) rfma(acc[u], s2m_sm[q * MS + g * MG + u], l);
        }
        const C rp = ldg_c(r + p), rh = ldg_c(rho + p);
#pragma unroll
        for (int u = 0; u < MG; ++u) {
            const int m = g * MG + u;
            if (m < MS) {
                C t = cadd(tile[m * ld + p], acc[u]);
                t.x -= rp.y; t.y += rp.x;                           // + i r_p
                tile[m * ld + p] = cmul(rh, t);
            }
        }
    }
    __syncthreads();
    fft_columns<EPT>(tile, MS, P, ld, tw);
    // W[k2][b M_L + m0 + m]: contiguous runs of MS along m for every k2
    C* dst = W + (size_t)b * M_L + m0;
    for (int idx = tid; idx < MS * P; idx += nthr) {
        const int k2 = idx / MS, m = idx % MS;
        dst[(size_t)k2 * Mg + m] = tile[m * ld + k2];
    }
}

// ---------------------------------------------------------------------------------------------
// One pass of the multi-pass Stockham FFT along rows of length M (§3 step 4):
// radix Rp, span Ns (product of the previous passes' radices). For j < M/Rp, k = j mod Ns:
//   v_t = x[j + t M/Rp] w_{Ns Rp}^{k t},  v = DFT_Rp(v),  y[(j - k) Rp + k + t Ns] = v_t.
// CTA = (chunk of c consecutive j, row). Element m of input row `row` is read at
//   in[row * in_row + (m / blk) * blk_stride + m % blk]
// which expresses both a plain row (blk = M) and the all-to-all receive layout
// [source rank][k2 local][m local] (blk = M/G, blk_stride = (P/G)(M/G), in_row = M/G).
// Output rows are plain: out[row * M + index].
// ---------------------------------------------------------------------------------------------
template <typename R, int EPT>
__global__ void __launch_bounds__(256)
k_fft_pass(const C2<R>* __restrict__ in, C2<R>* __restrict__ out, long long M, int Rp, long long Ns, int c,
           long long in_row, long long blk, long long blk_stride) {
    using C = C2<R>;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    const int ld = Rp + 1;
    C* tile = reinterpret_cast<C*>(smem_raw);                    // [c][Rp + 1]
    C* tw = tile + c * ld;                                        // [Rp]
    const int tid = threadIdx.x, nthr = blockDim.x;
    const long long row = blockIdx.y;
    const long long j0 = (long long)blockIdx.x * c;
    const long long stride = M / Rp;
    const long long span = Ns * Rp;

    fill_twiddles<R>(tw, Rp);
    const C* xin = in + row * in_row;
    for (int idx = tid; idx < c * Rp; idx += nthr) {
        const int t = idx / c, jj = idx % c;
        const long long m = j0 + jj + (long long)t * stride;
        C v = ldg_c(xin + (m / blk) * blk_stride + (m % blk));
        if (Ns > 1) {
            const long long k = (j0 + jj) % Ns;
            if (t) v = cmul(v, twiddle<R>((k * t) % span, span));
        }
        tile[jj * ld + t] = v;
    }
    __syncthreads();
    fft_columns<EPT>(tile, c, Rp, ld, tw);
    C* yout = out + row * M;
    if (Ns >= c) {
        for (int idx = tid; idx < c * Rp; idx += nthr) {
            const int t = idx / c, jj = idx % c;
            const long long j = j0 + jj, k = j % Ns;
            yout[(j - k) * Rp + k + (long long)t * Ns] = tile[jj * ld + t];
        }
    } else {
        const int ns = (int)Ns;
        for (int idx = tid; idx < c * Rp; idx += nthr) {
            const int jb = idx / (ns * Rp), rem = idx % (ns * Rp);
            const int t = rem / ns, k = rem % ns;
            yout[j0 * Rp + idx] = tile[(jb * ns + k) * ld + t];
        }
    }
}

}  // namespace fmmfft
