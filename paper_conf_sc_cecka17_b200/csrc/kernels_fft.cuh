// kernels_fft.cuh — the 2D FFT F_{M,P} of Alg. 1 line 16:
//   * k_post_pfft: L2T (line 14) + POST (line 15) + the M local P-point FFTs (§3 step 2),
//     writing W[k2][m] already transposed into the per-destination all-to-all layout
//     (the paper fuses POST into cuFFTXt's load callback; here the whole chain
//     L2T -> POST -> FFT_P -> transposed store is one kernel);
//   * k_fft_pass: one pass of a multi-pass Stockham FFT over rows of length M (§3 step 4),
//     the first pass reading the all-to-all receive layout directly.
// Both run the same shared-memory Stockham autosort FFT on a tile of columns, compiled for one
// transform length (template LLEN = log2 length): every stage's radix, shifts, masks and
// twiddle strides are compile-time constants; 8 elements per thread per stage.
#pragma once
#include <cooperative_groups.h>

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

// exp(-2 pi i e / 2^ls) for 0 <= e < 2^ls, exact argument (split above 2^24 for fp32)
__device__ __forceinline__ float2 twiddle_pow2(float, int e, int ls) {
    float s, c;
    if (ls <= 24) {
        sincospif(ldexpf((float)e, 1 - ls), &s, &c);
        return make_float2(c, -s);
    }
    const int hi = e & ~4095, lo = e & 4095;
    float s2, c2;
    sincospif(ldexpf((float)hi, 1 - ls), &s, &c);
    sincospif(ldexpf((float)lo, 1 - ls), &s2, &c2);
    return cmul(make_float2(c, -s), make_float2(c2, -s2));
}
__device__ __forceinline__ double2 twiddle_pow2(double, int e, int ls) {
    double s, c;
    sincospi(ldexp((double)e, 1 - ls), &s, &c);
    return make_double2(c, -s);
}

// One radix-E Stockham stage on a shared tile of columns of length 2^LLEN, column stride
// 2^LLEN + 1 (padding against bank conflicts). For each butterfly j < len/E, k = j mod Ns:
//   v_t = x[j + t len/E] w_{Ns E}^{k t};  v = DFT_E(v);  y[(j - k) E + k + t Ns] = v_t.
// In place: each thread keeps its 8/E butterflies in registers across a barrier.
// tw[u] = w_len^u, u < len. Lanes run over COLUMNS (consecutive columns, same butterfly j): the
// Stockham write y[(j - k) E + k + t Ns] then lands on a stride of the column pitch (P + 1
// complex: at most 2-way bank conflicts) instead of a stride of E elements within one column
// (up to 16-way for E = 8), and the warp's twiddle is a broadcast.
template <int E, int LLEN, int LNS, typename C>
__device__ __forceinline__ void stockham_stage(C* tile, int ncols, const C* tw) {
    constexpr int NB = 8 / E;
    constexpr int LE = E == 8 ? 3 : (E == 4 ? 2 : 1);
    constexpr int LPER = LLEN - LE;
    constexpr int LD = (1 << LLEN) + 1;
    constexpr int NS = 1 << LNS;
    constexpr int LTWS = LLEN - LNS - LE;                       // tw index = k t len / (Ns E)
    const int nthr = blockDim.x, tid = threadIdx.x;
    const int total = ncols << LPER;
    C v[NB][E];
#pragma unroll
    for (int k = 0; k < NB; ++k) {
        const int bf = tid + k * nthr;
        if (bf < total) {
            const int col = bf & (ncols - 1), j = bf / ncols;
            const C* x = tile + col * LD + j;
#pragma unroll
            for (int t = 0; t < E; ++t) v[k][t] = x[t << LPER];
            if constexpr (LNS > 0) {
                const int kk = j & (NS - 1);
#pragma unroll
                for (int t = 1; t < E; ++t) v[k][t] = cmul(v[k][t], tw[(kk * t) << LTWS]);
            }
            dftE<E>(v[k]);
        }
    }
    __syncthreads();
#pragma unroll
    for (int k = 0; k < NB; ++k) {
        const int bf = tid + k * nthr;
        if (bf < total) {
            const int col = bf & (ncols - 1), j = bf / ncols, kk = j & (NS - 1);
            C* y = tile + col * LD + ((j - kk) << LE) + kk;
#pragma unroll
            for (int t = 0; t < E; ++t) y[t << LNS] = v[k][t];
        }
    }
    __syncthreads();
}

// In-place FFT of every column: radix-8 stages, then one radix-4 or radix-2 stage.
template <int LLEN, int LNS = 0, typename C>
__device__ __forceinline__ void fft_columns(C* tile, int ncols, const C* tw) {
    if constexpr (LNS < LLEN) {
        constexpr int REM = LLEN - LNS;
        constexpr int LE = REM >= 3 ? 3 : REM;
        stockham_stage<1 << LE, LLEN, LNS>(tile, ncols, tw);
        fft_columns<LLEN, LNS + LE>(tile, ncols, tw);
    }
}

template <typename R>
__device__ __forceinline__ void fill_twiddles(C2<R>* tw, int llen) {
    for (int u = threadIdx.x; u < (1 << llen); u += blockDim.x) tw[u] = twiddle_pow2(R(0), u, llen);
}

// ---------------------------------------------------------------------------------------------
// L2T + POST + P-point FFT + transposed store (Alg. 1 lines 14-16, §3 step 2).
//   T_{pmb}  = T_near_{pmb} + L2T_{mq} L^L_{pqb}                       p >= 1
//   T_{pmb} <- rho_p (T_{pmb} + i r_p)                                   p >= 1   (R1)
//   W[k2][m] = sum_p w_P^{p k2} T_{pm}
// CTA = (leaf box b, m sub-tile of MS rows), MS*P/8 threads, P = 2^LP. W row k2 has length
// Mg = M/G (this rank's m range): element (k2, m_local) at W[k2 * Mg + m_local] — the
// all-to-all send layout [destination r][k2 local][m local] with k2 = r P/G + k2 local.
// ---------------------------------------------------------------------------------------------
template <typename R, int LP, int QT>
__global__ void __launch_bounds__(sizeof(R) == 4 ? 1024 : 512)
k_post_pfft(const C2<R>* __restrict__ Tn, const C2<R>* __restrict__ LL, const C2<R>* __restrict__ r,
            const C2<R>* __restrict__ rho, const R* __restrict__ s2m, C2<R>* __restrict__ W,
            int lML, int Qrt, int lMS, int Mg, int stage_L, int pmaj) {
    pdl_trigger();
    using C = C2<R>;
    constexpr int P = 1 << LP, LD = P + 1;
    constexpr int MG = 8;                                         // m per thread in L2T + POST
    extern __shared__ __align__(16) unsigned char smem_raw[];
    const int Q = QT ? QT : Qrt;
    const int MS = 1 << lMS, M_L = 1 << lML;
    C* tile = reinterpret_cast<C*>(smem_raw);                    // [MS][P + 1]
    C* tw = tile + MS * LD;                                       // [P]
    C* Lsm = tw + P;                                              // [Q][P] (pmaj: [P][Q + 1]) L^L of box b (if staged)
    R* s2m_sm = reinterpret_cast<R*>(Lsm + (stage_L ? (Q + 1) * P : 0)); // [Q][MS]  (16-byte aligned: MS % 8 == 0)
    const int tid = threadIdx.x, nthr = blockDim.x;
    const int lnsub = lML - lMS;
    const int b = blockIdx.x >> lnsub, m0 = (blockIdx.x & ((1 << lnsub) - 1)) << lMS;

    // constants (independent of the FMM stages): L2T rows of this m sub-tile, twiddles
    {
        constexpr int V = 16 / sizeof(R);                         // R per 16-byte copy
        const int nv = (Q * MS) / V, vpr = MS / V;
        for (int idx = tid; idx < nv; idx += nthr) {
            const int q = idx / vpr, c = idx - q * vpr;
            cp_async<16>(s2m_sm + q * MS + c * V, s2m + (size_t)q * M_L + m0 + c * V);
        }
    }
    fill_twiddles<R>(tw, LP);
    pdl_wait();                                                   // T_near / L^L / r from the FMM stages
    {
        // T_near [p][b][re/im][m] (p blocks of 2 nb M_L = 2 Mg reals) -> tile [m][p] (stride P + 1)
        const R* src = reinterpret_cast<const R*>(Tn) + ((size_t)b << (lML + 1)) + m0;
        for (int idx = tid; idx < (MS << LP); idx += nthr) {
            const int pp = idx >> lMS, m = idx & (MS - 1);
            cp_async_elem(&tile[m * LD + pp].x, src + (size_t)pp * 2 * Mg + m);
            cp_async_elem(&tile[m * LD + pp].y, src + (size_t)pp * 2 * Mg + M_L + m);
        }
        if (stage_L && pmaj) {                                    // [p][b][q] -> Lsm[p][Q + 1] (padded rows)
            const int nbt = Mg >> lML;
            for (int idx = tid; idx < Q * P; idx += nthr) {
                const int pp = idx / Q, q = idx - pp * Q;
                cp_async_elem(Lsm + pp * (Q + 1) + q, LL + ((size_t)pp * nbt + b) * Q + q);
            }
        } else if (stage_L) {
            const C* Lb = LL + (size_t)b * Q * P;
            constexpr int V = 16 / sizeof(C);
            for (int idx = tid; idx < Q * P / V; idx += nthr) cp_async<16>(Lsm + idx * V, Lb + idx * V);
        }
    }
    cp_async_wait_all();
    __syncthreads();

    // L2T + POST: thread (p, g) owns one p and MG consecutive m (L^L read once per q, the MG
    // L2T coefficients as two 16-byte broadcasts). MS * P / MG pairs, a multiple of nthr.
    const C* Lb = LL + (size_t)b * Q * P;
    for (int idx = tid; idx < (MS << LP) / MG; idx += nthr) {
        const int p = idx & (P - 1), g = idx >> LP;
        if (p == 0) continue;                                      // C_0 = I (R1)
        C acc[MG];
#pragma unroll
        for (int u = 0; u < MG; ++u) acc[u] = zero<C>();
        const R* a = s2m_sm + g * MG;
#pragma unroll 4
        for (int q = 0; q < Q; ++q) {
            const C l = stage_L ? (pmaj ? Lsm[p * (Q + 1) + q] : Lsm[q * P + p])
                                : (pmaj ? ldg_c(LL + ((size_t)p * (Mg >> lML) + b) * Q + q) : ldg_c(Lb + q * P + p));
            R av[MG];
            if constexpr (sizeof(R) == 4) {
                const float4 a0 = *reinterpret_cast<const float4*>(a + q * MS), a1 = *reinterpret_cast<const float4*>(a + q * MS + 4);
                av[0] = a0.x; av[1] = a0.y; av[2] = a0.z; av[3] = a0.w; av[4] = a1.x; av[5] = a1.y; av[6] = a1.z; av[7] = a1.w;
            } else {
#pragma unroll
                for (int u = 0; u < MG; u += 2) {
                    const double2 d = *reinterpret_cast<const double2*>(a + q * MS + u);
                    av[u] = d.x; av[u + 1] = d.y;
                }
            }
#pragma unroll
            for (int u = 0; u < MG; ++u) rfma(acc[u], av[u], l);
        }
        const C rp = ldg_c(r + p), rh = ldg_c(rho + p);
#pragma unroll
        for (int u = 0; u < MG; ++u) {
            C* t = tile + (g * MG + u) * LD + p;
            C v = cadd(*t, acc[u]);
            v.x -= rp.y; v.y += rp.x;                               // + i r_p
            *t = cmul(rh, v);
        }
    }
    __syncthreads();
    fft_columns<LP>(tile, MS, tw);
    // W[k2][b M_L + m0 + m]: contiguous runs of MS along m for every k2
    C* dst = W + ((size_t)b << lML) + m0;
    for (int idx = tid; idx < (MS << LP); idx += nthr) {
        const int k2 = idx >> lMS, m = idx & (MS - 1);
        dst[(size_t)k2 * Mg + m] = tile[m * LD + k2];
    }
}

// ---------------------------------------------------------------------------------------------
// One pass of the multi-pass Stockham FFT along rows of length M = 2^lM (§3 step 4):
// radix Rp = 2^LR, span Ns = 2^lNs (product of the previous passes' radices). For j < M/Rp,
// k = j mod Ns:
//   v_t = x[j + t M/Rp] w_{Ns Rp}^{k t},  v = DFT_Rp(v),  y[(j - k) Rp + k + t Ns] = v_t.
// CTA = (chunk of c = 2^lc consecutive j, row), c*Rp/8 threads. Input element m of row `row`
// is at in[row * in_row + (m >> lblk) * blk_stride + (m & (2^lblk - 1))], which expresses both a
// plain row (lblk = lM) and the all-to-all receive layout [source rank][k2 local][m local]
// (2^lblk = M/G, blk_stride = (P/G)(M/G), in_row = M/G). Output rows are plain.
// ---------------------------------------------------------------------------------------------
template <typename R, int LR>
__global__ void __launch_bounds__(sizeof(R) == 4 ? 1024 : 512)
k_fft_pass(const C2<R>* __restrict__ in, C2<R>* __restrict__ out, int lM, int lNs, int lc,
           int in_row, int lblk, int blk_stride, const C2<R>* __restrict__ dc) {
    pdl_trigger();
    using C = C2<R>;
    constexpr int Rp = 1 << LR, LD = Rp + 1;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    const int c = 1 << lc;
    C* tile = reinterpret_cast<C*>(smem_raw);                    // [c][Rp + 1]
    C* tw = tile + c * LD;                                        // [Rp]
    const int tid = threadIdx.x, nthr = blockDim.x;
    const size_t row = blockIdx.y;
    const int j0 = blockIdx.x << lc;
    const int lstride = lM - LR;
    const int Ns = 1 << lNs;
    const int lspan = lNs + LR;
    const int bmask = (1 << lblk) - 1;
    const C* xin = in + row * (size_t)in_row;
    const int total = c << LR;

    fill_twiddles<R>(tw, LR);                                     // independent of the predecessor
    pdl_wait();
    // 8 elements per thread: all loads issued before any is used
    C v[8];
#pragma unroll
    for (int u = 0; u < 8; ++u) {
        const int idx = tid + u * nthr;
        if (idx < total) {
            const int t = idx >> lc, jj = idx & (c - 1);
            const int m = j0 + jj + (t << lstride);
            v[u] = ldg_c(xin + (size_t)(m >> lblk) * blk_stride + (m & bmask));
        }
    }
#pragma unroll
    for (int u = 0; u < 8; ++u) {
        const int idx = tid + u * nthr;
        if (idx < total) {
            const int t = idx >> lc, jj = idx & (c - 1);
            C x = v[u];
            if (lNs > 0 && t) x = cmul(x, twiddle_pow2(R(0), ((j0 + jj) & (Ns - 1)) * t, lspan));
            tile[jj * LD + t] = x;
        }
    }
    __syncthreads();
    fft_columns<LR>(tile, c, tw);
    C* yout = out + (row << lM);
    if (lNs >= lc) {
#pragma unroll 4
        for (int idx = tid; idx < total; idx += nthr) {
            const int t = idx >> lc, jj = idx & (c - 1);
            const int j = j0 + jj, k = j & (Ns - 1);
            yout[((j - k) << LR) + k + (t << lNs)] = tile[jj * LD + t];
        }
    } else {
        const int lblkw = lNs + LR;
#pragma unroll 4
        for (int idx = tid; idx < total; idx += nthr) {
            const int jb = idx >> lblkw, rem = idx & ((1 << lblkw) - 1);
            const int t = rem >> lNs, k = rem & (Ns - 1);
            yout[(j0 << LR) + idx] = tile[((jb << lNs) + k) * LD + t];
        }
    }
    if (dc != nullptr && j0 == 0) {                              // the row's k = 0 output (R19)
        __syncthreads();
        if (tid == 0) yout[0] = dc[row];
    }
}

// ---------------------------------------------------------------------------------------------
// k_fft_row: the whole M-point FFT of one row in ONE pass (§3 step 4), for rows that fit
// in shared memory (M = 2^LLEN <= 2^14 complex64 / 2^13 complex128). Stockham autosort with a
// first stage of radix R0 = 2^(LLEN mod 4) (16 if that is 0) and radix-16 stages after it; a
// thread owns 16 elements per stage (16/r butterflies), M/16 threads per row:
//   stage (r, Ns): for j < M/r, k = j mod Ns:
//     v_t = x[j + t M/r] w_{r Ns}^{k t},  v = DFT_r(v),  y[(j - k) r + k + t Ns] = v_t.
// The first stage reads the row straight from global memory (the all-to-all receive layout as
// in k_fft_pass), the last (r = 16, Ns = M/16, so k = j) stores y[j + t M/16] — natural order —
// straight to global memory; in between, shared memory with one pad element per 16 (the
// stride-4 / stride-r write patterns land on distinct banks). Twiddles: w_M^u for u < M/16 from
// a host-computed (fp64) table; the powers w^t, t < 16, by a depth-4 product tree.
// ---------------------------------------------------------------------------------------------
template <typename C, typename Rr>
__device__ __forceinline__ C cmul_k(C a, Rr re, Rr im) {         // a * (re + i im), constants
    C r;
    r.x = a.x * re - a.y * im;
    r.y = a.x * im + a.y * re;
    return r;
}

// X[k] = sum_n v[n] w_16^{nk}, natural order in and out: 4 x 4 with inner twiddles w_16^{n2 k1}
template <typename C> __device__ __forceinline__ void dft16(C* v) {
    using R = decltype(v[0].x);
    const R c1 = (R)0.92387953251128675613, s1 = (R)0.38268343236508977173, h = (R)0.70710678118654752440;
    C a[4][4];
#pragma unroll
    for (int n2 = 0; n2 < 4; ++n2) {
        C t[4] = {v[n2], v[4 + n2], v[8 + n2], v[12 + n2]};
        dft4(t);
#pragma unroll
        for (int k1 = 0; k1 < 4; ++k1) a[n2][k1] = t[k1];
    }
    // w16^1 = (c1,-s1), w16^2 = (h,-h), w16^3 = (s1,-c1), w16^4 = -i, w16^6 = (-h,-h), w16^9 = (-c1,s1)
    a[1][1] = cmul_k(a[1][1], c1, -s1);
    a[1][2] = cmul_k(a[1][2], h, -h);
    a[1][3] = cmul_k(a[1][3], s1, -c1);
    a[2][1] = cmul_k(a[2][1], h, -h);
    a[2][2] = mul_mi(a[2][2]);
    a[2][3] = cmul_k(a[2][3], -h, -h);
    a[3][1] = cmul_k(a[3][1], s1, -c1);
    a[3][2] = cmul_k(a[3][2], -h, -h);
    a[3][3] = cmul_k(a[3][3], -c1, s1);
#pragma unroll
    for (int k1 = 0; k1 < 4; ++k1) {
        C t[4] = {a[0][k1], a[1][k1], a[2][k1], a[3][k1]};
        dft4(t);
#pragma unroll
        for (int k2 = 0; k2 < 4; ++k2) v[k1 + 4 * k2] = t[k2];
    }
}

template <int E, typename C> __device__ __forceinline__ void dftR(C* v) {
    if constexpr (E == 16) dft16(v);
    else dftE<E>(v);
}

// v[t] *= w^t for t = 1 .. E-1 (w^t by a product tree of depth <= 4)
template <int E, typename C> __device__ __forceinline__ void twiddle_powers(C* v, C w1) {
    C w[E];
    w[1] = w1;
#pragma unroll
    for (int t = 2; t < E; ++t) w[t] = (t & 1) ? cmul(w[t - 1], w1) : cmul(w[t / 2], w[t / 2]);
#pragma unroll
    for (int t = 1; t < E; ++t) v[t] = cmul(v[t], w[t]);
}

__device__ __forceinline__ constexpr int row_pad(int a) { return a + (a >> 4); }

template <typename R, int LLEN>
__global__ void __launch_bounds__(1 << (LLEN - 4))
k_fft_row(const C2<R>* __restrict__ in, C2<R>* __restrict__ out, const C2<R>* __restrict__ twM,
          int in_row, int lblk, int blk_stride, const C2<R>* __restrict__ dc) {
    using C = C2<R>;
    constexpr int M = 1 << LLEN, NT = M >> 4;
    constexpr int L0 = (LLEN & 3) ? (LLEN & 3) : 4, R0 = 1 << L0, NB0 = 16 / R0;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    C* x = reinterpret_cast<C*>(smem_raw);                        // [row_pad(M)]
    C* tw = x + row_pad(M);                                       // [M/16]  w_M^u
    const int tid = threadIdx.x;
    for (int u = tid; u < NT; u += NT) cp_async_elem(tw + u, twM + u);
    cp_async_commit();

    // ---- stage 0: radix R0, Ns = 1, from global (no twiddles)
    const C* xin = in + (size_t)blockIdx.x * in_row;
    const int bmask = (1 << lblk) - 1;
    C v[16];
#pragma unroll
    for (int b = 0; b < NB0; ++b) {
        const int j = tid + b * NT;
#pragma unroll
        for (int t = 0; t < R0; ++t) {
            const int m = j + t * (M / R0);
            v[b * R0 + t] = ldg_c(xin + (size_t)(m >> lblk) * blk_stride + (m & bmask));
        }
    }
#pragma unroll
    for (int b = 0; b < NB0; ++b) dftR<R0>(v + b * R0);
#pragma unroll
    for (int b = 0; b < NB0; ++b) {
        const int j = tid + b * NT;
#pragma unroll
        for (int t = 0; t < R0; ++t) x[row_pad(j * R0 + t)] = v[b * R0 + t];
    }
    cp_async_wait_all();
    __syncthreads();

    // ---- radix-16 stages, Ns = R0, 16 R0, ...; the last one (Ns = M/16) stores to global
    auto stage = [&](auto lnsc) {
        constexpr int LNS = decltype(lnsc)::value, NS = 1 << LNS;
        const int j = tid, k = j & (NS - 1);
#pragma unroll
        for (int t = 0; t < 16; ++t) v[t] = x[row_pad(j + t * NT)];
        twiddle_powers<16>(v, tw[k << (LLEN - 4 - LNS)]);
        dft16(v);
        if constexpr (LNS + 4 < LLEN) {
            __syncthreads();
#pragma unroll
            for (int t = 0; t < 16; ++t) x[row_pad(((j - k) << 4) + k + t * NS)] = v[t];
            __syncthreads();
        } else {
            C* y = out + ((size_t)blockIdx.x << LLEN);
#pragma unroll
            for (int t = 0; t < 16; ++t) y[j + t * NT] = v[t];
        }
    };
    stage(std::integral_constant<int, L0>{});
    if constexpr (L0 + 4 < LLEN) stage(std::integral_constant<int, L0 + 4>{});
    if constexpr (L0 + 8 < LLEN) stage(std::integral_constant<int, L0 + 8>{});
    static_assert(L0 + 12 >= LLEN, "k_fft_row: LLEN <= L0 + 12");
    if (dc != nullptr) {                                         // the row's k = 0 output (R19)
        __syncthreads();
        if (threadIdx.x == 0) out[(size_t)blockIdx.x << LLEN] = dc[blockIdx.x];
    }
}

// radix-E DFT in registers, E in {2, 4, 8, 16}
template <int E, typename C> __device__ __forceinline__ void dft_small(C* v) {
    if constexpr (E == 2) dft2(v);
    else if constexpr (E == 4) dft4(v);
    else if constexpr (E == 8) dft8(v);
    else dft16(v);
}

// ---------------------------------------------------------------------------------------------
// Large M (rows that do not fit one CTA's shared memory): the M-point FFT (§3 step 4) as a
// four-step split over 2 or 3 passes, each pass reading and writing HBM once with >= 64-byte runs.
// For M = M1 M2 (M3): n = n1 M2 M3 + n2 M3 + n3, k = k1 + M1 k2 + M1 M2 k3,
//   X[k] = sum_{n3} w_{M3}^{n3 k3} w_{M2 M3}^{n3 k2} sum_{n2} w_{M2}^{n2 k2} w_M^{n2' k1} sum_{n1} w_{M1}^{n1 k1} x[n],
// with n2' = n2 M3 + n3 the inner index of the first pass. A column pass (k_fft_col) takes
// sequences of length Ms = Mc Mi, FFTs the Mc-point columns (stride Mi) of CB adjacent inner
// indices at once and multiplies by w_{Ms}^{n_inner k_col}; the row pass (k_fft_rowt) FFTs CR
// contiguous rows of length Mr and stores them transposed, X[k_prefix + (M / Mr) k_last], CR
// consecutive prefixes at a time. Both use k_fft_row's scheme (radix R0 then radix-16 stages,
// 16 elements per thread, one pad element per 16) on CB (CR) columns side by side; the column
// stride CS = 16/CB (mod 16) makes the column-parallel accesses conflict-free.
// ---------------------------------------------------------------------------------------------
template <int LEN, int NCOL> __host__ __device__ constexpr int col_stride() {
    return ((row_pad(LEN) + 15) / 16) * 16 + 16 / NCOL;
}
template <typename R, int LC, int CB> __host__ __device__ constexpr size_t fft_col_smem() {
    return ((size_t)CB * col_stride<1 << LC, CB>() + ((1 << LC) >> 4)) * sizeof(C2<R>);
}

// radix-16 stage LNS (Ns = 2^LNS) of a 2^LL-point Stockham FFT on column xc, thread j of NT;
// the caller handles the last stage (LNS + 4 == LL)
template <int LL, int LNS, typename C>
__device__ __forceinline__ void row_stage_mid(C* xc, const C* tw, int j, C* v) {
    constexpr int NT = (1 << LL) >> 4, NS = 1 << LNS;
    const int k = j & (NS - 1);
#pragma unroll
    for (int t = 0; t < 16; ++t) v[t] = xc[row_pad(j + t * NT)];
    twiddle_powers<16>(v, tw[k << (LL - 4 - LNS)]);
    dft16(v);
    __syncthreads();
#pragma unroll
    for (int t = 0; t < 16; ++t) xc[row_pad(((j - k) << 4) + k + t * NS)] = v[t];
    __syncthreads();
}

template <typename R, int LC, int CB>
__global__ void __launch_bounds__(CB << (LC - 4))
k_fft_col(const C2<R>* __restrict__ in, C2<R>* __restrict__ out, int lMs, int lMi, int lSdiv, long long M,
          long long in_row, int lblk, long long blk_stride) {
    pdl_trigger();
    using C = C2<R>;
    constexpr int Mc = 1 << LC, NT = Mc >> 4, CS = col_stride<Mc, CB>();
    constexpr int L0 = (LC & 3) ? (LC & 3) : 4, R0 = 1 << L0, NB0 = 16 / R0;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    C* x = reinterpret_cast<C*>(smem_raw);                        // [CB][CS]
    C* tw = x + CB * CS;                                          // [Mc/16]  w_Mc^u
    const int tid = threadIdx.x, c = tid % CB, j = tid / CB;
    for (int u = tid; u < NT; u += blockDim.x) tw[u] = twiddle_pow2(R(0), u, LC);
    const long long s = blockIdx.y;
    const long long n2 = (long long)blockIdx.x * CB + c;          // inner index of this column
    const long long Mi = 1LL << lMi;
    const long long bmask = (1LL << lblk) - 1;
    const C* xin = in + s * in_row;
    C* xc = x + c * CS;
    pdl_wait();
    C v[16];
#pragma unroll
    for (int b = 0; b < NB0; ++b) {
        const int jj = j + b * NT;
#pragma unroll
        for (int t = 0; t < R0; ++t) {
            const long long m = (long long)(jj + t * (Mc / R0)) * Mi + n2;
            v[b * R0 + t] = ldg_c(xin + (m >> lblk) * blk_stride + (m & bmask));
        }
    }
#pragma unroll
    for (int b = 0; b < NB0; ++b) dftR<R0>(v + b * R0);
#pragma unroll
    for (int b = 0; b < NB0; ++b) {
        const int jj = j + b * NT;
#pragma unroll
        for (int t = 0; t < R0; ++t) xc[row_pad(jj * R0 + t)] = v[b * R0 + t];
    }
    __syncthreads();
    if constexpr (L0 + 4 < LC) row_stage_mid<LC, L0>(xc, tw, j, v);
    if constexpr (L0 + 8 < LC) row_stage_mid<LC, L0 + 4>(xc, tw, j, v);
    static_assert(L0 + 12 >= LC, "k_fft_col: LC <= L0 + 12");
    // last stage (Ns = Mc/16, k = j): natural order k_col = j + t NT, times w_Ms^{n2 k_col}
    constexpr int LNS = LC - 4;
#pragma unroll
    for (int t = 0; t < 16; ++t) v[t] = xc[row_pad(j + t * NT)];
    if constexpr (LNS > 0) twiddle_powers<16>(v, tw[j]);
    dft16(v);
    const long long Ms_mask = (1LL << lMs) - 1;
    const C wb = twiddle_pow2(R(0), (int)((n2 * j) & Ms_mask), lMs);
    twiddle_powers<16>(v, twiddle_pow2(R(0), (int)((n2 * NT) & Ms_mask), lMs));
    const long long hi = s >> lSdiv, lo = s & ((1LL << lSdiv) - 1);
    const long long kstride = Mi << lSdiv;
    C* y = out + hi * M + lo * Mi + n2;
#pragma unroll
    for (int t = 0; t < 16; ++t) y[(long long)(j + t * NT) * kstride] = cmul(v[t], wb);
}

template <typename R, int LL, int CR> __host__ __device__ constexpr size_t fft_rowt_smem() {
    return ((size_t)CR * col_stride<1 << LL, CR>() + ((1 << LL) >> 4)) * sizeof(C2<R>);
}

template <typename R, int LL, int CR>
__global__ void __launch_bounds__(CR << (LL - 4))
k_fft_rowt(const C2<R>* __restrict__ in, C2<R>* __restrict__ out, long long M, int lrpr, const C2<R>* __restrict__ dc) {
    pdl_trigger();
    using C = C2<R>;
    constexpr int Mr = 1 << LL, NT = Mr >> 4, CS = col_stride<Mr, CR>();
    constexpr int L0 = (LL & 3) ? (LL & 3) : 4, R0 = 1 << L0, NB0 = 16 / R0;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    C* x = reinterpret_cast<C*>(smem_raw);                        // [CR][CS]
    C* tw = x + CR * CS;                                          // [Mr/16]  w_Mr^u
    const int tid = threadIdx.x;
    for (int u = tid; u < NT; u += blockDim.x) tw[u] = twiddle_pow2(R(0), u, LL);
    const long long r0 = (long long)blockIdx.x * CR;              // first row (global)
    // stages 0 .. last-1: j fastest (row r = tid / NT), coalesced row loads
    const int jr = tid % NT, rr = tid / NT;
    C* xr = x + rr * CS;
    pdl_wait();
    C v[16];
    const C* xin = in + ((r0 + rr) << LL);
#pragma unroll
    for (int b = 0; b < NB0; ++b) {
        const int jj = jr + b * NT;
#pragma unroll
        for (int t = 0; t < R0; ++t) v[b * R0 + t] = ldg_c(xin + jj + t * (Mr / R0));
    }
#pragma unroll
    for (int b = 0; b < NB0; ++b) dftR<R0>(v + b * R0);
#pragma unroll
    for (int b = 0; b < NB0; ++b) {
        const int jj = jr + b * NT;
#pragma unroll
        for (int t = 0; t < R0; ++t) xr[row_pad(jj * R0 + t)] = v[b * R0 + t];
    }
    __syncthreads();
    if constexpr (L0 + 4 < LL) row_stage_mid<LL, L0>(xr, tw, jr, v);
    if constexpr (L0 + 8 < LL) row_stage_mid<LL, L0 + 4>(xr, tw, jr, v);
    static_assert(L0 + 12 >= LL, "k_fft_rowt: LL <= L0 + 12");
    // last stage: row fastest (r = tid % CR), stores of CR consecutive outputs per k
    constexpr int LNS = LL - 4;
    const int r = tid % CR, j = tid / CR;
    const C* xc = x + r * CS;
#pragma unroll
    for (int t = 0; t < 16; ++t) v[t] = xc[row_pad(j + t * NT)];
    if constexpr (LNS > 0) twiddle_powers<16>(v, tw[j]);
    dft16(v);
    const long long rg = r0 + r;
    const long long row = rg >> lrpr, pre = rg & ((1LL << lrpr) - 1);
    C* y = out + row * M + pre;
#pragma unroll
    for (int t = 0; t < 16; ++t) y[(long long)(j + t * NT) << lrpr] = v[t];
    if (dc != nullptr && (r0 & ((1LL << lrpr) - 1)) == 0) {     // this CTA holds the row's k = 0 output (R19)
        __syncthreads();
        if (tid == 0) out[(r0 >> lrpr) * M] = dc[r0 >> lrpr];
    }
}


// ---------------------------------------------------------------------------------------------
// The distributed radix-P Cooley-Tukey FFT (the six steps of P:283-310; the
// comparator that isolates the transposes the FMM-FFT saves): F_N = Pi_{M,P} (I_M x F_P) Pi_{P,M}
// T_{P,M} (I_P x F_M) Pi_{M,P}, N = M P, x block-distributed in natural order (rank g holds
// x[p + P m] for m in its block of M/G and every p).
//
// k_transpose_rc: step 1's local half, out[c][r] = in[r][c] for a rows x cols matrix (rank g's
// [m_local][p] block -> [p][m_local], so the all-to-all chunk of rank r is the contiguous rows
// p in r's block). 32 x 32 tiles through padded shared memory, coalesced both ways.
// ---------------------------------------------------------------------------------------------
template <typename R>
__global__ void __launch_bounds__(256)
k_transpose_rc(const C2<R>* __restrict__ in, C2<R>* __restrict__ out, long long rows, long long cols) {
    pdl_trigger();
    __shared__ C2<R> t[32][33];
    const long long r0 = (long long)blockIdx.y * 32, c0 = (long long)blockIdx.x * 32;
    pdl_wait();
    for (int k = threadIdx.y; k < 32; k += 8) {
        const long long r = r0 + k, c = c0 + threadIdx.x;
        if (r < rows && c < cols) t[k][threadIdx.x] = in[r * cols + c];
    }
    __syncthreads();
    for (int k = threadIdx.y; k < 32; k += 8) {
        const long long c = c0 + k, r = r0 + threadIdx.x;
        if (r < rows && c < cols) out[c * rows + r] = t[threadIdx.x][k];
    }
}

// ---------------------------------------------------------------------------------------------
// k_twiddle_chunk: steps 3 + 4's local half. Rank g holds X[p_local][k1] (rows p = g P/G +
// p_local, the M-point FFTs of step 2); multiplies by the twiddle T = w_N^{p k1} and writes the
// all-to-all send layout [r][p_local][k1_local] (k1 = r M/G + k1_local). The angle is reduced
// exactly in integers and evaluated in float64.
// ---------------------------------------------------------------------------------------------
template <typename R>
__global__ void __launch_bounds__(256)
k_twiddle_chunk(const C2<R>* __restrict__ X, C2<R>* __restrict__ W, long long M, int lMg, int lrows, long long p0, long long N) {
    pdl_trigger();
    pdl_wait();
    const long long total = M << lrows, Mg = 1LL << lMg;
    const long long stride = (long long)gridDim.x * blockDim.x;
    for (long long o = (long long)blockIdx.x * blockDim.x + threadIdx.x; o < total; o += stride) {
        const long long kl = o & (Mg - 1), pl = (o >> lMg) & ((1LL << lrows) - 1), r = o >> (lMg + lrows);
        const long long k1 = r * Mg + kl;
        const C2<R> v = X[pl * M + k1];
        const double2 w = twiddle_d(((p0 + pl) * k1) & (N - 1), N);
        W[o] = C2<R>{(R)(w.x * (double)v.x - w.y * (double)v.y), (R)(w.x * (double)v.y + w.y * (double)v.x)};
    }
}

// ---------------------------------------------------------------------------------------------
// Inverse transform (§8(f) NEXT-1): F_N^{-1} x = conj(F_N conj(x)) / N (F_N^{-1} = F_N^H / N),
// so the inverse plan conjugates its input into a workspace copy, runs the forward path and
// conjugates and scales the output in place: out[i] = scale * conj(in[i]). Two complex values
// per thread-iteration as one 16- (c64) or two 16-byte (c128) accesses.
// ---------------------------------------------------------------------------------------------
template <typename R>
__global__ void __launch_bounds__(256)
k_conj_scale(const C2<R>* in, C2<R>* out, long long n, R scale) {   // in == out allowed (no restrict / ldg)
    pdl_trigger();
    pdl_wait();
    const long long stride = (long long)gridDim.x * blockDim.x;
    for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; 2 * i < n; i += stride) {
        if constexpr (sizeof(R) == 4) {
            const float4 v = reinterpret_cast<const float4*>(in)[i];
            reinterpret_cast<float4*>(out)[i] = make_float4(scale * v.x, -scale * v.y, scale * v.z, -scale * v.w);
        } else {
            const double2 a = in[2 * i], b = in[2 * i + 1];
            out[2 * i] = make_double2(scale * a.x, -scale * a.y);
            out[2 * i + 1] = make_double2(scale * b.x, -scale * b.y);
        }
    }
}

// ---------------------------------------------------------------------------------------------
// k_dc_bins: the k1 = 0 output of every local M-FFT row, y[M k2] = sum_p w_P^{p k2} r_p — eq. (1)
// at k = M k2: sum_j x_j w_N^{j M k2} = sum_p w_P^{p k2} sum_m x_{p + P m} (reading R19). Through
// the FMM these P bins are the sums of the far field over all M targets, a sum with heavy
// cancellation (its terms ~ M / (pi d) against a net ~ M), so in float32 they carry ~1e-5 relative
// error at M = 2^22 (growing like sqrt M) while every other bin is at ~1e-6; the reductions r_p of
// Algorithm 1 line 11 hold the same quantities accurately. r_0 (p = 0 is no FMM) is
// the sum of M^L's slot 0 (S2M columns sum to 1): read from r[0] when the level kernels reduced it,
// else reduced here from M^L slot 0 (m0: m0_n values at stride m0_stride). Sums in float64. Writes
// dc[row] for this rank's rows; the last M-FFT pass (k_fft_rowt / k_fft_row / k_fft_pass) stores
// dc[row] as the row's k1 = 0 output, so this kernel runs off the critical path (side stream).
// ---------------------------------------------------------------------------------------------
template <typename R>
__global__ void __launch_bounds__(256)
k_dc_bins(C2<R>* __restrict__ y, const C2<R>* __restrict__ r, const C2<R>* __restrict__ m0, long long m0_n,
          long long m0_stride, int P, int rows, int row0, long long M, const double2* __restrict__ r0part, int nr0part) {
    pdl_trigger();
    __shared__ double2 red[8];
    __shared__ double2 rr[1024];                                  // r_p (r_0 replaced), then summed
    __shared__ double2 tw[1024];                                  // w_P^j, j < P
    const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
    for (int j = tid; j < P; j += blockDim.x) tw[j] = twiddle_d(j, P);
    pdl_wait();
    for (int j = tid; j < P; j += blockDim.x) rr[j] = make_double2((double)r[j].x, (double)r[j].y);
    if (nr0part > 0) {                                            // r_0 from the tree kernel's partial sums
        __syncthreads();
        if (tid == 0) {
            double2 t = make_double2(0.0, 0.0);
            for (int k = 0; k < nr0part; ++k) { t.x += r0part[k].x; t.y += r0part[k].y; }   // fixed order
            rr[0] = t;
        }
    }
    if (m0 != nullptr) {                                          // r_0 = sum of M^L slot 0
        double2 a = make_double2(0.0, 0.0);
        for (long long i0 = tid; i0 < m0_n; i0 += 8LL * blockDim.x) {   // 8 independent loads in flight
            C2<R> v[8];
#pragma unroll
            for (int u = 0; u < 8; ++u) {
                const long long i = i0 + (long long)u * blockDim.x;
                v[u] = i < m0_n ? m0[i * m0_stride] : C2<R>{R(0), R(0)};
            }
#pragma unroll
            for (int u = 0; u < 8; ++u) { a.x += (double)v[u].x; a.y += (double)v[u].y; }
        }
        for (int o = 16; o > 0; o >>= 1) {                        // fixed-order reduction: deterministic
            a.x += __shfl_xor_sync(0xffffffffu, a.x, o);
            a.y += __shfl_xor_sync(0xffffffffu, a.y, o);
        }
        if (lane == 0) red[wid] = a;
        __syncthreads();
        if (tid == 0) {
            double2 t = red[0];
            for (int w = 1; w < (int)(blockDim.x >> 5); ++w) { t.x += red[w].x; t.y += red[w].y; }
            rr[0] = t;
        }
    }
    __syncthreads();
    // one warp per output row: lanes over p, shuffle reduction
    const int row = blockIdx.x * (blockDim.x >> 5) + wid;
    if (row >= rows) return;
    const int k2 = row0 + row;
    double2 acc = make_double2(0.0, 0.0);
    for (int pp = lane; pp < P; pp += 32) {
        const double2 w = tw[(pp * k2) & (P - 1)], v = rr[pp];
        acc.x += w.x * v.x - w.y * v.y;
        acc.y += w.x * v.y + w.y * v.x;
    }
    for (int o = 16; o > 0; o >>= 1) {
        acc.x += __shfl_xor_sync(0xffffffffu, acc.x, o);
        acc.y += __shfl_xor_sync(0xffffffffu, acc.y, o);
    }
    if (lane == 0) y[row] = C2<R>{(R)acc.x, (R)acc.y};
}

// ---------------------------------------------------------------------------------------------
// k_r2c_post (FMMFFT_FLAG_REAL): real x of length N = 2H read as the complex
// vector z_j = x_{2j} + i x_{2j+1}; Z = F_H z comes from the complex plan. With a = Z_k,
// b = conj(Z_{H-k}) (Z_H = Z_0): E = (a + b)/2 (the DFT of the even samples), O = -i (a - b)/2
// (of the odd ones), and eq. (1) split by parity gives X_k = E + w_N^k O and
// X_{H-k} = conj(E - w_N^k O). Thread k <= H/2 reads Z_k and Z_{H-k} and writes both outputs,
// so every element is read and written once (coalesced, the second stream descending).
// ---------------------------------------------------------------------------------------------
template <typename R>
__global__ void __launch_bounds__(256)
k_r2c_post(const C2<R>* __restrict__ Z, C2<R>* __restrict__ X, long long H) {
    pdl_trigger();
    pdl_wait();
    const long long stride = (long long)gridDim.x * blockDim.x;
    for (long long k = (long long)blockIdx.x * blockDim.x + threadIdx.x; k <= H / 2; k += stride) {
        const C2<R> a = Z[k];
        const C2<R> zb = Z[k == 0 ? 0 : H - k];
        const R Er = R(0.5) * (a.x + zb.x), Ei = R(0.5) * (a.y - zb.y);   // (a + conj(zb)) / 2
        const R Or = R(0.5) * (a.y + zb.y), Oi = R(-0.5) * (a.x - zb.x);  // -i (a - conj(zb)) / 2
        R wr, wi;                                                        // w_N^k = exp(-2 pi i k / 2H)
        if constexpr (sizeof(R) == 4) {
            float sn, cs;
            sincospif(-(float)((double)k / (double)H), &sn, &cs);
            wr = cs; wi = sn;
        } else {
            double sn, cs;
            sincospi(-(double)k / (double)H, &sn, &cs);
            wr = cs; wi = sn;
        }
        const R tr = wr * Or - wi * Oi, ti = wr * Oi + wi * Or;            // w O
        X[k] = C2<R>{Er + tr, Ei + ti};
        X[H - k] = C2<R>{Er - tr, -(Ei - ti)};
    }
}

// k_r2c_post_dist: the same separation at G > 1 for rank g's block k = k0 + j, j < nl, with
// Z_{H-k} from the mirror exchange (Zm = rank G-1-g's block, Z_{H-k} = Zm[nl - j] for j > 0,
// zx = Z_{H-k0}); the last rank also writes X_H = Re Z_0 - Im Z_0 (Zm[0] = Z_0) at X[nl].
template <typename R>
__global__ void __launch_bounds__(256)
k_r2c_post_dist(const C2<R>* __restrict__ Z, const C2<R>* __restrict__ Zm, const C2<R>* __restrict__ zx,
                C2<R>* __restrict__ X, long long H, long long nl, long long k0, int last) {
    pdl_trigger();
    pdl_wait();
    const long long stride = (long long)gridDim.x * blockDim.x;
    for (long long j = (long long)blockIdx.x * blockDim.x + threadIdx.x; j < nl; j += stride) {
        const long long k = k0 + j;
        const C2<R> a = Z[j];
        const C2<R> zb = j == 0 ? zx[0] : Zm[nl - j];
        const R Er = R(0.5) * (a.x + zb.x), Ei = R(0.5) * (a.y - zb.y);
        const R Or = R(0.5) * (a.y + zb.y), Oi = R(-0.5) * (a.x - zb.x);
        R wr, wi;                                                        // w_N^k = exp(-2 pi i k / 2H)
        if constexpr (sizeof(R) == 4) {
            float sn, cs;
            sincospif(-(float)((double)k / (double)H), &sn, &cs);
            wr = cs; wi = sn;
        } else {
            double sn, cs;
            sincospi(-(double)k / (double)H, &sn, &cs);
            wr = cs; wi = sn;
        }
        X[j] = C2<R>{Er + wr * Or - wi * Oi, Ei + wr * Oi + wi * Or};
        if (last && j == 0) {
            const C2<R> z0 = Zm[0];
            X[nl] = C2<R>{z0.x - z0.y, R(0)};
        }
    }
}

// ---------------------------------------------------------------------------------------------
// k_c2r_pre (FMMFFT_FLAG_REAL | FMMFFT_FLAG_INVERSE): from X_k, k = 0..H, of a real signal of
// length N = 2H (X_{N-k} = conj(X_k)), with a = X_k, b = conj(X_{H-k}):
// E_k = (a + b)/2 and O_k = w_N^{-k} (a - b)/2 are the H-point spectra (scaled by 1/2) of the even
// and odd samples, so z = F_H^{-1} Z with Z_k = E_k + i O_k is z_j = x_{2j} + i x_{2j+1}, i.e. the
// N real outputs in place. Z_{H-k} = conj(E_k) + i conj(O_k). Writes conj(Z) (the inverse plan's
// input conjugation, fused): thread k <= H/2 writes k and H - k (k = 0: only Z_0).
// ---------------------------------------------------------------------------------------------
template <typename R>
__global__ void __launch_bounds__(256)
k_c2r_pre(const C2<R>* __restrict__ X, C2<R>* __restrict__ Zc, long long H) {
    pdl_trigger();
    pdl_wait();
    const long long stride = (long long)gridDim.x * blockDim.x;
    for (long long k = (long long)blockIdx.x * blockDim.x + threadIdx.x; k <= H / 2; k += stride) {
        C2<R> a = X[k];
        C2<R> xb = X[H - k];
        if (k == 0) a.y = xb.y = R(0);     // X_0, X_H of a real signal are real: Im ignored (fmmfft.h)
        const R Er = R(0.5) * (a.x + xb.x), Ei = R(0.5) * (a.y - xb.y);   // (a + conj(xb)) / 2
        const R Dr = R(0.5) * (a.x - xb.x), Di = R(0.5) * (a.y + xb.y);   // (a - conj(xb)) / 2
        R wr, wi;                                                        // w_N^{-k} = exp(+2 pi i k / 2H)
        if constexpr (sizeof(R) == 4) {
            float sn, cs;
            sincospif((float)((double)k / (double)H), &sn, &cs);
            wr = cs; wi = sn;
        } else {
            double sn, cs;
            sincospi((double)k / (double)H, &sn, &cs);
            wr = cs; wi = sn;
        }
        const R Or = wr * Dr - wi * Di, Oi = wr * Di + wi * Dr;            // O = w^{-k} D
        // Z_k = E + i O = (Er - Oi) + i (Ei + Or); stored conjugated
        Zc[k] = C2<R>{Er - Oi, -(Ei + Or)};
        // Z_{H-k} = conj(E) + i conj(O) = (Er + Oi) + i (Or - Ei); stored conjugated
        if (k != 0) Zc[H - k] = C2<R>{Er + Oi, Ei - Or};
    }
}

// k_c2r_pre_dist: the same at G > 1 for rank g's block k = k0 + j, j < nl, with X_{H-k} from the
// mirror exchange (Xm = rank G-1-g's block, X_{H-k} = Xm[nl - j] for j > 0, xx = X_{H-k0}, which
// is X_H for rank 0); writes conj(Z_k) for the rank's own k only.
template <typename R>
__global__ void __launch_bounds__(256)
k_c2r_pre_dist(const C2<R>* __restrict__ X, const C2<R>* __restrict__ Xm, const C2<R>* __restrict__ xx,
               C2<R>* __restrict__ Zc, long long H, long long nl, long long k0) {
    pdl_trigger();
    pdl_wait();
    const long long stride = (long long)gridDim.x * blockDim.x;
    for (long long j = (long long)blockIdx.x * blockDim.x + threadIdx.x; j < nl; j += stride) {
        const long long k = k0 + j;
        C2<R> a = X[j];
        C2<R> xb = j == 0 ? xx[0] : Xm[nl - j];
        if (k == 0) a.y = xb.y = R(0);     // X_0, X_H of a real signal are real: Im ignored (fmmfft.h)
        const R Er = R(0.5) * (a.x + xb.x), Ei = R(0.5) * (a.y - xb.y);
        const R Dr = R(0.5) * (a.x - xb.x), Di = R(0.5) * (a.y + xb.y);
        R wr, wi;                                                        // w_N^{-k}
        if constexpr (sizeof(R) == 4) {
            float sn, cs;
            sincospif((float)((double)k / (double)H), &sn, &cs);
            wr = cs; wi = sn;
        } else {
            double sn, cs;
            sincospi((double)k / (double)H, &sn, &cs);
            wr = cs; wi = sn;
        }
        const R Or = wr * Dr - wi * Di, Oi = wr * Di + wi * Dr;
        Zc[j] = C2<R>{Er - Oi, -(Ei + Or)};
    }
}

// ---------------------------------------------------------------------------------------------
// k_post_pfft_r: the same L2T + POST + P-point FFT + transposed store for P <= 32 with the whole
// P-point column of one m in one thread's registers (no shared-memory FFT tile, no barriers in
// the FFT): thread (box b, m) loads T_near[p][b][.][m] for all p (coalesced over m), adds
// L2T_{mq} L^L_{pqb} (L^L of its box broadcast from shared memory, two p per 16-byte load),
// applies POST, runs the P-point DFT in registers (radix 2/4/8/16, 32 = 2 x 16) and stores
// W[k2][b M_L + m] for every k2 (coalesced over m). CTA = NBX consecutive boxes x M_L threads.
// ---------------------------------------------------------------------------------------------
#ifndef FMMFFT_PPR_MINB
#define FMMFFT_PPR_MINB 4            // k_post_pfft_r CTAs per SM the register budget is sized for (3: 252 -> 4: 240 us at cfg3)
#endif
template <typename R, int LP, int QT>
__global__ void __launch_bounds__(256, FMMFFT_PPR_MINB)
k_post_pfft_r(const C2<R>* __restrict__ Tn, const C2<R>* __restrict__ LL, const C2<R>* __restrict__ r,
              const C2<R>* __restrict__ rho, const R* __restrict__ s2m, C2<R>* __restrict__ W, int lML, int Mg, int pmaj) {
    pdl_trigger();
    using C = C2<R>;
    constexpr int P = 1 << LP, Q = QT;
    const int M_L = 1 << lML;
    const int nbx = blockDim.x >> lML;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    C* Lsm = reinterpret_cast<C*>(smem_raw);                      // [nbx][Q][P]
    C* rr = Lsm + nbx * Q * P;                                     // [P] r_p
    C* rh = rr + P;                                                // [P] rho_p
    C* tw32 = rh + P;                                              // [16] w_32^k
    R* wsm = reinterpret_cast<R*>(tw32 + 16);                      // [Q][M_L] L2T_{mq} = S2M_{qm}
    const int tid = threadIdx.x, bx = tid >> lML, m = tid & (M_L - 1);
    const int b = blockIdx.x * nbx + bx;
    for (int idx = tid; idx < Q * M_L; idx += blockDim.x) cp_async_elem(wsm + idx, s2m + idx);
    if (tid < 16) tw32[tid] = twiddle_pow2(R(0), tid, 5);
    pdl_wait();                                                   // T_near / L^L / r from the FMM stages
    {
        constexpr int V = 16 / sizeof(C);
        if (pmaj) {                                               // [p][b][q] -> Lsm[bx][p][q]
            const int nbt = Mg >> lML;
            for (int idx = tid; idx < nbx * P * Q / V; idx += blockDim.x) {
                const int e = idx * V, row = e / Q, q = e - row * Q;  // row = bx P + p
                const int bxx = row / P, pp = row - bxx * P;
                cp_async<16>(Lsm + e, LL + ((size_t)pp * nbt + (size_t)blockIdx.x * nbx + bxx) * Q + q);
            }
        } else {
            const C* src = LL + (size_t)blockIdx.x * nbx * Q * P;
            for (int idx = tid; idx < nbx * Q * P / V; idx += blockDim.x) cp_async<16>(Lsm + idx * V, src + idx * V);
        }
        if (tid < P) { rr[tid] = ldg_c(r + tid); rh[tid] = ldg_c(rho + tid); }
    }
    C v[P];
    const R* tn = reinterpret_cast<const R*>(Tn) + ((size_t)b << (lML + 1)) + m;
#pragma unroll
    for (int p = 0; p < P; ++p) {
        v[p].x = __ldg(tn + (size_t)p * 2 * Mg);
        v[p].y = __ldg(tn + (size_t)p * 2 * Mg + M_L);
    }
    cp_async_wait_all();
    __syncthreads();
    // L2T accumulated straight into the column (q outer: one L2T coefficient register, the L^L
    // row of q a broadcast), then POST; p = 0 is the identity (C_0 = I, R1)
    const C* Lb = Lsm + bx * Q * P;
#pragma unroll 4
    for (int q = 0; q < Q; ++q) {
        const R wq = wsm[q * M_L + m];
#pragma unroll
        for (int p = 1; p < P; ++p) rfma(v[p], wq, pmaj ? Lb[p * Q + q] : Lb[q * P + p]);
    }
#pragma unroll
    for (int p = 1; p < P; ++p) {
        C t = v[p];
        t.x -= rr[p].y; t.y += rr[p].x;                            // + i r_p
        v[p] = cmul(rh[p], t);
    }
    // P-point DFT over p, natural order
    if constexpr (P <= 16) {
        dft_small<P>(v);
    } else {                                                      // 32 = 2 x 16: X[k] = E[k] + w^k O[k]
        C e[16], o[16];
#pragma unroll
        for (int t = 0; t < 16; ++t) { e[t] = v[2 * t]; o[t] = v[2 * t + 1]; }
        dft16(e); dft16(o);
#pragma unroll
        for (int k = 0; k < 16; ++k) {
            const C ow = cmul(o[k], tw32[k]);
            v[k] = cadd(e[k], ow);
            v[k + 16] = csub(e[k], ow);
        }
    }
    C* dst = W + ((size_t)b << lML) + m;
#pragma unroll
    for (int k2 = 0; k2 < P; ++k2) dst[(size_t)k2 * Mg] = v[k2];
}

}  // namespace fmmfft
