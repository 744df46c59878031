// kernel_s2t_tc.cuh — S2T (Alg. 1 line 3, §4.6) on the 5th-generation tensor
// cores, complex64, M_L = 64.
//
// For one FMM p and a tile of 64 consecutive leaf boxes b0..b0+63 the near field is the GEMM
//     D[n][i] = sum_{k < 192} A[n][k] * Toep_p[i][k],     Toep_p[i][k] = S2T_{p, (k - 64) - i}
// with rows n = 2 (b - b0) + c (box, re/im) — UMMA M = 128 — columns i < 64 (N = 64) and
// k = the position in the window [box b-1, b, b+1] (K = 192, the paper's -M_L <= j < 2 M_L).
// A[n][k] = S_{p, k mod 64, b - 1 + k div 64}.c is built in shared memory from the window of the
// p-major copy S'[p][b][m] that k_s2m writes (one contiguous bulk copy per CTA); Toep_p is
// precomputed per plan (fp64 -> tf32 hi/lo) in the UMMA K-major core-matrix layout and streamed
// with cp.async.bulk. Precision: 3xTF32, D = Ahi Bhi + Ahi Blo + Alo Bhi
// accumulated in fp32 in tensor memory (plain TF32 misses the 1e-5 bound).
// K is processed in 12 chunks of 16, double-buffered; one thread issues the 6 MMAs of a chunk
// (tcgen05.mma kind::tf32, M=128 N=64 K=8) and commits them to an mbarrier.
// p = 0 (the identity, R1) is a plain copy by its own CTAs.
#pragma once
#include "common.cuh"
#include "tcgen05.cuh"

namespace fmmfft {

constexpr int S2TC_BOXES = 64;                 // boxes per tile (UMMA M = 2 * 64)
constexpr int S2TC_CHUNK_K = 16;               // K per pipeline chunk
constexpr int S2TC_NCHUNK = 192 / S2TC_CHUNK_K;
constexpr int S2TC_LBO_A = 2064;               // bytes between K-halves of A (2048 + 16: bank skew)
constexpr int S2TC_A_BYTES = (S2TC_CHUNK_K / 4) * S2TC_LBO_A;   // one of hi / lo
constexpr int S2TC_B_BYTES = 64 * S2TC_CHUNK_K * 4;   // one of hi / lo, LBO 1024, SBO 128
constexpr int S2TC_TAB_FLOATS_PER_P = S2TC_NCHUNK * 2 * 64 * S2TC_CHUNK_K;   // [chunk][hi,lo][k4][r8][8][4]

constexpr int S2TC_SCOL_BYTES = ((S2TC_BOXES + 2) * 64 * 8 + 1023) / 1024 * 1024;   // staged S column
__host__ __device__ constexpr size_t s2tc_smem_bytes() {
    return (size_t)S2TC_SCOL_BYTES                       // staged S column (66 boxes x 64 m, float2)
           + 2 * (2 * S2TC_A_BYTES)                      // A hi/lo, double-buffered
           + 2 * (2 * S2TC_B_BYTES)                      // B hi/lo, double-buffered
           + 64;                                         // mbarriers + TMEM address
}

__global__ void __launch_bounds__(256, 2)
k_s2t_tc(const float2* __restrict__ Sp, const float2* __restrict__ S, const float2* __restrict__ haloL,
         const float2* __restrict__ haloR, float2* __restrict__ Tn, const float* __restrict__ toep, int P, int nb, int G) {
    pdl_trigger();
    pdl_wait();
    extern __shared__ __align__(1024) unsigned char smem_tc[];
    float2* Scol = reinterpret_cast<float2*>(smem_tc);                           // [66][64]
    unsigned char* Abase = smem_tc + S2TC_SCOL_BYTES;                            // 2 x (hi, lo)
    unsigned char* Bbase = Abase + 2 * 2 * S2TC_A_BYTES;                          // 2 x (hi, lo)
    uint64_t* bar = reinterpret_cast<uint64_t*>(Bbase + 2 * 2 * S2TC_B_BYTES);    // [0,1] B load, [2,3] mma, [4] S
    uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bar + 5);
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int b0 = blockIdx.x * S2TC_BOXES;
    const int p = blockIdx.y;
    const size_t box = (size_t)64 * P;

    if (p == 0) {                                                // C_0 = I: T[., ., 0] = S[., ., 0]
        for (int o = tid; o < S2TC_BOXES * 64; o += blockDim.x)
            Tn[((size_t)b0 * 64 + o) * P] = S[((size_t)b0 * 64 + o) * P];
        return;
    }
    if (tid == 0) {
        for (int k = 0; k < 5; ++k) tc::mbar_init(&bar[k], 1);
        tc::fence_barrier_init();
    }
    if (warp == 0) tc::tmem_alloc<64>(tmem_slot);
    tc::tc_fence_before();
    __syncthreads();
    tc::tc_fence_after();
    const uint32_t tmem = *tmem_slot;
    const float* tp = toep + (size_t)p * S2TC_TAB_FLOATS_PER_P;
    const float2* spp = Sp + (size_t)p * nb * 64;                // S'[p][b][m]
    // window boxes b0-1 .. b0+64: the interior ones in one bulk copy from S'
    const int ilo = max(b0 - 1, 0), ihi = min(b0 + S2TC_BOXES + 1, nb);   // [ilo, ihi)
    if (tid == 0) {
        tc::mbar_expect_tx(&bar[4], (uint32_t)(ihi - ilo) * 512);
        tc::bulk_g2s(Scol + (ilo - (b0 - 1)) * 64, spp + (size_t)ilo * 64, (uint32_t)(ihi - ilo) * 512, &bar[4]);
        for (int c = 0; c < 2; ++c) {                            // B chunks 0 and 1
            tc::mbar_expect_tx(&bar[c], 2 * S2TC_B_BYTES);
            tc::bulk_g2s(Bbase + c * 2 * S2TC_B_BYTES, tp + (size_t)c * 2 * 64 * S2TC_CHUNK_K, 2 * S2TC_B_BYTES, &bar[c]);
        }
    }
    // edge boxes -1 / nb: neighbour halos (G > 1) or the periodic wrap (G = 1)
    if (b0 == 0 || b0 + S2TC_BOXES == nb) {
        for (int o = tid; o < 2 * 64; o += blockDim.x) {
            const int side = o >> 6, m = o & 63;
            const int bb = side ? b0 + S2TC_BOXES : b0 - 1;
            if (bb >= 0 && bb < nb) continue;
            const int u = bb - (b0 - 1);
            if (G == 1) Scol[u * 64 + m] = spp[(size_t)(bb < 0 ? nb - 1 : 0) * 64 + m];
            else Scol[u * 64 + m] = (bb < 0 ? haloL : haloR)[(size_t)m * P + p];
        }
    }
    tc::mbar_wait(&bar[4], 0);
    __syncthreads();
    (void)box;

    constexpr uint32_t IDESC = tc::idesc_tf32(128, 64);
    for (int c = 0; c < S2TC_NCHUNK; ++c) {
        const int buf = c & 1;
        unsigned char* Ahi = Abase + buf * 2 * S2TC_A_BYTES;
        unsigned char* Alo = Ahi + S2TC_A_BYTES;
        unsigned char* Bhi = Bbase + buf * 2 * S2TC_B_BYTES;
        unsigned char* Blo = Bhi + S2TC_B_BYTES;
        if (c >= 2) {
            tc::mbar_wait(&bar[2 + buf], ((c - 2) >> 1) & 1);    // MMAs of chunk c-2 done: buffers free
            if (tid == 0) {
                tc::mbar_expect_tx(&bar[buf], 2 * S2TC_B_BYTES);
                tc::bulk_g2s(Bhi, tp + (size_t)c * 2 * 64 * S2TC_CHUNK_K, 2 * S2TC_B_BYTES, &bar[buf]);
            }
        }
        // build A chunk c: rows n = 2 bl + cc, K columns kk = 4 k4 + j (window k = 16 c + kk)
        const int kb = (S2TC_CHUNK_K * c) >> 6;                  // window box offset 0, 1, 2
        const int m0 = (S2TC_CHUNK_K * c) & 63;
        {
            const int k4 = tid & 3, bl = tid >> 2;               // 64 boxes x 4 k4
            const float4* sp = reinterpret_cast<const float4*>(Scol + (bl + kb) * 64 + m0 + 4 * k4);
            const float4 u0 = sp[0], u1 = sp[1];                 // (re, im) of 4 consecutive m
            const float re[4] = {u0.x, u0.z, u1.x, u1.z}, im[4] = {u0.y, u0.w, u1.y, u1.w};
            float4 rh, rl, ih, il;
            float* prh = &rh.x; float* prl = &rl.x; float* pih = &ih.x; float* pil = &il.x;
#pragma unroll
            for (int j = 0; j < 4; ++j) {
                const float h1 = tc::to_tf32(re[j]); prh[j] = h1; prl[j] = re[j] - h1;
                const float h2 = tc::to_tf32(im[j]); pih[j] = h2; pil[j] = im[j] - h2;
            }
            const int n = 2 * bl;                                // re row; im row = n + 1
            const int offr = k4 * S2TC_LBO_A + (n >> 3) * 128 + (n & 7) * 16;
            *reinterpret_cast<float4*>(Ahi + offr) = rh;
            *reinterpret_cast<float4*>(Alo + offr) = rl;
            *reinterpret_cast<float4*>(Ahi + offr + 16) = ih;
            *reinterpret_cast<float4*>(Alo + offr + 16) = il;
        }
        tc::fence_proxy_async();
        __syncthreads();
        if (tid == 0) {
            tc::mbar_wait(&bar[buf], (c >> 1) & 1);              // B chunk landed
            tc::tc_fence_after();
#pragma unroll
            for (int st = 0; st < S2TC_CHUNK_K / 8; ++st) {
                const uint64_t ah = tc::umma_desc_kmajor(Ahi + 2 * st * S2TC_LBO_A, S2TC_LBO_A, 128);
                const uint64_t al = tc::umma_desc_kmajor(Alo + 2 * st * S2TC_LBO_A, S2TC_LBO_A, 128);
                const uint64_t bh = tc::umma_desc_kmajor(Bhi + 2 * st * 1024, 1024, 128);
                const uint64_t bl_ = tc::umma_desc_kmajor(Blo + 2 * st * 1024, 1024, 128);
                const uint32_t acc0 = (c | st) ? 1u : 0u;
                tc::mma_tf32(tmem, ah, bh, IDESC, acc0);
                tc::mma_tf32(tmem, ah, bl_, IDESC, 1u);
                tc::mma_tf32(tmem, al, bh, IDESC, 1u);
            }
            tc::mma_commit(&bar[2 + buf]);
        }
        __syncwarp();
    }
    tc::mbar_wait(&bar[2 + ((S2TC_NCHUNK - 1) & 1)], ((S2TC_NCHUNK - 1) >> 1) & 1);
    tc::tc_fence_after();
    // epilogue: warps w and w+4 read TMEM lanes 32 (w mod 4) .. +31, columns [32 (w / 4), +32)
    {
        const int q = warp & 3, half = warp >> 2;
        float v[32];
        tc::tmem_ld32(tmem + ((uint32_t)(32 * q) << 16) + 32 * half, v);
        const int n = 32 * q + lane, bl = n >> 1;
        const bool is_re = (lane & 1) == 0;
        float2* trow = Tn + ((size_t)(b0 + bl) * 64) * P + p;
#pragma unroll
        for (int k = 0; k < 32; ++k) {
            const float other = __shfl_xor_sync(0xffffffffu, v[k], 1);
            // even lane writes columns k < 16 of the pair, odd lane k >= 16
            if ((k < 16) == is_re) {
                const int i = 32 * half + k;
                trow[(size_t)i * P] = is_re ? make_float2(v[k], other) : make_float2(other, v[k]);
            }
        }
    }
    tc::tc_fence_before();
    __syncthreads();
    if (warp == 0) tc::tmem_dealloc<64>(tmem);
}

}  // namespace fmmfft
