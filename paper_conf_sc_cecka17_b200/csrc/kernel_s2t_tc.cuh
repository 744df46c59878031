// kernel_s2t_tc.cuh — S2T (Alg. 1 line 3, §4.6) on the 5th-generation tensor
// cores, complex64, M_L = 64.
//
// The near field of leaf box b for FMM p is
//     T[b][i] = sum_{j=-64}^{127} K_p[j - i] S_window[j],   K_p[k] = cot(pi (p + P k) / N),
// the window being boxes b-1, b, b+1. Split by source box (segment s = 0, 1, 2 <-> box b-1+s):
//     T[b][i] = sum_{s<3} sum_{m<64} A[b - 1 + s][m] B_s[i][m],   B_s[i][m] = K_p[(s-1) 64 + m - i],
// with A[b][m] = S_{p m b} (one real component at a time; the operator is real).
// For a tile of 128 consecutive boxes this is three accumulating GEMMs (UMMA M = 128 boxes,
// N = 64 outputs i, K = 64 points m) whose A operands are the SAME shared-memory rows shifted by
// one box: A is stored K-major with 8-row core-matrix groups packed back to back (SBO = 128 B), so
// row r sits at r x 16 bytes and "the rows of boxes b0-1+s .. b0+126+s" is the descriptor of row
// s — a 16-byte offset. The A buffer holds 130 rows (boxes b0-1 .. b0+128): the data is used once,
// never Toeplitz-expanded, and the accumulator already holds T (no shift in the epilogue).
// B_s is the per-p Toeplitz operator, precomputed per plan in fp64 and split into tf32 hi + lo.
// Precision: 3xTF32, T = Ahi Bhi + Ahi Blo + Alo Bhi accumulated in fp32 in tensor memory (plain
// TF32 misses the 1e-5 bound): 9 MMAs (M=128, N=64, K=8) per K step and component.
//
// CTA = a contiguous run of (FMM p, 128-box tile) work items — (p - 1) ntile + t, split evenly
// over one CTA per SM, so every SM gets the same number of tiles (a run crosses at most a few p;
// the operator B_p is reloaded when p changes, after the previous tile's MMAs completed) —
// warp-specialised, 9 warps:
//   warps 0-3  build A (re/im x hi/lo, K chunks of 16 in a 2-slot ring) from the p-major copy
//              S'[p][b][m] (the next chunk prefetched into registers); halo rows from the
//              neighbouring boxes (periodic wrap at G = 1, the halo buffers at rank edges);
//   warp 8     loads the operator B_p (bulk copies, one mbarrier per K chunk) and issues the MMAs,
//              committing each chunk's MMAs to the slot's mbarrier;
//   warps 4-7  (TMEM lane quarters 0-3) the epilogue: tcgen05.ld of T (re and im accumulators),
//              coalesced stores through a 32 x 32 shared-memory transpose per warp.
// Two TMEM accumulator sets (2 x 256 columns: per component Ahi[Bhi|Blo] in 128 columns, Alo Bhi
// added to the first 64): the epilogue of tile t overlaps the MMAs of t+1.
// Output T_near is p-major and planar per box: [p][b][re/im][m] (what k_post_pfft reads).
// p = 0 (the identity, R1) is written by k_s2m.
#pragma once
#include "common.cuh"
#include "tcgen05.cuh"

#ifndef STAMP
#define STAMP(i) do {} while (0)                          // timing probes (scripts/micro/bench_s2t_tc.cu)
#endif

namespace fmmfft {

constexpr int S2TC_BOXES = 128;                           // boxes per tile (UMMA M)
constexpr int S2TC_ROWS = S2TC_BOXES + 2;                 // + halo boxes b0-1, b0+128
constexpr int S2TC_KC = 16;                               // K (m) per A chunk
constexpr int S2TC_NKC = 64 / S2TC_KC;
constexpr int S2TC_LBO_A = S2TC_ROWS * 16;                // bytes between k4 columns of A (2080)
constexpr int S2TC_A_PART = (S2TC_KC / 4) * S2TC_LBO_A;   // one (component, hi/lo) part of a chunk
constexpr int S2TC_A_SLOT = 4 * S2TC_A_PART;              // [re/im][hi/lo] parts
constexpr int S2TC_N = 192;                               // operator rows (segment, i)
constexpr int S2TC_B_K4 = (S2TC_N / 8) * 128;             // bytes per k4 column of B (24 core matrices)
constexpr int S2TC_B_BYTES = 16 * S2TC_B_K4;              // one of hi / lo (K = 64)
constexpr int S2TC_TAB_FLOATS_PER_P = 2 * S2TC_B_BYTES / 4;   // [k4 16][r8 48][8][4], rows (s, hi/lo, i)
// B rows per k4 column: for each shift s the 64 hi rows then the 64 lo rows, so [Bhi_s; Blo_s] is
// ONE N = 128 operand: Ahi x [Bhi_s | Blo_s] is one MMA into 128 TMEM columns (the two products
// summed in the epilogue) and Alo x Bhi_s (N = 64, the same descriptor) accumulates into the first
// 64 — 2 MMAs per (shift, component, K step) instead of 3, and A_hi is read once.
constexpr int S2TC_B_K4N = (2 * S2TC_N / 8) * 128;         // bytes per k4 column (48 core matrices)
#ifndef S2TC_BW
#define S2TC_BW 8                                         // A-builder warps (4: 168 registers, S2T 369 us at cfg3; 8: 128 registers, 283 us)
#endif
constexpr int S2TC_BT = S2TC_BW * 32;                     // builder threads
#ifndef S2TC_EW
#define S2TC_EW 4                                         // epilogue warps (4, or 8: two per TMEM lane quarter)
#endif
constexpr int S2TC_THREADS = (S2TC_BW + S2TC_EW + 1) * 32;  // builders, epilogue warps, the MMA warp
constexpr int S2TC_MMA_WARP = S2TC_BW + S2TC_EW;

struct S2tcSmem {                                         // byte offsets
    static constexpr int B = 0;
    static constexpr int A = B + 2 * S2TC_B_BYTES;              // 2-slot ring of K chunks
    static constexpr int XT = A + 2 * S2TC_A_SLOT;              // per-warp transpose [4][32][33] floats
    static constexpr int BAR = XT + S2TC_EW * 32 * 33 * 4;      // 12 mbarriers
    static constexpr int TSLOT = BAR + 12 * 8;
    static constexpr int TOTAL = TSLOT + 16;
};
__host__ __device__ constexpr size_t s2tc_smem_bytes() { return (size_t)S2tcSmem::TOTAL; }

template <int PF>                                          // A-chunk prefetch distance (1 or 2)
__global__ void __launch_bounds__(S2TC_THREADS, 1)
k_s2t_tc(const float2* __restrict__ Sp, const float2* __restrict__ haloL, const float2* __restrict__ haloR,
         float* __restrict__ Tn, const float* __restrict__ toep, int P, int nb, int G) {
    pdl_trigger();
    pdl_wait();
    STAMP(0);
    extern __shared__ __align__(1024) unsigned char smem_tc[];
    unsigned char* Bsm = smem_tc + S2tcSmem::B;
    unsigned char* Asm = smem_tc + S2tcSmem::A;
    float* Xt = reinterpret_cast<float*>(smem_tc + S2tcSmem::XT);
    uint64_t* bar = reinterpret_cast<uint64_t*>(smem_tc + S2tcSmem::BAR);
    uint64_t* bfull = bar;                                       // [4] operator chunk landed
    uint64_t* cfull = bar + 4;                                   // [2] A slot built (128 arrivals)
    uint64_t* cempty = bar + 6;                                  // [2] MMAs of A slot done (commit)
    uint64_t* afull = bar + 8;                                   // [2] accumulators complete (commit)
    uint64_t* aempty = bar + 10;                                 // [2] accumulators read (128 arrivals)
    uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(smem_tc + S2tcSmem::TSLOT);

    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int ntile = nb / S2TC_BOXES;
    const long long W = (long long)(P - 1) * ntile;              // work items (p - 1) ntile + t
    const int w0 = (int)(W * blockIdx.x / gridDim.x), w1 = (int)(W * (blockIdx.x + 1) / gridDim.x);
    if (w0 >= w1) return;
    const int nit = w1 - w0;
    const size_t pblk = (size_t)nb * 64;                         // elements per p block of S' / T

    if (tid == 0) {
        for (int k = 0; k < 12; ++k) tc::mbar_init(&bar[k], (k == 4 || k == 5) ? (unsigned)S2TC_BT : (k >= 10 ? (unsigned)(S2TC_EW * 32) : 1u));
        tc::fence_barrier_init();
    }
    if (warp == 0) tc::tmem_alloc<512>(tmem_slot);
    tc::tc_fence_before();
    __syncthreads();
    tc::tc_fence_after();
    const uint32_t tmem = *tmem_slot;
    STAMP(1);

    if (warp < S2TC_BW) {
        // ------------------------------------------------------------ A builders (128 threads)
        // item j: row r = idx >> 2 (box b0 - 1 + r), k4 = idx & 3, idx = tid + S2TC_BT j < 4 x 130
        constexpr int NJ = (4 * S2TC_ROWS + S2TC_BT - 1) / S2TC_BT;   // 5 (3 with 8 builder warps)
        float4 sv[2][NJ][2];                                     // two chunks in flight (prefetch distance 2)
        auto load_chunk = [&](float4 (&svb)[NJ][2], int p, int t, int kc) {
            const float2* spp = Sp + (size_t)p * pblk;
#pragma unroll
            for (int j = 0; j < NJ; ++j) {
                const int idx = tid + S2TC_BT * j;
                if (idx < 4 * S2TC_ROWS) {
                    const int r = idx >> 2, k4 = idx & 3;
                    const int g = t * S2TC_BOXES - 1 + r;        // global box (within this rank)
                    const int m = S2TC_KC * kc + 4 * k4;
                    if (g >= 0 && g < nb) {
                        const float4* src = reinterpret_cast<const float4*>(spp + (size_t)g * 64 + m);
                        svb[j][0] = __ldg(src);
                        svb[j][1] = __ldg(src + 1);
                    } else if (G == 1) {                         // periodic wrap (R8)
                        const float4* src = reinterpret_cast<const float4*>(spp + (size_t)((g + nb) % nb) * 64 + m);
                        svb[j][0] = __ldg(src);
                        svb[j][1] = __ldg(src + 1);
                    } else {                                     // neighbour rank's box ([m][P] layout)
                        const float2* h = (g < 0 ? haloL : haloR) + (size_t)m * P + p;
                        const float2 a = __ldg(h), b = __ldg(h + P), c = __ldg(h + 2 * P), d = __ldg(h + 3 * P);
                        svb[j][0] = make_float4(a.x, a.y, b.x, b.y);
                        svb[j][1] = make_float4(c.x, c.y, d.x, d.y);
                    }
                }
            }
        };
        // (p, t) of the tile being built and of the next one (no division in the pacing loop)
        int pc = w0 / ntile + 1, tc_ = w0 - (pc - 1) * ntile;
        load_chunk(sv[0], pc, tc_, 0);
        if (PF == 2) load_chunk(sv[1], pc, tc_, 1);
        for (int it = 0; it < nit; ++it) {
            const int pn = tc_ + 1 == ntile ? pc + 1 : pc, tn = tc_ + 1 == ntile ? 0 : tc_ + 1;
#pragma unroll
            for (int kc = 0; kc < S2TC_NKC; ++kc) {
                const int gi = it * S2TC_NKC + kc, slot = gi & 1, use = gi >> 1;
                if (use > 0) tc::mbar_wait(&cempty[slot], (use - 1) & 1);   // MMAs done with this slot
                unsigned char* As = Asm + slot * S2TC_A_SLOT;
#pragma unroll
                for (int j = 0; j < NJ; ++j) {
                    const int idx = tid + S2TC_BT * j;
                    if (idx < 4 * S2TC_ROWS) {
                        const int r = idx >> 2, k4 = idx & 3;
                        const float4 u0 = sv[kc & 1][j][0], u1 = sv[kc & 1][j][1];   // (re, im) of 4 consecutive m
                        const float re[4] = {u0.x, u0.z, u1.x, u1.z}, im[4] = {u0.y, u0.w, u1.y, u1.w};
                        float4 rh, rl, ihv, il;
                        float* prh = &rh.x; float* prl = &rl.x; float* pih = &ihv.x; float* pil = &il.x;
#pragma unroll
                        for (int q = 0; q < 4; ++q) {
                            // lo rounded to nearest too (the MMA would truncate it: 2^-21 vs 2^-22)
                            const float h1 = tc::to_tf32(re[q]); prh[q] = h1; prl[q] = tc::to_tf32(re[q] - h1);
                            const float h2 = tc::to_tf32(im[q]); pih[q] = h2; pil[q] = tc::to_tf32(im[q] - h2);
                        }
                        const int off = k4 * S2TC_LBO_A + r * 16;   // [c][hi/lo][k4][row][16 B]
                        *reinterpret_cast<float4*>(As + 0 * S2TC_A_PART + off) = rh;
                        *reinterpret_cast<float4*>(As + 1 * S2TC_A_PART + off) = rl;
                        *reinterpret_cast<float4*>(As + 2 * S2TC_A_PART + off) = ihv;
                        *reinterpret_cast<float4*>(As + 3 * S2TC_A_PART + off) = il;
                    }
                }
                tc::fence_proxy_async();
                tc::mbar_arrive(&cfull[slot]);
                if (it < 2) STAMP(41 + 4 * it + kc);
                // prefetch chunk kc + PF (into the buffer just consumed when PF = 2; S2TC_NKC is even)
                if (kc + PF < S2TC_NKC) load_chunk(sv[(kc + PF) & 1], pc, tc_, kc + PF);
                else if (it + 1 < nit) load_chunk(sv[(kc + PF) & 1], pn, tn, kc + PF - S2TC_NKC);
            }
            pc = pn;
            tc_ = tn;
        }
    } else if (warp == S2TC_MMA_WARP) {
        // ------------------------------------------------------------ operator loads + MMA issue
        if (lane == 0) {
            auto load_B = [&](int p) {
                const float* tp = toep + (size_t)p * S2TC_TAB_FLOATS_PER_P;
                for (int kc = 0; kc < S2TC_NKC; ++kc) {          // B chunk kc: k4 in [4 kc, 4 kc + 4), hi and lo
                    tc::mbar_expect_tx(&bfull[kc], 4 * S2TC_B_K4N);
                    tc::bulk_g2s(Bsm + kc * 4 * S2TC_B_K4N, tp + kc * S2TC_B_K4N, 4 * S2TC_B_K4N, &bfull[kc]);
                }
            };
            int pcur = w0 / ntile + 1, bphase = 0;
            bool bnew = true;                                    // wait for the B chunks at the next tile
            load_B(pcur);
            constexpr uint32_t IDESC128 = tc::idesc_tf32(128, 128), IDESC64 = tc::idesc_tf32(128, 64);
            for (int it = 0; it < nit; ++it) {
                const int buf = it & 1;
                const int pit = (w0 + it) / ntile + 1;
                if (pit != pcur) {                               // next FMM: reload B_p once tile it-1's MMAs completed
                    tc::mbar_wait(&afull[(it - 1) & 1], ((it - 1) >> 1) & 1);
                    tc::tc_fence_after();
                    pcur = pit;
                    bphase ^= 1;
                    bnew = true;
                    load_B(pcur);
                }
                if (it >= 2) tc::mbar_wait(&aempty[buf], ((it >> 1) + 1) & 1);   // epilogue of tile it-2 done
                for (int kc = 0; kc < S2TC_NKC; ++kc) {
                    const int gi = it * S2TC_NKC + kc, slot = gi & 1, use = gi >> 1;
                    if (bnew) tc::mbar_wait(&bfull[kc], bphase);
                    tc::mbar_wait(&cfull[slot], use & 1);
                    tc::tc_fence_after();
                    const unsigned char* As = Asm + slot * S2TC_A_SLOT;
#pragma unroll
                    for (int st = 0; st < S2TC_KC / 8; ++st) {
                        const unsigned char* bk = Bsm + (4 * kc + 2 * st) * S2TC_B_K4N;
#pragma unroll
                        for (int c = 0; c < 2; ++c) {
                            const uint32_t d = tmem + (uint32_t)(buf * 256 + c * 128);
                            const unsigned char* ahp = As + (2 * c) * S2TC_A_PART + 2 * st * S2TC_LBO_A;
                            const unsigned char* alp = As + (2 * c + 1) * S2TC_A_PART + 2 * st * S2TC_LBO_A;
#pragma unroll
                            for (int s = 0; s < 3; ++s) {        // rows of boxes b0-1+s ..: 16-byte offset
                                const uint64_t ah = tc::umma_desc_kmajor(ahp + 16 * s, S2TC_LBO_A, 128);
                                const uint64_t al = tc::umma_desc_kmajor(alp + 16 * s, S2TC_LBO_A, 128);
                                const uint64_t b2 = tc::umma_desc_kmajor(bk + s * 2048, S2TC_B_K4N, 128);   // [Bhi_s; Blo_s]
                                tc::mma_tf32(d, ah, b2, IDESC128, (kc | st | s) ? 1u : 0u);
                                tc::mma_tf32(d, al, b2, IDESC64, 1u);                                      // Alo Bhi_s
                            }
                        }
                    }
                    tc::mma_commit(&cempty[slot]);
                    if (it < 2) STAMP(2 + 4 * it + kc);
                }
                bnew = false;
                tc::mma_commit(&afull[buf]);
            }
        }
    } else {
        // ------------------------------------------------------------ epilogue (warps 4-7)
        // warp q reads TMEM lanes 32 q .. 32 q + 31 = boxes b0 + 32 q + lane
        const int q = warp & 3;
        const int eh = (warp - S2TC_BW) >> 2;                   // with 8 epilogue warps: which 2 of the 4 chunks
        float* xt = Xt + (warp - S2TC_BW) * 32 * 33;
        for (int it = 0; it < nit; ++it) {
            const int w = w0 + it, buf = it & 1;
            const int p = w / ntile + 1, t = w - (p - 1) * ntile;
            if (it < 4) STAMP(20 + 4 * it);
            tc::mbar_wait(&afull[buf], (it >> 1) & 1);
            tc::tc_fence_after();
            if (it < 4) STAMP(21 + 4 * it);
            // planar [p][b][c][m]: rows of boxes b0 + 32 q + r, r < 32
            float* tw = Tn + ((size_t)p * nb + (size_t)t * S2TC_BOXES + 32 * q) * 128;
#pragma unroll 1
            for (int ch = (S2TC_EW == 8 ? 2 * eh : 0); ch < (S2TC_EW == 8 ? 2 * eh + 2 : 4); ++ch) {   // (component, i half)
                const int c = ch >> 1, h = ch & 1;
                float v[32];
                tc::tmem_ld32(tmem + ((uint32_t)(32 * q) << 16) + (uint32_t)(buf * 256 + c * 128 + 32 * h), v);
                {   // + the Ahi Blo half (columns 64..127 of the component)
                    float v2[32];
                    tc::tmem_ld32(tmem + ((uint32_t)(32 * q) << 16) + (uint32_t)(buf * 256 + c * 128 + 64 + 32 * h), v2);
#pragma unroll
                    for (int k = 0; k < 32; ++k) v[k] += v2[k];
                }
                if (ch == (S2TC_EW == 8 ? 2 * eh + 1 : 3)) {     // this warp's reads done: accumulators free for tile it + 2
                    tc::tc_fence_before();
                    tc::mbar_arrive(&aempty[buf]);
                }
#pragma unroll
                for (int k = 0; k < 32; ++k) xt[lane * 33 + k] = v[k];
                __syncwarp();
#pragma unroll
                for (int r = 0; r < 32; ++r) tw[(size_t)r * 128 + c * 64 + 32 * h + lane] = xt[r * 33 + lane];
                __syncwarp();
            }
            if (it < 4) STAMP(22 + 4 * it);
        }
    }
    tc::tc_fence_before();
    __syncthreads();
    STAMP(40);
    if (warp == 0) tc::tmem_dealloc<512>(tmem);
}

}  // namespace fmmfft
