// Phase timing of k_tree_pc alone (cfg2 shape by default; random data, timing only):
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -I include -o /tmp/btp scripts/micro/bench_tree_pc.cu
//   /tmp/btp [L] [B] [P]
#include <cstdio>
#include <cstdlib>
__device__ long long g_ts[64];
#define TSTAMP(i) do { if (blockIdx.x == 0 && threadIdx.x == 0) g_ts[i] = clock64(); } while (0)
#include "../../paper_conf_sc_cecka17_b200/csrc/kernels_fmm.cuh"
using namespace fmmfft;
int main(int argc, char** argv) {
    const int L = argc > 1 ? atoi(argv[1]) : 8, B = argc > 2 ? atoi(argv[2]) : 2, P = argc > 3 ? atoi(argv[3]) : 64;
    constexpr int Q = 16, CL = 2, NTH = 512;
    const size_t QQ = Q * Q, nbB = 1u << B, tabB = (nbB - 3) * QQ;
    auto H = [&](int l) { return ((size_t)1 << l) / CL; };
    size_t cplx = 32 + nbB * Q + (nbB / CL) * Q + H(L) * Q + H(L - 1) * Q;
    for (int l = B + 1; l <= L; ++l) cplx += (H(l) + 6) * Q;
    const size_t smem = (2 * QQ + tabB + (size_t)(L - B) * 4 * QQ) * 4 + QQ * 8 + cplx * 8;
    TreePArgs a{};
    for (int l = B; l <= L; ++l) {
        cudaMalloc(&a.M[l], ((size_t)1 << l) * Q * P * 8); cudaMemset(a.M[l], 0, ((size_t)1 << l) * Q * P * 8);
        cudaMalloc(&a.Lx[l], ((size_t)1 << l) * Q * P * 8);
        void* t; const size_t te = (l == B ? tabB : 4 * QQ) * P;
        cudaMalloc(&t, te * 4); cudaMemset(t, 0, te * 4); a.tab[l] = t;
    }
    cudaMalloc(&a.r, P * 8);
    a.L = L; a.B = B; a.dbg = 0;
    float* m2m; cudaMalloc(&m2m, 2 * QQ * 4); cudaMemset(m2m, 0, 2 * QQ * 4);
    auto kern = k_tree_pc<Q, NTH, CL>;
    cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    cudaLaunchConfig_t cfg{};
    cfg.gridDim = dim3((P - 1) * CL); cfg.blockDim = dim3(NTH); cfg.dynamicSmemBytes = smem;
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    for (int i = 0; i < 3; ++i) cudaLaunchKernelEx(&cfg, kern, a, (const float*)m2m, P, (int)tabB);
    cudaEventRecord(e0);
    for (int i = 0; i < 20; ++i) cudaLaunchKernelEx(&cfg, kern, a, (const float*)m2m, P, (int)tabB);
    cudaEventRecord(e1); cudaEventSynchronize(e1);
    float ms; cudaEventElapsedTime(&ms, e0, e1);
    printf("k_tree_pc L=%d B=%d P=%d smem=%zu: %.2f us/launch (%s)\n", L, B, P, smem, ms * 1e3 / 20, cudaGetErrorString(cudaGetLastError()));
    long long ts[64]; cudaMemcpyFromSymbol(ts, g_ts, sizeof ts);
    const char* nm[] = {"start", "staged", "up done", "cluster sync 1", "exchange+sync 2", "base", "down l=B+1"};
    for (int i = 1; i < 6 + L - B + 1; ++i) if (i != 6)
        printf("  %-16s +%6lld cyc  (%6lld)\n", i < 7 ? nm[i] : "down", ts[i] - ts[0], ts[i] - ts[i - 1]);
    for (int i = 29; i < 30 + L; ++i) if (ts[i] > ts[0]) printf("  up stamp %2d      +%6lld cyc\n", i, ts[i] - ts[0]);
    return 0;
}
