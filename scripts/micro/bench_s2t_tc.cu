// Micro-benchmark of k_s2t_tc alone (timing only; values are random, no parity here):
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -DS2TC_STAMPS -o /tmp/bs scripts/micro/bench_s2t_tc.cu
//   /tmp/bs [nb] [P] [ctas]  (the (p, tile) work items split evenly over `ctas` CTAs, default 148)
#include <cstdio>
#include <cstdlib>
#include <vector>
#ifdef S2TC_STAMPS
__device__ long long g_stamp[128];
#define STAMP(i) do { if (blockIdx.x == 0 && blockIdx.y == 0 && (threadIdx.x == 0 || threadIdx.x == 128 || threadIdx.x == 256)) g_stamp[i] = clock64(); } while (0)
#else
#define STAMP(i) do {} while (0)
#endif
#include "../../paper_conf_sc_cecka17_b200/csrc/kernel_s2t_tc.cuh"
using namespace fmmfft;
int main(int argc, char** argv) {
    int nb = argc > 1 ? atoi(argv[1]) : 256, P = argc > 2 ? atoi(argv[2]) : 64, ctas = argc > 3 ? atoi(argv[3]) : 148;
    size_t n = (size_t)nb * 64 * P;
    float2 *Sp, *Tn; float *toep, *kf;
    cudaMalloc(&Sp, n * 8); cudaMalloc(&Tn, n * 8);
    cudaMalloc(&toep, (size_t)P * S2TC_TAB_FLOATS_PER_P * 4); cudaMalloc(&kf, (size_t)P * 1024);
    cudaMemset(Sp, 0, n * 8); cudaMemset(toep, 0, (size_t)P * S2TC_TAB_FLOATS_PER_P * 4); cudaMemset(kf, 0, (size_t)P * 1024);
    cudaFuncSetAttribute(k_s2t_tc<2>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)s2tc_smem_bytes());
    cudaFuncSetAttribute(k_s2t_tc<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)s2tc_smem_bytes());
    const long long work = (long long)(P - 1) * (nb / S2TC_BOXES);
    if (ctas > work) ctas = (int)work;
    const bool many = work > ctas;
    dim3 grid(ctas);
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    for (int i = 0; i < 5; ++i) (many ? k_s2t_tc<2> : k_s2t_tc<1>)<<<grid, S2TC_THREADS, s2tc_smem_bytes()>>>(Sp, Sp, Sp, (float*)Tn, toep, P, nb, 1);
    cudaEventRecord(a);
    const int R = 50;
    for (int i = 0; i < R; ++i) (many ? k_s2t_tc<2> : k_s2t_tc<1>)<<<grid, S2TC_THREADS, s2tc_smem_bytes()>>>(Sp, Sp, Sp, (float*)Tn, toep, P, nb, 1);
    cudaEventRecord(b); cudaEventSynchronize(b);
    float ms; cudaEventElapsedTime(&ms, a, b);
    printf("nb=%d P=%d ctas=%d: %.2f us/launch  err=%s\n", nb, P, ctas, ms * 1e3 / R,
           cudaGetErrorString(cudaGetLastError()));
#ifdef S2TC_STAMPS
    long long st[128]; cudaMemcpyFromSymbol(st, g_stamp, sizeof st);
    for (int i = 1; i < 80; ++i) if (st[i]) printf("stamp %2d: +%lld\n", i, st[i] - st[0]);
#endif
    return 0;
}
