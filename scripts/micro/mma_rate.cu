// tcgen05.mma kind::tf32 SS-mode issue rate vs N (M = 128, K = 8 per instruction), one CTA per SM.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o /tmp/mr scripts/micro/mma_rate.cu
#include <cstdio>
#include "../../paper_conf_sc_cecka17_b200/csrc/tcgen05.cuh"
using namespace fmmfft;
template <int N>
__global__ void k(long long* out, int reps, int lbo_a) {
    extern __shared__ __align__(1024) unsigned char sm[];
    __shared__ uint64_t bar;
    __shared__ uint32_t slot;
    if (threadIdx.x == 0) { tc::mbar_init(&bar, 1); tc::fence_barrier_init(); }
    if (threadIdx.x < 32) tc::tmem_alloc<256>(&slot);
    for (int i = threadIdx.x; i < 160 * 1024 / 4; i += blockDim.x) reinterpret_cast<float*>(sm)[i] = 0.f;
    tc::fence_proxy_async();
    tc::tc_fence_before(); __syncthreads(); tc::tc_fence_after();
    const uint32_t tmem = slot;
    if (threadIdx.x == 0) {
        constexpr uint32_t ID = tc::idesc_tf32(128, N);
        const uint64_t a = tc::umma_desc_kmajor(sm, lbo_a, 128);
        const uint64_t b = tc::umma_desc_kmajor(sm + 65536, N / 8 * 128, 128);
        long long t0 = clock64();
        for (int r = 0; r < reps; ++r) tc::mma_tf32(tmem, a, b, ID, 1u);
        tc::mma_commit(&bar);
        tc::mbar_wait(&bar, 0);
        long long t1 = clock64();
        if (blockIdx.x == 0) out[0] = t1 - t0;
    }
    tc::tc_fence_before(); __syncthreads();
    if (threadIdx.x < 32) tc::tmem_dealloc<256>(tmem);
}
template <int N> void run(long long* d, int lbo) {
    cudaFuncSetAttribute(k<N>, cudaFuncAttributeMaxDynamicSharedMemorySize, 160 * 1024);
    const int reps = 2048;
    k<N><<<148, 128, 160 * 1024>>>(d, reps, lbo);
    long long c; cudaMemcpy(&c, d, 8, cudaMemcpyDeviceToHost);
    printf("N=%3d lboA=%d: %.1f cycles/MMA (floor %d), %.0f B/clk smem operand reads  %s\n", N, lbo, (double)c / reps,
           128 * N / 256, (128.0 * 8 * 4 + N * 8 * 4) * reps / c, cudaGetErrorString(cudaGetLastError()));
}
int main() {
    long long* d; cudaMalloc(&d, 8);
    run<64>(d, 2048); run<128>(d, 2048); run<192>(d, 2048); run<256>(d, 2048);
    run<64>(d, 2080); run<192>(d, 2080);
    return 0;
}
