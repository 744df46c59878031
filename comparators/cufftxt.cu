// cufftxt.cu — the library comparator of BASELINE.json's metric ("speedup vs cuFFTXt"): a 1D C2C
// cuFFT plan spread over nGPU devices of one process (cufftXtSetGPUs), timed on the same input.
// NOT part of the FMM-FFT product path (the product is libfmmfft.so); bench.py loads this only to
// time the comparator, in a separate process on rank 0.
//
//   int cufftxt_bench(N, ngpu, dbl, iters, in_host, out_host, ms[2], err, errlen)
//     in_host: N interleaved complex (float2 / double2) in natural order;
//     out_host: N complex, the transform in natural order (after the reorder);
//     ms[0]: ms per cufftXtExecDescriptor (output left in cuFFT's shuffled multi-GPU order),
//     ms[1]: ms per exec + cufftXtMemcpy device-to-device into a natural-order descriptor.
//   Host wall clock around `iters` back-to-back executes, every device synchronised at both ends.
#include <cuda_runtime.h>
#include <cufft.h>
#include <cufftXt.h>

#include <chrono>
#include <cstdio>

#define CK(x)                                                                                     \
    do {                                                                                          \
        auto r_ = (x);                                                                            \
        if ((int)r_ != 0) {                                                                       \
            snprintf(err, errlen, "%s failed: %d (%s:%d)", #x, (int)r_, __FILE__, __LINE__);      \
            rc = 1;                                                                               \
            goto done;                                                                            \
        }                                                                                         \
    } while (0)

static void sync_all(int n) {
    for (int g = 0; g < n; ++g) {
        cudaSetDevice(g);
        cudaDeviceSynchronize();
    }
}

extern "C" __attribute__((visibility("default"))) int cufftxt_bench(long long N, int ngpu, int dbl, int iters,
                                                                     const void* in_host, void* out_host,
                                                                     double* ms, char* err, int errlen) {
    int rc = 0;
    cufftHandle plan = 0;
    cudaLibXtDesc *d = nullptr, *dn = nullptr;
    int gpus[16];
    size_t ws[16];
    const cufftType ty = dbl ? CUFFT_Z2Z : CUFFT_C2C;
    err[0] = 0;
    if (ngpu < 2 || ngpu > 16) { snprintf(err, errlen, "cufftXt multi-GPU needs 2..16 GPUs"); return 1; }
    for (int g = 0; g < ngpu; ++g) gpus[g] = g;
    CK(cufftCreate(&plan));
    CK(cufftXtSetGPUs(plan, ngpu, gpus));
    CK(cufftMakePlan1d(plan, (int)N, ty, 1, ws));
    CK(cufftXtMalloc(plan, &d, CUFFT_XT_FORMAT_INPLACE));
    CK(cufftXtMalloc(plan, &dn, CUFFT_XT_FORMAT_INPLACE));
    CK(cufftXtMemcpy(plan, d, const_cast<void*>(in_host), CUFFT_COPY_HOST_TO_DEVICE));
    for (int k = 0; k < 2; ++k) {                       // [0]: exec only; [1]: exec + reorder
        for (int w = 0; w < 3; ++w) {
            CK(cufftXtExecDescriptor(plan, d, d, CUFFT_FORWARD));
            CK(cufftXtMemcpy(plan, d, const_cast<void*>(in_host), CUFFT_COPY_HOST_TO_DEVICE));
        }
        sync_all(ngpu);
        double total = 0;
        for (int it = 0; it < iters; ++it) {
            CK(cufftXtMemcpy(plan, d, const_cast<void*>(in_host), CUFFT_COPY_HOST_TO_DEVICE));   // untimed refill
            sync_all(ngpu);
            auto t0 = std::chrono::steady_clock::now();
            CK(cufftXtExecDescriptor(plan, d, d, CUFFT_FORWARD));
            if (k == 1) CK(cufftXtMemcpy(plan, dn, d, CUFFT_COPY_DEVICE_TO_DEVICE));
            sync_all(ngpu);
            total += std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
        }
        ms[k] = total / iters;
    }
    CK(cufftXtMemcpy(plan, out_host, dn, CUFFT_COPY_DEVICE_TO_HOST));
done:
    if (d) cufftXtFree(d);
    if (dn) cufftXtFree(dn);
    if (plan) cufftDestroy(plan);
    return rc;
}
