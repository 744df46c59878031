// common.cuh — shared device helpers of the FMM-FFT library (sm_100a).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

namespace fmmfft {

// Complex storage is interleaved (re, im) — the paper's array-of-structs layout
// and the ABI's float2 / double2.
template <typename R> struct cplx;
template <> struct cplx<float> { using type = float2; };
template <> struct cplx<double> { using type = double2; };
template <typename R> using C2 = typename cplx<R>::type;

// Blackwell packs two fp32 lanes per instruction (FADD2 / FMUL2 / FFMA2, PTX .f32x2): a complex
// value is one float2 register pair, and a real operator entry times complex data is a single
// FFMA2 with the scalar broadcast — the FMM's whole arithmetic shape.
__device__ __forceinline__ float2 cadd(float2 a, float2 b) { return __fadd2_rn(a, b); }
__device__ __forceinline__ double2 cadd(double2 a, double2 b) { return make_double2(a.x + b.x, a.y + b.y); }
__device__ __forceinline__ float2 csub(float2 a, float2 b) { return __fadd2_rn(a, make_float2(-b.x, -b.y)); }
__device__ __forceinline__ double2 csub(double2 a, double2 b) { return make_double2(a.x - b.x, a.y - b.y); }
__device__ __forceinline__ float2 cmul(float2 a, float2 b) {
    return make_float2(fmaf(a.x, b.x, -a.y * b.y), fmaf(a.x, b.y, a.y * b.x));
}
__device__ __forceinline__ double2 cmul(double2 a, double2 b) {
    return make_double2(fma(a.x, b.x, -a.y * b.y), fma(a.x, b.y, a.y * b.x));
}
// a += k * b for real k (the FMM operators are real)
__device__ __forceinline__ void rfma(float2& a, float k, float2 b) { a = __ffma2_rn(make_float2(k, k), b, a); }
__device__ __forceinline__ void rfma(double2& a, double k, double2 b) { a.x = fma(k, b.x, a.x); a.y = fma(k, b.y, a.y); }
__device__ __forceinline__ float2 czero(float2) { return make_float2(0.f, 0.f); }
__device__ __forceinline__ double2 czero(double2) { return make_double2(0.0, 0.0); }
template <typename C> __device__ __forceinline__ C zero();
template <> __device__ __forceinline__ float2 zero<float2>() { return make_float2(0.f, 0.f); }
template <> __device__ __forceinline__ double2 zero<double2>() { return make_double2(0.0, 0.0); }

// multiply by -i (used by the radix-4 butterfly): (x + iy)(-i) = y - ix
__device__ __forceinline__ float2 mul_mi(float2 a) { return make_float2(a.y, -a.x); }
__device__ __forceinline__ double2 mul_mi(double2 a) { return make_double2(a.y, -a.x); }

// w = exp(-2 pi i num / den) for integers 0 <= num < den, den a power of two; the argument
// 2 num / den is exact in floating point, and sincospi(f) is correctly rounded to ~1 ulp.
__device__ __forceinline__ float2 twiddle_f(long long num, long long den) {
    float s, c;
    sincospif(2.0f * (float)num / (float)den, &s, &c);
    return make_float2(c, -s);
}
__device__ __forceinline__ double2 twiddle_d(long long num, long long den) {
    double s, c;
    sincospi(2.0 * (double)num / (double)den, &s, &c);
    return make_double2(c, -s);
}
template <typename R> __device__ __forceinline__ C2<R> twiddle(long long num, long long den);
template <> __device__ __forceinline__ float2 twiddle<float>(long long num, long long den) { return twiddle_f(num, den); }
template <> __device__ __forceinline__ double2 twiddle<double>(long long num, long long den) { return twiddle_d(num, den); }

__device__ __forceinline__ float2 ldg_c(const float2* p) { return __ldg(p); }
__device__ __forceinline__ double2 ldg_c(const double2* p) { return __ldg(p); }

// cp.async (LDGSTS): global -> shared without a register round trip, so a thread can have many
// copies in flight; cp_async_wait_all() + __syncthreads() publishes them.
template <int BYTES>
__device__ __forceinline__ void cp_async(void* smem, const void* gmem) {
    const unsigned sa = (unsigned)__cvta_generic_to_shared(smem);
    if constexpr (BYTES == 16)
        asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"(sa), "l"(gmem) : "memory");
    else
        asm volatile("cp.async.ca.shared.global [%0], [%1], %2;\n" ::"r"(sa), "l"(gmem), "n"(BYTES) : "memory");
}
template <typename T>
__device__ __forceinline__ void cp_async_elem(T* smem, const T* gmem) { cp_async<sizeof(T)>(smem, gmem); }
__device__ __forceinline__ void cp_async_wait_all() { asm volatile("cp.async.wait_all;\n" ::: "memory"); }
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;\n" ::: "memory"); }
template <int N> __device__ __forceinline__ void cp_async_wait_group() {
    asm volatile("cp.async.wait_group %0;\n" ::"n"(N) : "memory");
}

// Programmatic dependent launch: let the next kernel in the stream start scheduling its CTAs
// (call early), and wait until the previous kernel's results are complete and visible (call
// before the first read of them and before any global write).
// The explicit early trigger is compiled out: dependents then launch when every CTA of the
// predecessor has exited (the implicit trigger), which still hides the launch gap but never parks
// dependent CTAs on SMs the predecessor's later waves (or the side stream) need.
#ifdef FMMFFT_EARLY_PDL_TRIGGER
__device__ __forceinline__ void pdl_trigger() { asm volatile("griddepcontrol.launch_dependents;\n" ::: "memory"); }
#else
__device__ __forceinline__ void pdl_trigger() {}
#endif
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;\n" ::: "memory"); }

}  // namespace fmmfft
