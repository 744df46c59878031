// fmmfft.cu — plan / execute orchestration and the C ABI of include/fmmfft.h.
//
// One process per GPU (NCCL over NVLink/NVSwitch between ranks), or G "virtual ranks" on one
// GPU with device-to-device copies standing in for NCCL (FMMFFT_FLAG_VIRTUAL, for testing the
// partitioned data flow). The stage sequence per execute is Algorithm 1
// followed by the distributed 2D FFT with its single all-to-all:
//
//   comm_S    S halo (line 2)                          NCCL send/recv | D2D | none (G = 1)
//   near_up   S2T + S2M (lines 1, 3)                   k_near_up
//   m2m       M2M for l = L-1 .. l_g (line 5)          k_m2m per level
//   comm_M    M^l halos for l > l_g (line 7) + all-gather of level l_g (line 9, reading R16)
//   top       M2M l_g-1 .. B on the gathered level, M2L-B (line 10), REDUCE (line 11),
//             M2L + L2L for B < l <= l_g (replicated top of the tree)
//   down      M2L-l (line 8) + L2L (line 13) for l = l_g+1 .. L   k_down per level
//   post_pfft L2T + POST + P-point FFTs + transposed store (lines 14-16)
//   a2a       the one all-to-all transpose (line 16)
//   mfft      P/G M-point FFTs, multi-pass Stockham (line 16)
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <string>
#include <vector>

#include "../../include/fmmfft.h"
#include "common.cuh"
#include "kernels_fft.cuh"
#include "kernels_fmm.cuh"
#include "nccl_loader.hpp"

namespace fmmfft {

// ------------------------------------------------------------------ errors
static thread_local std::string g_last_error;

static fmmfft_status_t fail(fmmfft_status_t st, const char* fmt, ...) {
    char buf[512];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof buf, fmt, ap);
    va_end(ap);
    g_last_error = buf;
    return st;
}

#define CUDA_TRY(expr)                                                                          \
    do {                                                                                        \
        cudaError_t e_ = (expr);                                                                \
        if (e_ != cudaSuccess)                                                                  \
            return fail(e_ == cudaErrorMemoryAllocation ? FMMFFT_ALLOC_FAILED : FMMFFT_CUDA_ERROR, \
                        "%s failed: %s (%s:%d)", #expr, cudaGetErrorString(e_), __FILE__, __LINE__); \
    } while (0)

#define NCCL_TRY(expr)                                                                          \
    do {                                                                                        \
        ncclResult_t r_ = (expr);                                                               \
        if (r_ != ncclSuccess)                                                                  \
            return fail(FMMFFT_NCCL_ERROR, "%s failed: %s", #expr, nccl().GetErrorString(r_));  \
    } while (0)

#define LAUNCH_CHECK() CUDA_TRY(cudaGetLastError())

// ------------------------------------------------------------------ communicator
struct Comm {
    ncclComm_t comm = nullptr;
    int rank = 0, size = 0, device = -1;
};
static Comm g_comm;

// ------------------------------------------------------------------ host operator tables (fp64)
// These are the product's own tables (computed here in C++); they share nothing with oracle/.
static std::vector<double> cheb_nodes(int Q) {            // z_j = cos((2j+1) pi / (2Q))
    std::vector<double> z(Q);
    for (int j = 0; j < Q; ++j) z[j] = std::cos((2.0 * j + 1.0) * M_PI / (2.0 * Q));
    return z;
}
static double lagr(const std::vector<double>& z, int i, double t) {   // l_i(t)
    double v = 1.0;
    for (size_t k = 0; k < z.size(); ++k)
        if ((int)k != i) v *= (t - z[k]) / (z[i] - z[k]);
    return v;
}
static double cotpi(double x) { return std::cos(M_PI * x) / std::sin(M_PI * x); }  // cot(pi x)

// ------------------------------------------------------------------ plan
enum Stage { ST_COMM_S, ST_NEAR, ST_M2M, ST_COMM_M, ST_TOP, ST_DOWN, ST_PFFT, ST_A2A, ST_MFFT, ST_COUNT };
static const char* kStageNames[ST_COUNT] = {"comm_S", "near_up", "m2m", "comm_M", "top",
                                            "down", "post_pfft", "a2a", "mfft"};

struct RankBufs {
    int g = 0;
    void* Tn = nullptr;      // [nb][M_L][P]   S2T output (T_near)
    void* tmp = nullptr;     // M-FFT ping-pong buffer
    void* W = nullptr;       // [k2][Mg]       P-FFT output = all-to-all send buffer
    void* Rcv = nullptr;     // all-to-all receive buffer (G > 1)
    void* haloL = nullptr;   // S box -1  (G > 1)
    void* haloR = nullptr;   // S box nb  (G > 1)
    void* r = nullptr;       // [P] reductions
    void* din = nullptr;     // execute_host staging
    void* dout = nullptr;
    std::vector<void*> Mpad, Lloc, Mfull, Lfull;   // indexed by level
};

}  // namespace fmmfft

struct fmmfft_plan_s {
    long long N = 0, M = 0, Mg = 0;
    int P = 0, G = 0, B = 0, Q = 0, M_L = 0, L = 0, lg = 0, nb = 0;
    fmmfft_precision_t prec = FMMFFT_C64;
    unsigned flags = 0;
    bool virt = false;
    int device = -1;
    size_t esz = 0, rsz = 0;
    // device tables
    void* s2m = nullptr;
    void* m2m = nullptr;
    void* s2t = nullptr;
    void* rho = nullptr;
    void* m2lB = nullptr;
    std::vector<void*> m2l;          // by level
    std::vector<fmmfft::RankBufs> ranks;
    std::vector<int> radices;        // M-FFT passes
    size_t ws_bytes = 0;
    int kernels = 0;
    cudaEvent_t ev[fmmfft::ST_COUNT + 1] = {};
    cudaStream_t last_stream = nullptr;
    bool have_times = false;
    std::vector<void*> allocs;
};

namespace fmmfft {

static fmmfft_status_t dalloc(fmmfft_plan_s* p, void** ptr, size_t bytes) {
    if (bytes == 0) bytes = 16;
    cudaError_t e = cudaMalloc(ptr, bytes);
    if (e != cudaSuccess) return fail(FMMFFT_ALLOC_FAILED, "cudaMalloc(%zu) failed: %s", bytes, cudaGetErrorString(e));
    p->allocs.push_back(*ptr);
    p->ws_bytes += bytes;
    CUDA_TRY(cudaMemset(*ptr, 0, bytes));
    return FMMFFT_SUCCESS;
}

template <typename R>
static fmmfft_status_t upload(fmmfft_plan_s* p, void** dst, const std::vector<double>& v) {
    std::vector<R> h(v.begin(), v.end());
    fmmfft_status_t st = dalloc(p, dst, h.size() * sizeof(R));
    if (st) return st;
    CUDA_TRY(cudaMemcpy(*dst, h.data(), h.size() * sizeof(R), cudaMemcpyHostToDevice));
    return FMMFFT_SUCCESS;
}

static int ilog2(long long v) { int l = 0; while ((1LL << l) < v) ++l; return l; }
static bool pow2(long long v) { return v > 0 && (v & (v - 1)) == 0; }

template <typename R>
static fmmfft_status_t build_tables(fmmfft_plan_s* p) {
    const int Q = p->Q, M_L = p->M_L, P = p->P;
    const long long N = p->N;
    const auto z = cheb_nodes(Q);
    fmmfft_status_t st;
    // S2M_{qm} = l_q(s_m), s_m = -1 + (2m+1)/M_L; L2T = S2M^T
    std::vector<double> s2m((size_t)Q * M_L);
    for (int q = 0; q < Q; ++q)
        for (int m = 0; m < M_L; ++m) s2m[(size_t)q * M_L + m] = lagr(z, q, -1.0 + (2.0 * m + 1.0) / M_L);
    if ((st = upload<R>(p, &p->s2m, s2m))) return st;
    // M2M = [M2M^- M2M^+], M2M^{-+}_{qk} = l_q((z_k -+ 1)/2); L2L = M2M^T
    std::vector<double> m2m((size_t)Q * 2 * Q);
    for (int q = 0; q < Q; ++q)
        for (int k = 0; k < 2 * Q; ++k)
            m2m[(size_t)q * 2 * Q + k] = lagr(z, q, (z[k % Q] + (k < Q ? -1.0 : 1.0)) / 2.0);
    if ((st = upload<R>(p, &p->m2m, m2m))) return st;
    // S2T_{pk} = cot(pi (p + P k)/N), p > 0; delta_{k0} for p = 0, layout [k][p]
    const int nK = 4 * M_L - 1;
    std::vector<double> s2t((size_t)nK * P, 0.0);
    for (int ki = 0; ki < nK; ++ki) {
        const long long k = ki - (2 * M_L - 1);
        for (int pp = 0; pp < P; ++pp)
            s2t[(size_t)ki * P + pp] = pp == 0 ? (k == 0 ? 1.0 : 0.0) : cotpi((double)(pp + (long long)P * k) / (double)N);
    }
    if ((st = upload<R>(p, &p->s2t, s2t))) return st;
    // M2L^l_{pijs} = cot(pi/2^l (z_j/2 - z_i/2 + s) + pi p/N) for FMM p (slot = p),
    // layout [s][i][j][p]; s in {-3, -2, 2, 3} for l > B, and 2..2^B-2 at the base
    p->m2l.assign(p->L + 1, nullptr);
    const int shifts[4] = {-3, -2, 2, 3};
    for (int lev = p->B; lev <= p->L; ++lev) {
        const bool base = lev == p->B;
        const int ns = base ? (1 << p->B) - 3 : 4;
        std::vector<double> t((size_t)ns * Q * Q * P, 0.0);
        for (int si = 0; si < ns; ++si) {
            const int s = base ? 2 + si : shifts[si];
            for (int i = 0; i < Q; ++i)
                for (int j = 0; j < Q; ++j)
                    for (int pp = 1; pp < P; ++pp)
                        t[(((size_t)si * Q + i) * Q + j) * P + pp] =
                            cotpi((z[j] / 2 - z[i] / 2 + s) / (double)(1LL << lev) + (double)pp / (double)N);
        }
        if ((st = upload<R>(p, base ? &p->m2lB : &p->m2l[lev], t))) return st;
    }
    // rho_p = exp(-i pi p/P) sin(pi p/P) / M, interleaved complex; rho_0 unused
    std::vector<double> rho(2 * (size_t)P);
    for (int pp = 0; pp < P; ++pp) {
        const double sn = std::sin(M_PI * pp / P) / (double)p->M;
        rho[2 * pp] = pp ? std::cos(M_PI * pp / P) * sn : 1.0;
        rho[2 * pp + 1] = pp ? -std::sin(M_PI * pp / P) * sn : 0.0;
    }
    return upload<R>(p, &p->rho, rho);
}

static constexpr int kTileF = 8192, kTileD = 4096;   // shared FFT tile (elements)

static void plan_radices(fmmfft_plan_s* p) {
    const int maxbits = p->prec == FMMFFT_C64 ? 10 : 9;
    const int bits = ilog2(p->M);
    const int n = std::max(1, (bits + maxbits - 1) / maxbits);
    p->radices.clear();
    int left = bits;
    for (int i = 0; i < n; ++i) {
        const int b = (left + (n - i) - 1) / (n - i);
        p->radices.push_back(1 << b);
        left -= b;
    }
}

static fmmfft_status_t alloc_rank(fmmfft_plan_s* p, RankBufs& rb) {
    const size_t e = p->esz;
    const long long n_local = p->N / p->G;
    const size_t QP = (size_t)p->Q * p->P;
    fmmfft_status_t st;
    if ((st = dalloc(p, &rb.Tn, n_local * e))) return st;
    if ((st = dalloc(p, &rb.W, n_local * e))) return st;
    if ((st = dalloc(p, &rb.tmp, n_local * e))) return st;
    if (p->G > 1) {
        if ((st = dalloc(p, &rb.Rcv, n_local * e))) return st;
        if ((st = dalloc(p, &rb.haloL, (size_t)p->M_L * p->P * e))) return st;
        if ((st = dalloc(p, &rb.haloR, (size_t)p->M_L * p->P * e))) return st;
    }
    if ((st = dalloc(p, &rb.r, (size_t)p->P * e))) return st;
    rb.Mpad.assign(p->L + 1, nullptr);
    rb.Lloc.assign(p->L + 1, nullptr);
    rb.Mfull.assign(p->L + 1, nullptr);
    rb.Lfull.assign(p->L + 1, nullptr);
    for (int lev = p->lg; lev <= p->L; ++lev) {
        const long long nbl = (1LL << lev) / p->G;
        if ((st = dalloc(p, &rb.Mpad[lev], (nbl + 4) * QP * e))) return st;
        if ((st = dalloc(p, &rb.Lloc[lev], nbl * QP * e))) return st;
    }
    for (int lev = p->B; lev <= p->lg; ++lev) {
        if (p->G == 1 && lev == p->lg) {
            rb.Mfull[lev] = (char*)rb.Mpad[lev] + 2 * QP * e;     // G = 1: the "gather" is the identity
        } else if ((st = dalloc(p, &rb.Mfull[lev], ((size_t)1 << lev) * QP * e))) {
            return st;
        }
        if (lev < p->lg && (st = dalloc(p, &rb.Lfull[lev], ((size_t)1 << lev) * QP * e))) return st;
    }
    return FMMFFT_SUCCESS;
}

static void destroy_plan(fmmfft_plan_s* p) {
    for (void* a : p->allocs) cudaFree(a);
    for (auto& ev : p->ev)
        if (ev) cudaEventDestroy(ev);
    delete p;
}

static int count_kernels(const fmmfft_plan_s* p) {
    int k = 1;                          // near_up
    k += p->L - p->lg;                  // m2m (distributed levels)
    k += p->lg - p->B;                  // m2m on the gathered top
    k += 2;                             // base M2L + reduce
    k += p->lg - p->B;                  // replicated down levels
    k += p->L - p->lg;                  // distributed down levels
    k += 1;                             // post_pfft
    k += (int)p->radices.size();        // M-FFT passes
    return k * (p->virt ? p->G : 1);
}

// ------------------------------------------------------------------ execute
template <typename R>
struct Exec {
    using C = C2<R>;
    fmmfft_plan_s* p;
    cudaStream_t s;
    std::vector<const C*> in;    // per rank
    std::vector<C*> out;

    static constexpr int IB = sizeof(R) == 4 ? 16 : 8;
    static constexpr int EPT = sizeof(R) == 4 ? 32 : 16;
    static constexpr int TILE = sizeof(R) == 4 ? kTileF : kTileD;
    int PC() const { return std::min(p->P, sizeof(R) == 4 ? 32 : 16); }
    size_t QP() const { return (size_t)p->Q * p->P; }
    int nb_at(int lev) const { return (int)((1LL << lev) / p->G); }
    C* interior(void* pad) const { return (C*)pad + 2 * QP(); }
    ncclDataType_t nt() const { return sizeof(R) == 4 ? ncclFloat : ncclDouble; }

    fmmfft_status_t mark(int stage) {
        if (p->flags & FMMFFT_FLAG_PROFILE) CUDA_TRY(cudaEventRecord(p->ev[stage], s));
        return FMMFFT_SUCCESS;
    }

    // ---- comm_S: S halo (line 2)
    fmmfft_status_t comm_S() {
        if (p->G == 1) return FMMFFT_SUCCESS;
        const size_t box = (size_t)p->M_L * p->P;
        const int G = p->G;
        if (p->virt) {
            for (int g = 0; g < G; ++g) {
                RankBufs& rb = p->ranks[g];
                const C* left = in[(g - 1 + G) % G];
                const C* right = in[(g + 1) % G];
                CUDA_TRY(cudaMemcpyAsync(rb.haloL, left + (size_t)(p->nb - 1) * box, box * sizeof(C), cudaMemcpyDeviceToDevice, s));
                CUDA_TRY(cudaMemcpyAsync(rb.haloR, right, box * sizeof(C), cudaMemcpyDeviceToDevice, s));
            }
            return FMMFFT_SUCCESS;
        }
        RankBufs& rb = p->ranks[0];
        const int g = g_comm.rank, lf = (g - 1 + G) % G, rt = (g + 1) % G;
        NcclApi& n = nccl();
        NCCL_TRY(n.GroupStart());
        NCCL_TRY(n.Send(in[0], 2 * box, nt(), lf, g_comm.comm, s));
        NCCL_TRY(n.Send(in[0] + (size_t)(p->nb - 1) * box, 2 * box, nt(), rt, g_comm.comm, s));
        NCCL_TRY(n.Recv(rb.haloR, 2 * box, nt(), rt, g_comm.comm, s));
        NCCL_TRY(n.Recv(rb.haloL, 2 * box, nt(), lf, g_comm.comm, s));
        NCCL_TRY(n.GroupEnd());
        return FMMFFT_SUCCESS;
    }

    // ---- near_up: S2T + S2M
    fmmfft_status_t near_up() {
        const int PC_ = PC(), nib = p->M_L / IB;
        const int threads = PC_ * nib;
        const int npc = p->P / PC_;
        const int target = 2 * 148 * 2;
        const int bpc = std::max(1, (int)((long long)p->nb * npc / target));
        const dim3 grid((p->nb + bpc - 1) / bpc, npc);
        const size_t smem = (size_t)3 * p->M_L * PC_ * sizeof(C) + (size_t)(4 * p->M_L - 1) * PC_ * sizeof(R) +
                            (size_t)p->Q * p->M_L * sizeof(R);
        CUDA_TRY(cudaFuncSetAttribute(k_near_up<R, IB>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
        for (RankBufs& rb : p->ranks) {
            const C* S = in[p->virt ? rb.g : 0];
            const size_t box = (size_t)p->M_L * p->P;
            const C* hl = p->G == 1 ? S + (size_t)(p->nb - 1) * box : (const C*)rb.haloL;
            const C* hr = p->G == 1 ? S : (const C*)rb.haloR;
            k_near_up<R, IB><<<grid, threads, smem, s>>>(S, hl, hr, (C*)rb.Tn, interior(rb.Mpad[p->L]),
                                                       (const R*)p->s2t, (const R*)p->s2m, p->P, p->M_L,
                                                       p->Q, p->nb, bpc, PC_);
            LAUNCH_CHECK();
        }
        return FMMFFT_SUCCESS;
    }

    fmmfft_status_t launch_m2m(const C* inl, C* outl, int nb_out) {
        const long long total = (long long)nb_out * QP();
        const int threads = 256;
        const int blocks = (int)std::min<long long>((total + threads - 1) / threads, 148LL * 16);
        const size_t smem = (size_t)2 * p->Q * p->Q * sizeof(R);
        k_m2m<R><<<blocks, threads, smem, s>>>(inl, outl, (const R*)p->m2m, p->P, p->Q, nb_out);
        LAUNCH_CHECK();
        return FMMFFT_SUCCESS;
    }

    // ---- m2m on own boxes, l = L-1 .. l_g
    fmmfft_status_t m2m_local() {
        fmmfft_status_t st;
        for (int lev = p->L - 1; lev >= p->lg; --lev)
            for (RankBufs& rb : p->ranks)
                if ((st = launch_m2m(interior(rb.Mpad[lev + 1]), interior(rb.Mpad[lev]), nb_at(lev)))) return st;
        return FMMFFT_SUCCESS;
    }

    // ---- comm_M: halos (2 boxes per side) for l in (l_g, L] and all-gather of level l_g
    fmmfft_status_t comm_M() {
        if (p->G == 1) return FMMFFT_SUCCESS;
        const size_t QPc = QP();
        const int G = p->G;
        const long long nlg = nb_at(p->lg);
        if (p->virt) {
            for (int g = 0; g < G; ++g) {
                RankBufs& rb = p->ranks[g];
                RankBufs& lf = p->ranks[(g - 1 + G) % G];
                RankBufs& rt = p->ranks[(g + 1) % G];
                for (int lev = p->lg + 1; lev <= p->L; ++lev) {
                    const int nbl = nb_at(lev);
                    CUDA_TRY(cudaMemcpyAsync(rb.Mpad[lev], (C*)lf.Mpad[lev] + (size_t)nbl * QPc, 2 * QPc * sizeof(C), cudaMemcpyDeviceToDevice, s));
                    CUDA_TRY(cudaMemcpyAsync((C*)rb.Mpad[lev] + (size_t)(nbl + 2) * QPc, (C*)rt.Mpad[lev] + 2 * QPc, 2 * QPc * sizeof(C), cudaMemcpyDeviceToDevice, s));
                }
                for (int src = 0; src < G; ++src)
                    CUDA_TRY(cudaMemcpyAsync((C*)rb.Mfull[p->lg] + (size_t)src * nlg * QPc, interior(p->ranks[src].Mpad[p->lg]),
                                             nlg * QPc * sizeof(C), cudaMemcpyDeviceToDevice, s));
            }
            return FMMFFT_SUCCESS;
        }
        RankBufs& rb = p->ranks[0];
        const int g = g_comm.rank, lf = (g - 1 + G) % G, rt = (g + 1) % G;
        NcclApi& n = nccl();
        NCCL_TRY(n.GroupStart());
        for (int lev = p->lg + 1; lev <= p->L; ++lev) {
            const int nbl = nb_at(lev);
            C* pad = (C*)rb.Mpad[lev];
            NCCL_TRY(n.Send(pad + 2 * QPc, 4 * QPc, nt(), lf, g_comm.comm, s));              // own boxes 0,1 -> left
            NCCL_TRY(n.Send(pad + (size_t)nbl * QPc, 4 * QPc, nt(), rt, g_comm.comm, s));    // own boxes nb-2, nb-1 -> right
            NCCL_TRY(n.Recv(pad + (size_t)(nbl + 2) * QPc, 4 * QPc, nt(), rt, g_comm.comm, s));
            NCCL_TRY(n.Recv(pad, 4 * QPc, nt(), lf, g_comm.comm, s));
        }
        NCCL_TRY(n.GroupEnd());
        NCCL_TRY(n.AllGather(interior(rb.Mpad[p->lg]), rb.Mfull[p->lg], 2 * nlg * QPc, nt(), g_comm.comm, s));
        return FMMFFT_SUCCESS;
    }

    fmmfft_status_t launch_down(const C* src, long long src_base, int src_mod, const C* parent, long long par_base,
                                C* outp, long long tgt_base, int ntg, int lev) {
        const bool base = lev == p->B;
        const int nshift = base ? (1 << p->B) - 3 : 3;
        const R* tab = (const R*)(base ? p->m2lB : p->m2l[lev]);
        const long long total = (long long)ntg * QP();
        const int threads = 256;
        const int blocks = (int)std::min<long long>((total + threads - 1) / threads, 148LL * 16);
        const size_t smem = (size_t)2 * p->Q * p->Q * sizeof(R);
        k_down<R><<<blocks, threads, smem, s>>>(src, src_base, src_mod, parent, par_base, outp, tgt_base, ntg, tab, nshift,
                                                base ? 1 : 0, 1 << p->B, (const R*)p->m2m, p->P, p->Q);
        LAUNCH_CHECK();
        return FMMFFT_SUCCESS;
    }

    // ---- top: replicated levels l_g .. B
    fmmfft_status_t top() {
        fmmfft_status_t st;
        for (RankBufs& rb : p->ranks) {
            const int g = p->virt ? rb.g : g_comm.rank * (p->G > 1);
            for (int lev = p->lg - 1; lev >= p->B; --lev)
                if ((st = launch_m2m((C*)rb.Mfull[lev + 1], (C*)rb.Mfull[lev], 1 << lev))) return st;
            // M2L-B: targets = own boxes if l_g == B, else all 2^B boxes
            if (p->lg == p->B) {
                if ((st = launch_down((C*)rb.Mfull[p->B], 0, 1 << p->B, nullptr, 0, (C*)rb.Lloc[p->B],
                                      (long long)g * nb_at(p->B), nb_at(p->B), p->B))) return st;
            } else {
                if ((st = launch_down((C*)rb.Mfull[p->B], 0, 1 << p->B, nullptr, 0, (C*)rb.Lfull[p->B], 0, 1 << p->B, p->B)))
                    return st;
            }
            k_reduce<R><<<(p->P + 127) / 128, 128, 0, s>>>((C*)rb.Mfull[p->B], (C*)rb.r, p->P, p->Q, 1 << p->B);
            LAUNCH_CHECK();
            for (int lev = p->B + 1; lev <= p->lg; ++lev) {
                if (lev < p->lg) {
                    if ((st = launch_down((C*)rb.Mfull[lev], 0, 1 << lev, (C*)rb.Lfull[lev - 1], 0, (C*)rb.Lfull[lev], 0,
                                          1 << lev, lev))) return st;
                } else {
                    if ((st = launch_down((C*)rb.Mfull[lev], 0, 1 << lev, (C*)rb.Lfull[lev - 1], 0, (C*)rb.Lloc[lev],
                                          (long long)g * nb_at(lev), nb_at(lev), lev))) return st;
                }
            }
        }
        return FMMFFT_SUCCESS;
    }

    // ---- down: distributed levels l_g+1 .. L
    fmmfft_status_t down() {
        fmmfft_status_t st;
        for (int lev = p->lg + 1; lev <= p->L; ++lev) {
            for (RankBufs& rb : p->ranks) {
                const int g = p->virt ? rb.g : g_comm.rank * (p->G > 1);
                const long long nbl = nb_at(lev), nbp = nb_at(lev - 1);
                const C* src;
                long long src_base;
                int mod;
                if (p->G == 1) { src = interior(rb.Mpad[lev]); src_base = 0; mod = 1 << lev; }
                else { src = (C*)rb.Mpad[lev]; src_base = g * nbl - 2; mod = 0; }
                if ((st = launch_down(src, src_base, mod, (C*)rb.Lloc[lev - 1], g * nbp, (C*)rb.Lloc[lev], g * nbl, (int)nbl,
                                      lev))) return st;
            }
        }
        return FMMFFT_SUCCESS;
    }

    // ---- L2T + POST + P-FFT
    fmmfft_status_t post_pfft() {
        const int MS = std::min(p->M_L, std::max(1, TILE / p->P));
        const size_t smem = (size_t)MS * (p->P + 1) * sizeof(C) + (size_t)p->P * sizeof(C) + (size_t)p->Q * MS * sizeof(R);
        CUDA_TRY(cudaFuncSetAttribute(k_post_pfft<R, EPT>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
        const int blocks = p->nb * (p->M_L / MS);
        for (RankBufs& rb : p->ranks) {
            k_post_pfft<R, EPT><<<blocks, 256, smem, s>>>((const C*)rb.Tn, (const C*)rb.Lloc[p->L], (const C*)rb.r,
                                                         (const C*)p->rho, (const R*)p->s2m, (C*)rb.W, p->P, p->M_L, p->Q, MS,
                                                         p->Mg);
            LAUNCH_CHECK();
        }
        return FMMFFT_SUCCESS;
    }

    // ---- the all-to-all: chunk r of W (k2 in r's block, own m) -> rank r's Rcv slot g
    fmmfft_status_t a2a() {
        if (p->G == 1) return FMMFFT_SUCCESS;
        const int G = p->G;
        const size_t chunk = (size_t)(p->P / G) * p->Mg;
        if (p->virt) {
            for (int r = 0; r < G; ++r)
                for (int src = 0; src < G; ++src)
                    CUDA_TRY(cudaMemcpyAsync((C*)p->ranks[r].Rcv + src * chunk, (C*)p->ranks[src].W + r * chunk,
                                             chunk * sizeof(C), cudaMemcpyDeviceToDevice, s));
            return FMMFFT_SUCCESS;
        }
        RankBufs& rb = p->ranks[0];
        NcclApi& n = nccl();
        NCCL_TRY(n.GroupStart());
        for (int r = 0; r < G; ++r) {
            NCCL_TRY(n.Send((C*)rb.W + r * chunk, 2 * chunk, nt(), r, g_comm.comm, s));
            NCCL_TRY(n.Recv((C*)rb.Rcv + r * chunk, 2 * chunk, nt(), r, g_comm.comm, s));
        }
        NCCL_TRY(n.GroupEnd());
        return FMMFFT_SUCCESS;
    }

    // ---- M-point FFTs over the P/G local rows
    fmmfft_status_t mfft() {
        const int n = (int)p->radices.size();
        const long long rows = p->P / p->G;
        for (RankBufs& rb : p->ranks) {
            C* dst = out[p->virt ? rb.g : 0];
            const C* src = (const C*)(p->G > 1 ? rb.Rcv : rb.W);
            long long Ns = 1;
            for (int i = 0; i < n; ++i) {
                const int Rp = p->radices[i];
                C* o = ((n - 1 - i) % 2 == 0) ? dst : (C*)rb.tmp;
                const long long nj = p->M / Rp;
                int c = (int)std::min<long long>(TILE / Rp, nj);
                while (c > 8 && (nj / c) * rows < 2 * 148) c /= 2;
                long long in_row = p->M, blk = p->M, blk_stride = 0;
                if (i == 0 && p->G > 1) {
                    in_row = p->Mg; blk = p->Mg; blk_stride = (long long)(p->P / p->G) * p->Mg;
                    c = (int)std::min<long long>(c, p->Mg);
                }
                const size_t smem = (size_t)c * (Rp + 1) * sizeof(C) + (size_t)Rp * sizeof(C);
                CUDA_TRY(cudaFuncSetAttribute(k_fft_pass<R, EPT>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
                const dim3 grid((unsigned)(nj / c), (unsigned)rows);
                k_fft_pass<R, EPT><<<grid, 256, smem, s>>>(src, o, p->M, Rp, Ns, c, in_row, blk, blk_stride);
                LAUNCH_CHECK();
                src = o;
                Ns *= Rp;
            }
        }
        return FMMFFT_SUCCESS;
    }

    fmmfft_status_t run() {
        fmmfft_status_t st;
#define STEP(stage, call) if ((st = mark(stage))) return st; if ((st = call)) return st;
        STEP(ST_COMM_S, comm_S())
        STEP(ST_NEAR, near_up())
        STEP(ST_M2M, m2m_local())
        STEP(ST_COMM_M, comm_M())
        STEP(ST_TOP, top())
        STEP(ST_DOWN, down())
        STEP(ST_PFFT, post_pfft())
        STEP(ST_A2A, a2a())
        STEP(ST_MFFT, mfft())
#undef STEP
        return mark(ST_COUNT);
    }
};

template <typename R>
static fmmfft_status_t execute_t(fmmfft_plan_s* p, const void* in, void* out, cudaStream_t s) {
    Exec<R> ex{p, s, {}, {}};
    const long long nl = p->N / p->G;
    if (p->virt) {
        for (int g = 0; g < p->G; ++g) {
            ex.in.push_back((const C2<R>*)in + g * nl);
            ex.out.push_back((C2<R>*)out + g * nl);
        }
    } else {
        ex.in.push_back((const C2<R>*)in);
        ex.out.push_back((C2<R>*)out);
    }
    fmmfft_status_t st = ex.run();
    p->last_stream = s;
    p->have_times = st == FMMFFT_SUCCESS && (p->flags & FMMFFT_FLAG_PROFILE);
    return st;
}

}  // namespace fmmfft

using namespace fmmfft;

// ====================================================================== C ABI
extern "C" {

const char* fmmfft_last_error(void) { return g_last_error.c_str(); }
const char* fmmfft_version(void) { return "fmmfft-b200 0.1 (sm_100a)"; }
const char* fmmfft_stage_name(int i) { return (i >= 0 && i < ST_COUNT) ? kStageNames[i] : ""; }

fmmfft_status_t fmmfft_get_unique_id(unsigned char id[128]) {
    if (!id) return fail(FMMFFT_INVALID_VALUE, "id is NULL");
    NcclApi& n = nccl();
    if (!n.ok) return fail(FMMFFT_NCCL_ERROR, "NCCL unavailable: %s", n.err.c_str());
    ncclUniqueId u;
    NCCL_TRY(n.GetUniqueId(&u));
    static_assert(sizeof(u.internal) == 128, "NCCL unique id size");
    memcpy(id, u.internal, 128);
    return FMMFFT_SUCCESS;
}

fmmfft_status_t fmmfft_comm_init(int rank, int G, const unsigned char id[128]) {
    if (!id || G < 1 || rank < 0 || rank >= G) return fail(FMMFFT_INVALID_VALUE, "bad rank/G/id (rank=%d G=%d)", rank, G);
    NcclApi& n = nccl();
    if (!n.ok) return fail(FMMFFT_NCCL_ERROR, "NCCL unavailable: %s", n.err.c_str());
    if (g_comm.comm) return fail(FMMFFT_INVALID_VALUE, "communicator already initialised");
    ncclUniqueId u;
    memcpy(u.internal, id, 128);
    int dev = 0;
    CUDA_TRY(cudaGetDevice(&dev));
    NCCL_TRY(n.CommInitRank(&g_comm.comm, G, u, rank));
    g_comm.rank = rank;
    g_comm.size = G;
    g_comm.device = dev;
    return FMMFFT_SUCCESS;
}

fmmfft_status_t fmmfft_comm_destroy(void) {
    if (!g_comm.comm) return FMMFFT_SUCCESS;
    NCCL_TRY(nccl().CommDestroy(g_comm.comm));
    g_comm = Comm{};
    return FMMFFT_SUCCESS;
}

fmmfft_status_t fmmfft_plan_ex(fmmfft_plan_t* plan, long long N, int P, int G, int B, int Q,
                               fmmfft_precision_t precision, int M_L, unsigned flags) {
    if (!plan) return fail(FMMFFT_INVALID_VALUE, "plan is NULL");
    *plan = nullptr;
    if (precision != FMMFFT_C64 && precision != FMMFFT_C128) return fail(FMMFFT_INVALID_VALUE, "bad precision");
    if (!pow2(N) || !pow2(P) || !pow2(M_L)) return fail(FMMFFT_INVALID_VALUE, "N, P, M_L must be powers of two");
    if (P < 2 || P > 2048) return fail(FMMFFT_INVALID_VALUE, "need 2 <= P <= 2048 (P=%d)", P);
    if (!(G == 1 || G == 2 || G == 4 || G == 8)) return fail(FMMFFT_INVALID_VALUE, "G must be 1, 2, 4 or 8");
    if (P % G) return fail(FMMFFT_INVALID_VALUE, "P %% G != 0");
    if (M_L < 16 || M_L > 128) return fail(FMMFFT_INVALID_VALUE, "need 16 <= M_L <= 128");
    if (Q < 2 || Q > 32) return fail(FMMFFT_INVALID_VALUE, "need 2 <= Q <= 32");
    if (N % ((long long)P * M_L)) return fail(FMMFFT_INVALID_VALUE, "N must be a multiple of P*M_L");
    const long long nleaf = N / ((long long)P * M_L);
    const int L = ilog2(nleaf);
    if (B < 2 || L < B) return fail(FMMFFT_INVALID_VALUE, "need L >= B >= 2 (L=%d, B=%d)", L, B);
    if (B > 10) return fail(FMMFFT_UNSUPPORTED, "B > 10 not supported");
    if (nleaf % G) return fail(FMMFFT_INVALID_VALUE, "2^L %% G != 0");
    const bool virt = (flags & FMMFFT_FLAG_VIRTUAL) != 0;
    if (G > 1 && !virt) {
        if (!g_comm.comm) return fail(FMMFFT_NOT_INITIALIZED, "G > 1 needs fmmfft_comm_init");
        if (g_comm.size != G) return fail(FMMFFT_INVALID_VALUE, "G=%d differs from the communicator size %d", G, g_comm.size);
    }
    int dev = 0;
    CUDA_TRY(cudaGetDevice(&dev));
    cudaDeviceProp prop;
    CUDA_TRY(cudaGetDeviceProperties(&prop, dev));
    if (prop.major != 10 || prop.minor != 0)
        return fail(FMMFFT_UNSUPPORTED, "device %s is sm_%d%d; this build is sm_100a only", prop.name, prop.major, prop.minor);

    fmmfft_plan_s* p = new fmmfft_plan_s;
    p->N = N; p->P = P; p->G = G; p->B = B; p->Q = Q; p->M_L = M_L; p->L = L;
    p->M = N / P; p->Mg = p->M / G; p->prec = precision; p->flags = flags; p->virt = virt; p->device = dev;
    p->nb = (int)(nleaf / G);
    p->lg = std::min(std::max(B, ilog2(G) + 1), L);
    if (G == 1) p->lg = B;
    p->esz = precision == FMMFFT_C64 ? 8 : 16;
    p->rsz = p->esz / 2;
    plan_radices(p);
    fmmfft_status_t st = precision == FMMFFT_C64 ? build_tables<float>(p) : build_tables<double>(p);
    if (!st) {
        const int nr = virt ? G : 1;
        p->ranks.resize(nr);
        for (int g = 0; g < nr && !st; ++g) {
            p->ranks[g].g = virt ? g : (G > 1 ? g_comm.rank : 0);
            st = alloc_rank(p, p->ranks[g]);
        }
    }
    if (!st && (flags & FMMFFT_FLAG_PROFILE)) {
        for (auto& ev : p->ev) {
            cudaError_t e = cudaEventCreate(&ev);
            if (e != cudaSuccess) { st = fail(FMMFFT_CUDA_ERROR, "cudaEventCreate: %s", cudaGetErrorString(e)); break; }
        }
    }
    if (!st) {
        cudaError_t e = cudaDeviceSynchronize();
        if (e != cudaSuccess) st = fail(FMMFFT_CUDA_ERROR, "plan setup: %s", cudaGetErrorString(e));
    }
    if (st) { destroy_plan(p); return st; }
    p->kernels = count_kernels(p);
    *plan = p;
    return FMMFFT_SUCCESS;
}

fmmfft_status_t fmmfft_plan(fmmfft_plan_t* plan, long long N, int P, int G, int B, int Q, fmmfft_precision_t precision) {
    return fmmfft_plan_ex(plan, N, P, G, B, Q, precision, 64, 0u);
}

fmmfft_status_t fmmfft_execute(fmmfft_plan_t p, const void* in, void* out, void* stream) {
    if (!p) return fail(FMMFFT_INVALID_VALUE, "plan is NULL");
    if (!in || !out) return fail(FMMFFT_INVALID_VALUE, "in/out is NULL");
    const size_t bytes = (size_t)(p->virt ? p->N : p->N / p->G) * p->esz;
    const char* a = (const char*)in;
    const char* b = (const char*)out;
    if (a < b + bytes && b < a + bytes) return fail(FMMFFT_INVALID_VALUE, "in and out overlap");
    if (((uintptr_t)in | (uintptr_t)out) & 15) return fail(FMMFFT_INVALID_VALUE, "in/out must be 16-byte aligned");
    cudaPointerAttributes at;
    if (cudaPointerGetAttributes(&at, in) != cudaSuccess || at.type != cudaMemoryTypeDevice ||
        cudaPointerGetAttributes(&at, out) != cudaSuccess || at.type != cudaMemoryTypeDevice) {
        cudaGetLastError();
        return fail(FMMFFT_INVALID_VALUE, "in/out must be device pointers");
    }
    cudaStream_t s = (cudaStream_t)stream;
    return p->prec == FMMFFT_C64 ? execute_t<float>(p, in, out, s) : execute_t<double>(p, in, out, s);
}

fmmfft_status_t fmmfft_execute_host(fmmfft_plan_t p, const void* in_host, void* out_host, void* stream) {
    if (!p || !in_host || !out_host) return fail(FMMFFT_INVALID_VALUE, "NULL argument");
    const size_t bytes = (size_t)(p->virt ? p->N : p->N / p->G) * p->esz;
    RankBufs& rb = p->ranks[0];
    if (!rb.din) {
        fmmfft_status_t st;
        if ((st = dalloc(p, &rb.din, bytes))) return st;
        if ((st = dalloc(p, &rb.dout, bytes))) return st;
    }
    cudaStream_t s = (cudaStream_t)stream;
    CUDA_TRY(cudaMemcpyAsync(rb.din, in_host, bytes, cudaMemcpyHostToDevice, s));
    fmmfft_status_t st = p->prec == FMMFFT_C64 ? execute_t<float>(p, rb.din, rb.dout, s) : execute_t<double>(p, rb.din, rb.dout, s);
    if (st) return st;
    CUDA_TRY(cudaMemcpyAsync(out_host, rb.dout, bytes, cudaMemcpyDeviceToHost, s));
    return FMMFFT_SUCCESS;
}

fmmfft_status_t fmmfft_destroy(fmmfft_plan_t p) {
    if (!p) return FMMFFT_SUCCESS;
    cudaDeviceSynchronize();
    destroy_plan(p);
    return FMMFFT_SUCCESS;
}

fmmfft_status_t fmmfft_get_info(fmmfft_plan_t p, fmmfft_info_t* info) {
    if (!p || !info) return fail(FMMFFT_INVALID_VALUE, "NULL argument");
    info->N = p->N; info->P = p->P; info->G = p->G; info->B = p->B; info->Q = p->Q; info->M_L = p->M_L;
    info->L = p->L; info->precision = p->prec; info->M = p->M; info->level_gather = p->lg;
    info->n_stages = ST_COUNT; info->workspace_bytes = p->ws_bytes; info->kernels_per_execute = p->kernels;
    return FMMFFT_SUCCESS;
}

fmmfft_status_t fmmfft_stage_times(fmmfft_plan_t p, float* ms, int n, int* n_out) {
    if (!p || !ms || !n_out) return fail(FMMFFT_INVALID_VALUE, "NULL argument");
    if (!(p->flags & FMMFFT_FLAG_PROFILE) || !p->have_times) return fail(FMMFFT_INVALID_VALUE, "plan not profiled / not executed");
    CUDA_TRY(cudaEventSynchronize(p->ev[ST_COUNT]));
    const int k = std::min(n, (int)ST_COUNT);
    for (int i = 0; i < k; ++i) CUDA_TRY(cudaEventElapsedTime(&ms[i], p->ev[i], p->ev[i + 1]));
    *n_out = k;
    return FMMFFT_SUCCESS;
}

fmmfft_status_t fmmfft_debug_buffer(fmmfft_plan_t p, int rank, int which, int level, const void** ptr, size_t* bytes) {
    if (!p || !ptr || !bytes) return fail(FMMFFT_INVALID_VALUE, "NULL argument");
    if (rank < 0 || rank >= (int)p->ranks.size()) return fail(FMMFFT_INVALID_VALUE, "bad rank");
    RankBufs& rb = p->ranks[rank];
    const size_t nl = (size_t)(p->N / p->G), QP = (size_t)p->Q * p->P;
    switch (which) {
        case 0: *ptr = rb.Tn; *bytes = nl * p->esz; return FMMFFT_SUCCESS;
        case 3: *ptr = rb.W; *bytes = nl * p->esz; return FMMFFT_SUCCESS;
        case 4: *ptr = rb.r; *bytes = (size_t)p->P * p->esz; return FMMFFT_SUCCESS;
        case 1:
        case 2: {
            if (level < p->B || level > p->L) return fail(FMMFFT_INVALID_VALUE, "level out of range");
            if (level >= p->lg) {
                const size_t nbl = (size_t)((1LL << level) / p->G);
                *ptr = which == 1 ? (const void*)((char*)rb.Mpad[level] + 2 * QP * p->esz) : rb.Lloc[level];
                *bytes = nbl * QP * p->esz;
            } else {
                *ptr = which == 1 ? rb.Mfull[level] : rb.Lfull[level];
                *bytes = ((size_t)1 << level) * QP * p->esz;
            }
            return FMMFFT_SUCCESS;
        }
        default: return fail(FMMFFT_INVALID_VALUE, "bad buffer id");
    }
}

}  // extern "C"
