// fmmfft.cu — plan / execute orchestration and the C ABI of include/fmmfft.h.
//
// One process per GPU (NCCL over NVLink/NVSwitch between ranks), or G "virtual ranks" on one
// GPU with device-to-device copies standing in for NCCL (FMMFFT_FLAG_VIRTUAL, for testing the
// partitioned data flow). The stage sequence per execute is Algorithm 1
// followed by the distributed 2D FFT with its single all-to-all:
//
//   comm_S    S halo (line 2)                          NCCL send/recv | D2D | none (G = 1)
//   near_up   S2T + S2M (lines 1, 3)                   k_near_up
//   m2m       M2M for l = L-1 .. l_g (line 5)          k_up (up to 4 levels per launch)
//   comm_M    M^l halos for l > l_g (line 7) + all-gather of level l_g (line 9, reading R16)
//   top       M2M l_g-1 .. B on the gathered level, M2L-B (line 10) + REDUCE (line 11),
//             M2L + L2L for B < l <= l_g (replicated top of the tree)
//   down      M2L-l (line 8) + L2L (line 13) for l = l_g+1 .. L   k_tree_down + k_m2l_lvl
//   post_pfft L2T + POST + P-point FFTs + transposed store (lines 14-16)
//   a2a       the one all-to-all transpose (line 16)
//   mfft      P/G M-point FFTs, multi-pass Stockham (line 16)
//
// The whole sequence is captured once per (in, out) pair into a CUDA graph (on a plan-owned
// stream) and replayed on the caller's stream: one launch per execute instead of ~20.
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <atomic>
#include <mutex>
#include <string>
#include <type_traits>
#include <utility>
#include <vector>

#include "../../include/fmmfft.h"
#include "common.cuh"
#include "kernels_fft.cuh"
#include "kernels_fmm.cuh"
#include "kernel_s2t_tc.cuh"
#include "kernel_s2t_fft.cuh"
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

#define LAUNCH_CHECK() do { ++nlaunch; CUDA_TRY(cudaGetLastError()); } while (0)

// compile-time dispatch of a runtime value onto a list of template values
template <int... Vs, typename F>
static bool dispatch(int v, F&& f) {
    bool hit = false;
    ((v == Vs ? (f(std::integral_constant<int, Vs>{}), hit = true) : false), ...);
    return hit;
}

// Launch with programmatic dependent launch allowed: the kernel's CTAs may be scheduled while
// its stream predecessor drains (each kernel triggers griddepcontrol.launch_dependents at its start
// and waits in griddepcontrol.wait before touching the predecessor's results).
static bool g_pdl = [] {
    // Opt-in: measured on cfg2 (bench20) PDL cost 20 us/step (863 vs 1043 GFLOP/s) -- early
    // dependent CTAs park in griddepcontrol.wait on SMs the side-stream S2T needs.
    const char* e = getenv("FMMFFT_PDL");
    return e && e[0] == '1';
}();

template <typename... KArgs, typename... Args>
static cudaError_t launch_pdl(void (*kern)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t st, Args&&... args) {
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = grid;
    cfg.blockDim = block;
    cfg.dynamicSmemBytes = smem;
    cfg.stream = st;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = at;
    cfg.numAttrs = g_pdl ? 1 : 0;
    return cudaLaunchKernelEx(&cfg, kern, std::forward<Args>(args)...);
}

// Plain stream-ordered launch (for kernels whose CTAs fill an SM: launched early they would sit in
// griddepcontrol.wait holding the SMs their predecessor and the side stream need).
template <typename... KArgs, typename... Args>
static cudaError_t launch_plain(void (*kern)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t st, Args&&... args) {
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = grid;
    cfg.blockDim = block;
    cfg.dynamicSmemBytes = smem;
    cfg.stream = st;
    cfg.attrs = nullptr;
    cfg.numAttrs = 0;
    return cudaLaunchKernelEx(&cfg, kern, std::forward<Args>(args)...);
}

// Launch of a kernel with compile-time cluster dimensions, asking the scheduler to spread the
// cluster's CTAs over distinct SMs (small CTAs would otherwise be packed onto one SM).
template <typename... KArgs, typename... Args>
static cudaError_t launch_cluster(void (*kern)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t st, Args&&... args) {
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = grid;
    cfg.blockDim = block;
    cfg.dynamicSmemBytes = smem;
    cfg.stream = st;
    cudaLaunchAttribute at[2];
    at[0].id = cudaLaunchAttributeClusterSchedulingPolicyPreference;
    at[0].val.clusterSchedulingPolicyPreference = cudaClusterSchedulingPolicySpread;
    at[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[1].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = at;
    cfg.numAttrs = g_pdl ? 2 : 1;
    return cudaLaunchKernelEx(&cfg, kern, std::forward<Args>(args)...);
}

// makes `dev` current for a scope, restoring the caller's device on exit
struct DeviceGuard {
    int prev = -1;
    cudaError_t err = cudaSuccess;
    explicit DeviceGuard(int dev) {
        err = cudaGetDevice(&prev);
        if (err == cudaSuccess && prev != dev) err = cudaSetDevice(dev);
        else prev = -1;
    }
    ~DeviceGuard() { if (prev >= 0) cudaSetDevice(prev); }
};

// ------------------------------------------------------------------ communicator
struct Comm {
    ncclComm_t comm = nullptr;
    int rank = 0, size = 0, device = -1;
};
static Comm g_comm;
static std::atomic<int> g_comm_plans{0};    // live plans holding g_comm.comm (comm_destroy refuses)

// One point-to-point transfer of a rank's exchange, exactly the arguments of its ncclSend /
// ncclRecv (n complex elements). Every exchange (S halo, M^l halos, the all-to-all) is first
// written as the per-rank list of these; NCCL plans issue their own rank's list in one group,
// virtual plans execute every rank's list by matching the k-th send g -> q with the k-th receive
// at q from g (NCCL's in-order matching per peer pair), so the virtual data flow exercises the
// very pointer and count arithmetic the NCCL branch issues.
struct P2P { bool send; int peer; void* ptr; size_t n; };
struct Gather { const void* send; void* recv; size_t n; };    // ncclAllGather(send, recv, n)

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
// Stages on the main stream (consecutive events), plus S2T on the side stream (its own pair).
enum Stage { ST_COMM_S, ST_NEAR, ST_M2M, ST_COMM_M, ST_TOP, ST_DOWN, ST_PFFT, ST_A2A, ST_MFFT, ST_COUNT };
static const char* kStageNames[ST_COUNT + 1] = {"comm_S", "s2m", "m2m", "comm_M", "top",
                                                "down", "post_pfft", "a2a", "mfft", "s2t"};

struct RankBufs {
    int g = 0;
    void* Tn = nullptr;      // [P][nb][2][M_L] S2T output (T_near, p-major, planar re/im per box)
    void* tmp = nullptr;     // M-FFT ping-pong buffer
    void* Sp = nullptr;      // S'[p][b][m]: p-major copy of the input for the tensor-core S2T
    void* W = nullptr;       // [k2][Mg]       P-FFT output = all-to-all send buffer
    void* Rcv = nullptr;     // all-to-all receive buffer (G > 1)
    void* haloL = nullptr;   // S box -1  (G > 1)
    void* haloR = nullptr;   // S box nb  (G > 1)
    void* r = nullptr;       // [P] reductions
    void* dc = nullptr;      // [P/G] the k1 = 0 outputs of this rank's M-FFT rows (k_dc_bins, R19)
    void* r0p = nullptr;     // [(P-1) top_cl] double2 partial sums of r_0 (wide trees with the cluster top)
    void* cin = nullptr;     // conj(in) (inverse plans)
    void* rz = nullptr;      // Z = F_{N/2} z (real-input plans, FMMFFT_FLAG_REAL)
    void* mir = nullptr;     // real plans, G > 1: the mirror block (rank G-1-g's Z or X block)
    void* xtra = nullptr;    //   and the one element A[(G-g) N/(2G)] (mirror exchange)
    void* din = nullptr;     // execute_host staging
    void* dout = nullptr;
    std::vector<void*> Mpad, Lloc, Mfull, Lfull;   // indexed by level
};

struct GraphEntry {
    const void* in = nullptr;
    void* out = nullptr;
    cudaGraphExec_t exec = nullptr;
    int nlaunch = 0;
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
    int PCn = 0, PCd = 0;            // p-chunks of near_up and of the tree kernels
    int s2t_chunk = 0, m2l_chunk = 0, m2lB_chunk = 0;   // table chunk strides (elements)
    // device tables
    void* s2m = nullptr;
    void* s2mT = nullptr;            // S2M^T [M_L][Qp], Qp = Q rounded up to 4 (k_s2m)
    void* m2m = nullptr;
    void* s2t = nullptr;
    void* rho = nullptr;
    void* m2lB = nullptr;
    std::vector<void*> m2l;          // by level
    std::vector<void*> m2l_pmaj;     // p-major copies for the fused per-p tree (G = 1), by level
    bool tree_p = false;             // use k_tree_p for the far field
    int tree_cl = 1;                 // k_tree_pc: CTAs per FMM (cluster), 1 = not used
    int top_L = 0;                   // > 0: wide tree (G = 1) whose levels B..top_L run on k_tree_pc
    int top_cl = 0;                  //   with clusters of top_cl CTAs; levels > top_L per level
    bool s2m_w = false;              // S2M on k_s2m_w (complex64, M_L = 64, P % 16 == 0)
    bool s2m_m2m = false;            //   with the first M2M level (L -> L-1) fused into it
    bool s2m_sym = false;            //   and the reflection-symmetric (even / odd) S2M (Q % 8 == 0)
    int fs_lc1 = 0, fs_lc2 = 0, fs_lr = 0;   // four-step large-M FFT: column pass bits (2nd: 0 = none), row pass bits
    bool inverse = false;            // FMMFFT_FLAG_INVERSE: x = F_N^{-1} y
    bool real = false;               // FMMFFT_FLAG_REAL: N (below) is the complex length H = N_real / 2
    bool pmaj = false;               // M^L / L^L p-major [p][b][q] between k_s2m, k_tree_pc and post_pfft
    bool direct = false;             // FMMFFT_FLAG_DIRECT: plain four-step FFT of length N, no FMM
    bool s2t_tc = false;             // S2T on tcgen05 (k_s2t_tc): complex64, M_L = 64, nb % 128 == 0
    bool s2t_fft = false;            // S2T as a fast convolution (k_s2t_fft, NEXT-4): M_L = 64, nb % 32 == 0
    bool s2t_dmma = false;           // complex128 S2T direct sum on the FP64 tensor pipe (k_s2t_dmma)
    void* s2tf_h = nullptr;          // its kernel spectra H_s = DFT_128(h_s) / 128, [p][s][cc][k1][t']
    void* toep = nullptr;            // its Toeplitz hi/lo operand table
    bool row_fft1 = false;           // M-point FFTs in one pass per row (k_fft_row), M fits smem
    void* twM = nullptr;             // its twiddles w_M^u, u < M/16
    std::vector<fmmfft::RankBufs> ranks;
    std::vector<int> radices;        // M-FFT passes
    size_t ws_bytes = 0;
    int kernels = 0;
    cudaEvent_t ev[fmmfft::ST_COUNT + 1] = {};
    cudaEvent_t ev_s2t[2] = {};      // S2T on the side stream (profiling)
    cudaEvent_t fork = nullptr, join = nullptr;   // side-stream fork / join
    cudaEvent_t fork2 = nullptr;     // S' ready (tensor-core S2T)
    cudaStream_t side = nullptr;     // S2T runs here, concurrently with the far field
    cudaEvent_t cs_done = nullptr;   // S halo exchange (side stream) complete: orders NCCL work
    cudaEvent_t dc_fork = nullptr, dc_join = nullptr;   // k_dc_bins on the side stream (after top)
    ncclComm_t comm = nullptr;       // G > 1 (non-virtual): the communicator, bound at plan time;
                                     // virtual + FMMFFT_FLAG_VIRTUAL_NCCL: a 1-rank communicator
    int comm_rank = 0;
    bool vnccl = false;              // virtual ranks exchange through NCCL self send / recv
    bool have_times = false;
    bool use_graph = true;
    cudaStream_t cap_stream = nullptr;
    std::vector<fmmfft::GraphEntry> graphs;
    std::vector<void*> allocs;
};

namespace fmmfft {

static fmmfft_status_t dalloc(fmmfft_plan_s* p, void** ptr, size_t bytes) {
    if (bytes == 0) bytes = 16;
    bytes = (bytes + 255) & ~(size_t)255;
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
static int pad16(int elems, int esz) { return ((elems * esz + 15) / 16) * 16 / esz; }

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
    {
        const int Qp = (Q + 3) / 4 * 4;
        std::vector<double> s2mT((size_t)M_L * Qp, 0.0);
        for (int q = 0; q < Q; ++q)
            for (int m = 0; m < M_L; ++m) s2mT[(size_t)m * Qp + q] = s2m[(size_t)q * M_L + m];
        if ((st = upload<R>(p, &p->s2mT, s2mT))) return st;
    }
    // M2M = [M2M^- M2M^+], M2M^{-+}_{qk} = l_q((z_k -+ 1)/2); L2L = M2M^T
    std::vector<double> m2m((size_t)Q * 2 * Q);
    for (int q = 0; q < Q; ++q)
        for (int k = 0; k < 2 * Q; ++k)
            m2m[(size_t)q * 2 * Q + k] = lagr(z, q, (z[k % Q] + (k < Q ? -1.0 : 1.0)) / 2.0);
    if ((st = upload<R>(p, &p->m2m, m2m))) return st;
    // S2T_{pk} = cot(pi (p + P k)/N), p > 0; delta_{k0} for p = 0,
    // layout [chunk][k][pl] for near_up's p-chunk PCn
    const int nK = 4 * M_L - 1, PCn = p->PCn;
    p->s2t_chunk = pad16(nK * PCn, sizeof(R));
    std::vector<double> s2t((size_t)(P / PCn) * p->s2t_chunk, 0.0);
    for (int pp = 0; pp < P; ++pp)
        for (int ki = 0; ki < nK; ++ki) {
            const long long k = ki - (2 * M_L - 1);
            s2t[(size_t)(pp / PCn) * p->s2t_chunk + (size_t)ki * PCn + pp % PCn] =
                pp == 0 ? (k == 0 ? 1.0 : 0.0) : cotpi((double)(pp + (long long)P * k) / (double)N);
        }
    if ((st = upload<R>(p, &p->s2t, s2t))) return st;
    // M2L^l_{pijs} = cot(pi/2^l (z_j/2 - z_i/2 + s) + pi p/N) for FMM p (slot = p),
    // layout [chunk][s][i][j][pl]; s in {-3, -2, 2, 3} for l > B, 2..2^B-2 at the base
    const int PCd = p->PCd;
    p->m2l.assign(p->L + 1, nullptr);
    p->m2l_pmaj.assign(p->L + 1, nullptr);
    const int shifts[4] = {-3, -2, 2, 3};
    for (int lev = p->B; lev <= p->L; ++lev) {
        const bool base = lev == p->B;
        const int ns = base ? (1 << p->B) - 3 : 4;
        const int chunk = pad16(ns * Q * Q * PCd, sizeof(R));
        (base ? p->m2lB_chunk : p->m2l_chunk) = chunk;
        std::vector<double> t((size_t)(P / PCd) * chunk, 0.0);
        for (int si = 0; si < ns; ++si) {
            const int s = base ? 2 + si : shifts[si];
            for (int i = 0; i < Q; ++i)
                for (int j = 0; j < Q; ++j)
                    for (int pp = 1; pp < P; ++pp)
                        t[(size_t)(pp / PCd) * chunk + (((size_t)si * Q + i) * Q + j) * PCd + pp % PCd] =
                            cotpi((z[j] / 2 - z[i] / 2 + s) / (double)(1LL << lev) + (double)pp / (double)N);
        }
        if ((st = upload<R>(p, base ? &p->m2lB : &p->m2l[lev], t))) return st;
        {                                                  // [p][s][j][i] (i fastest): k_tree_p*, k_down_narrow
            std::vector<double> tp((size_t)P * ns * Q * Q, 0.0);
            for (int pp = 0; pp < P; ++pp)
                for (int si = 0; si < ns; ++si)
                    for (int i = 0; i < Q; ++i)
                        for (int j = 0; j < Q; ++j)
                            tp[(size_t)pp * ns * Q * Q + ((size_t)si * Q + j) * Q + i] =
                                t[(size_t)(pp / PCd) * chunk + (((size_t)si * Q + i) * Q + j) * PCd + pp % PCd];
            if ((st = upload<R>(p, &p->m2l_pmaj[lev], tp))) return st;
        }
    }
    // tensor-core S2T operator (kernel_s2t_tc.cuh): B_p[(s, i)][m] = S2T_{p, (s-1) 64 + m - i},
    // split into tf32 hi + lo, UMMA K-major core-matrix layout [hi/lo][k4][r8][8][4] per p
    if (p->s2t_tc) {
        auto tf32 = [](double v) {                     // round to nearest (ties away), tf32 precision
            float f = (float)v;
            uint32_t u;
            memcpy(&u, &f, 4);
            u = (u + 0x1000u) & 0xFFFFE000u;
            memcpy(&f, &u, 4);
            return f;
        };
        std::vector<float> tb((size_t)P * S2TC_TAB_FLOATS_PER_P, 0.f);
        for (int pp = 1; pp < P; ++pp) {
            for (int k4 = 0; k4 < 16; ++k4)
                for (int r = 0; r < S2TC_N; ++r)
                    for (int kk = 0; kk < 4; ++kk) {
                        const int seg = r / 64, i = r % 64, m = 4 * k4 + kk;
                        const long long d = (long long)(seg - 1) * 64 + m - i;
                        const double v = cotpi((double)(pp + (long long)P * d) / (double)N);
                        const float hi = tf32(v);
                        const float lo = tf32(v - (double)hi);
                        // rows (seg, hi/lo, i): [Bhi_seg; Blo_seg] contiguous along N
                        for (int hl = 0; hl < 2; ++hl) {
                            const int row = seg * 128 + hl * 64 + i;
                            const size_t e = (size_t)pp * S2TC_TAB_FLOATS_PER_P + ((size_t)k4 * (2 * S2TC_N / 8) + row / 8) * 32 + (row % 8) * 4 + kk;
                            tb[e] = hl ? lo : hi;
                        }
                    }
        }
        fmmfft_status_t st2 = dalloc(p, &p->toep, tb.size() * sizeof(float));
        if (st2) return st2;
        CUDA_TRY(cudaMemcpy(p->toep, tb.data(), tb.size() * sizeof(float), cudaMemcpyHostToDevice));
    }
    // fast-convolution S2T (kernel_s2t_fft.cuh): h_s[n mod 128] = S2T_{p, 64 s - n} for
    // n in [-63, 63] (s = -1, 0, 1), h_s[64] = 0; H_s[f] = sum_n h_s[n] w_128^{f n} / 128 (float64,
    // exact angle reduction f n mod 128), stored [p][s][cc][k1][t'] with f = 2 t' + cc + 16 k1
    if (p->s2t_fft) {
        std::vector<double> cs(128), sn(128);
        for (int k = 0; k < 128; ++k) { cs[k] = std::cos(2 * M_PI * k / 128.0); sn[k] = -std::sin(2 * M_PI * k / 128.0); }
        std::vector<double> H((size_t)P * S2TF_H_PER_P * 2, 0.0);
        for (int pp = 0; pp < P; ++pp)
            for (int s = -1; s <= 1; ++s) {
                double h[128];
                for (int n = 0; n < 128; ++n) {
                    const int lag = n <= 63 ? n : n - 128;          // n = 64: unused slot
                    const long long k = 64LL * s - lag;
                    h[n] = n == 64 ? 0.0
                                   : (pp == 0 ? (k == 0 ? 1.0 : 0.0) : cotpi((double)(pp + (long long)P * k) / (double)N));
                }
                for (int f = 0; f < 128; ++f) {
                    double re = 0, im = 0;
                    for (int n = 0; n < 128; ++n) { re += h[n] * cs[(f * n) & 127]; im += h[n] * sn[(f * n) & 127]; }
                    const int k2 = f & 15, k1 = f >> 4, tt = k2 >> 1, cc = k2 & 1;
                    const size_t e = (size_t)pp * S2TF_H_PER_P + (size_t)(s + 1) * 128 + (cc * 8 + k1) * 8 + tt;
                    H[2 * e] = re / 128.0;
                    H[2 * e + 1] = im / 128.0;
                }
            }
        if ((st = upload<R>(p, &p->s2tf_h, H))) return st;
    }
    // rho_p = exp(-i pi p/P) sin(pi p/P) / M, interleaved complex; rho_0 unused
    std::vector<double> rho(2 * (size_t)P);
    for (int pp = 0; pp < P; ++pp) {
        const double sn = std::sin(M_PI * pp / P) / (double)p->M;
        rho[2 * pp] = pp ? std::cos(M_PI * pp / P) * sn : 1.0;
        rho[2 * pp + 1] = pp ? -std::sin(M_PI * pp / P) * sn : 0.0;
    }
    if ((st = upload<R>(p, &p->rho, rho))) return st;
    if (p->row_fft1) {                                   // w_M^u = exp(-2 pi i u / M), u < M/16
        std::vector<double> tw(2 * (p->M / 16));
        for (long long u = 0; u < p->M / 16; ++u) {
            tw[2 * u] = std::cos(2 * M_PI * (double)u / (double)p->M);
            tw[2 * u + 1] = -std::sin(2 * M_PI * (double)u / (double)p->M);
        }
        if ((st = upload<R>(p, &p->twM, tw))) return st;
    }
    return FMMFFT_SUCCESS;
}

#ifndef FMMFFT_TILE_F
#define FMMFFT_TILE_F 2048
#endif
#ifndef FMMFFT_TILE_D
#define FMMFFT_TILE_D 2048
#endif
// shared FFT tile (elements) of k_post_pfft / k_fft_pass: 2048 = 256 threads per CTA, several CTAs
// per SM overlap their load / compute / store phases (measured: 8192 -> 4096 -> 2048 = 98 -> 65 -> 59 us at P = 128)
static constexpr int kTileF = FMMFFT_TILE_F, kTileD = FMMFFT_TILE_D;
template <typename R> static constexpr int kRowFftMax = sizeof(R) == 4 ? 14 : 13;   // k_fft_row: whole row in smem
// four-step passes: largest pass length (log2) and columns (rows) per CTA for a pass of 2^l points
template <typename R> __host__ __device__ constexpr int fs_max() { return sizeof(R) == 4 ? 11 : 10; }
template <typename R> __host__ __device__ constexpr int fs_cols(int l) { return l <= fs_max<R>() - 2 ? 16 : 8; }

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

// four-step split of a 2^lM-point row into passes of <= 2^mx points (2 or 3 passes; none if the
// row is too short or too long)
static void choose_fourstep(fmmfft_plan_s* p, int lM, int mx) {
    p->fs_lr = p->fs_lc1 = p->fs_lc2 = 0;
    if (lM < 10 || lM > 3 * mx) return;
    if (lM <= 2 * mx) {
        p->fs_lr = std::min(mx, (lM + 1) / 2);
        p->fs_lc1 = lM - p->fs_lr;
    } else {
        p->fs_lr = std::min(mx, (lM + 2) / 3);
        p->fs_lc1 = std::min(mx, (lM - p->fs_lr + 1) / 2);
        p->fs_lc2 = lM - p->fs_lr - p->fs_lc1;
    }
    if (p->fs_lc1 < 5 || p->fs_lr < 5 || (p->fs_lc2 && p->fs_lc2 < 5)) p->fs_lr = p->fs_lc1 = p->fs_lc2 = 0;
}

// the M-point row FFT kernels for p->M, p->P / p->G rows: one pass per row in shared memory
// (k_fft_row, M <= 2^14 / 2^13) when there are enough rows to fill the GPU, else the four-step
// column + transposing row passes, else the multi-pass Stockham kernel (short rows).
// FMMFFT_MFFT=pass forces k_fft_pass, =fs the four-step (test knobs).
static void plan_mfft(fmmfft_plan_s* p) {
    plan_radices(p);
    const int lM = ilog2(p->M);
    const char* e = getenv("FMMFFT_MFFT");
    const bool pass = e && e[0] == 'p', fs = e && e[0] == 'f';
    p->row_fft1 = !pass && lM >= 8 && lM <= (p->prec == FMMFFT_C64 ? 14 : 13);
    const bool few_rows = p->P / p->G < 148 && lM >= 13;
    if ((fs && lM >= 10) || few_rows) p->row_fft1 = false;
    // 11-bit passes (1 CTA per SM) measured slower than 3 passes of <= 10 bits
#ifndef FMMFFT_FS_MX
#define FMMFFT_FS_MX 10
#endif
    if (!pass && !p->row_fft1) choose_fourstep(p, lM, FMMFFT_FS_MX);
}

static fmmfft_status_t alloc_rank(fmmfft_plan_s* p, RankBufs& rb) {
    const size_t e = p->esz;
    const long long n_local = p->N / p->G;
    const size_t QP = (size_t)p->Q * p->P;
    fmmfft_status_t st;
    if ((st = dalloc(p, &rb.Tn, n_local * e))) return st;
    if ((st = dalloc(p, &rb.W, n_local * e))) return st;
    if ((st = dalloc(p, &rb.tmp, n_local * e))) return st;
    if (p->s2t_tc && (st = dalloc(p, &rb.Sp, n_local * e))) return st;
    if (p->inverse && (st = dalloc(p, &rb.cin, n_local * e))) return st;
    if (p->G > 1) {
        if ((st = dalloc(p, &rb.Rcv, n_local * e))) return st;
        if ((st = dalloc(p, &rb.haloL, (size_t)p->M_L * p->P * e))) return st;
        if ((st = dalloc(p, &rb.haloR, (size_t)p->M_L * p->P * e))) return st;
    }
    if ((st = dalloc(p, &rb.r, (size_t)p->P * e))) return st;
    if ((st = dalloc(p, &rb.dc, (size_t)(p->P / p->G) * e))) return st;
    if (p->top_L && (st = dalloc(p, &rb.r0p, (size_t)(p->P - 1) * p->top_cl * 16))) return st;
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
    for (auto& g : p->graphs)
        if (g.exec) cudaGraphExecDestroy(g.exec);
    for (void* a : p->allocs) cudaFree(a);
    for (auto& ev : p->ev)
        if (ev) cudaEventDestroy(ev);
    for (auto& ev : p->ev_s2t)
        if (ev) cudaEventDestroy(ev);
    if (p->fork) cudaEventDestroy(p->fork);
    if (p->join) cudaEventDestroy(p->join);
    if (p->fork2) cudaEventDestroy(p->fork2);
    if (p->cs_done) cudaEventDestroy(p->cs_done);
    if (p->dc_fork) cudaEventDestroy(p->dc_fork);
    if (p->dc_join) cudaEventDestroy(p->dc_join);
    if (p->comm) --g_comm_plans;
    if (p->side) cudaStreamDestroy(p->side);
    if (p->cap_stream) cudaStreamDestroy(p->cap_stream);
    delete p;
}

#ifndef FMMFFT_NEAR_IB_D
#define FMMFFT_NEAR_IB_D 8           // complex128 k_near_up: outputs per thread (register block)
#endif

#ifndef FMMFFT_NARROW_FORCE
#define FMMFFT_NARROW_FORCE 0        // 1: narrow kernels for the top of every tree, per-level kernels below
#endif

// Raise every kernel's dynamic shared memory cap once per device (function attributes are
// per device; not legal during capture). Called with the plan's device current.
template <typename R>
static fmmfft_status_t init_kernel_attrs() {
    constexpr int kMaxDev = 64;
    static std::once_flag once_dev[kMaxDev];
    static cudaError_t err_dev[kMaxDev] = {};
    int cur = 0;
    CUDA_TRY(cudaGetDevice(&cur));
    if (cur < 0 || cur >= kMaxDev) return fail(FMMFFT_UNSUPPORTED, "device ordinal %d", cur);
    cudaError_t& err = err_dev[cur];
    std::call_once(once_dev[cur], [&err] {
        int dev = 0, optin = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
        auto set = [&](const void* f) {
            cudaFuncAttributes fa;
            cudaError_t e = cudaFuncGetAttributes(&fa, f);
            if (e == cudaSuccess)
                e = cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, optin - (int)fa.sharedSizeBytes);
            if (e != cudaSuccess && err == cudaSuccess) err = e;
        };
        constexpr int IB = sizeof(R) == 4 ? 16 : FMMFFT_NEAR_IB_D;
        auto per_pc = [&](auto pc) {
            constexpr int PCv = decltype(pc)::value;
            set((const void*)k_near_up<R, IB, PCv>);
            for (int lml = 4; lml <= 7; ++lml)
                dispatch<4, 5, 6, 7>(lml, [&](auto v) { set((const void*)k_s2m<R, PCv, decltype(v)::value>); });
            if constexpr (PCv <= (sizeof(R) == 4 ? 16 : 8)) {
                set((const void*)k_up<R, PCv>);
                set((const void*)k_base<R, 4, PCv>);
                set((const void*)k_base<R, 8, PCv>);
                set((const void*)k_base<R, 16, PCv>);
                set((const void*)k_base<R, 32, PCv>);
                set((const void*)k_tree_down<R, PCv, 1>);
                set((const void*)k_tree_down<R, PCv, 2>);
                set((const void*)k_tree_down<R, PCv, 4>);
                set((const void*)k_tree_down<R, PCv, 8>);
                set((const void*)k_tree_down<R, PCv, 16>);
            }
        };
        for (int pc = 2; pc <= (sizeof(R) == 4 ? 32 : 16); pc *= 2) dispatch<2, 4, 8, 16, 32>(pc, per_pc);
        if constexpr (sizeof(R) == 4) {
            set((const void*)k_tree_pc<16, 512, 2>);
            set((const void*)k_tree_pc<8, 512, 2>);
            set((const void*)k_tree_pc<16, 512, 4>);
            set((const void*)k_tree_pc<8, 512, 4>);
            set((const void*)k_tree_pc<16, 512, 8>);
            set((const void*)k_tree_pc<8, 512, 8>);
        }
        if constexpr (sizeof(R) == 4) { set((const void*)k_s2t_tc<1>); set((const void*)k_s2t_tc<2>); }
        set((const void*)k_s2t_fft<R>);
        set((const void*)k_s2m_w<R>);
        set((const void*)k_base_sg<R, 4, sizeof(R) == 4 ? 8 : 4, 4>);
        for (int lp = 1; lp <= 5; ++lp)
            dispatch<1, 2, 3, 4, 5>(lp, [&](auto v) {
                set((const void*)k_post_pfft_r<R, decltype(v)::value, 8>);
                set((const void*)k_post_pfft_r<R, decltype(v)::value, 16>);
                set((const void*)k_post_pfft_r<R, decltype(v)::value, 24>);
            });
        set((const void*)k_up_narrow<R, 8>);
        set((const void*)k_up_narrow<R, 16>);
        set((const void*)k_up_narrow<R, 24>);
        set((const void*)k_down_narrow<R, 8>);
        set((const void*)k_down_narrow<R, 16>);
        set((const void*)k_down_narrow<R, 24>);
        if constexpr (sizeof(R) == 8) {
            set((const void*)k_m2l_dmma<8>); set((const void*)k_m2l_dmma<16>); set((const void*)k_m2l_dmma<24>);
            set((const void*)k_m2m_dmma<8>); set((const void*)k_m2m_dmma<16>); set((const void*)k_m2m_dmma<24>);
        }
        set((const void*)k_m2l_lvl<R, 8>);
        set((const void*)k_m2m_lvl<R, 8>);
        set((const void*)k_m2m_lvl<R, 16>);
        set((const void*)k_m2m_lvl<R, 24>);
        set((const void*)k_m2l_lvl<R, 16>);
        set((const void*)k_m2l_lvl<R, 24>);
        set((const void*)k_tree_p<R, 1>);
        set((const void*)k_tree_p<R, 2>);
        set((const void*)k_tree_p<R, 4>);
        set((const void*)k_tree_p<R, 8>);
        for (int lp = 1; lp <= 11; ++lp)
            dispatch<1, 2, 3, 4, 5, 6, 7, 8, 9, 10, 11>(lp, [&](auto v) {
                set((const void*)k_post_pfft<R, decltype(v)::value, 0>);
                set((const void*)k_post_pfft<R, decltype(v)::value, 8>);
                set((const void*)k_post_pfft<R, decltype(v)::value, 16>);
                set((const void*)k_post_pfft<R, decltype(v)::value, 24>);
            });
        for (int lr = 1; lr <= 10; ++lr)
            dispatch<1, 2, 3, 4, 5, 6, 7, 8, 9, 10>(lr, [&](auto v) { set((const void*)k_fft_pass<R, decltype(v)::value>); });
        for (int l = 5; l <= fs_max<R>(); ++l)
            dispatch<5, 6, 7, 8, 9, 10, 11>(l, [&](auto v) {
                constexpr int LV = decltype(v)::value;
                if constexpr (LV <= fs_max<R>()) {
                    set((const void*)k_fft_col<R, LV, fs_cols<R>(LV)>);
                    set((const void*)k_fft_rowt<R, LV, fs_cols<R>(LV)>);
                }
            });
        for (int ll = 8; ll <= kRowFftMax<R>; ++ll)
            dispatch<8, 9, 10, 11, 12, 13, 14>(ll, [&](auto v) {
                if constexpr (decltype(v)::value <= kRowFftMax<R>) set((const void*)k_fft_row<R, decltype(v)::value>);
            });
    });
    CUDA_TRY(err);
    return FMMFFT_SUCCESS;
}

// shared memory of k_tree_p: the multipole pyramid + M2M + all M2L tables of one FMM
static size_t tree_p_smem(const fmmfft_plan_s* p, int threads) {
    (void)threads;
    const size_t Q = p->Q;
    const size_t npyr = (((size_t)2 << p->L) - ((size_t)1 << p->B)) * Q;
    const size_t tabs = ((size_t)(1 << p->B) - 3) * Q * Q + (size_t)(p->L - p->B) * 4 * Q * Q;
    return npyr * p->esz + (4 * Q * Q + tabs) * p->rsz + 32 * p->esz;
}

// shared memory of k_tree_pc (cluster of CL CTAs per FMM)
static size_t tree_pc_smem(const fmmfft_plan_s* p, int CL, int Lt = -1) {
    const int L = Lt >= 0 ? Lt : p->L;                  // the tree's (top) leaf level
    const size_t Q = p->Q, QQ = Q * Q, nbB = (size_t)1 << p->B;
    const size_t tabB = (nbB - 3) * QQ;
    auto H = [&](int l) { return ((size_t)1 << l) / CL; };
    size_t cplx = 32 + nbB * Q + (nbB / CL) * Q + H(L) * Q + (L > 0 ? H(L - 1) : 0) * Q;
    for (int l = p->B + 1; l <= L; ++l) cplx += (H(l) + 6) * Q;
    return (2 * QQ + tabB + (size_t)(L - p->B) * 4 * QQ) * 4 + QQ * 8 + cplx * 8;
}

// ------------------------------------------------------------------ execute
template <typename R>
struct Exec {
    using C = C2<R>;
    fmmfft_plan_s* p;
    cudaStream_t s;
    std::vector<const C*> in;    // per rank
    std::vector<C*> out;
    int nlaunch = 0;             // kernels launched by this execute (all virtual ranks)

    static constexpr int IB = sizeof(R) == 4 ? 16 : FMMFFT_NEAR_IB_D;
    static constexpr int TILE = sizeof(R) == 4 ? kTileF : kTileD;
    size_t QP() const { return (size_t)p->Q * p->P; }
    int nb_at(int lev) const { return (int)((1LL << lev) / p->G); }
    C* interior(void* pad) const { return (C*)pad + 2 * QP(); }
    ncclDataType_t nt() const { return sizeof(R) == 4 ? ncclFloat : ncclDouble; }
    int grank(const RankBufs& rb) const { return p->virt ? rb.g : p->comm_rank; }

    template <typename F> bool with_pcd(F&& f) const {
        if constexpr (sizeof(R) == 4) return dispatch<2, 4, 8, 16>(p->PCd, f);
        else return dispatch<2, 4, 8>(p->PCd, f);
    }

    // the stream of the near field (S halo + S2T): concurrent with the far field, except in
    // profiled plans, which serialise it on the main stream so every stage's events bracket only
    // its own kernels (fmmfft_stage_times: s2t measured alone, s2m excludes it)
    cudaStream_t side() const { return (p->flags & FMMFFT_FLAG_PROFILE) ? s : p->side; }

    // stage boundary event; inside a graph capture it must be an "external" record to become a
    // real event-record node (a plain record during capture only expresses a dependency)
    fmmfft_status_t mark(int stage) {
        if (p->flags & FMMFFT_FLAG_PROFILE)
            CUDA_TRY(cudaEventRecordWithFlags(p->ev[stage], s, p->use_graph ? cudaEventRecordExternal : cudaEventRecordDefault));
        return FMMFFT_SUCCESS;
    }

    // ---- the exchanges, written once per rank as the NCCL arguments (P2P lists) --------------
    int gidx(const RankBufs& rb) const { return p->virt ? rb.g : 0; }   // index into in[] / out[]

    // S halo (line 2): rank g sends its box 0 to the left neighbour (whose right halo it
    // is) and its last box to the right one; receives haloR from the right, haloL from the left
    std::vector<P2P> sched_S(const RankBufs& rb) const {
        const size_t box = (size_t)p->M_L * p->P;
        const int G = p->G, g = grank(rb), lf = (g - 1 + G) % G, rt = (g + 1) % G;
        C* S = const_cast<C*>(in[gidx(rb)]);
        return {{true, lf, S, box}, {true, rt, S + (size_t)(p->nb - 1) * box, box},
                {false, rt, rb.haloR, box}, {false, lf, rb.haloL, box}};
    }

    // M^l halos for l > l_g (line 7): two boxes per side per level, all levels in one
    // group; Mpad[l] = [2 left halo | nbl own | 2 right halo] boxes of Q P each
    std::vector<P2P> sched_M(const RankBufs& rb) const {
        const size_t QPc = QP();
        const int G = p->G, g = grank(rb), lf = (g - 1 + G) % G, rt = (g + 1) % G;
        std::vector<P2P> v;
        for (int lev = p->lg + 1; lev <= p->L; ++lev) {
            const size_t nbl = (size_t)nb_at(lev);
            C* pad = (C*)rb.Mpad[lev];
            v.push_back({true, lf, pad + 2 * QPc, 2 * QPc});              // own boxes 0, 1 -> left
            v.push_back({true, rt, pad + nbl * QPc, 2 * QPc});            // own boxes nbl-2, nbl-1 -> right
            v.push_back({false, rt, pad + (nbl + 2) * QPc, 2 * QPc});
            v.push_back({false, lf, pad, 2 * QPc});
        }
        return v;
    }

    // all-gather of level l_g (line 9 / reading R16)
    Gather sched_gather(const RankBufs& rb) const {
        return {interior(rb.Mpad[p->lg]), rb.Mfull[p->lg], (size_t)nb_at(p->lg) * QP()};
    }

    // the one all-to-all (line 16): chunk r of W (k2 in r's block, own m) -> rank r's
    // receive slot g
    std::vector<P2P> sched_A2A(const RankBufs& rb) const {
        const size_t chunk = (size_t)(p->P / p->G) * p->Mg;
        std::vector<P2P> v;
        for (int r = 0; r < p->G; ++r) {
            v.push_back({true, r, (C*)rb.W + r * chunk, chunk});
            v.push_back({false, r, (C*)rb.Rcv + r * chunk, chunk});
        }
        return v;
    }

    // real plans, G > 1: the mirror exchange. Output k of rank g needs A[H - k] (H = N/2, A = Z
    // for the forward, A = X for the inverse): for k in g's block those are rank G-1-g's block
    // (reversed, minus its first element) and the one element A[(G-g) H/G] — rank (G-g) mod G's
    // first (R2C: A[H] = Z[0], rank 0's own), or for C2R at g = 0 X_H, rank G-1's extra slot
    std::vector<P2P> sched_mirror(const RankBufs& rb, const C* own, bool c2r) const {
        const int G = p->G, g = grank(rb);
        const size_t nl = (size_t)(p->N / G);
        C* a = const_cast<C*>(own);
        std::vector<P2P> v;
        v.push_back({true, G - 1 - g, a, nl});                          // mirror block first
        if (!c2r) v.push_back({true, (G - g) % G, a, 1});
        else {
            if (g == G - 1) v.push_back({true, 0, a + nl, 1});           // X_H -> rank 0
            if (g > 0) v.push_back({true, G - g, a, 1});
        }
        v.push_back({false, G - 1 - g, rb.mir, nl});
        v.push_back({false, c2r ? (g == 0 ? G - 1 : G - g) : (G - g) % G, rb.xtra, 1});
        return v;
    }

    // issue one exchange on stream st: NCCL group (one process per GPU), or every virtual rank's
    // list matched send-to-receive and executed as device copies (or NCCL self send / receive on
    // a 1-rank communicator, FMMFFT_FLAG_VIRTUAL_NCCL)
    template <typename Sched>
    fmmfft_status_t exchange(Sched sched, cudaStream_t st) {
        NcclApi& n = nccl();
        if (!p->virt) {
            const std::vector<P2P> v = sched(p->ranks[0]);
            NCCL_TRY(n.GroupStart());
            for (const P2P& o : v) {
                if (o.send) NCCL_TRY(n.Send(o.ptr, 2 * o.n, nt(), o.peer, p->comm, st));
                else        NCCL_TRY(n.Recv(o.ptr, 2 * o.n, nt(), o.peer, p->comm, st));
            }
            NCCL_TRY(n.GroupEnd());
            return FMMFFT_SUCCESS;
        }
        const int G = p->G;
        std::vector<std::vector<P2P>> all(G);
        for (RankBufs& rb : p->ranks) all[rb.g] = sched(rb);
        std::vector<size_t> cur((size_t)G * G, 0);            // (receiver, sender) -> next receive op
        std::vector<std::pair<const P2P*, const P2P*>> pairs;
        for (int g = 0; g < G; ++g)
            for (const P2P& o : all[g]) {
                if (!o.send) continue;
                const std::vector<P2P>& rv = all[o.peer];
                size_t& k = cur[(size_t)o.peer * G + g];
                while (k < rv.size() && (rv[k].send || rv[k].peer != g)) ++k;
                if (k == rv.size()) return fail(FMMFFT_INVALID_VALUE, "exchange: send %d->%d has no receive", g, o.peer);
                if (rv[k].n != o.n) return fail(FMMFFT_INVALID_VALUE, "exchange: %d->%d sends %zu, receives %zu", g, o.peer, o.n, rv[k].n);
                pairs.push_back({&o, &rv[k]});
                ++k;
            }
        size_t nrecv = 0;
        for (auto& v : all) for (const P2P& o : v) nrecv += !o.send;
        if (nrecv != pairs.size()) return fail(FMMFFT_INVALID_VALUE, "exchange: %zu receives, %zu sends", nrecv, pairs.size());
        if (p->vnccl) {
            NCCL_TRY(n.GroupStart());
            for (auto& pr : pairs) {
                NCCL_TRY(n.Send(pr.first->ptr, 2 * pr.first->n, nt(), 0, p->comm, st));
                NCCL_TRY(n.Recv(pr.second->ptr, 2 * pr.second->n, nt(), 0, p->comm, st));
            }
            NCCL_TRY(n.GroupEnd());
            return FMMFFT_SUCCESS;
        }
        for (auto& pr : pairs)
            CUDA_TRY(cudaMemcpyAsync(pr.second->ptr, pr.first->ptr, pr.first->n * sizeof(C), cudaMemcpyDeviceToDevice, st));
        return FMMFFT_SUCCESS;
    }

    fmmfft_status_t allgather(cudaStream_t st) {
        NcclApi& n = nccl();
        if (!p->virt) {
            const Gather a = sched_gather(p->ranks[0]);
            NCCL_TRY(n.AllGather(a.send, a.recv, 2 * a.n, nt(), p->comm, st));
            return FMMFFT_SUCCESS;
        }
        if (p->vnccl) NCCL_TRY(n.GroupStart());
        for (RankBufs& dst : p->ranks) {
            const Gather d = sched_gather(dst);
            for (RankBufs& src : p->ranks) {
                const Gather a = sched_gather(src);
                if (a.n != d.n) return fail(FMMFFT_INVALID_VALUE, "allgather: counts differ");
                C* to = (C*)d.recv + (size_t)src.g * a.n;
                if (p->vnccl) {
                    NCCL_TRY(n.Send(a.send, 2 * a.n, nt(), 0, p->comm, st));
                    NCCL_TRY(n.Recv(to, 2 * a.n, nt(), 0, p->comm, st));
                } else {
                    CUDA_TRY(cudaMemcpyAsync(to, a.send, a.n * sizeof(C), cudaMemcpyDeviceToDevice, st));
                }
            }
        }
        if (p->vnccl) NCCL_TRY(n.GroupEnd());
        return FMMFFT_SUCCESS;
    }

    // ---- comm_S: S halo (line 2) on the side stream, ahead of S2T (overlaps S2M)
    fmmfft_status_t comm_S(cudaStream_t st) {
        if (p->G == 1) return FMMFFT_SUCCESS;
        return exchange([this](const RankBufs& rb) { return sched_S(rb); }, st);
    }

    // record a stage-boundary-style event on an arbitrary stream (S2T's own pair)
    fmmfft_status_t mark_on(cudaEvent_t e, cudaStream_t st) {
        if (p->flags & FMMFFT_FLAG_PROFILE)
            CUDA_TRY(cudaEventRecordWithFlags(e, st, p->use_graph ? cudaEventRecordExternal : cudaEventRecordDefault));
        return FMMFFT_SUCCESS;
    }

    // ---- near field: S2M on the main stream; S2T forked onto the side stream (joined before
    // post_pfft), so the far field and the near field run concurrently
    fmmfft_status_t near_up() {
        fmmfft_status_t st;
        const int PCs = std::min(p->P, sizeof(R) == 4 ? 32 : 16);
        constexpr int PCW = s2mw_pc<R>();
        // complex64 (complex128's S2M is DFMA-bound with Q = 24: k_s2m measured faster, 1.68 vs 2.12 ms)
        if (p->s2m_w) {                                  // warp-per-box S2M (k_s2m_w)
            const int Qp = (p->Q + 3) / 4 * 4;
            const long long tasks = (long long)p->nb * (p->P / PCW);
            int bpw = (int)std::max<long long>(1, std::min<long long>(8, tasks / (S2MW_WARPS * 148 * 4)));
            if (p->s2m_m2m) bpw = std::max(2, bpw & ~1);                // sibling pairs within one warp
            const dim3 grid((unsigned)((p->nb + (long long)S2MW_WARPS * bpw - 1) / ((long long)S2MW_WARPS * bpw)), (unsigned)(p->P / PCW));
            for (RankBufs& rb : p->ranks) {
                const C* S = in[p->virt ? rb.g : 0];
                launch_pdl(k_s2m_w<R>, grid, S2MW_WARPS * 32, s2mw_smem<R>(Qp), s, S, interior(rb.Mpad[p->L]), (const R*)p->s2mT,
                           p->P, p->Q, (C*)rb.Sp, (C*)rb.Tn, p->nb, (int)p->pmaj, bpw,
                           p->s2m_m2m ? interior(rb.Mpad[p->L - 1]) : (C*)nullptr, (const R*)p->m2m, (int)p->s2m_sym);
                LAUNCH_CHECK();
            }
        } else
        for (RankBufs& rb : p->ranks) {
            const C* S = in[p->virt ? rb.g : 0];
            const int Qp = (p->Q + 3) / 4 * 4;
            // boxes per CTA (k_s2m NBX <= 2; nb is even or 1): 1 unless that gives > 4 CTAs per SM
            int nbx = (long long)p->nb * (p->P / PCs) > 4 * 148 ? 2 : 1;
            if (p->nb < 2) nbx = 1;
            const size_t smem = (size_t)2 * p->M_L * (PCs + 1) * sizeof(C) + (size_t)Qp * p->M_L * sizeof(R);
            const dim3 grid((unsigned)(p->nb / nbx), (unsigned)(p->P / PCs));
            dispatch<2, 4, 8, 16, 32>(PCs, [&](auto pc) {
                constexpr int PCv = decltype(pc)::value;
                if constexpr (!(sizeof(R) == 8 && PCv > 16))
                    dispatch<4, 5, 6, 7>(ilog2(p->M_L), [&](auto lml) {
                        launch_pdl(k_s2m<R, PCv, decltype(lml)::value>, grid, PCv * (Qp / 4) * nbx, smem, s, S, interior(rb.Mpad[p->L]),
                                   (const R*)p->s2mT, p->P, p->Q, (C*)rb.Sp, (C*)rb.Tn, p->nb, nbx, (int)p->pmaj);
                    });
            });
            LAUNCH_CHECK();
        }
        // fork after S2M (so S2M runs alone; the tensor-core S2T needs its S'): S2T on the side
        // stream, behind the S halo exchange already queued there (G > 1)
        CUDA_TRY(cudaEventRecord(p->fork2, s));
        CUDA_TRY(cudaStreamWaitEvent(side(), p->fork2, 0));
        if ((st = mark_on(p->ev_s2t[0], side()))) return st;
        if (p->s2t_fft) {                                      // fast convolution (k_s2t_fft, NEXT-4)
            const long long nchunk = p->nb / S2TF_CHUNK;
            // chunks per CTA: >= ~4 waves of 148 SMs x 4 CTAs, at most 16 (prologue = 1/cpc of a chunk)
            const int cpc = (int)std::max<long long>(1, std::min<long long>(16, nchunk * p->P / (148 * 16)));
            for (RankBufs& rb : p->ranks) {
                const C* S = in[p->virt ? rb.g : 0];
                const size_t box = (size_t)p->M_L * p->P;
                const C* hl = p->G == 1 ? S + (size_t)(p->nb - 1) * box : (const C*)rb.haloL;
                const C* hr = p->G == 1 ? S : (const C*)rb.haloR;
                launch_pdl(k_s2t_fft<R>, dim3((unsigned)p->P, (unsigned)((nchunk + cpc - 1) / cpc)), S2TF_THREADS,
                           s2tf_smem_bytes<R>(), side(), S, hl, hr, (R*)rb.Tn, (const C*)p->s2tf_h, p->P, p->nb, cpc);
                LAUNCH_CHECK();
            }
            if ((st = mark_on(p->ev_s2t[1], side()))) return st;
            CUDA_TRY(cudaEventRecord(p->join, side()));
            return FMMFFT_SUCCESS;
        }
        if constexpr (sizeof(R) == 4) {
            if (p->s2t_tc) {                                   // tensor cores (tcgen05, 3xTF32)
                const long long work = (long long)(p->P - 1) * (p->nb / S2TC_BOXES);
                // one CTA per SM (TMEM + ~180 KB of shared memory); the (p, tile) items split evenly
                // over (P - 1) floor(148 / (P - 1)) CTAs, so a CTA's run stays within one p (B_p
                // loaded once) and the few SMs left over run the far field meanwhile (measured:
                // all 148 SMs on S2T, with B_p reloads, was 334 -> 354 us at cfg3)
                // (fewer CTAs, leaving SMs to the far field, measured slower at cfg3: 105 CTAs 1.66 ms,
                // 60 CTAs 1.73 ms, vs 1.64 ms)
                const int ctas = (int)std::min<long long>((long long)(p->P - 1) * std::max(1, 148 / (p->P - 1)), work);
                for (RankBufs& rb : p->ranks) {
                    // several tiles per CTA: A chunks prefetched two ahead; one tile: one ahead (the
                    // first chunk's loads alone, so the first MMAs start sooner)
                    if (work > ctas)
                        launch_pdl(k_s2t_tc<2>, dim3((unsigned)ctas), S2TC_THREADS, s2tc_smem_bytes(), side(), (const C*)rb.Sp,
                                   (const C*)rb.haloL, (const C*)rb.haloR, (float*)rb.Tn, (const float*)p->toep, p->P, p->nb, p->G);
                    else
                        launch_pdl(k_s2t_tc<1>, dim3((unsigned)ctas), S2TC_THREADS, s2tc_smem_bytes(), side(), (const C*)rb.Sp,
                                   (const C*)rb.haloL, (const C*)rb.haloR, (float*)rb.Tn, (const float*)p->toep, p->P, p->nb, p->G);
                    LAUNCH_CHECK();
                }
                if ((st = mark_on(p->ev_s2t[1], side()))) return st;
                CUDA_TRY(cudaEventRecord(p->join, side()));
                return FMMFFT_SUCCESS;
            }
        }
        if constexpr (sizeof(R) == 8) {
            if (p->s2t_dmma) {                                 // FP64 tensor pipe (mma.sync f64), k_s2t_dmma
                constexpr int NB = 32;
                for (RankBufs& rb : p->ranks) {
                    const C* S = in[p->virt ? rb.g : 0];
                    const size_t box = (size_t)p->M_L * p->P;
                    const C* hl = p->G == 1 ? S + (size_t)(p->nb - 1) * box : (const C*)rb.haloL;
                    const C* hr = p->G == 1 ? S : (const C*)rb.haloR;
                    launch_pdl(k_s2t_dmma<NB>, dim3((unsigned)p->P, (unsigned)(p->nb / NB)), NB * 4, 0, side(),
                               (const double2*)S, (const double2*)hl, (const double2*)hr, (double2*)rb.Tn,
                               (const double*)p->s2t, p->s2t_chunk, p->PCn, p->P, p->nb);
                    LAUNCH_CHECK();
                }
                if ((st = mark_on(p->ev_s2t[1], side()))) return st;
                CUDA_TRY(cudaEventRecord(p->join, side()));
                return FMMFFT_SUCCESS;
            }
        }
        const int PC_ = p->PCn, nib = p->M_L / IB;
        const int threads = PC_ * nib;
        const int npc = p->P / PC_;
        const int target = 2 * 148 * 2;
        const int bpc = std::max(1, (int)((long long)p->nb * npc / target));
        const dim3 grid((p->nb + bpc - 1) / bpc, npc);
        const size_t smem = (size_t)4 * p->M_L * PC_ * sizeof(C) + (size_t)p->s2t_chunk * sizeof(R) +
                            (size_t)p->Q * p->M_L * sizeof(R);
        for (RankBufs& rb : p->ranks) {
            const C* S = in[p->virt ? rb.g : 0];
            const size_t box = (size_t)p->M_L * p->P;
            const C* hl = p->G == 1 ? S + (size_t)(p->nb - 1) * box : (const C*)rb.haloL;
            const C* hr = p->G == 1 ? S : (const C*)rb.haloR;
            auto go = [&](auto pc) {
                constexpr int PCv = decltype(pc)::value;
                if constexpr (sizeof(R) == 8 && PCv > 16) return;
                else
                    launch_pdl(k_near_up<R, IB, PCv>, grid, threads, smem, side(), S, hl, hr, (C*)rb.Tn, nullptr,
                                                                            (const R*)p->s2t, p->s2t_chunk, (const R*)p->s2m,
                                                                            p->P, p->M_L, p->Q, p->nb, bpc);
            };
            dispatch<2, 4, 8, 16, 32>(PC_, go);
            LAUNCH_CHECK();
        }
        if ((st = mark_on(p->ev_s2t[1], side()))) return st;
        CUDA_TRY(cudaEventRecord(p->join, side()));
        return FMMFFT_SUCCESS;
    }

    // join the side stream (S2T) before the near and far fields are combined
    fmmfft_status_t join_near() {
        CUDA_TRY(cudaStreamWaitEvent(s, p->join, 0));
        return FMMFFT_SUCCESS;
    }

    // M2M for levels from..to (from > to) starting at `inl` (level `from`, nb_from boxes),
    // writing level l to outs(l); k_up handles up to 4 levels per launch.
    template <typename OutF>
    fmmfft_status_t launch_up(const C* inl, int from, int to, long long nb_from, OutF outs) {
        const int PC_ = p->PCd;
        int cur = from;
        const C* src = inl;
        long long nbc = nb_from;
        // wide levels: one register-blocked k_m2m_lvl launch per level (>= 2 tiles of parents)
        constexpr int PCl = lvl_pc<R>();
        const bool lvl_ok = (p->Q == 8 || p->Q == 16 || p->Q == 24) && p->PCd % PCl == 0 && p->P % PCl == 0;
        int optin = 0;
        CUDA_TRY(cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, p->device));
        while (lvl_ok && cur > to && (nbc >> 1) >= 2 * lvl_nt<R, 16>() &&
               ((long long)((nbc >> 1) / lvl_nt<R, 16>()) * (p->P / PCl) >= 148 || (FMMFFT_NARROW_FORCE && narrow_ok() && !narrow_up_fits(nbc)))) {
            C* o = (C*)outs(cur - 1);
            const int nsub = p->P / PCl;
            dispatch<8, 16, 24>(p->Q, [&](auto qv) {
                constexpr int QV = decltype(qv)::value;
                const int ntiles = (int)((nbc >> 1) / lvl_nt<R, QV>());
                const size_t smem = m2m_lvl_smem<R, QV>();
                const int per_sm = std::max(1, std::min(2, (int)((size_t)(optin + 1024) / (smem + 1024))));
                const int nseg = (int)std::max(1LL, std::min<long long>(ntiles, (148LL * per_sm + nsub - 1) / nsub));
                if constexpr (sizeof(R) == 8)                // FP64 tensor pipe
                    launch_pdl(k_m2m_dmma<QV>, dim3((unsigned)nseg, (unsigned)nsub), 256, smem, s, (const C*)src, o,
                               (const double*)p->m2m, p->P, ntiles);
                else
                    launch_pdl(k_m2m_lvl<R, QV>, dim3((unsigned)nseg, (unsigned)nsub), lvl_threads<R, QV>(), smem, s, src, o,
                               (const R*)p->m2m, p->P, ntiles);
            });
            LAUNCH_CHECK();
            src = o;
            nbc >>= 1;
            --cur;
        }
        if (cur > to && narrow_ok() && narrow_up_fits(nbc)) {   // every remaining level in one launch
            NarrowUp no{};
            for (int l = to; l < cur; ++l) no.out[l] = outs(l);
            const size_t smem = narrow_up_smem((int)nbc);
            dispatch<8, 16, 24>(p->Q, [&](auto qv) {
                constexpr int QV = decltype(qv)::value;
                launch_pdl(k_up_narrow<R, QV>, (unsigned)p->P, 256, smem, s, src, no, cur - 1, to, (int)nbc,
                           (const R*)p->m2m, p->P);
            });
            LAUNCH_CHECK();
            return FMMFFT_SUCCESS;
        }
        while (cur > to) {
            int h = std::min(4, cur - to);
            while ((1LL << h) > nbc) --h;
            UpOut uo{};
            for (int l = 1; l <= h; ++l) uo.lev[l - 1] = outs(cur - l);
            const size_t smem = ((size_t)1 << h) * p->Q * PC_ * sizeof(C) + (size_t)2 * p->Q * p->Q * sizeof(R);
            const dim3 grid((unsigned)(nbc >> h), (unsigned)(p->P / PC_));
            with_pcd([&](auto pc) {
                constexpr int PCv = decltype(pc)::value;
                launch_pdl(k_up<R, PCv>, grid, PCv * p->Q, smem, s, src, uo, h, (const R*)p->m2m, p->P, p->Q);
            });
            LAUNCH_CHECK();
            src = (const C*)outs(cur - h);
            nbc >>= h;
            cur -= h;
        }
        return FMMFFT_SUCCESS;
    }

    // k_up_narrow / k_down_narrow keep a whole narrow subtree of one FMM on chip (<= 200 KB)
    bool narrow_ok() const { return p->Q == 8 || p->Q == 16 || p->Q == 24; }
    bool narrow_up_fits(long long nin) const { return nin <= 1024 && narrow_up_smem((int)nin) <= 200 * 1024; }
    bool narrow_down_fits(long long nmax) const { return nmax <= 1024 && narrow_down_smem((int)nmax) <= 200 * 1024; }
    size_t narrow_down_smem(int nmax) const {
        const size_t bsc = (size_t)(2 * p->Q + 2) / 2;
        return (size_t)10 * p->Q * p->Q * sizeof(R) + ((size_t)4 * (nmax / 2 + 2) + 2 * (size_t)nmax) * bsc * sizeof(C);
    }
    size_t narrow_up_smem(int nin) const {
        const size_t bsc = (size_t)(2 * p->Q + 2) / 2;
        return (size_t)2 * p->Q * p->Q * sizeof(R) + ((size_t)nin + nin / 2) * bsc * sizeof(C);
    }

    // ---- the whole far field per FMM p in one launch (G = 1): M2M, M2L-B, REDUCE, M2L + L2L
    fmmfft_status_t tree_p() {
        for (RankBufs& rb : p->ranks) {
            TreePArgs a{};
            for (int lev = p->B; lev <= p->L; ++lev) {
                a.M[lev] = interior(rb.Mpad[lev]);
                a.Lx[lev] = rb.Lloc[lev];
                a.tab[lev] = p->m2l_pmaj[lev];
            }
            a.r = rb.r;
            a.L = p->L;
            a.B = p->B;
            a.dbg = (p->flags & FMMFFT_FLAG_DEBUG) ? 1 : 0;
            a.pmaj = p->pmaj ? 1 : 0;
            a.p0 = 1;
            const int tabB = ((1 << p->B) - 3) * p->Q * p->Q;
            // complex64, Q = 16 or 8: each FMM on a cluster of 2 CTAs (k_tree_pc)
            if constexpr (sizeof(R) == 4) {
                if (p->tree_cl > 1) {
                    const size_t smem = tree_pc_smem(p, p->tree_cl);
                    const unsigned grid = (unsigned)((p->P - 1) * p->tree_cl);
                    dispatch<2, 4, 8>(p->tree_cl, [&](auto cl) {
                        constexpr int CL = decltype(cl)::value;
                        if (p->Q == 16) launch_cluster(k_tree_pc<16, 512, CL>, grid, 512, smem, s, a, (const float*)p->m2m, p->P, tabB);
                        else            launch_cluster(k_tree_pc<8, 512, CL>, grid, 512, smem, s, a, (const float*)p->m2m, p->P, tabB);
                    });
                    LAUNCH_CHECK();
                    continue;
                }
            }
            const int threads = sizeof(R) == 4 ? 1024 : 512;
            const int maxo = (int)((((long long)p->Q << p->L) + threads - 1) / threads);
            const size_t smem = tree_p_smem(p, threads);
            dispatch<1, 2, 4, 8>(maxo <= 1 ? 1 : maxo <= 2 ? 2 : maxo <= 4 ? 4 : 8, [&](auto mo) {
                constexpr int MO = decltype(mo)::value;
                launch_plain(k_tree_p<R, MO>, p->P - 1, threads, smem, s, a, (const R*)p->m2m, p->P, p->Q, tabB);
            });
            LAUNCH_CHECK();
        }
        return FMMFFT_SUCCESS;
    }

    // ---- wide trees (G = 1): levels B..top_L of each FMM on a cluster (k_tree_pc with top_L as
    // its leaf level: M^{top_L} from the per-level M2M in, L^{top_L} for the per-level M2L out)
    fmmfft_status_t tree_top() {
        for (RankBufs& rb : p->ranks) {
            TreePArgs a{};
            for (int lev = p->B; lev <= p->top_L; ++lev) {
                a.M[lev] = interior(rb.Mpad[lev]);
                a.Lx[lev] = rb.Lloc[lev];
                a.tab[lev] = p->m2l_pmaj[lev];
            }
            a.r = rb.r;
            a.L = p->top_L;
            a.B = p->B;
            a.dbg = (p->flags & FMMFFT_FLAG_DEBUG) ? 1 : 0;
            a.pmaj = 0;
            a.p0 = 1;
            a.r0part = rb.r0p;                              // r_0 (R19): partial sums of M^{top_L} slot 0
            const int tabB = ((1 << p->B) - 3) * p->Q * p->Q;
            const size_t smem = tree_pc_smem(p, p->top_cl, p->top_L);
            const unsigned grid = (unsigned)((p->P - 1) * p->top_cl);
            auto go = [&](auto cl) {
                constexpr int CL = decltype(cl)::value;
                if (p->Q == 16) launch_cluster(k_tree_pc<16, 512, CL>, grid, 512, smem, s, a, (const float*)p->m2m, p->P, tabB);
                else            launch_cluster(k_tree_pc<8, 512, CL>, grid, 512, smem, s, a, (const float*)p->m2m, p->P, tabB);
            };
            dispatch<2, 4, 8>(p->top_cl, go);
            LAUNCH_CHECK();
        }
        return FMMFFT_SUCCESS;
    }

    // ---- m2m on own boxes, l = L-1 .. l_g
    fmmfft_status_t m2m_local() {
        if (p->tree_p) return FMMFFT_SUCCESS;
        fmmfft_status_t st;
        for (RankBufs& rb : p->ranks) {
            auto outs = [&](int l) -> void* { return interior(rb.Mpad[l]); };
            // (the first level L -> L-1 already came out of k_s2m_w when p->s2m_m2m)
            const int from = p->s2m_m2m ? p->L - 1 : p->L;
            if ((st = launch_up(interior(rb.Mpad[from]), from, p->top_L ? p->top_L : p->lg, nb_at(from), outs))) return st;
        }
        return FMMFFT_SUCCESS;
    }

    // ---- comm_M: halos (2 boxes per side) for l in (l_g, L] and all-gather of level l_g
    fmmfft_status_t comm_M() {
        if (p->G == 1) return FMMFFT_SUCCESS;
        fmmfft_status_t st;
        // NCCL work is issued in one order on every rank: the S halo (side stream) first
        CUDA_TRY(cudaStreamWaitEvent(s, p->cs_done, 0));
        if (p->L > p->lg && (st = exchange([this](const RankBufs& rb) { return sched_M(rb); }, s))) return st;
        return allgather(s);
    }

    // M2L-B + REDUCE on the gathered base level (sources: all 2^B boxes, periodic)
    fmmfft_status_t launch_base(RankBufs& rb, C* outp, long long tgt_base, int ntg) {
        const int nbB = 1 << p->B;
        {   // all shifts staged at once, shift groups in parallel (k_base_sg)
            constexpr int PCb = sizeof(R) == 4 ? 8 : 4, SG = 4, NTb = 4;
            const size_t smem = (size_t)nbB * p->Q * PCb * sizeof(C) + (size_t)SG * NTb * p->Q * PCb * sizeof(C) +
                                (size_t)(nbB - 3) * p->Q * p->Q * PCb * sizeof(R);
            if (nbB >= 4 && p->PCd % PCb == 0 && p->P % PCb == 0 && smem <= 200 * 1024 && PCb * p->Q * SG <= 1024) {
                const dim3 grid((unsigned)(p->P / PCb), (unsigned)((ntg + NTb - 1) / NTb));
                launch_pdl(k_base_sg<R, NTb, PCb, SG>, grid, PCb * p->Q * SG, smem, s, (const C*)rb.Mfull[p->B], outp,
                           (C*)rb.r, (int)tgt_base, ntg, (const R*)p->m2lB, p->m2lB_chunk, p->PCd, nbB, p->P, p->Q);
                LAUNCH_CHECK();
                return FMMFFT_SUCCESS;
            }
        }
        const int PC_ = p->PCd;
        const size_t smem = ((size_t)nbB + 1) * p->Q * PC_ * sizeof(C) + (size_t)p->Q * p->Q * PC_ * sizeof(R);
        if (ntg <= 32 && smem <= 200 * 1024) {
            const int NTr = 4;                          // targets per CTA (grid y spans them)
            const unsigned gy = (unsigned)((ntg + NTr - 1) / NTr);
            with_pcd([&](auto pc) {
                constexpr int PCv = decltype(pc)::value;
                dispatch<4>(NTr, [&](auto ntv) {
                    constexpr int NTv = decltype(ntv)::value;
                    launch_pdl(k_base<R, NTv, PCv>, dim3((unsigned)(p->P / PCv), gy), PCv * p->Q, smem, s, (const C*)rb.Mfull[p->B], outp, (C*)rb.r,
                                                                           (int)tgt_base, ntg, (const R*)p->m2lB,
                                                                           p->m2lB_chunk, nbB, p->P, p->Q);
                });
            });
            LAUNCH_CHECK();
            return FMMFFT_SUCCESS;
        }
        const long long total = (long long)ntg * QP();
        const int blocks = (int)std::min<long long>((total + 255) / 256, 148LL * 16);
        launch_pdl(k_base_generic<R>, blocks, 256, 0, s, (const C*)rb.Mfull[p->B], outp, tgt_base, ntg, (const R*)p->m2lB,
                                                  p->m2lB_chunk, PC_, nbB, p->P, p->Q);
        LAUNCH_CHECK();
        launch_pdl(k_reduce<R>, (p->P + 127) / 128, 128, 0, s, (C*)rb.Mfull[p->B], (C*)rb.r, p->P, p->Q, nbB);
        LAUNCH_CHECK();
        return FMMFFT_SUCCESS;
    }

    // ---- top: replicated levels l_g .. B
    fmmfft_status_t top() {
        if (p->tree_p) return tree_p();
        if constexpr (sizeof(R) == 4)
            if (p->top_L) return tree_top();
        fmmfft_status_t st;
        for (RankBufs& rb : p->ranks) {
            const int g = grank(rb);
            if (p->lg > p->B) {
                auto outs = [&](int l) -> void* { return rb.Mfull[l]; };
                if ((st = launch_up((C*)rb.Mfull[p->lg], p->lg, p->B, 1LL << p->lg, outs))) return st;
            }
            // M2L-B (+ REDUCE): targets = own boxes if l_g == B, else all 2^B boxes
            if (p->lg == p->B) {
                if ((st = launch_base(rb, (C*)rb.Lloc[p->B], (long long)g * nb_at(p->B), nb_at(p->B)))) return st;
            } else {
                if ((st = launch_base(rb, (C*)rb.Lfull[p->B], 0, 1 << p->B))) return st;
            }
        }
        return FMMFFT_SUCCESS;
    }

    // level l's source / output placement (global box indices -> buffers)
    TreeLevel level_io(RankBufs& rb, int lev, long long g) const {
        TreeLevel tl{};
        const long long nbl = nb_at(lev);
        tl.tab = p->m2l[lev];
        if (p->G == 1) {
            tl.src = interior(rb.Mpad[lev]); tl.src_base = 0; tl.src_mod = 1 << lev;
            tl.out = rb.Lloc[lev]; tl.out_base = 0;
        } else if (lev <= p->lg) {
            tl.src = rb.Mfull[lev]; tl.src_base = 0; tl.src_mod = 1 << lev;
            if (lev == p->lg) { tl.out = rb.Lloc[lev]; tl.out_base = g * nbl; }
            else { tl.out = rb.Lfull[lev]; tl.out_base = 0; }
        } else {
            tl.src = rb.Mpad[lev]; tl.src_base = g * nbl - 2; tl.src_mod = 0;
            tl.out = rb.Lloc[lev]; tl.out_base = g * nbl;
        }
        return tl;
    }

    // first level handled by the per-level kernel k_m2l_lvl (levels with >= 2 tiles per rank);
    // the levels above it go to k_tree_down. FMMFFT_DOWN=tree keeps every level in k_tree_down.
    int lvl_first() const {
        if (!(p->Q == 8 || p->Q == 16 || p->Q == 24)) return p->L + 1;
        constexpr int PCl = lvl_pc<R>();
        if (p->PCd % PCl || p->P % PCl) return p->L + 1;
        // a level goes to k_m2l_lvl once its tiles x p sub-chunks fill the GPU; narrower levels
        // are latency-bound there (one tile per CTA) and cheaper inside k_tree_down's single launch
        const int nsub = p->P / PCl;
        for (int lev = std::max(p->B, p->lg) + 1; lev <= p->L; ++lev)
            if (nb_at(lev) >= 2 * lvl_nt<R, 16>() && (long long)(nb_at(lev) / lvl_nt<R, 16>()) * nsub >= 148) return lev;
        return p->L + 1;
    }

    // ---- down: M2L + L2L for every level B+1 .. L: k_tree_down over the upper levels (one
    // launch, per leaf range), then one k_m2l_lvl launch per wide level
    // targets of level lev on this rank: all 2^lev boxes (G = 1, or the replicated levels < l_g),
    // else the rank's own boxes
    std::pair<long long, int> narrow_targets(long long g, int lev) const {
        if (p->G == 1 || lev < p->lg) return {0, 1 << lev};
        return {g * nb_at(lev), nb_at(lev)};
    }

    fmmfft_status_t down() {
        if (p->L == p->B || p->tree_p) return FMMFFT_SUCCESS;
        if (p->top_L) return p->top_L < p->L ? down_levels(p->top_L + 1) : FMMFFT_SUCCESS;
        int lnew = lvl_first();
        if (narrow_ok()) {                           // k_down_narrow up to the widest level that fits
            int lnar = p->B, nmax = 0;
            for (int lev = p->B + 1; lev < lnew; ++lev) {
                const int n = narrow_targets(0, lev).second;
                if (!narrow_down_fits(std::max(nmax, n))) break;
                nmax = std::max(nmax, n);
                lnar = lev;
            }
            constexpr int PCl = lvl_pc<R>();
            const bool lvl_usable = p->PCd % PCl == 0 && p->P % PCl == 0;
            if (lnar > p->B && (lnar == lnew - 1 || FMMFFT_NARROW_FORCE) && (lnar == p->L || lvl_usable)) {
                for (RankBufs& rb : p->ranks) {
                    const long long g = grank(rb);
                    NarrowArgs na{};
                    for (int lev = p->B + 1; lev <= lnar; ++lev) {
                        const TreeLevel tl = level_io(rb, lev, g);
                        NarrowLevel& nl = na.lev[lev];
                        nl.src = tl.src; nl.src_base = tl.src_base; nl.src_mod = tl.src_mod;
                        nl.tab = p->m2l_pmaj[lev]; nl.out_base = tl.out_base;
                        // only the last level leaves the chip (the per-level kernels' parent / the leaf
                        // L^L); debug plans keep every level for the stage tests
                        nl.out = (lev == lnar || (p->flags & FMMFFT_FLAG_DEBUG)) ? tl.out : nullptr;
                        const auto ft = narrow_targets(g, lev);
                        nl.f = ft.first; nl.n = ft.second;
                    }
                    if (p->lg == p->B) { na.par0 = rb.Lloc[p->B]; na.par0_base = g * nb_at(p->B); }
                    else { na.par0 = rb.Lfull[p->B]; na.par0_base = 0; }
                    na.lstart = p->B + 1;
                    na.Lv = lnar;
                    na.nmax = nmax;
                    dispatch<8, 16, 24>(p->Q, [&](auto qv) {
                        constexpr int QV = decltype(qv)::value;
                        launch_pdl(k_down_narrow<R, QV>, (unsigned)(p->P - 1), 256, narrow_down_smem(nmax), s, na,
                                   (const R*)p->m2m, p->P);
                    });
                    LAUNCH_CHECK();
                }
                return down_levels(lnar + 1);
            }
        }
        const int Lv = lnew - 1;                     // k_tree_down's (virtual) leaf level
        const int PC_ = p->PCd;
        const int npc = p->P / PC_;
        const int QPC = p->Q * PC_;
        int optin = 0;
        CUDA_TRY(cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, p->device));
        for (RankBufs& rb : p->ranks) {
            const long long g = grank(rb);
            if (Lv > p->B) {
                const int nbv = nb_at(Lv);
                auto smem_of = [&](int nr, int db) {
                    return (size_t)(1 + db) * p->m2l_chunk * sizeof(R) + (size_t)(1 + db) * (nr + 6) * QPC * sizeof(C) +
                           (size_t)nr * QPC * sizeof(C) + (size_t)(nr / 2 + 1) * QPC * sizeof(C) + (size_t)2 * p->Q * p->Q * sizeof(R);
                };
                int NR = std::min(16, nbv);
                while (NR > 1 && (long long)(nbv / NR) * npc < 148) NR /= 2;
                while (NR > 1 && smem_of(NR, 0) > (size_t)optin) NR /= 2;
                const int db = smem_of(NR, 1) <= (size_t)optin ? 1 : 0;
                const size_t smem = smem_of(NR, db);
                TreeDownArgs a{};
                for (int lev = p->B + 1; lev <= Lv; ++lev) a.lev[lev] = level_io(rb, lev, g);
                if (p->lg == p->B) { a.par0 = rb.Lloc[p->B]; a.par0_base = g * nb_at(p->B); }
                else { a.par0 = rb.Lfull[p->B]; a.par0_base = 0; }
                a.leaf0 = g * nbv;
                a.lstart = p->B + 1;
                a.L = Lv;
                const dim3 grid((unsigned)(nbv / NR), (unsigned)npc);
                with_pcd([&](auto pc) {
                    constexpr int PCv = decltype(pc)::value;
                    dispatch<1, 2, 4, 8, 16>(NR, [&](auto nr) {
                        constexpr int NRv = decltype(nr)::value;
                        launch_pdl(k_tree_down<R, PCv, NRv>, grid, PCv * p->Q, smem, s, a, (const R*)p->m2m, p->P, p->Q,
                                                                                p->m2l_chunk, db);
                    });
                });
                LAUNCH_CHECK();
            }
        }
        return down_levels(lnew);
    }

    // one k_m2l_lvl launch per level first..L (wide levels: M2L + L2L, register-blocked)
    fmmfft_status_t down_levels(int first) {
        int optin = 0;
        CUDA_TRY(cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, p->device));
        for (RankBufs& rb : p->ranks) {
            const long long g = grank(rb);
            for (int lev = first; lev <= p->L; ++lev) {
                const TreeLevel tl = level_io(rb, lev, g);
                LvlArgs la{};
                la.src = tl.src; la.src_base = tl.src_base; la.src_mod = tl.src_mod;
                la.out = tl.out; la.out_base = tl.out_base;
                if (lev - 1 == p->B) {
                    if (p->lg == p->B) { la.par = rb.Lloc[p->B]; la.par_base = g * nb_at(p->B); }
                    else { la.par = rb.Lfull[p->B]; la.par_base = 0; }
                } else {
                    const TreeLevel tp = level_io(rb, lev - 1, g);
                    la.par = tp.out; la.par_base = tp.out_base;
                }
                la.tab = tl.tab; la.tab_chunk = p->m2l_chunk; la.PCd = p->PCd;
                la.tgt0 = g * nb_at(lev);
                constexpr int PCl = lvl_pc<R>();
                const int nsub = p->P / PCl;
                bool ok = dispatch<8, 16, 24>(p->Q, [&](auto qv) {
                    constexpr int QV = decltype(qv)::value;
                    constexpr int NT = lvl_nt<R, QV>();
                    la.ntiles = nb_at(lev) / NT;
                    const size_t smem = lvl_smem<R, QV>();
                    const int per_sm = std::max(1, std::min(2, (int)((size_t)(optin + 1024) / (smem + 1024))));
                    const int target = 148 * per_sm;
                    const int nseg = (int)std::max(1LL, std::min<long long>(la.ntiles, (target + nsub - 1) / nsub));
                    if constexpr (sizeof(R) == 8)            // FP64 tensor pipe
                        launch_pdl(k_m2l_dmma<QV>, dim3((unsigned)nseg, (unsigned)nsub), 256, smem, s, la, (const double*)p->m2m, p->P);
                    else
                        launch_pdl(k_m2l_lvl<R, QV>, dim3((unsigned)nseg, (unsigned)nsub), lvl_threads<R, QV>(), smem, s, la,
                                   (const R*)p->m2m, p->P);
                });
                if (!ok) return fail(FMMFFT_UNSUPPORTED, "k_m2l_lvl: Q=%d", p->Q);
                LAUNCH_CHECK();
            }
        }
        return FMMFFT_SUCCESS;
    }

    // ---- L2T + POST + P-FFT
    fmmfft_status_t post_pfft() {
        // P <= 32 (and a specialised Q): the register-resident variant, one thread per (box, m)
        if (p->P <= 32 && p->P >= 2 && (p->Q == 8 || p->Q == 16 || p->Q == 24) && p->M_L <= 256) {
            const int nbx = std::max(1, std::min(p->nb, 256 / p->M_L));
            if (p->nb % nbx == 0) {
                const size_t smem = ((size_t)nbx * p->Q * p->P + 2 * p->P + 16) * sizeof(C) + (size_t)p->Q * p->M_L * sizeof(R);
                for (RankBufs& rb : p->ranks) {
                    bool ok = dispatch<1, 2, 3, 4, 5>(ilog2(p->P), [&](auto lp) {
                        constexpr int LP = decltype(lp)::value;
                        dispatch<8, 16, 24>(p->Q, [&](auto qv) {
                            launch_pdl(k_post_pfft_r<R, LP, decltype(qv)::value>, (unsigned)(p->nb / nbx), nbx * p->M_L, smem, s,
                                       (const C*)rb.Tn, (const C*)rb.Lloc[p->L], (const C*)rb.r, (const C*)p->rho,
                                       (const R*)p->s2m, (C*)rb.W, ilog2(p->M_L), (int)p->Mg, (int)p->pmaj);
                        });
                    });
                    if (!ok) return fail(FMMFFT_UNSUPPORTED, "k_post_pfft_r: P=%d", p->P);
                    LAUNCH_CHECK();
                }
                return FMMFFT_SUCCESS;
            }
        }
        // m sub-tile per CTA: the whole P-point FFT tile, split further (down to 16) while that
        // leaves fewer than ~4 CTAs per SM (small N: latency-bound, more CTAs in flight)
        int MS = std::min(p->M_L, std::max(8, TILE / p->P));     // >= 8: the L2T phase owns 8 m per thread
        while (MS > 16 && (long long)p->nb * (p->M_L / MS) < 4 * 148) MS /= 2;
        const int threads = std::min(sizeof(R) == 4 ? 1024 : 512, std::max(32, MS * p->P / 8));
        size_t smem = (size_t)MS * (p->P + 1) * sizeof(C) + (size_t)p->P * sizeof(C) + (size_t)p->Q * MS * sizeof(R);
        const int stage_L = smem + (size_t)(p->Q + 1) * p->P * sizeof(C) <= 160 * 1024;   // stage L^L of the box
        if (stage_L) smem += (size_t)(p->Q + 1) * p->P * sizeof(C);
        const int blocks = p->nb * (p->M_L / MS);
        for (RankBufs& rb : p->ranks) {
            const int qt = (p->Q == 8 || p->Q == 16 || p->Q == 24) ? p->Q : 0;
            dispatch<1, 2, 3, 4, 5, 6, 7, 8, 9, 10, 11>(ilog2(p->P), [&](auto lp) {
                constexpr int LP = decltype(lp)::value;
                dispatch<0, 8, 16, 24>(qt, [&](auto qv) {
                    launch_pdl(k_post_pfft<R, LP, decltype(qv)::value>, blocks, threads, smem, s, (const C*)rb.Tn,
                               (const C*)rb.Lloc[p->L], (const C*)rb.r, (const C*)p->rho, (const R*)p->s2m, (C*)rb.W,
                               ilog2(p->M_L), p->Q, ilog2(MS), (int)p->Mg, stage_L, (int)p->pmaj);
                });
            });
            LAUNCH_CHECK();
        }
        return FMMFFT_SUCCESS;
    }

    // ---- the all-to-all: chunk r of W (k2 in r's block, own m) -> rank r's Rcv slot g
    fmmfft_status_t a2a() {
        if (p->G == 1) return FMMFFT_SUCCESS;
        return exchange([this](const RankBufs& rb) { return sched_A2A(rb); }, s);
    }

    // one column pass of the four-step M-FFT (k_fft_col): nseq sequences of length 2^lMs
    // (lMi_ >= 0: inner count given explicitly, then lMs only sets the twiddle w_{2^lMs}; 0 = none)
    fmmfft_status_t col_pass(const C* in_, C* out_, int LCv, int lMs, int lSdiv, long long in_row, int lblk,
                             long long blk_stride, long long nseq, int lMi_ = -1) {
        const int lMi = lMi_ >= 0 ? lMi_ : lMs - LCv;
        bool ok = dispatch<5, 6, 7, 8, 9, 10, 11>(LCv, [&](auto lc) {
            constexpr int LC = decltype(lc)::value;
            constexpr int CB = fs_cols<R>(LC);
            if constexpr (LC <= fs_max<R>()) {
                launch_pdl(k_fft_col<R, LC, CB>, dim3((unsigned)((1LL << lMi) / CB), (unsigned)nseq), CB << (LC - 4),
                           fft_col_smem<R, LC, CB>(), s, in_, out_, lMs, lMi, lSdiv, (long long)p->M, in_row, lblk, blk_stride);
            }
        });
        if (!ok) return fail(FMMFFT_UNSUPPORTED, "k_fft_col: 2^%d", LCv);
        LAUNCH_CHECK();
        return FMMFFT_SUCCESS;
    }

    // ---- M-point FFTs over the P/G local rows (line 16): from the all-to-all receive
    // layout (G > 1: [src][row][m_local(src)]) or the P-FFT output [row][m] (G = 1), into `dst`
    // (default: the caller's output) in natural order
    fmmfft_status_t mfft(const C* src_override = nullptr, bool to_tn = false) {
        fmmfft_status_t st_;
        const int n = (int)p->radices.size();
        const long long rows = p->P / p->G;
        const int lM = ilog2(p->M);
        for (RankBufs& rb : p->ranks) {
            C* dst = to_tn ? (C*)rb.Tn : out[gidx(rb)];
            const C* dcp = p->direct ? nullptr : (const C*)rb.dc;    // the rows' k = 0 outputs (R19)
            const C* src = src_override ? src_override : (const C*)(p->G > 1 ? rb.Rcv : rb.W);
            if (src_override == in[0] && p->virt) src = in[gidx(rb)];
            long long in_row = p->M, blk_stride = 0;
            int lblk = 62;
            if (p->G > 1 && src_override != in[0]) { in_row = p->Mg; lblk = ilog2(p->Mg); blk_stride = (p->P / p->G) * p->Mg; }
            if (p->fs_lr) {                      // four-step: column pass(es) + transposing row pass
                // (running every pass of a group of rows back to back, so the group's intermediate
                // stays in L2, measured slower at cfg3: 499 -> 524-538 us for groups of 4 / 2 rows)
                const int npass = p->fs_lc2 ? 3 : 2;
                C* a1out = npass == 3 ? dst : (C*)rb.tmp;
                if ((st_ = col_pass(src, a1out, p->fs_lc1, lM, 0, in_row, lblk, blk_stride, rows))) return st_;
                const C* bsrc = a1out;
                if (npass == 3) {
                    const int lMs = lM - p->fs_lc1;
                    if ((st_ = col_pass(dst, (C*)rb.tmp, p->fs_lc2, lMs, p->fs_lc1, 1LL << lMs, 62, 0, rows << p->fs_lc1))) return st_;
                    bsrc = (const C*)rb.tmp;
                }
                const int lrpr = lM - p->fs_lr;
                const long long trows = rows << lrpr;
                bool ok = dispatch<5, 6, 7, 8, 9, 10, 11>(p->fs_lr, [&](auto ll) {
                    constexpr int LL = decltype(ll)::value;
                    constexpr int CR = fs_cols<R>(LL);
                    if constexpr (LL <= fs_max<R>())
                        launch_pdl(k_fft_rowt<R, LL, CR>, (unsigned)(trows / CR), CR << (LL - 4), fft_rowt_smem<R, LL, CR>(), s,
                                   bsrc, dst, (long long)p->M, lrpr, dcp);
                });
                if (!ok) return fail(FMMFFT_UNSUPPORTED, "k_fft_rowt: 2^%d", p->fs_lr);
                LAUNCH_CHECK();
                continue;
            }
            if (p->row_fft1) {                   // one pass per row, the row in shared memory
                const size_t smem = ((size_t)p->M + p->M / 16 + p->M / 16) * sizeof(C);
                dispatch<8, 9, 10, 11, 12, 13, 14>(lM, [&](auto ll) {
                    constexpr int LL = decltype(ll)::value;
                    if constexpr (LL <= kRowFftMax<R>)
                        launch_pdl(k_fft_row<R, LL>, (unsigned)rows, 1 << (LL - 4), smem, s, src, dst, (const C*)p->twM,
                                   (int)in_row, lblk == 62 ? lM : lblk, (int)blk_stride, dcp);
                });
                LAUNCH_CHECK();
                continue;
            }
            int lNs = 0;
            for (int i = 0; i < n; ++i) {
                const int Rp = p->radices[i], lR = ilog2(Rp);
                C* o = ((n - 1 - i) % 2 == 0) ? dst : (C*)rb.tmp;
                const long long nj = p->M / Rp;
                long long c = std::min<long long>(TILE / Rp, nj);
                while (c > 8 && c * Rp > 2048 && (nj / c) * rows < 2 * 148) c /= 2;
                int ir = (int)p->M, lb = lM, bs = 0;
                if (i == 0 && blk_stride) {
                    ir = (int)in_row; lb = lblk; bs = (int)blk_stride;
                    c = std::min<long long>(c, p->Mg);
                }
                const int threads = (int)std::min<long long>(sizeof(R) == 4 ? 1024 : 512, std::max<long long>(32, c * Rp / 8));
                const size_t smem = (size_t)c * (Rp + 1) * sizeof(C) + (size_t)Rp * sizeof(C);
                const dim3 grid((unsigned)(nj / c), (unsigned)rows);
                dispatch<1, 2, 3, 4, 5, 6, 7, 8, 9, 10>(lR, [&](auto lr) {
                    constexpr int LR = decltype(lr)::value;
                    launch_pdl(k_fft_pass<R, LR>, grid, threads, smem, s, src, o, lM, lNs, ilog2(c), ir, lb, bs,
                               i == n - 1 ? dcp : (const C*)nullptr);
                });
                LAUNCH_CHECK();
                src = o;
                lNs += lR;
            }
        }
        return FMMFFT_SUCCESS;
    }

    // the k1 = 0 bins of the local M-FFT rows from the reductions r_p (k_dc_bins, reading R19): on
    // the side stream once r is known (after top), into rb.dc; the last M-FFT pass stores them
    fmmfft_status_t dc_bins() {
        const int rows = p->P / p->G;
        CUDA_TRY(cudaEventRecord(p->dc_fork, s));
        CUDA_TRY(cudaStreamWaitEvent(side(), p->dc_fork, 0));
        for (RankBufs& rb : p->ranks) {
            // r_0: reduced by the per-level kernels (k_base*), or here from M^L's slot 0 when the
            // fused per-FMM far field (p = 1..P-1 only) ran
            const C* m0 = nullptr;
            long long m0_n = 0, m0_stride = 0;
            if (p->tree_p) {
                m0 = interior(rb.Mpad[p->L]);
                m0_n = (long long)p->nb * p->Q;
                m0_stride = p->pmaj ? 1 : p->P;
            }
            launch_pdl(k_dc_bins<R>, (unsigned)((rows + 7) / 8), 256, 0, side(), (C*)rb.dc, (const C*)rb.r, m0, m0_n,
                       m0_stride, p->P, rows, grank(rb) * rows, (long long)p->M, (const double2*)rb.r0p,
                       p->top_L ? (p->P - 1) * p->top_cl : 0);
            LAUNCH_CHECK();
        }
        CUDA_TRY(cudaEventRecord(p->dc_join, side()));
        return FMMFFT_SUCCESS;
    }

    // inverse plans: y <- scale * conj(x) over this rank's N/G elements
    fmmfft_status_t conj_scale(const C* x, C* y, R scale) {
        const long long n = p->N / p->G;
        const unsigned blocks = (unsigned)std::min<long long>((n / 2 + 255) / 256, 148LL * 8);
        launch_pdl(k_conj_scale<R>, blocks, 256, 0, s, x, y, n, scale);
        LAUNCH_CHECK();
        return FMMFFT_SUCCESS;
    }

    // real-input plans: X_k, k = 0..H, from Z = F_H z (k_r2c_post)
    fmmfft_status_t r2c_post(const C* Z, C* X) {
        const long long H = p->N;
        const unsigned blocks = (unsigned)std::min<long long>((H / 2 + 256) / 256, 148LL * 8);
        launch_pdl(k_r2c_post<R>, blocks, 256, 0, s, Z, X, H);
        LAUNCH_CHECK();
        return FMMFFT_SUCCESS;
    }

    fmmfft_status_t run() {
        fmmfft_status_t st;
        if (p->real && p->inverse) {                    // C2R: conj(Z) -> forward -> conj / H = z
            const long long H = p->N;
            if (p->G > 1 && (st = exchange([this](const RankBufs& rb) { return sched_mirror(rb, in[gidx(rb)], true); }, s)))
                return st;
            for (RankBufs& rb : p->ranks) {
                const int g = gidx(rb);
                C* Zc = (C*)rb.cin;
                if (p->G == 1) {
                    const unsigned blocks = (unsigned)std::min<long long>((H / 2 + 256) / 256, 148LL * 8);
                    launch_pdl(k_c2r_pre<R>, blocks, 256, 0, s, in[g], Zc, H);
                } else {
                    const long long nl = H / p->G;
                    const unsigned blocks = (unsigned)std::min<long long>((nl + 255) / 256, 148LL * 8);
                    launch_pdl(k_c2r_pre_dist<R>, blocks, 256, 0, s, in[g], (const C*)rb.mir, (const C*)rb.xtra, Zc, H, nl,
                               (long long)grank(rb) * nl);
                }
                LAUNCH_CHECK();
                in[g] = Zc;
            }
            if ((st = run_forward())) return st;
            for (RankBufs& rb : p->ranks)
                if ((st = conj_scale(out[gidx(rb)], out[gidx(rb)], R(1) / (R)H))) return st;
            return FMMFFT_SUCCESS;
        }
        if (p->real) {                                  // z_j = x_{2j} + i x_{2j+1}: the input as is
            std::vector<C*> X = out;
            for (RankBufs& rb : p->ranks) out[gidx(rb)] = (C*)rb.rz;
            if ((st = run_forward())) return st;
            if (p->G == 1) return r2c_post(out[0], X[0]);
            if ((st = exchange([this](const RankBufs& rb) { return sched_mirror(rb, (const C*)rb.rz, false); }, s))) return st;
            for (RankBufs& rb : p->ranks) {
                const long long nl = p->N / p->G;
                const unsigned blocks = (unsigned)std::min<long long>((nl + 255) / 256, 148LL * 8);
                launch_pdl(k_r2c_post_dist<R>, blocks, 256, 0, s, (const C*)rb.rz, (const C*)rb.mir, (const C*)rb.xtra,
                           X[gidx(rb)], p->N, nl, (long long)grank(rb) * nl, (int)(grank(rb) == p->G - 1));
                LAUNCH_CHECK();
            }
            return FMMFFT_SUCCESS;
        }
        if (p->inverse)                                 // F^{-1} x = conj(F conj(x)) / N
            for (RankBufs& rb : p->ranks) {
                const int g = p->virt ? rb.g : 0;
                if ((st = conj_scale(in[g], (C*)rb.cin, R(1)))) return st;
                in[g] = (const C*)rb.cin;
            }
        if ((st = run_forward())) return st;
        if (p->inverse)
            for (RankBufs& rb : p->ranks) {
                const int g = p->virt ? rb.g : 0;
                if ((st = conj_scale(out[g], out[g], R(1) / (R)p->N))) return st;
            }
        return FMMFFT_SUCCESS;
    }

    // ---- the distributed radix-P Cooley-Tukey FFT with three all-to-alls (FMMFFT_FLAG_DIRECT,
    // G > 1): the same exchange schedule, M-FFT kernels and column
    // pass as the FMM-FFT, so the two differ only in the FMM vs the two extra transposes
    fmmfft_status_t run_direct_dist() {
        fmmfft_status_t st;
        const long long Mg = p->Mg, rows = p->P / p->G;
        auto a2a_ = [this]() { return exchange([this](const RankBufs& rb) { return sched_A2A(rb); }, s); };
        for (RankBufs& rb : p->ranks) {                 // (1) [m_local][p] -> [p][m_local]
            const dim3 grid((unsigned)((p->P + 31) / 32), (unsigned)((Mg + 31) / 32));
            launch_pdl(k_transpose_rc<R>, grid, dim3(32, 8), 0, s, in[gidx(rb)], (C*)rb.W, Mg, (long long)p->P);
            LAUNCH_CHECK();
        }
        if ((st = a2a_())) return st;                   //     transpose P-major -> M-major
        if ((st = mfft(nullptr, true))) return st;      // (2) P/G local M-point FFTs -> Tn
        for (RankBufs& rb : p->ranks) {                 // (3) twiddle + (4)'s send layout
            const unsigned blocks = (unsigned)std::min<long long>((p->M * rows + 255) / 256, 148LL * 8);
            launch_pdl(k_twiddle_chunk<R>, blocks, 256, 0, s, (const C*)rb.Tn, (C*)rb.W, (long long)p->M, ilog2(Mg),
                       ilog2(rows), (long long)grank(rb) * rows, p->N);
            LAUNCH_CHECK();
        }
        if ((st = a2a_())) return st;                   //     transpose M-major -> P-major
        for (RankBufs& rb : p->ranks)                   // (5) M/G local P-point FFTs (columns of [p][k1_local])
            if ((st = col_pass((const C*)rb.Rcv, (C*)rb.W, ilog2(p->P), 0, 0, 0, 62, 0, 1, ilog2(Mg)))) return st;
        if ((st = a2a_())) return st;                   // (6) transpose P-major -> M-major
        for (RankBufs& rb : p->ranks)                   //     [src][k2_local][k1_local] -> y[k1 + M k2]
            for (int src = 0; src < p->G; ++src)
                CUDA_TRY(cudaMemcpy2DAsync(out[gidx(rb)] + src * Mg, (size_t)p->M * sizeof(C), (const C*)rb.Rcv + src * rows * Mg,
                                           (size_t)Mg * sizeof(C), (size_t)Mg * sizeof(C), (size_t)rows, cudaMemcpyDeviceToDevice, s));
        return FMMFFT_SUCCESS;
    }

    fmmfft_status_t run_forward() {
        fmmfft_status_t st;
        if (p->direct) return p->G > 1 ? run_direct_dist() : mfft(in[0]);
#define STEP(stage, call) if ((st = mark(stage))) return st; if ((st = call)) return st;
        if ((st = mark(ST_COMM_S))) return st;
        if (p->G > 1) {                                 // S halo on the side stream (overlaps S2M)
            CUDA_TRY(cudaEventRecord(p->fork, s));
            CUDA_TRY(cudaStreamWaitEvent(side(), p->fork, 0));
            if ((st = comm_S(side()))) return st;
            CUDA_TRY(cudaEventRecord(p->cs_done, side()));
        }
        STEP(ST_NEAR, near_up())
        STEP(ST_M2M, m2m_local())
        STEP(ST_COMM_M, comm_M())
        STEP(ST_TOP, top())
        if ((st = dc_bins())) return st;
        STEP(ST_DOWN, down())
        if ((st = join_near())) return st;
        STEP(ST_PFFT, post_pfft())
        STEP(ST_A2A, a2a())
        if ((st = mark(ST_MFFT))) return st;
        CUDA_TRY(cudaStreamWaitEvent(s, p->dc_join, 0));
        if ((st = mfft())) return st;
#undef STEP
        return mark(ST_COUNT);
    }
};

template <typename R>
static fmmfft_status_t execute_t(fmmfft_plan_s* p, const void* in, void* out, cudaStream_t s) {
    // replay a captured graph for this (in, out) pair
    if (p->use_graph) {
        for (auto& ge : p->graphs)
            if (ge.in == in && ge.out == out) {
                CUDA_TRY(cudaGraphLaunch(ge.exec, s));
                p->kernels = ge.nlaunch;
                p->have_times = (p->flags & FMMFFT_FLAG_PROFILE) != 0;
                return FMMFFT_SUCCESS;
            }
    }
    const long long nl = p->N / p->G;
    auto make = [&](cudaStream_t st) {
        Exec<R> ex{p, st, {}, {}};
        if (p->virt) {
            for (int g = 0; g < p->G; ++g) {
                ex.in.push_back((const C2<R>*)in + g * nl);
                ex.out.push_back((C2<R>*)out + g * nl);
            }
        } else {
            ex.in.push_back((const C2<R>*)in);
            ex.out.push_back((C2<R>*)out);
        }
        return ex;
    };
    if (!p->use_graph) {
        Exec<R> ex = make(s);
        fmmfft_status_t st = ex.run();
        p->kernels = ex.nlaunch;
        p->have_times = st == FMMFFT_SUCCESS && (p->flags & FMMFFT_FLAG_PROFILE);
        return st;
    }
    // capture on the plan's own stream (the caller's may be the legacy default stream)
    Exec<R> ex = make(p->cap_stream);
    CUDA_TRY(cudaStreamBeginCapture(p->cap_stream, cudaStreamCaptureModeRelaxed));
    fmmfft_status_t st = ex.run();
    cudaGraph_t graph = nullptr;
    cudaError_t e = cudaStreamEndCapture(p->cap_stream, &graph);
    if (st) {
        if (graph) cudaGraphDestroy(graph);
        return st;
    }
    CUDA_TRY(e);
    cudaGraphExec_t exec = nullptr;
    e = cudaGraphInstantiate(&exec, graph, 0);
    cudaGraphDestroy(graph);
    CUDA_TRY(e);
    if (p->graphs.size() >= 8) {
        cudaGraphExecDestroy(p->graphs.front().exec);
        p->graphs.erase(p->graphs.begin());
    }
    p->graphs.push_back(GraphEntry{in, out, exec, ex.nlaunch});
    CUDA_TRY(cudaGraphLaunch(exec, s));
    p->kernels = ex.nlaunch;
    p->have_times = (p->flags & FMMFFT_FLAG_PROFILE) != 0;
    return FMMFFT_SUCCESS;
}

}  // namespace fmmfft

using namespace fmmfft;

// ====================================================================== C ABI
// ---------------------------------------------------------------- autotuner
static double tune_error(int Q, fmmfft_precision_t prec) {
    const double trunc = 1.7e-3 * std::pow(6.3, -(double)(Q - 2));      // oracle Q sweep
    return std::max(trunc, prec == FMMFFT_C64 ? 2.6e-7 : 3e-14);
}

// roofline model of one execute (seconds), per GPU: HBM passes, S2T flops on the tensor pipe
// (c64) or FFMA / DFMA, the tree's flops at the register-blocked kernels' measured efficiency,
// and a per-launch latency
static double tune_model(long long N, int P, int G, int B, int Q, int M_L, fmmfft_precision_t prec) {
    const double esz = prec == FMMFFT_C64 ? 8 : 16;
    const double n = (double)N / G, fmm = (double)(P - 1) / P;
    const int L = ilog2(N / ((long long)P * M_L));
    const double hbm = 6.4e12, alu = prec == FMMFFT_C64 ? 74e12 : 37e12;
    const double tc = prec == FMMFFT_C64 ? 279e12 * 0.25 : 0.0;        // 3xTF32, smem-operand bound
    const int lM = ilog2(N / P);
    const int mpass = lM <= 14 ? 1 : (lM <= 22 ? 2 : 3);
    double t = (2 + 2 + 2 * mpass) * n * esz / hbm;                    // s2m, post_pfft, M-FFT passes
    if (prec == FMMFFT_C64) t += n * esz / hbm;                         // the S' copy
    const double s2t = 6.0 * 2 * M_L * fmm * n;
    t += prec == FMMFFT_C64 && M_L == 64 ? s2t / tc : s2t / (0.35 * alu);
    const double far = 2.0 * (20.0 * Q * Q / M_L + 4.0 * Q) * fmm * n;
    t += far / (0.3 * alu) + ((1 << B) * ((1 << B) - 3)) * 4.0 * Q * Q * (P - 1) / (0.05 * alu);
    const int launches = 6 + 2 * std::max(0, L - B);
    t += launches * 4e-6;
    if (G > 1) t += (double)(G - 1) / G * n * esz / 700e9;              // the all-to-all over NVLink
    return t;
}

template <typename R>
static fmmfft_status_t tune_measure(long long N, int P, int B, int Q, int M_L, fmmfft_precision_t prec, float* ms) {
    fmmfft_plan_t pl = nullptr;
    fmmfft_status_t st = fmmfft_plan_ex(&pl, N, P, 1, B, Q, prec, M_L, 0u);
    if (st) return st;
    void *x = nullptr, *y = nullptr;
    const size_t bytes = (size_t)N * sizeof(C2<R>);
    cudaStream_t s = nullptr;
    cudaEvent_t e0 = nullptr, e1 = nullptr;
    cudaError_t e = cudaMalloc(&x, bytes);
    if (e == cudaSuccess) e = cudaMalloc(&y, bytes);
    if (e == cudaSuccess) e = cudaMemset(x, 0x3c, bytes);               // finite values (~1e-2 .. 1)
    if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
    if (e == cudaSuccess) e = cudaEventCreate(&e0);
    if (e == cudaSuccess) e = cudaEventCreate(&e1);
    if (e != cudaSuccess) st = fail(FMMFFT_CUDA_ERROR, "autotune scratch: %s", cudaGetErrorString(e));
    for (int i = 0; i < 3 && !st; ++i) st = fmmfft_execute(pl, x, y, s);
    if (!st) {
        cudaEventRecord(e0, s);
        for (int i = 0; i < 5 && !st; ++i) st = fmmfft_execute(pl, x, y, s);
        cudaEventRecord(e1, s);
        e = cudaEventSynchronize(e1);
        float t = 0;
        if (e == cudaSuccess) e = cudaEventElapsedTime(&t, e0, e1);
        if (e != cudaSuccess) st = fail(FMMFFT_CUDA_ERROR, "autotune timing: %s", cudaGetErrorString(e));
        *ms = t / 5;
    }
    if (e0) cudaEventDestroy(e0);
    if (e1) cudaEventDestroy(e1);
    if (s) cudaStreamDestroy(s);
    if (x) cudaFree(x);
    if (y) cudaFree(y);
    fmmfft_destroy(pl);
    return st;
}

extern "C" {

const char* fmmfft_last_error(void) { return g_last_error.c_str(); }
const char* fmmfft_version(void) { return "fmmfft-b200 0.2 (sm_100a)"; }
const char* fmmfft_stage_name(int i) { return (i >= 0 && i <= ST_COUNT) ? kStageNames[i] : ""; }

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
    if (g_comm_plans > 0) return fail(FMMFFT_INVALID_VALUE, "%d live plan(s) use the communicator: destroy them first", (int)g_comm_plans);
    NCCL_TRY(nccl().CommDestroy(g_comm.comm));
    g_comm = Comm{};
    return FMMFFT_SUCCESS;
}

// FMMFFT_FLAG_DIRECT: the in-house Cooley-Tukey comparator — the same
// four-step FFT kernels (k_fft_col + k_fft_rowt) on the whole length-N vector, no FMM.
// FMMFFT_FLAG_DIRECT: the in-house Cooley-Tukey comparator — no FMM. G = 1: the
// four-step FFT kernels (k_fft_col + k_fft_rowt) on the whole length-N vector. G > 1: the
// distributed radix-P six-step FFT with its three all-to-alls, P = 2^ceil(log2 N / 2)
// clamped to the column pass's range, the same exchange schedule (NCCL or virtual ranks).
static fmmfft_status_t plan_direct(fmmfft_plan_t* plan, long long N, int G, fmmfft_precision_t precision, unsigned flags) {
    if (!pow2(N)) return fail(FMMFFT_INVALID_VALUE, "N must be a power of two");
    if (!(G == 1 || G == 2 || G == 4 || G == 8)) return fail(FMMFFT_INVALID_VALUE, "G must be 1, 2, 4 or 8");
    if (flags & FMMFFT_FLAG_PROFILE) return fail(FMMFFT_UNSUPPORTED, "FMMFFT_FLAG_DIRECT: no profile");
    const bool virt = (flags & FMMFFT_FLAG_VIRTUAL) != 0, vnccl = (flags & FMMFFT_FLAG_VIRTUAL_NCCL) != 0;
    if (G == 1 && (virt || vnccl)) return fail(FMMFFT_UNSUPPORTED, "FMMFFT_FLAG_DIRECT: virtual ranks need G > 1");
    if (vnccl && !virt) return fail(FMMFFT_INVALID_VALUE, "FMMFFT_FLAG_VIRTUAL_NCCL needs FMMFFT_FLAG_VIRTUAL");
    if ((G > 1 && !virt) || vnccl) {
        if (!g_comm.comm) return fail(FMMFFT_NOT_INITIALIZED, "G > 1 needs fmmfft_comm_init");
        if (g_comm.size != (vnccl ? 1 : G)) return fail(FMMFFT_INVALID_VALUE, "communicator size %d", g_comm.size);
    }
    int dev = 0;
    CUDA_TRY(cudaGetDevice(&dev));
    cudaDeviceProp prop;
    CUDA_TRY(cudaGetDeviceProperties(&prop, dev));
    if (prop.major != 10 || prop.minor != 0) return fail(FMMFFT_UNSUPPORTED, "sm_100a only");
    fmmfft_status_t st = precision == FMMFFT_C64 ? init_kernel_attrs<float>() : init_kernel_attrs<double>();
    if (st) return st;
    const int lN = ilog2(N), lPmax = precision == FMMFFT_C64 ? 11 : 10;
    const int lP = G == 1 ? 0 : std::max(5, std::min(lPmax, (lN + 1) / 2));
    if (G > 1 && (lN - lP < 8 || (1LL << (lN - lP)) % G || (1LL << lP) % G || (N >> lP) / G < 16))
        return fail(FMMFFT_UNSUPPORTED, "FMMFFT_FLAG_DIRECT: N = 2^%d too small for G = %d", lN, G);
    if (N / G > (1LL << 30)) return fail(FMMFFT_UNSUPPORTED, "N/G > 2^30 per rank not supported");
    fmmfft_plan_s* p = new fmmfft_plan_s;
    p->N = N; p->P = 1 << lP; p->M = N >> lP; p->G = G; p->Mg = p->M / G; p->prec = precision; p->flags = flags;
    p->device = dev; p->virt = virt; p->direct = true;
    p->inverse = (flags & FMMFFT_FLAG_INVERSE) != 0;
    p->esz = precision == FMMFFT_C64 ? 8 : 16;
    p->rsz = p->esz / 2;
    if ((G > 1 && !virt) || vnccl) {
        p->comm = g_comm.comm;
        p->comm_rank = g_comm.rank;
        p->vnccl = vnccl;
        ++g_comm_plans;
    }
    if (G == 1) {
        choose_fourstep(p, lN, lPmax);
        if (!p->fs_lr) { destroy_plan(p); return fail(FMMFFT_UNSUPPORTED, "FMMFFT_FLAG_DIRECT: need 2^10 <= N <= 2^%d", precision == FMMFFT_C64 ? 33 : 30); }
    } else {
        plan_mfft(p);
        if (p->row_fft1) {                               // k_fft_row's twiddles w_M^u, u < M/16
            std::vector<double> tw(2 * (p->M / 16));
            for (long long u = 0; u < p->M / 16; ++u) {
                tw[2 * u] = std::cos(2 * M_PI * (double)u / (double)p->M);
                tw[2 * u + 1] = -std::sin(2 * M_PI * (double)u / (double)p->M);
            }
            st = precision == FMMFFT_C64 ? upload<float>(p, &p->twM, tw) : upload<double>(p, &p->twM, tw);
        }
    }
    const char* g_env = getenv("FMMFFT_NO_GRAPH");
    p->use_graph = !(g_env && g_env[0] == '1');
    const int nr = virt ? G : 1;
    const size_t nl = (size_t)(N / G) * p->esz;
    p->ranks.resize(nr);
    for (int g = 0; g < nr && !st; ++g) {
        RankBufs& rb = p->ranks[g];
        rb.g = virt ? g : p->comm_rank;
        st = dalloc(p, &rb.tmp, nl);
        if (!st && p->inverse) st = dalloc(p, &rb.cin, nl);
        if (!st && G > 1) st = dalloc(p, &rb.W, nl);
        if (!st && G > 1) st = dalloc(p, &rb.Rcv, nl);
        if (!st && G > 1) st = dalloc(p, &rb.Tn, nl);
    }
    if (!st) {
        cudaError_t e = cudaStreamCreateWithFlags(&p->cap_stream, cudaStreamNonBlocking);
        if (e != cudaSuccess) st = fail(FMMFFT_CUDA_ERROR, "stream setup: %s", cudaGetErrorString(e));
    }
    if (st) { destroy_plan(p); return st; }
    *plan = p;
    return FMMFFT_SUCCESS;
}

static fmmfft_status_t plan_complex(fmmfft_plan_t* plan, long long N, int P, int G, int B, int Q,
                                    fmmfft_precision_t precision, int M_L, unsigned flags) {
    if (!plan) return fail(FMMFFT_INVALID_VALUE, "plan is NULL");
    *plan = nullptr;
    if (precision != FMMFFT_C64 && precision != FMMFFT_C128) return fail(FMMFFT_INVALID_VALUE, "bad precision");
    if (flags & FMMFFT_FLAG_DIRECT) return plan_direct(plan, N, G, precision, flags);
    if (precision != FMMFFT_C64 && precision != FMMFFT_C128) return fail(FMMFFT_INVALID_VALUE, "bad precision");
    if (!pow2(N) || !pow2(P) || !pow2(M_L)) return fail(FMMFFT_INVALID_VALUE, "N, P, M_L must be powers of two");
    // k_post_pfft holds >= 8 m-rows of all P points in one CTA's shared memory tile
    const int Pmax = precision == FMMFFT_C64 ? 1024 : 512;
    if (P < 2 || P > Pmax) return fail(FMMFFT_INVALID_VALUE, "need 2 <= P <= %d (P=%d)", Pmax, P);
    if (!(G == 1 || G == 2 || G == 4 || G == 8)) return fail(FMMFFT_INVALID_VALUE, "G must be 1, 2, 4 or 8");
    if (P % G) return fail(FMMFFT_INVALID_VALUE, "P %% G != 0");
    if (M_L < 16 || M_L > 128) return fail(FMMFFT_INVALID_VALUE, "need 16 <= M_L <= 128");
    if (Q < 2 || Q > 32) return fail(FMMFFT_INVALID_VALUE, "need 2 <= Q <= 32");
    if (N % ((long long)P * M_L)) return fail(FMMFFT_INVALID_VALUE, "N must be a multiple of P*M_L");
    if (N / G > (1LL << 30)) return fail(FMMFFT_UNSUPPORTED, "N/G > 2^30 per rank not supported");
    const long long nleaf = N / ((long long)P * M_L);
    const int L = ilog2(nleaf);
    if (B < 2 || L < B) return fail(FMMFFT_INVALID_VALUE, "need L >= B >= 2 (L=%d, B=%d)", L, B);
    if (B > 10) return fail(FMMFFT_UNSUPPORTED, "B > 10 not supported");
    if (nleaf % G) return fail(FMMFFT_INVALID_VALUE, "2^L %% G != 0");
    const bool virt = (flags & FMMFFT_FLAG_VIRTUAL) != 0;
    const bool vnccl = (flags & FMMFFT_FLAG_VIRTUAL_NCCL) != 0;
    if (vnccl && !virt) return fail(FMMFFT_INVALID_VALUE, "FMMFFT_FLAG_VIRTUAL_NCCL needs FMMFFT_FLAG_VIRTUAL");
    if ((G > 1 && !virt) || vnccl) {
        if (!g_comm.comm) return fail(FMMFFT_NOT_INITIALIZED, "G > 1 needs fmmfft_comm_init");
        const int want = vnccl ? 1 : G;
        if (g_comm.size != want) return fail(FMMFFT_INVALID_VALUE, "communicator size %d, need %d", g_comm.size, want);
    }
    int dev = 0;
    CUDA_TRY(cudaGetDevice(&dev));
    if (((G > 1 && !virt) || vnccl) && g_comm.device != dev)
        return fail(FMMFFT_INVALID_VALUE, "current device %d differs from the communicator's device %d", dev, g_comm.device);
    cudaDeviceProp prop;
    CUDA_TRY(cudaGetDeviceProperties(&prop, dev));
    if (prop.major != 10 || prop.minor != 0)
        return fail(FMMFFT_UNSUPPORTED, "device %s is sm_%d%d; this build is sm_100a only", prop.name, prop.major, prop.minor);
    fmmfft_status_t st = precision == FMMFFT_C64 ? init_kernel_attrs<float>() : init_kernel_attrs<double>();
    if (st) return st;

    fmmfft_plan_s* p = new fmmfft_plan_s;
    p->N = N; p->P = P; p->G = G; p->B = B; p->Q = Q; p->M_L = M_L; p->L = L;
    p->inverse = (flags & FMMFFT_FLAG_INVERSE) != 0;
    p->M = N / P; p->Mg = p->M / G; p->prec = precision; p->flags = flags; p->virt = virt; p->device = dev;
    if ((G > 1 && !virt) || vnccl) {
        p->comm = g_comm.comm;
        p->comm_rank = g_comm.rank;
        p->vnccl = vnccl;
        ++g_comm_plans;
    }
    p->nb = (int)(nleaf / G);
    p->lg = std::min(std::max(B, ilog2(G) + 1), L);
    if (G == 1) p->lg = B;
    p->esz = precision == FMMFFT_C64 ? 8 : 16;
    p->rsz = p->esz / 2;
    p->PCn = std::min(P, precision == FMMFFT_C64 ? 32 : 16);
    p->PCd = std::min(P, precision == FMMFFT_C64 ? 16 : 8);
    // fused per-FMM far field (k_tree_p) for single-GPU plans whose tree fits one CTA's
    // shared memory and at most 8 outputs per thread per level
    {
        const int threads = precision == FMMFFT_C64 ? 1024 : 512;
        int optin = 0;
        cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
        const size_t scratch = (((size_t)3 * Q) << (L > 0 ? L - 1 : 0)) * p->esz + (size_t)2 * Q * Q * p->rsz;
        p->tree_p = (G == 1) && ((long long)Q << L) <= 8LL * threads && tree_p_smem(p, threads) + scratch <= (size_t)optin;
        // FMMFFT_TREE=w: the per-level (wide-tree) kernels even where the fused far field fits
        if (const char* e = getenv("FMMFFT_TREE")) p->tree_p = p->tree_p && e[0] != 'w';
        // complex64, Q = 8 / 16: each FMM's tree on a cluster of 2 CTAs (k_tree_pc); else one CTA
        // per FMM (k_tree_p)
        if (p->tree_p && precision == FMMFFT_C64 && (Q == 16 || Q == 8) && tree_pc_smem(p, 2) <= (size_t)optin) p->tree_cl = 2;
        // (clusters of 4 measured slower at cfg2: the fused far field 29 -> 41 us)
        // wide trees at G = 1 (complex64, Q = 8 / 16): the levels below the first wide level (the
        // per-level kernels' launch-latency-bound top: k_up, k_base, k_tree_down) as ONE k_tree_pc
        // launch, each FMM's top subtree on a cluster of 8 (else 4, 2) CTAs, levels B..top_L
        // entirely on chip; FMMFFT_TOP=w keeps the per-level kernels
        const char* et = getenv("FMMFFT_TOP");
        if (!p->tree_p && G == 1 && precision == FMMFFT_C64 && (Q == 16 || Q == 8) && L > B && !(et && et[0] == 'w') &&
            (P % 8) == 0) {
            int lt = L;                                     // = lvl_first - 1 (Exec::lvl_first at G = 1)
            for (int lev = B + 1; lev <= L; ++lev)
                if ((1LL << lev) >= 64 && (long long)((1LL << lev) / 32) * (P / 8) >= 148) { lt = lev - 1; break; }
            for (int cl : {8, 4, 2})
                if (lt > B && (2LL << B) >= 2LL * cl && tree_pc_smem(p, cl, lt) <= (size_t)optin) {
                    p->top_L = lt;
                    p->top_cl = cl;
                    break;
                }
        }
    }
    // S2T kernel: complex64 with M_L = 64 and whole 128-box tiles per rank -> tensor cores
    // (k_s2t_tc, 3xTF32 on tcgen05); other M_L = 64 plans (32-box chunks) -> the fast convolution
    // (k_s2t_fft, NEXT-4: measured 5.77 -> 5.15 ms against the FP64 tensor-pipe direct sum at cfg4,
    // and 1.03 ms vs 1.85 ms for the FFMA2 kernel at cfg3's complex64 shape); else k_near_up.
    // FMMFFT_S2T=tc | fft | dmma (complex128 direct sum on mma.sync f64) | simt (k_near_up) overrides
    {
        const bool tc_ok = precision == FMMFFT_C64 && M_L == 64 && (p->nb % S2TC_BOXES) == 0;
        const bool fft_ok = M_L == 64 && (p->nb % S2TF_CHUNK) == 0;
        const char* e = getenv("FMMFFT_S2T");
        const char k = (e && *e) ? e[0] : 0;            // 0: the default choice
        p->s2t_tc = tc_ok && (k == 't' || k == 0);
        p->s2t_fft = fft_ok && (k == 'f' || ((k == 0 || k == 't') && !tc_ok));
        p->s2t_dmma = precision == FMMFFT_C128 && M_L == 64 && (p->nb % 32) == 0 && !p->s2t_fft && k != 's';
    }
    // the cluster far field gathers M^L and scatters L^L one FMM (one p) at a time: keep both
    // p-major so those are contiguous runs (debug plans keep [b][q][p] for the stage buffers)
    p->pmaj = p->tree_p && p->tree_cl > 1 && L > B && !(flags & FMMFFT_FLAG_DEBUG);
    // complex64 only: complex128's S2M is DFMA-bound at Q = 24 (k_s2m_w measured 2.12 ms vs 1.68 ms
    // for k_s2m; with the symmetric S2M and the fused M2M level 4.2 ms, step 21.2 -> 22.7 ms)
    p->s2m_sym = Q % 8 == 0 && !getenv("FMMFFT_S2M_NOSYM");
    p->s2m_w = precision == FMMFFT_C64 && M_L == 64 && P % 16 == 0 && !getenv("FMMFFT_S2M_OLD");
    // NEXT-4 kernel fusion: the first upward level from the S2M kernel's registers
    // (saves one read of M^L and a launch); per-level trees only, levels L-1 >= the gathered / top level
    p->s2m_m2m = p->s2m_w && !p->tree_p && !p->pmaj && L - 1 >= std::max(p->lg, p->top_L) && L - 1 >= B &&
                 (p->nb % 2) == 0 && !getenv("FMMFFT_S2M_NOFUSE");
    const char* g_env = getenv("FMMFFT_NO_GRAPH");
    p->use_graph = !(g_env && g_env[0] == '1');
    plan_mfft(p);
    st = precision == FMMFFT_C64 ? build_tables<float>(p) : build_tables<double>(p);
    if (!st) {
        const int nr = virt ? G : 1;
        p->ranks.resize(nr);
        for (int g = 0; g < nr && !st; ++g) {
            p->ranks[g].g = virt ? g : p->comm_rank;
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
        // the far field (main stream) is the critical path: it gets the higher priority, the near
        // field on the side stream fills the SMs it leaves idle
        int lo = 0, hi = 0;
        cudaDeviceGetStreamPriorityRange(&lo, &hi);
        cudaError_t e = cudaStreamCreateWithPriority(&p->cap_stream, cudaStreamNonBlocking, hi);
        if (e == cudaSuccess) e = cudaStreamCreateWithPriority(&p->side, cudaStreamNonBlocking, lo);
        if (e == cudaSuccess) e = cudaEventCreateWithFlags(&p->fork, cudaEventDisableTiming);
        if (e == cudaSuccess) e = cudaEventCreateWithFlags(&p->join, cudaEventDisableTiming);
        if (e == cudaSuccess) e = cudaEventCreateWithFlags(&p->fork2, cudaEventDisableTiming);
        if (e == cudaSuccess) e = cudaEventCreateWithFlags(&p->cs_done, cudaEventDisableTiming);
        if (e == cudaSuccess) e = cudaEventCreateWithFlags(&p->dc_fork, cudaEventDisableTiming);
        if (e == cudaSuccess) e = cudaEventCreateWithFlags(&p->dc_join, cudaEventDisableTiming);
        if (e == cudaSuccess && (flags & FMMFFT_FLAG_PROFILE)) {
            e = cudaEventCreate(&p->ev_s2t[0]);
            if (e == cudaSuccess) e = cudaEventCreate(&p->ev_s2t[1]);
        }
        if (e != cudaSuccess) st = fail(FMMFFT_CUDA_ERROR, "stream/event setup: %s", cudaGetErrorString(e));
    }
    if (!st) {
        cudaError_t e = cudaDeviceSynchronize();
        if (e != cudaSuccess) st = fail(FMMFFT_CUDA_ERROR, "plan setup: %s", cudaGetErrorString(e));
    }
    if (st) { destroy_plan(p); return st; }
    *plan = p;
    return FMMFFT_SUCCESS;
}

fmmfft_status_t fmmfft_autotune(long long N, int G, fmmfft_precision_t precision, double tol, int measure, fmmfft_tune_t* best) {
    if (!best) return fail(FMMFFT_INVALID_VALUE, "best is NULL");
    if (precision != FMMFFT_C64 && precision != FMMFFT_C128) return fail(FMMFFT_INVALID_VALUE, "bad precision");
    if (!pow2(N) || !(G == 1 || G == 2 || G == 4 || G == 8)) return fail(FMMFFT_INVALID_VALUE, "N a power of two, G in {1,2,4,8}");
    if (measure && G != 1) return fail(FMMFFT_INVALID_VALUE, "measured autotuning is single-GPU (G = 1); use the model for G > 1");
    int Q = 0;
    for (int q : {8, 16, 24})
        if (tune_error(q, precision) * 4 <= tol) { Q = q; break; }
    if (!Q) return fail(FMMFFT_INVALID_VALUE, "no Q in {8,16,24} reaches tol=%g at this precision", tol);
    const int M_L = 64;
    *best = fmmfft_tune_t{0, 0, Q, M_L, 0.f, tune_error(Q, precision), 0};
    double best_t = 1e30;
    for (int P = std::max(2, G); P <= (precision == FMMFFT_C64 ? 1024 : 512); P *= 2) {
        if (P % G || N % ((long long)P * M_L)) continue;
        const long long nleaf = N / ((long long)P * M_L);
        if (nleaf % G) continue;
        const int L = ilog2(nleaf);
        for (int B = 2; B <= 4; ++B) {
            if (L < B) continue;
            double t;
            if (measure) {
                float ms = 0;
                const fmmfft_status_t st = precision == FMMFFT_C64 ? tune_measure<float>(N, P, B, Q, M_L, precision, &ms)
                                                                   : tune_measure<double>(N, P, B, Q, M_L, precision, &ms);
                if (st == FMMFFT_UNSUPPORTED || st == FMMFFT_INVALID_VALUE) continue;   // not a valid plan here
                if (st) return st;
                t = ms * 1e-3;
            } else {
                t = tune_model(N, P, G, B, Q, M_L, precision);
            }
            ++best->candidates;
            if (t < best_t) { best_t = t; best->P = P; best->B = B; best->ms = (float)(t * 1e3); }
        }
    }
    if (!best->P) return fail(FMMFFT_INVALID_VALUE, "no valid (P, B) for N=%lld, G=%d with M_L=64", N, G);
    return FMMFFT_SUCCESS;
}

// FMMFFT_FLAG_REAL (SURVEY §8(f) NEXT-1, C = 1): N real inputs read as the complex vector
// z_j = x_{2j} + i x_{2j+1} of length H = N/2, the complex plan of length H (FMM or DIRECT), then
// k_r2c_post; at G > 1 the mirror exchange (sched_mirror) + k_r2c_post_dist.
fmmfft_status_t fmmfft_plan_ex(fmmfft_plan_t* plan, long long N, int P, int G, int B, int Q,
                               fmmfft_precision_t precision, int M_L, unsigned flags) {
    if (!(flags & FMMFFT_FLAG_REAL)) return plan_complex(plan, N, P, G, B, Q, precision, M_L, flags);
    if (!plan) return fail(FMMFFT_INVALID_VALUE, "plan is NULL");
    *plan = nullptr;
    if (N < 4 || (N & 1)) return fail(FMMFFT_INVALID_VALUE, "FMMFFT_FLAG_REAL: N must be even");
    fmmfft_status_t st = plan_complex(plan, N / 2, P, G, B, Q, precision, M_L, flags);
    if (st) return st;
    fmmfft_plan_s* p = *plan;
    p->real = true;
    for (RankBufs& rb : p->ranks) {
        const size_t nl = (size_t)(N / 2 / G);
        if ((st = dalloc(p, &rb.rz, nl * p->esz)) ||
            (G > 1 && ((st = dalloc(p, &rb.mir, nl * p->esz)) || (st = dalloc(p, &rb.xtra, p->esz))))) {
            destroy_plan(p);
            *plan = nullptr;
            return st;
        }
    }
    return FMMFFT_SUCCESS;
}

fmmfft_status_t fmmfft_plan(fmmfft_plan_t* plan, long long N, int P, int G, int B, int Q, fmmfft_precision_t precision) {
    return fmmfft_plan_ex(plan, N, P, G, B, Q, precision, 64, 0u);
}

fmmfft_status_t fmmfft_execute(fmmfft_plan_t p, const void* in, void* out, void* stream) {
    if (!p) return fail(FMMFFT_INVALID_VALUE, "plan is NULL");
    if (!in || !out) return fail(FMMFFT_INVALID_VALUE, "in/out is NULL");
    const size_t nb = (size_t)(p->virt ? p->N : p->N / p->G) * p->esz;
    const size_t half = nb + (p->real ? p->esz : 0);        // real plans: N/2 + 1 complex values
    const size_t bytes = p->real && p->inverse ? half : nb, obytes = p->real && p->inverse ? nb : half;
    const char* a = (const char*)in;
    const char* b = (const char*)out;
    if (a < b + obytes && b < a + bytes) return fail(FMMFFT_INVALID_VALUE, "in and out overlap");
    if (((uintptr_t)in | (uintptr_t)out) & 15) return fail(FMMFFT_INVALID_VALUE, "in/out must be 16-byte aligned");
    cudaPointerAttributes at, bt;
    if (cudaPointerGetAttributes(&at, in) != cudaSuccess || at.type != cudaMemoryTypeDevice ||
        cudaPointerGetAttributes(&bt, out) != cudaSuccess || bt.type != cudaMemoryTypeDevice) {
        cudaGetLastError();
        return fail(FMMFFT_INVALID_VALUE, "in/out must be device pointers");
    }
    if (at.device != p->device || bt.device != p->device)
        return fail(FMMFFT_INVALID_VALUE, "in/out live on device %d/%d, the plan on device %d", at.device, bt.device, p->device);
    DeviceGuard guard(p->device);
    if (guard.err != cudaSuccess) return fail(FMMFFT_CUDA_ERROR, "cudaSetDevice(%d): %s", p->device, cudaGetErrorString(guard.err));
    cudaStream_t s = (cudaStream_t)stream;
    return p->prec == FMMFFT_C64 ? execute_t<float>(p, in, out, s) : execute_t<double>(p, in, out, s);
}

fmmfft_status_t fmmfft_execute_host(fmmfft_plan_t p, const void* in_host, void* out_host, void* stream) {
    if (!p || !in_host || !out_host) return fail(FMMFFT_INVALID_VALUE, "NULL argument");
    const size_t nb = (size_t)(p->virt ? p->N : p->N / p->G) * p->esz;
    const size_t half = nb + (p->real ? p->esz : 0);        // real plans: N/2 + 1 complex values
    const size_t bytes = p->real && p->inverse ? half : nb, obytes = p->real && p->inverse ? nb : half;
    DeviceGuard guard(p->device);
    if (guard.err != cudaSuccess) return fail(FMMFFT_CUDA_ERROR, "cudaSetDevice(%d): %s", p->device, cudaGetErrorString(guard.err));
    RankBufs& rb = p->ranks[0];
    if (!rb.din) {
        fmmfft_status_t st;
        if ((st = dalloc(p, &rb.din, bytes))) return st;
        if ((st = dalloc(p, &rb.dout, obytes))) return st;
    }
    cudaStream_t s = (cudaStream_t)stream;
    CUDA_TRY(cudaMemcpyAsync(rb.din, in_host, bytes, cudaMemcpyHostToDevice, s));
    fmmfft_status_t st = p->prec == FMMFFT_C64 ? execute_t<float>(p, rb.din, rb.dout, s) : execute_t<double>(p, rb.din, rb.dout, s);
    if (st) return st;
    CUDA_TRY(cudaMemcpyAsync(out_host, rb.dout, obytes, cudaMemcpyDeviceToHost, s));
    return FMMFFT_SUCCESS;
}

fmmfft_status_t fmmfft_destroy(fmmfft_plan_t p) {
    if (!p) return FMMFFT_SUCCESS;
    DeviceGuard guard(p->device);
    cudaDeviceSynchronize();
    destroy_plan(p);
    return FMMFFT_SUCCESS;
}

fmmfft_status_t fmmfft_get_info(fmmfft_plan_t p, fmmfft_info_t* info) {
    if (!p || !info) return fail(FMMFFT_INVALID_VALUE, "NULL argument");
    info->N = p->real ? 2 * p->N : p->N; info->P = p->P; info->G = p->G; info->B = p->B; info->Q = p->Q; info->M_L = p->M_L;
    info->L = p->L; info->precision = p->prec; info->M = p->M; info->level_gather = p->lg;
    info->n_stages = ST_COUNT + 1; info->workspace_bytes = p->ws_bytes; info->kernels_per_execute = p->kernels;
    info->variant = (p->tree_p ? FMMFFT_VARIANT_TREE_FUSED : 0u) | (p->s2t_tc ? FMMFFT_VARIANT_S2T_TC : 0u) |
                    (p->s2t_fft ? FMMFFT_VARIANT_S2T_FFT : 0u) |
                    (p->s2m_w ? FMMFFT_VARIANT_S2M_WARP : 0u) | (p->top_L ? FMMFFT_VARIANT_TOP_CLUSTER : 0u) |
                    (p->s2m_m2m ? FMMFFT_VARIANT_S2M_M2M : 0u) | (p->s2m_w && p->s2m_sym ? FMMFFT_VARIANT_S2M_SYM : 0u) |
                    (p->row_fft1 ? FMMFFT_VARIANT_ROW_FFT1 : 0u) | (p->fs_lr ? FMMFFT_VARIANT_FOURSTEP : 0u) |
                    (!p->tree_p && !p->direct ? FMMFFT_VARIANT_DOWN_LVL : 0u) |
                    (p->pmaj ? FMMFFT_VARIANT_PMAJ : 0u);
    info->top_level = p->top_L;
    return FMMFFT_SUCCESS;
}

fmmfft_status_t fmmfft_stage_times(fmmfft_plan_t p, float* ms, int n, int* n_out) {
    if (!p || !ms || !n_out) return fail(FMMFFT_INVALID_VALUE, "NULL argument");
    if (!(p->flags & FMMFFT_FLAG_PROFILE) || !p->have_times) return fail(FMMFFT_INVALID_VALUE, "plan not profiled / not executed");
    CUDA_TRY(cudaEventSynchronize(p->ev[ST_COUNT]));
    const int k = std::min(n, (int)ST_COUNT + 1);
    for (int i = 0; i < k && i < ST_COUNT; ++i) CUDA_TRY(cudaEventElapsedTime(&ms[i], p->ev[i], p->ev[i + 1]));
    float s2t = 0.f;
    if (!p->direct) CUDA_TRY(cudaEventElapsedTime(&s2t, p->ev_s2t[0], p->ev_s2t[1]));
    if (k > ST_NEAR) ms[ST_NEAR] = std::max(0.f, ms[ST_NEAR] - s2t);     // S2T ran serialised inside it
    if (k > ST_COUNT) ms[ST_COUNT] = s2t;
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
