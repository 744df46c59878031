/*
 * fmmfft.h — C ABI of the B200-native FMM-FFT (Cecka, "Low Communication FMM-Accelerated FFT
 * on GPUs", SC17). Citations "P:<lines>" point into the paper text.
 *
 * WHAT IS COMPUTED. The forward, unnormalised, in-order 1D complex DFT of length N,
 *     y_k = sum_{j<N} x_j w_N^{jk},  w_N = exp(-2 pi i / N)            (eq. 1)
 * by the FMM-FFT factorisation F_N = F_{M,P} H^_{M,P}, N = M P          (eq. 2):
 * P-1 interleaved periodic 1D FMMs with the cotangent kernel (Algorithm 1),
 * the POST scaling (line 15), and an M x P 2D FFT with ONE all-to-all transpose (line 16,
 * P:389-399). The FMM uses Q Chebyshev nodes per box, M_L points per leaf box,
 * leaf level L = log2(N / (P M_L)) and base level B (Table 1).
 *
 * DATA. Input and output are interleaved complex (float2 for FMMFFT_C64, double2 for
 * FMMFFT_C128), block-distributed in natural order: rank g of G holds x[g N/G, (g+1) N/G)
 * and receives y[g N/G, (g+1) N/G). For G = 1 these are the whole vectors.
 *
 * OWNERSHIP. The plan owns every workspace buffer (halos, tree, transpose buffers, operator
 * tables) and, for G > 1, uses the communicator set up by fmmfft_comm_init. Caller-owned
 * buffers are never retained after a call returns (execution is stream-ordered: they must stay
 * valid until the stream reaches the end of the enqueued work).
 *
 * ERRORS. Every entry point returns an fmmfft_status_t; no C++ exception crosses the
 * boundary. On failure fmmfft_last_error() returns a thread-local message. Invalid arguments
 * return FMMFFT_INVALID_VALUE and leave outputs untouched.
 *
 * THREADING. A plan is not re-entrant: no concurrent execute on one plan. Different plans
 * may be used from different threads.
 */
#ifndef FMMFFT_H
#define FMMFFT_H

#include <stddef.h>
#include <stdint.h>

#if defined(__GNUC__)
#define FMMFFT_API __attribute__((visibility("default")))
#else
#define FMMFFT_API
#endif

#ifdef __cplusplus
extern "C" {
#endif

typedef struct fmmfft_plan_s* fmmfft_plan_t;

/* Arithmetic type. C64 = complex64 storage, fp32 arithmetic; C128 = complex128, fp64. */
typedef enum { FMMFFT_C64 = 0, FMMFFT_C128 = 1 } fmmfft_precision_t;

typedef enum {
    FMMFFT_SUCCESS = 0,
    FMMFFT_INVALID_VALUE = 1,   /* an argument violates the contract below                 */
    FMMFFT_UNSUPPORTED = 2,     /* valid in the paper, not supported by this build / device */
    FMMFFT_ALLOC_FAILED = 3,    /* device or host allocation failed                          */
    FMMFFT_CUDA_ERROR = 4,      /* a CUDA runtime call or kernel launch failed               */
    FMMFFT_NCCL_ERROR = 5,      /* NCCL missing or an NCCL call failed                       */
    FMMFFT_NOT_INITIALIZED = 6  /* G > 1 without fmmfft_comm_init                            */
} fmmfft_status_t;

/* Plan flags (fmmfft_plan_ex). */
#define FMMFFT_FLAG_VIRTUAL 1u  /* G "virtual ranks" in this process on the current device:
                                   the distributed data flow (halos, all-gather, all-to-all)
                                   runs with device-to-device copies instead of NCCL. in/out
                                   are then the FULL length-N vectors. For testing the
                                   partitioned algorithm on one GPU. */
#define FMMFFT_FLAG_VIRTUAL_NCCL 64u  /* with FMMFFT_FLAG_VIRTUAL: the virtual ranks' exchanges go
                                   through NCCL (ncclSend / ncclRecv to self, ncclGroupStart/End,
                                   captured in the execute graph) on a 1-rank communicator
                                   (fmmfft_comm_init(0, 1, id) on this device) instead of device
                                   copies — the NCCL transport on one GPU (else NOT_INITIALIZED
                                   / INVALID_VALUE). */
#define FMMFFT_FLAG_PROFILE 2u  /* record CUDA events around every stage (fmmfft_stage_times) */
#define FMMFFT_FLAG_DEBUG 4u    /* keep every level's M^l / L^l in the buffers fmmfft_debug_buffer
                                   returns. Without it the fused single-GPU far field
                                   (FMMFFT_VARIANT_TREE_FUSED) keeps levels < L on chip only, and
                                   those debug buffers hold stale data. */
#define FMMFFT_FLAG_DIRECT 16u  /* no FMM: the plain four-step (Cooley-Tukey) FFT of length N with
                                   the same M-FFT kernels, as the in-house comparator (SURVEY §8(f)
                                   NEXT-3). G = 1 only (else FMMFFT_UNSUPPORTED); P, B, Q, M_L are
                                   ignored; 2^10 <= N <= 2^33 (c64) / 2^30 (c128); combinable with
                                   FMMFFT_FLAG_INVERSE. */
#define FMMFFT_FLAG_INVERSE 8u  /* the inverse transform x_j = (1/N) sum_k y_k exp(+2 pi i jk/N)
                                   (F_N^{-1} = F_N^H / N): the same FMM-FFT
                                   path on conj(input), its output conjugated and scaled by 1/N
                                   (two extra elementwise passes, k_conj_scale). Same layouts,
                                   distribution and error bounds as the forward plan. */

#define FMMFFT_FLAG_REAL 32u    /* real-input forward transform (C = 1):
                                   X_k = sum_j x_j exp(-2 pi i jk/N), k = 0..N/2, for REAL x
                                   (eq. 1; the other half is conj(X_{N-k})).
                                   N is the real length (even); in = N reals (float / double by
                                   precision, 16-byte aligned), out = N/2 + 1 complex values
                                   (must not overlap in). The N reals are read in place as the
                                   complex vector z_j = x_{2j} + i x_{2j+1}, transformed by the
                                   complex plan of length N/2 (P, B, Q, M_L — or DIRECT — apply
                                   to THAT length), then one elementwise pass (k_r2c_post)
                                   separates the even / odd halves. With FMMFFT_FLAG_INVERSE:
                                   the complex-to-real inverse x_j = (1/N) sum_{k<N} X_k
                                   exp(+2 pi i jk/N) of a Hermitian spectrum given as X_0..X_{N/2}
                                   (in = N/2 + 1 complex, out = N reals; the imaginary parts of
                                   X_0 and X_{N/2} are ignored): one elementwise pass (k_c2r_pre)
                                   builds the length-N/2 spectrum of z_j = x_{2j} + i x_{2j+1},
                                   then the inverse complex plan writes z = the N reals in place.
                                   G > 1: x block-distributed (rank g holds reals
                                   [g N/G, (g+1) N/G)); rank g's out holds X_k for k in
                                   [g N/(2G), (g+1) N/(2G)) plus one slot, written only by rank
                                   G-1 with X_{N/2} (so every rank's out is N/(2G) + 1 complex;
                                   VIRTUAL plans: one array X_0..X_{N/2}); the inverse takes the
                                   same distribution. One extra exchange per execute: rank g
                                   receives rank G-1-g's block and one element (the pairing of
                                   k with N/2 - k crosses ranks).
                                   fmmfft_get_info reports the real N; M, L, ... describe the
                                   complex plan. */

/* ---------------------------------------------------------------- communicator (G > 1)
 * One process per GPU. Rank 0 calls fmmfft_get_unique_id and broadcasts the 128 bytes (e.g.
 * through torch.distributed); every rank then calls fmmfft_comm_init with its rank, the
 * world size G and that id. Binds the communicator to the CURRENT CUDA device. NCCL is loaded
 * at run time (dlopen "libnccl.so.2"); FMMFFT_NCCL_ERROR if it cannot be found. */
FMMFFT_API fmmfft_status_t fmmfft_get_unique_id(unsigned char id[128]);
FMMFFT_API fmmfft_status_t fmmfft_comm_init(int rank, int G, const unsigned char id[128]);
FMMFFT_API fmmfft_status_t fmmfft_comm_destroy(void);  /* INVALID_VALUE while a plan created on the
                                                           communicator is alive */

/* ---------------------------------------------------------------- plans
 * fmmfft_plan: N = M P points, P FMMs interleaved (P - 1 non-trivial), G ranks, base level
 * B, Q Chebyshev nodes, M_L = 64 (the paper's large-N leaf size).
 * fmmfft_plan_ex: same with an explicit M_L and flags.
 * Requirements (else FMMFFT_INVALID_VALUE):
 *   N, P, M_L powers of two; P >= 2; G in {1, 2, 4, 8}; P % G == 0; N % (P M_L) == 0;
 *   L = log2(N / (P M_L)) >= B >= 2; 2^L % G == 0; 2 <= Q <= 32;
 *   16 <= M_L <= 128; P <= 1024 (complex64) / 512 (complex128); M = N / P >= 2 G.
 *   Without FMMFFT_FLAG_VIRTUAL and G > 1, fmmfft_comm_init must have been called with the
 *   same G (else FMMFFT_NOT_INITIALIZED). The device must be sm_100 (else UNSUPPORTED).
 * Collective when G > 1 (non-virtual): every rank creates its plan with identical arguments.
 * Allocates all device workspace and uploads the operator tables (computed in fp64 on the
 * host: S2M/L2T, M2M/L2L P:630-800, S2T P:843-860, M2L P:902-947, rho_p P:374). */
FMMFFT_API fmmfft_status_t fmmfft_plan(fmmfft_plan_t* plan, long long N, int P, int G, int B, int Q,
                            fmmfft_precision_t precision);
FMMFFT_API fmmfft_status_t fmmfft_plan_ex(fmmfft_plan_t* plan, long long N, int P, int G, int B, int Q,
                               fmmfft_precision_t precision, int M_L, unsigned flags);

/* ---------------------------------------------------------------- parameter autotuner
 * pick (P, B, Q, M_L) for (N, G, precision) and a relative-l2 error target
 * `tol` (the paper searches its parameter space per N, Figs. 6-9).
 *   Q: the smallest of {8, 16, 24} whose predicted error meets tol with a 4x margin — the
 *      truncation model e(Q) = 1.7e-3 * 6.3^-(Q-2) fitted to the oracle's Q sweep (DESIGN.md §2,
 *      geometric decay, saturating near Q = 18) — plus the arithmetic floor
 *      (2.6e-7 complex64, 3e-14 complex128). FMMFFT_INVALID_VALUE if no Q reaches tol.
 *   M_L = 64 (the tensor-core S2T's tile), P over the powers of two with G | P,
 *      L = log2(N/(P M_L)) >= B and G | 2^L, B over {2, 3, 4} (B <= L).
 *   measure != 0 (G = 1 only): every candidate plan is built and timed on the current device
 *      (3 warm-up + 5 timed executes, CUDA events, on a scratch input) — the fastest wins;
 *      measure == 0: ranked by a roofline model (HBM passes, tensor / FFMA2 flops, per-launch
 *      latency), host only, no device work.
 * best->ms is the measured (or modelled) time of the winner, best->error its predicted error,
 * best->candidates the number of (P, B) pairs considered. */
typedef struct {
    int P, B, Q, M_L;
    float ms;
    double error;
    int candidates;
} fmmfft_tune_t;

FMMFFT_API fmmfft_status_t fmmfft_autotune(long long N, int G, fmmfft_precision_t precision, double tol, int measure,
                                           fmmfft_tune_t* best);

/* Forward transform. in, out: device pointers on the plan's device, N/G complex elements
 * each (N for a virtual plan), 16-byte aligned, non-overlapping (else INVALID_VALUE).
 * in is not modified. Asynchronous on `stream` (a cudaStream_t; NULL = legacy default
 * stream); no host synchronisation. Collective when G > 1. */
FMMFFT_API fmmfft_status_t fmmfft_execute(fmmfft_plan_t plan, const void* in, void* out, void* stream);

/* End-to-end variant with HOST buffers (pinned for full overlap; pageable works): copies
 * in -> device, executes, copies the result -> out, all enqueued on `stream`. The caller
 * synchronises the stream before reading out. */
FMMFFT_API fmmfft_status_t fmmfft_execute_host(fmmfft_plan_t plan, const void* in_host, void* out_host,
                                    void* stream);

FMMFFT_API fmmfft_status_t fmmfft_destroy(fmmfft_plan_t plan);

/* ---------------------------------------------------------------- introspection */
typedef struct {
    long long N;
    int P, G, B, Q, M_L, L, precision;
    long long M;            /* N / P                                               */
    int level_gather;       /* l_g = max(B, log2 G + 1): finest all-gathered level (R16) */
    int n_stages;           /* entries reported by fmmfft_stage_times               */
    size_t workspace_bytes; /* device bytes owned by the plan (all virtual ranks)   */
    int kernels_per_execute;/* kernels this library launched in the last execute (0 before) */
    unsigned variant;       /* kernel variants the plan chose: FMMFFT_VARIANT_* bits below  */
    int top_level;          /* FMMFFT_VARIANT_TOP_CLUSTER: levels B..top_level of every FMM run
                               in one cluster kernel, levels above it per level (else 0)  */
} fmmfft_info_t;

#define FMMFFT_VARIANT_TREE_FUSED 1u  /* far field as one per-FMM kernel (G = 1, tree fits smem) */
#define FMMFFT_VARIANT_S2T_TC     2u  /* near field on tcgen05 tensor cores (3xTF32)             */
#define FMMFFT_VARIANT_S2M_WARP 256u  /* S2M (+ the S' copy) one warp per box (k_s2m_w)            */
#define FMMFFT_VARIANT_S2M_M2M 1024u  /* the first M2M level (L -> L-1) fused into k_s2m_w         */
#define FMMFFT_VARIANT_S2M_SYM 2048u  /* S2M by the reflection symmetry (even / odd halves)        */
#define FMMFFT_VARIANT_TOP_CLUSTER 512u /* wide tree (G = 1): the top levels of each FMM on a CTA
                                         cluster (k_tree_pc), the wide levels per level            */
#define FMMFFT_VARIANT_S2T_FFT  128u  /* near field as a fast convolution: per-box DFT_128, 3
                                         kernel spectra, inverse DFT_128 (k_s2t_fft, NEXT-4)       */
#define FMMFFT_VARIANT_ROW_FFT1   4u  /* M-point FFTs as one single-pass kernel per row        */
#define FMMFFT_VARIANT_FOURSTEP   8u  /* long rows: column pass(es) + transposing row pass     */
#define FMMFFT_VARIANT_DOWN_LVL  32u  /* wide levels on the per-level M2M / M2L kernels        */
#define FMMFFT_VARIANT_PMAJ      64u  /* leaf M^L / L^L stored p-major [p][b][q] (the cluster far
                                         field; never with FMMFFT_FLAG_DEBUG): the debug buffers of
                                         level L then hold that layout instead of [b][q][p]      */

FMMFFT_API fmmfft_status_t fmmfft_get_info(fmmfft_plan_t plan, fmmfft_info_t* info);

/* Per-stage device times (ms) of the LAST execute of a plan created with
 * FMMFFT_FLAG_PROFILE (else INVALID_VALUE); synchronises that execute's stream. Stage i's
 * name is fmmfft_stage_name(i): comm_S, s2m, m2m, comm_M, top, down, post_pfft, a2a, mfft —
 * consecutive intervals of the stream — and s2t, the near field. A profiled plan runs the near
 * field (S halo + S2T) serialised on the main stream instead of concurrently on its side
 * stream, so each interval holds only its own kernels (s2m excludes the S2T that follows it).
 * n = capacity of ms[]; returns the count in *n_out. */
FMMFFT_API fmmfft_status_t fmmfft_stage_times(fmmfft_plan_t plan, float* ms, int n, int* n_out);
FMMFFT_API const char* fmmfft_stage_name(int i);

/* Internal buffers after an execute, for stage-by-stage parity tests. `which`:
 *   0 = T_near  [p][b][re/im][m]  (S2T output, N/G complex as 2N/G reals: p-major, planar per box)
 *   1 = M^l     [b][q][p]  (multipoles of level `level`, own boxes; slot p = FMM p)
 *   2 = L^l     [b][q][p]  (local expansions of level `level`, own boxes)
 *   3 = W       [k2][m]    (P-point FFT output before the transpose, N/G complex)
 *   4 = r       [p]        (reductions r_p, slot p = FMM p; P complex)
 * Returns a device pointer and its size in bytes; rank selects the virtual rank. */
FMMFFT_API fmmfft_status_t fmmfft_debug_buffer(fmmfft_plan_t plan, int rank, int which, int level,
                                    const void** ptr, size_t* bytes);

/* Thread-local message of the last failure in this thread ("" if none). */
FMMFFT_API const char* fmmfft_last_error(void);
FMMFFT_API const char* fmmfft_version(void);

#ifdef __cplusplus
}
#endif
#endif /* FMMFFT_H */
