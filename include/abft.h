/*
 * abft.h — C-ABI of the B200-native Enhanced Online-ABFT Cholesky (libabft.so).
 *
 * Operation (§III, §IV): factor an SPD n x n FP64 matrix A = L L^T while the
 * matrix carries two column checksums per nb x nb block (chk1 = v1^T T, chk2 = v2^T T with
 * v1 = [1..1], v2 = [1, 2, .., nb]; §IV.A). The checksums are carried through
 * POTRF (Alg. 2), TRSM and the SYRK/GEMM trailing update
 * (PAPER.md:137-153). Every block is re-verified before it is read (V1-V6 schedule,
 * SURVEY.md §8c / DESIGN.md §2); a detected error is located from d2/d1
 * and corrected in place. The MAGMA dpotrf_gpu interface is kept: the
 * matrix is already in GPU memory, lower storage, overwritten by L.
 *
 * Conventions for every entry point:
 *  - FP64, column-major, lower triangle (uplo = 'L'). The strictly upper triangle of A is
 *    never read or written.
 *  - Pointers are DEVICE pointers unless stated otherwise; `stream` is a cudaStream_t
 *    (declared here as struct CUstream_st* so that this header needs no CUDA include).
 *  - Everything is stream-ordered on `stream`. A call synchronises the stream exactly once,
 *    at its end, and only when it must fill a host report (rep != NULL).
 *  - Return value: 0 OK; -i if argument i is invalid (LAPACK style, 1-based);
 *    ABFT_UNCORRECTABLE (1); ABFT_NOT_SPD (2); ABFT_ERR_CUDA (3); ABFT_ERR_NCCL (4).
 *    No C++ exception crosses this boundary. When rep == NULL the call is fully asynchronous
 *    and statuses 1/2 are not observable (use a report to learn them).
 *  - Version-1 restriction: n % nb == 0 (all of the paper's sizes are multiples);
 *    otherwise the nb argument is reported invalid.
 */
#ifndef ABFT_H
#define ABFT_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

struct CUstream_st;
typedef struct CUstream_st* abft_stream_t;

/* status codes */
#define ABFT_OK 0
#define ABFT_UNCORRECTABLE 1
#define ABFT_NOT_SPD 2
#define ABFT_ERR_CUDA 3
#define ABFT_ERR_NCCL 4

/* injection hooks ("computation error" = output
 * corruption of an operation, "memory error" = storage corruption between verification and use) */
#define ABFT_HOOK_REST 0       /* storage error at the start of iteration k (k = N: before V6)  */
#define ABFT_HOOK_POTRF_OUT 1  /* corrupt the output of POTRF(k) / Alg. 2                         */
#define ABFT_HOOK_TRSM_OUT 2   /* corrupt the output of the panel TRSM(k)                          */
#define ABFT_HOOK_UPDATE_OUT 3 /* corrupt the output of the trailing update of iteration k        */
#define ABFT_HOOK_RECV 4       /* (multi-GPU) corrupt rank `rank`'s received copy of panel k      */
#define ABFT_TGT_DATA 0        /* row, col = global element of A (row >= col)                     */
#define ABFT_TGT_CHK 1         /* row = checksum row nchk I + t (t < nchk; nchk = 2 unless options
                                  say 3), col = global column (col/nb <= I)                       */

/* checks (where an event was raised) and event kinds */
#define ABFT_V1 1   /* pre-read check of the diagonal tile (k,k) before POTRF                */
#define ABFT_V2 2   /* pre-read check of panel tiles (i>k, k) before TRSM                     */
#define ABFT_V3 3   /* check of L_kk against the Alg.-2 checksums                             */
#define ABFT_V4 4   /* check of the solved panel before the trailing update reads it          */
#define ABFT_V5 5   /* check of every trailing tile after update k                            */
#define ABFT_V6 6   /* final sweep over L                                                      */
#define ABFT_V4R 7  /* (multi-GPU) receiver re-check of the broadcast panel                   */
#define ABFT_V7 8   /* (left-looking order) the L blocks a SYRK/GEMM is about to read (Table I) */
#define ABFT_KIND_DATA 1          /* one data element located (row = d2/d1 - 1) and corrected   */
#define ABFT_KIND_NONFINITE 2     /* non-finite delta; located by argmax |X| and corrected       */
#define ABFT_KIND_CHK1 3          /* checksum row 1 corrupted; recomputed from the data          */
#define ABFT_KIND_CHK2 4          /* checksum row 2 corrupted; recomputed from the data          */
#define ABFT_KIND_UNCORRECTABLE 5 /* more errors in a tile column than the checksums locate:
                                     abort (status 1)                                          */
#define ABFT_KIND_CHK3 6          /* (nchk = 3) checksum row 3 corrupted; recomputed from the data */

typedef struct abft_inject_spec {
    int32_t k, hook, target, pad0;
    int64_t row, col;
    uint64_t xor_mask;  /* XOR-ed into the 64-bit pattern of the stored double */
    int32_t rank, pad1; /* RECV only */
} abft_inject_spec_t;   /* host array, terminated by an entry with k = -1 */

typedef struct abft_event {
    int32_t k, check, tile_i, tile_j;
    int32_t row, col;   /* inside the tile; the stored (lower) element for diagonal tiles;
                           row = -1 / -2 / -4 for CHK1 / CHK2 / CHK3, -3 for UNCORRECTABLE  */
    int32_t kind, rank;   /* rank that ran the check: owner of block column tile_j (receiver for V4R) */
    double delta1, delta2;
} abft_event_t;

typedef struct abft_report {
    int64_t info;       /* LAPACK info: 1-based order of the first non-positive leading minor */
    int64_t n_checks, n_detected, n_data, n_nonfinite, n_chk1, n_chk2, n_uncorrectable;
                        /* n_chk2 counts repairs of checksum rows 2 and 3                  */
    int64_t n_events;   /* events raised (may exceed cap; only cap are stored)               */
    int64_t cap;        /* capacity of `events` (set by the caller)                          */
    abft_event_t* events; /* HOST array owned by the caller, sorted by (k, check, J, I, col, row) */
    double seconds;     /* device time of the call (CUDA events on `stream`)                 */
    int64_t reruns;     /* Online / Offline schemes: re-executions after an uncorrectable error */
    double max_noise_ratio; /* max over every column that PASSED a check of max(|d1|/tau1, |d2|/tau2):
                               the fault-free rounding noise relative to the threshold of reading A4
                               (how much margin C_tau = 64 leaves; the oracle's max_ratio)          */
} abft_report_t;

typedef struct abft_options {
    int32_t abft_enabled; /* 1: Enhanced Online-ABFT; 0: the same kernels with every checksum
                             operation, check and encode removed (overhead baseline)            */
    int32_t K;            /* Opt. 3: V5 every K iterations; 1 = every one   */
    double c_tau;         /* threshold constant C_tau of reading A4 (default 64)               */
    int32_t lookahead;    /* reserved (0/1)                                                    */
    int32_t profile;      /* 1: time every phase with CUDA events on `stream` (abft_last_profile) */
    int32_t mode;         /* ABFT_MODE_ENHANCED (default), _ONLINE, _OFFLINE or _ENHANCED_REDO    */
    int32_t order;        /* ABFT_ORDER_RIGHT (default: trailing update + look-ahead) or
                             ABFT_ORDER_LEFT (MAGMA's Alg. 1, Table I checks)     */
    int32_t nchk;         /* checksum rows per block: 0 or 2 (the paper's choice) or 3: the
                             third row v3 = [1, 4, .., nb^2] locates and corrects up to TWO errors
                             in a column of a block ("m+1 column checksums ... up to m errors",
                             P:121; reading B10 of DESIGN.md: ambiguous pairs are UNCORRECTABLE).
                             nchk = 3: right-looking Enhanced scheme on one GPU (else -8)         */
    int32_t prows;        /* multi-GPU only (abft_potrf_dist / _dist_sim): process-grid rows Pr of a
                             2D block-cyclic distribution of the nranks = Pr x Pc ranks;
                             0 or 1 = the 1D column-cyclic distribution. Must divide nranks, <= 15;
                             Pr > 1 needs the peer-memory transport or the one-device harness (-11) */
} abft_options_t;
#define ABFT_ORDER_RIGHT 0
#define ABFT_ORDER_LEFT 1

/* Schemes (§II.B, §III; Table VII/VIII compare them):
 *  ENHANCED  verify every block before it is read (V1..V6) — errors are corrected in place.
 *  ONLINE    verify each operation's result after it (V3, V4, V5) + a final sweep (V6): computing
 *            errors are corrected; a storage error between a verification and the next read
 *            propagates, and the call re-runs the factorisation once from a saved copy of A.
 *  OFFLINE   checksums carried through, verified only at the end (V6); any detection re-runs.  */
#define ABFT_MODE_ENHANCED 0
#define ABFT_MODE_ONLINE 1
#define ABFT_MODE_OFFLINE 2
#define ABFT_MODE_ENHANCED_REDO 3   /* Enhanced + one re-run from a saved copy of A on UNCORRECTABLE
                                       (more errors in a block column than two checksums locate,
                                       PAPER.md:121; the paper's re-do)          */

/* Per-phase device time of the last abft_potrf* call on this thread with options.profile = 1.
 * Phases: 0 encode, 1 V1/V2, 2 POTRF+inverse, 3 TRSM (+Alg. 2 rows), 4 V3, 5 V4, 6 panel
 * write-back, 7 trailing update (data rows), 8 trailing update (checksum rows), 9 V5, 10 V6,
 * 11 injection, 12 main stream waiting for the look-ahead panel. flops / bytes are the
 * ALGORITHMIC counts of DESIGN.md §6 (not executed ones). */
#define ABFT_NPHASE 13
typedef struct abft_profile {
    int32_t nphase, pad;
    double ms[16];
    int64_t launches[16];   /* event-timed instances of the phase */
    double flops[16];
    double bytes[16];
} abft_profile_t;
int abft_last_profile(abft_profile_t* out);
const char* abft_phase_name(int phase);

/* Checksum encoding (§IV.A, cost 2n^2).
 * A: n x n lower (lda >= max(1,n)); chk: 2N x n output (ldchk >= 2N, N = n/nb): row 2I is
 * v1^T T(I,J), row 2I+1 is v2^T T(I,J) for I >= J (diagonal tiles as sym(tril(T)));
 * scales: output, n + 2N doubles = [s_i = sqrt(A_ii) | S1_I | S2_I] (threshold scales, A4).
 * Errors: -1 n<0, -2 nb<1 or n%nb, -3 A NULL, -4 lda, -5 chk NULL, -6 ldchk, -7 scales NULL. */
int abft_encode(int64_t n, int64_t nb, const double* A, int64_t lda, double* chk, int64_t ldchk,
                double* scales, abft_stream_t stream);

/* One detect/locate/correct sweep (§IV.C) over every lower tile I >= J.
 * factored = 1 checks L (diagonal tiles as tril), 0 checks an unfactored matrix (sym).
 * correct = 0 only reports. Events carry k = -1, check = V6 (factored) or V5.
 * rep may be NULL (no sync). Errors as abft_encode, -8 factored, -9 correct. */
int abft_verify(int64_t n, int64_t nb, double* A, int64_t lda, double* chk, int64_t ldchk,
                const double* scales, int factored, int correct, abft_stream_t stream,
                abft_report_t* rep);

/* Enhanced Online-ABFT Cholesky, A = L L^T in place (lower). Workspace (checksums, scales,
 * panel buffer, event buffer: about n*nb + 2n^2/nb doubles) is allocated with cudaMallocAsync
 * on `stream` and freed before return (except in graph mode, see abft_graph_release). inj: HOST list (NULL = none), validated up front
 * (-6 on an out-of-range target/hook). rep: HOST report (NULL = asynchronous, no report).
 * Errors: -1 n, -2 nb, -3 A, -4 lda, -6 inj. */
int abft_potrf(int64_t n, int64_t nb, double* A, int64_t lda, abft_stream_t stream,
               const abft_inject_spec_t* inj, abft_report_t* rep);

/* As abft_potrf with options (NULL = defaults: ABFT on, K = 1, C_tau = 64). -8 bad options. */
int abft_potrf_ex(int64_t n, int64_t nb, double* A, int64_t lda, abft_stream_t stream,
                  const abft_inject_spec_t* inj, abft_report_t* rep, const abft_options_t* opt);

/* End-to-end variant on HOST memory (A_host: n x n column-major, lda >= n; pinned memory
 * recommended — the overlapped write-back below is used only for page-locked A_host, a
 * pageable buffer takes the plain copy-factor-copy path): copies A to the device, factors with
 * abft_potrf_ex, copies L back, then
 * synchronises. On the direct fault-free right-looking path (no injections, n above the graph-
 * mode threshold) only the block columns from their diagonal blocks down go to the device (the
 * strict upper triangle outside the diagonal blocks is never read, as in LAPACK uplo = 'L'), and
 * each block column of L is copied back on a copy stream as soon as its panel is written back,
 * overlapped with the remaining updates; if
 * the final sweep V6 corrected anything, or the call failed, the whole matrix is copied again
 * after the factorisation (ABFT_HOST_OVERLAP set in the environment disables the overlap).
 * Same errors as abft_potrf_ex. */
int abft_potrf_host(int64_t n, int64_t nb, double* A_host, int64_t lda, abft_stream_t stream,
                    const abft_inject_spec_t* inj, abft_report_t* rep, const abft_options_t* opt);

/* Synthetic SPD input of reading A15 (the same counter-based generator as synthetic/):
 * A[i,j] = A[j,i] = U(splitmix64(seed*n^2 + max(i,j)*n + min(i,j))), A[i,i] += n.
 * Writes the full n x n matrix. Errors: -1 n, -3 A, -4 lda. */
int abft_gen_spd(int64_t n, uint64_t seed, double* A, int64_t lda, abft_stream_t stream);

/* ---- multi-GPU (one process per GPU, block-cyclic tiles, panel broadcast) ---------------------
 * abft_nccl_id: fill 128 bytes (ncclUniqueId) on rank 0, share them out of band.
 * abft_comm_init: create the communicator for `rank` of `nranks` on the current device.
 * abft_potrf_dist: 1D (options.prows <= 1): rank r owns block columns {j : j mod nranks == r},
 * stored contiguously in A_local (n x (n_local_cols) column-major, lda_local >= n, local block
 * column t is global block column t*nranks + r). 2D (options.prows = Pr > 1, Pc = nranks / Pr,
 * rank r = pr * Pc + pc): rank r owns the tiles (I, J) with I mod Pr = pr and J mod Pc = pc; it
 * stores the block columns {j : j mod Pc == pc} contiguously and full height (global rows, local
 * block column t = global t*Pc + pc), reads and writes only its own tiles (the other rows are
 * workspace). Per iteration the diagonal block's owner factors it and pushes inv(L_kk) to the other
 * ranks of its process column, each of those solves and checks its own panel tiles and pushes them
 * to every rank; every rank re-checks the tiles it received (V4R). Same semantics and report as
 * abft_potrf; events of all ranks are gathered into rank 0's report (other ranks report their
 * own); an event's rank is the owner of the checked tile (the receiver for V4R). Errors as
 * abft_potrf, 4 NCCL. */
int abft_nccl_id(void* id128);
int abft_comm_init(void** comm, int nranks, const void* id128, int rank);
int abft_comm_destroy(void* comm);
int abft_potrf_dist(int64_t n, int64_t nb, double* A_local, int64_t lda_local, void* comm, int rank,
                    int nranks, abft_stream_t stream, const abft_inject_spec_t* inj,
                    abft_report_t* rep, const abft_options_t* opt);

/* Peer-memory transport (NEXT-3 groundwork; also how two ranks share ONE device in the tests,
 * where NCCL refuses duplicate devices): each rank exports one device arena of cap_bytes (+256
 * bytes of flags) through CUDA IPC; the panel broadcast is a pull of the owner's panel straight
 * out of its arena (peer loads over NVLink/NVSwitch between GPUs), the all-reduces and the
 * all-gather are peer reads in rank order, all synchronised by device-side release/acquire flags
 * on the caller's stream (no host round trip). cap_bytes must hold the largest message: the
 * packed panel, (n - nb) nb + 2 n + 8 doubles.
 * abft_comm_init_ipc: allocate + export; handle_out receives this rank's 64-byte handle.
 * abft_comm_attach_ipc: handles = nranks x 64 bytes (all ranks' handles, rank order) -> map peers.
 * The resulting comm is used with abft_potrf_dist and released with abft_comm_destroy, like an
 * NCCL one. Errors: -1 comm, -2 nranks (1..64) / handles, -3 rank, -4 cap_bytes, -5 handle_out;
 * ABFT_ERR_CUDA if the device refuses the export / mapping. */
int abft_comm_init_ipc(void** comm, int nranks, int rank, int64_t cap_bytes, void* handle_out);
int abft_comm_attach_ipc(void* comm, const void* handles);
/* abft_potrf_dist errors: -1 n, -2 nb, -3 A_local, -4 lda_local, -5 comm (or its rank/size
 * disagree with rank/nranks), -6 rank, -7 nranks, -9 inj, -11 options; ABFT_ERR_NCCL on a failed
 * collective. Depth-1 look-ahead across ranks: the owner of block column k+1 updates it first and
 * factors + broadcasts panel k+1 on a high-priority stream while every rank finishes update k
 * (DESIGN.md §5). */

/* Test harness of the multi-GPU algorithm on ONE device: runs the nranks ranks of
 * abft_potrf_dist in one process, in lock-step, with the NCCL broadcast replaced by device-to-
 * device copies (A_locals[r]: rank r's local block columns, same layout as abft_potrf_dist).
 * Everything else — ownership, the owner's panel, the receivers' RECV hook and V4R re-check,
 * the per-rank trailing updates, V5/V6 on owned tiles, the merged report — is the code the NCCL
 * path runs. Errors: -1 n, -2 nb, -3 nranks, -4 A_locals, -5 lda_local, -6 inj (as -9 there). */
int abft_potrf_dist_sim(int64_t n, int64_t nb, int nranks, double* const* A_locals, int64_t lda_local,
                        abft_stream_t stream, const abft_inject_spec_t* inj, abft_report_t* rep,
                        const abft_options_t* opt);
/* (2D, options.prows > 1: A_locals[r] holds the block columns of process column r mod Pc, full
 * height, as abft_potrf_dist; the owners push their panel rows into the other ranks' buffers.) */

/* Diagnostics: the trailing-update GEMM on its own (for benchmarking the dominant kernel):
 * C = beta C + alpha A B^T over the lower triangle (lower = 1: r >= c, requires N <= M) or all
 * of C (lower = 0). A: M x K, B: N x K, column-major device buffers. Errors: -1 bad sizes. */
int abft_dev_gemm_nt(int64_t M, int64_t N, int64_t K, const double* A, int64_t lda, const double* B,
                     int64_t ldb, double* C, int64_t ldc, double alpha, double beta, int lower,
                     abft_stream_t stream);

/* Diagnostics: the diagonal-block factorisation alone (POTRF + inverse of an nb x nb SPD block):
 * A (lower, overwritten by L), Li (nb x nb, ld nb) receives inv(L). Returns ABFT_NOT_SPD (2) on a
 * non-positive pivot. Synchronises `stream`. */
int abft_dev_chol_inv(int64_t nb, double* A, int64_t lda, double* Li, abft_stream_t stream);

/* Diagnostics: abft_dev_chol_inv through the one-launch task-graph path with a per-task trace:
 * trace_host (cap >= 4 x tasks, host) receives per task {type | i<<8 | j<<16 | b<<24 | smid<<32 |
 * cta<<48, fetch ns, start ns (dependencies met), end ns} (%globaltimer). Returns the number of
 * tasks, -1 if nb does not take the task path or cap is too small, -2 if the factorisation failed. */
int abft_dev_chol_trace(int64_t nb, double* A, int64_t lda, double* Li, uint64_t* trace_host, int64_t cap,
                        abft_stream_t stream);

/* Graph mode. A fault-free Enhanced (or ABFT-off) right-looking abft_potrf / abft_potrf_ex call
 * without the per-phase profiler is captured once into a CUDA graph (both streams) and replayed
 * on later calls with the same device, n, nb, A, lda, options and report capacity: no host launch
 * cost, shorter dependent-launch gaps on the panel chain. OWNERSHIP EXCEPTION to abft_potrf's
 * "workspace freed before return": in graph mode the workspace (about n nb + 3 n^2 / nb doubles
 * plus the fused-V5 partials) belongs to the cached graph, per host thread (one entry), and stays
 * allocated until the key changes or this call releases it. Default for n <= 12288 (measured
 * faster there, slower above); ABFT_GRAPH=0 / 1 in the environment forces direct launches /
 * graph mode. Returns 0. */
int abft_graph_release(void);

/* Diagnostics: kernel launches issued by the last call on this thread, a static version string,
 * and the text of the last CUDA error seen on this thread (empty if none). */
int64_t abft_last_launch_count(void);
const char* abft_version(void);
const char* abft_last_error(void);

#ifdef __cplusplus
}
#endif
#endif /* ABFT_H */
