// common.cuh — shared device-side types of libabft (CUDA path only; the oracle has its own).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "../../include/abft.h"

#define ABFT_EPS 0x1p-52  /* DBL_EPSILON (reading A17) */
#define ABFT_RHO 0x1p-30  /* relative slack of the location test (reading A6) */
#define ABFT_RHO2 0x1p-40 /* relative slack of the two-error residual (reading B10, nchk = 3) */

namespace abft {

// A flagged column produced by a check's recalculation pass (phase 1), resolved by phase 2.
struct Flag {
    int32_t I, J, c, part;   // part: which StageArgs of a two-part check launch raised it
    double d1, d2, r1, r2, d3, r3;   // d3, r3: third checksum (nchk = 3), else 0
};

constexpr int kFlagCap = 8192;
constexpr int kMaxFix = 1024;   // corrections held per tile by phase 2 (beyond: UNCORRECTABLE)

// A correction decided by phase 2: the stored element (or checksum) and its new value.
struct Fix { double* p; double* p2; double val; };

// Flagged columns pending resolution (phase 1 -> phase 2), and phase 2's per-tile correction list
// (in global memory, so that the check kernel keeps a small shared-memory footprint and can sit
// next to two update CTAs on an SM). One list per concurrent stream.
struct FlagList {
    int32_t nflag, overflow;
    Flag flags[kFlagCap];
    Fix fix[kMaxFix];
};

// Device-resident run state. One per abft_* call.
struct DevState {
    int32_t abort;        // set by UNCORRECTABLE / NOT_SPD: every later kernel returns at entry
    int32_t status;       // ABFT_OK / ABFT_UNCORRECTABLE / ABFT_NOT_SPD
    long long info;       // LAPACK info (1-based)
    unsigned long long nev;        // events raised
    unsigned long long n_checks;   // tile checks run
    long long n_detected, n_data, n_nonfinite, n_chk1, n_chk2, n_unc;
    unsigned long long max_ratio_bits;   // max over passing columns of max(|d1|/tau1, |d2|/tau2)
                                         // (fault-free noise margin, as the oracle's max_ratio)
    unsigned int done[4];                // per flag list: CTAs of the running check launch that
                                         // finished phase 1 (the last one resolves the flags)
    FlagList fl[3];       // [0]: main stream, [1]: look-ahead panel stream, [2]: panel side stream (V2)
};

// Where the tiles of a check stage live (DESIGN.md §5 "data layout").
enum StageKind : int32_t {
    SK_COLUMN = 0,     // V1/V2: tiles (k..N-1, k) in A, unfactored; checksums in chk
    SK_DIAG_FACT = 1,  // V3: tile (k,k) in A, factored; checksums in W rows mB, mB+1
    SK_PANEL = 2,      // V4/V4R: tiles (k+1..N-1, k) in W (data rows), checksums in W (chk rows)
    SK_TRAIL = 3,      // V5: tiles (I,J), k < J <= I, in A, unfactored; checksums in chk
    SK_ALL = 4,        // V6 / abft_verify: all tiles I >= J in A; factored per flag
    SK_TRAIL_OFF = 5,  // V5, off-diagonal trailing tiles, recalculation from the GEMM's fused partials
    SK_TRAIL_DIAG = 6, // V5, diagonal trailing tiles (J, J), J in [j_lo, j_hi), re-read as sym(tril)
    SK_LEFT_L = 7,     // V7 (left-looking): L tiles (I, J), J < k, I in [k, k + j_hi), factored
    SK_COL_DIAG = 8,   // V1 alone: tile (k, k) in A, unfactored (the part POTRF reads)
    SK_COL_BELOW = 9,  // V2 alone: tiles (k+1..N-1, k) in A, unfactored (runs concurrently with POTRF)
};

struct StageArgs {
    int32_t kind, V, k, factored;   // k: iteration (-1 for abft_verify); V: event check code
    int32_t correct, rank, encode, pad;
    int64_t n, nb, N;
    double* A; int64_t lda;         // global matrix (or local columns in dist mode)
    double* chk; int64_t ldc;       // checksum matrix 2N x n(local)
    double* W; int64_t ldw;         // packed panel buffer (SK_DIAG_FACT, SK_PANEL)
    int64_t mB;                     // rows of data in W (m * nb)
    const double* s; const double* S1; const double* S2;  // threshold scales
    const double* S3;               // (nchk = 3) sum of (i+1)^2 s_i over block I
    int32_t nchk, pad3;             // checksum rows per block: 2 or 3 (reading B10)
    double c_tau;
    int32_t col_owner_mod, col_owner_rank;  // dist: local column mapping (1, 0 on one GPU)
    // dist, 2D block-cyclic (NEXT-3): tile (I, J) belongs to this rank iff J % col_owner_mod ==
    // col_owner_rank and I % row_owner_mod == row_owner_rank (rows stay global: every rank stores its
    // block columns full height and maintains only its own tiles); own_invert = 1 selects the tiles
    // this rank does NOT own (V4R: the received panel tiles)
    int32_t row_owner_mod, row_owner_rank;
    int32_t own_invert;
    int32_t flist;                  // flag list used by this stage (one per stream)
    int64_t j_lo, j_hi;             // SK_TRAIL*: block columns [j_lo, j_hi)
    const double* cs; int64_t cs_ld, cs_nslab, cs_slab_rows;   // SK_TRAIL_OFF: fused partials
    DevState* st;
    abft_event_t* ev; int64_t ev_cap;
};

// Tile view: data pointer, leading dim, checksum row pointers with stride.
struct TileView {
    double* T; int64_t ldt;
    double* c1; double* c2; int64_t ldc;
    double* c3;                     // third checksum row (nchk = 3) or nullptr
    bool diag, factored;
};

__host__ __device__ __forceinline__ int64_t stage_count(const StageArgs& a) {
    const int64_t N = a.N, k = a.k;
    switch (a.kind) {
        case SK_COLUMN: return N - k;
        case SK_COL_DIAG: return 1;
        case SK_COL_BELOW: return N - k - 1;
        case SK_DIAG_FACT: return 1;
        case SK_PANEL: return N - k - 1;
        case SK_TRAIL: {
            const int64_t lo = a.j_lo, hi = a.j_hi;
            return hi <= lo ? 0 : (hi - lo) * N - (hi * (hi - 1) - lo * (lo - 1)) / 2;
        }
        case SK_TRAIL_DIAG: return a.j_hi > a.j_lo ? a.j_hi - a.j_lo : 0;
        case SK_LEFT_L: return (int64_t)a.k * a.j_hi;
        case SK_TRAIL_OFF: {
            const int64_t lo = a.j_lo, hi = a.j_hi;
            return hi <= lo ? 0 : (hi - lo) * (N - 1) - (hi * (hi - 1) - lo * (lo - 1)) / 2;
        }
        default: return N * (N + 1) / 2;
    }
}

// Column-major tile enumeration over block columns J >= j0 where column J holds N - J - d tiles
// (d = 0: I >= J, d = 1: I > J): the column J and the offset rem inside it of tile t, in closed form
// (a root of the quadratic prefix count, corrected by at most a step or two) — every CTA of a check
// launch decodes its tile, and a per-column loop cost up to N iterations per thread.
__host__ __device__ __forceinline__ int64_t tiles_before(int64_t J, int64_t j0, int64_t N, int64_t d) {
    return (J - j0) * (N - d) - (J * (J - 1) - j0 * (j0 - 1)) / 2;
}
__host__ __device__ __forceinline__ void decode_cols(int64_t t, int64_t j0, int64_t N, int64_t d, int64_t& J,
                                                     int64_t& rem) {
    const double a = (double)(N - d) + 0.5;
    const double C = (double)j0 * (double)(N - d) - 0.5 * (double)j0 * (double)(j0 - 1);
    const double disc = a * a - 2.0 * ((double)t + C);
    int64_t j = (int64_t)(a - sqrt(disc > 0.0 ? disc : 0.0));
    if (j < j0) j = j0;
    while (j > j0 && tiles_before(j, j0, N, d) > t) --j;
    while (tiles_before(j + 1, j0, N, d) <= t) ++j;
    J = j;
    rem = t - tiles_before(j, j0, N, d);
}

// t-th tile of the stage, in the oracle's check order (column-major over tiles).
__device__ __forceinline__ void stage_tile(const StageArgs& a, int64_t t, int64_t& I, int64_t& J) {
    const int64_t N = a.N, k = a.k;
    switch (a.kind) {
        case SK_COLUMN: I = k + t; J = k; return;
        case SK_COL_DIAG: I = k; J = k; return;
        case SK_COL_BELOW: I = k + 1 + t; J = k; return;
        case SK_DIAG_FACT: I = k; J = k; return;
        case SK_PANEL: I = k + 1 + t; J = k; return;
        case SK_TRAIL_DIAG: I = J = a.j_lo + t; return;
        case SK_LEFT_L: J = t / a.j_hi; I = k + t % a.j_hi; return;
        case SK_TRAIL_OFF: {   // column-major over (I > J), J in [j_lo, j_hi)
            int64_t rem;
            decode_cols(t, a.j_lo, N, 1, J, rem);
            I = J + 1 + rem; return;
        }
        default: {             // column-major over (I >= J), J from j_lo (SK_TRAIL) or 0
            int64_t rem;
            decode_cols(t, (a.kind == SK_TRAIL) ? a.j_lo : 0, N, 0, J, rem);
            I = J + rem; return;
        }
    }
}

// Does this rank check tile (I, J) in this stage (dist ownership; always true on one GPU)?
__device__ __forceinline__ bool tile_mine(const StageArgs& a, int64_t I, int64_t J) {
    const bool own = (J % a.col_owner_mod == a.col_owner_rank) && (I % a.row_owner_mod == a.row_owner_rank);
    return a.own_invert ? !own : own;
}

// Local column offset of global block column J (1D block-cyclic in dist mode).
__device__ __forceinline__ int64_t local_col(const StageArgs& a, int64_t J) {
    return (J / a.col_owner_mod) * a.nb;
}

__device__ __forceinline__ TileView stage_view(const StageArgs& a, int64_t I, int64_t J) {
    TileView v;
    const int64_t B = a.nb, nc = a.nchk;
    v.diag = (I == J);
    switch (a.kind) {
        case SK_DIAG_FACT:
            v.T = a.A + local_col(a, J) * a.lda + I * B; v.ldt = a.lda;
            v.c1 = a.W + a.mB; v.c2 = v.c1 + 1; v.ldc = a.ldw;
            v.factored = true; break;
        case SK_PANEL:
            v.T = a.W + (I - a.k - 1) * B; v.ldt = a.ldw;
            v.c1 = a.W + a.mB + nc + nc * (I - a.k - 1); v.c2 = v.c1 + 1; v.ldc = a.ldw;
            v.diag = false; v.factored = true; break;
        case SK_COLUMN:
        case SK_COL_DIAG:
        case SK_COL_BELOW:
        case SK_TRAIL:
        case SK_TRAIL_OFF:
        case SK_TRAIL_DIAG:
            v.T = a.A + local_col(a, J) * a.lda + I * B; v.ldt = a.lda;
            v.c1 = a.chk + local_col(a, J) * a.ldc + nc * I; v.c2 = v.c1 + 1; v.ldc = a.ldc;
            v.factored = false; break;
        default:
            v.T = a.A + local_col(a, J) * a.lda + I * B; v.ldt = a.lda;
            v.c1 = a.chk + local_col(a, J) * a.ldc + nc * I; v.c2 = v.c1 + 1; v.ldc = a.ldc;
            v.factored = a.factored != 0; break;
    }
    v.c3 = nc == 3 ? v.c1 + 2 : nullptr;
    return v;
}

// X(r,c) of the check: sym(tril(T)) for an unfactored diagonal tile, tril(T) if factored.
__device__ __forceinline__ double view_x(const TileView& v, int64_t r, int64_t c) {
    if (v.diag) {
        if (r >= c) return v.T[c * v.ldt + r];
        return v.factored ? 0.0 : v.T[r * v.ldt + c];
    }
    return v.T[c * v.ldt + r];
}
__device__ __forceinline__ double* view_store(const TileView& v, int64_t r, int64_t c) {
    if (v.diag && r < c) return &v.T[r * v.ldt + c];
    return &v.T[c * v.ldt + r];
}

// Thresholds of reading A4, evaluated with explicit round-to-nearest ops (no FMA contraction)
// so that a decision depends only on (d1, d2) and the scales.
__device__ __forceinline__ void thresholds(const StageArgs& a, int64_t I, int64_t g, bool factored,
                                           double& tau1, double& tau2, double& tau3) {
    const double base = a.c_tau * ABFT_EPS;  // exact: power-of-two scaling
    const double sc = factored ? 1.0 : a.s[g];
    tau1 = __dmul_rn(__dmul_rn(base, a.S1[I]), sc);
    tau2 = __dmul_rn(__dmul_rn(base, a.S2[I]), sc);
    tau3 = a.nchk == 3 ? __dmul_rn(__dmul_rn(base, a.S3[I]), sc) : 0.0;
}

__device__ __forceinline__ bool dfinite(double x) { return isfinite(x); }

// The run's abort flag as ONE decision per CTA. The flag can be raised by a kernel on another
// stream while this CTA starts; threads that read it independently could disagree, and a CTA
// whose warps split (some return, some wait at a barrier or on an mbarrier) hangs. Every kernel
// with CTA-level synchronisation checks the flag through this helper at entry.
__device__ __forceinline__ bool cta_aborted(const int32_t* flag) {
    __shared__ int s_abort;
    if (threadIdx.x == 0) s_abort = *(volatile const int32_t*)flag;
    __syncthreads();
    return s_abort != 0;
}

// One FP64 tensor-core MMA (SASS DMMA.8x8x4): C(8x8) += A(8x4) B(4x8). Fragments: lane holds
// A[lane/4][lane%4], B[k = lane%4][n = lane/4], C[lane/4][2 (lane%4) + {0, 1}].
__device__ __forceinline__ void dmma(double& c0, double& c1, double a, double b) {
    asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};\n"
                 : "+d"(c0), "+d"(c1) : "d"(a), "d"(b));
}

}  // namespace abft

// Per-column partial checksums of an updated trailing tile, written by the GEMM epilogue
// (fused V5 recalculation): slab s = global_row / slab_rows, column g (global):
//   p[s * ld + g] = sum over the slab's rows of C_new,  p[(nslab + s) * ld + g] = weighted sum,
// weights = (row index inside its nb-block) + 1.
namespace abft {
struct ColSumOut {
    double* p; int64_t ld, nslab;   // rows [0, nslab) v1, [nslab, 2 nslab) v2, [2 nslab, 3 nslab) v3
    int64_t row0, col0;   // global row of C's row 0; partial-array column of C's column 0
    int64_t nb;
    int64_t slab_rows;    // rows per slab (set by the GEMM launcher: its warp-tile height)
    int64_t colg0;        // GLOBAL column of C's column 0 (block-diagonal test; = col0 on one GPU)
    int64_t nchk;         // 3: also the v3 partials (weights (row in block + 1)^2)
};
}  // namespace abft

// UPDATE_OUT injections applied inside the update GEMM's epilogue (reading A21: after the
// update, before the fused V5 partials and the store). Coordinates are relative to the launch's
// C (seg 0, data rows) or C2 (seg 1, checksum rows), in its local columns.
namespace abft {
struct EpiInjOp { int64_t r, c; uint64_t mask; int32_t seg, pad; };
constexpr int kMaxEpiInj = 4;
struct EpiInj { int32_t n, pad; EpiInjOp op[kMaxEpiInj]; };
}  // namespace abft

// Host helpers
#define ABFT_CUDA_TRY(expr)                                   \
    do {                                                      \
        cudaError_t _e = (expr);                              \
        if (_e != cudaSuccess) { abft_set_error(_e, #expr); return ABFT_ERR_CUDA; } \
    } while (0)

void abft_set_error(cudaError_t e, const char* what);
void abft_count_launch(int n = 1);

// Collective transport of the multi-GPU path: NCCL (dist.cu) — one rank per process.
struct DistTransport {
    int rank = 0, nranks = 1;
    virtual ~DistTransport() {}
    virtual int bcast(void* buf, size_t bytes, int root, cudaStream_t s) = 0;       // in place
    virtual int allreduce_sum(double* buf, size_t count, cudaStream_t s) = 0;
    virtual int allreduce_max(double* buf, size_t count, cudaStream_t s) = 0;
    virtual int allgather(const void* send, void* recv, size_t bytes, cudaStream_t s) = 0;
    // Push mode (peer-memory transports, NEXT-3): the transport owns every rank's two panel
    // receive buffers, mapped into every rank, so the owner's write-back kernel stores the panel
    // straight into its peers' buffers (no separate broadcast pass). nullptr: not supported.
    virtual double* recv_buf(int r, int slot) { (void)r; (void)slot; return nullptr; }
    virtual size_t recv_capacity() const { return 0; }   // doubles per receive buffer
    virtual int wait_free(int64_t panel, cudaStream_t s) { (void)panel; (void)s; return 0; }   // owner: peers done with the slot
    virtual int post_panel(int64_t panel, cudaStream_t s) { (void)panel; (void)s; return 0; }  // owner: panel stored
    virtual int wait_panel(int root, int64_t panel, cudaStream_t s) { (void)root; (void)panel; (void)s; return 0; }
    virtual int mark_free(int64_t value, cudaStream_t s) { (void)value; (void)s; return 0; }     // this rank's reads done
    // 2D block-cyclic push mode: the diagonal block's owner stores inv(L_kk) into the receive
    // buffers of its process column and publishes it (post_li); those ranks wait for it (wait_li)
    // start of one factorisation with N block columns: flag-based transports move their flag
    // values to a fresh range, so that flags left by an earlier call on this comm cannot satisfy
    // this call's waits
    virtual int begin_call(int64_t N, cudaStream_t s) { (void)N; (void)s; return 0; }
    virtual int post_li(int64_t panel, cudaStream_t s) { (void)panel; (void)s; return 0; }
    virtual int wait_li(int root, int64_t panel, cudaStream_t s) { (void)root; (void)panel; (void)s; return 0; }
};
// The owner's write-back of panel k fused with the push to its peers: data rows -> A panel,
// checksum rows -> chk, the whole W (+ abort slot `slot`) -> every peer's receive buffer (util.cu).
// 2D block-cyclic (rmod > 1): only the rows of this rank's tiles (data block b with b % rmod ==
// dphase, checksum block c with c % rmod == cphase, two checksum rows per block) are written.
int launch_panel_out(const double* W, int64_t ldw, int64_t mB, int64_t ncrows, int64_t B, double* Apanel,
                     int64_t lda, double* chk, int64_t ldc, double* const* peers, int npeer, const int32_t* abort_flag,
                     cudaStream_t s, int64_t rmod = 1, int64_t dphase = 0, int64_t cphase = 0, int slot = 0);
// The 1D block-cyclic driver (abft.cu). ranks: local ranks driven by this call — one with a
// transport (NCCL, one process per GPU) or all P of them with tp == nullptr (single-process
// simulation on one device: the broadcast becomes a device-to-device copy).
struct DistLocal { int rank; double* A; int64_t lda; };
int run_dist(int64_t n, int64_t nb, int P, const DistLocal* locals, int nlocal, DistTransport* tp,
             cudaStream_t s, const abft_inject_spec_t* inj, abft_report_t* rep, const abft_options_t* opt);

// DMMA GEMM launcher (gemm.cu). Returns 1 if the fused column partials `cs` were written
// (warp-specialised path with 128-row tiles aligned to nb), 0 otherwise.
int launch_gemm(int64_t M, int64_t N, int64_t K, const double* A, int64_t lda, const double* B,
                int64_t ldb, double* C, int64_t ldc, double alpha, double beta, bool transB, int mask,
                int krange, int64_t nb, int64_t q_tile0, int64_t c_tile0, const int32_t* abort_flag,
                cudaStream_t s, int force_tile = 0, abft::ColSumOut* cs = nullptr, int nchk = 2);
// The trailing update with the checksum rows as a second row segment of the same launch.
// cstride > 1: C's column block t (and the B operand's row block t) is global block t * cstride
// (a rank's 1D block-cyclic local columns in one launch); returns -1 if the shapes do not allow it.
// Panel TRSM + its checksum rows in one launch (second row segment); returns 1 if fused.
int launch_trsm_with_chk(int64_t mB, int64_t B, const double* Ap, int64_t lda, const double* Li, double* W,
                         int64_t ldw, int64_t M2, const double* A2, int64_t lda2, const int32_t* abort_flag,
                         cudaStream_t s, int64_t rstride = 1, int64_t rfirst = 0);
// rstride > 1 (2D block-cyclic): only the data-row blocks rfirst + u * rstride (relative to C's row
// 0) are computed — this rank's tiles; the checksum segment is computed for every row.
// Returns a bit mask: 1 = the fused V5 partials were written, 2 = the epilogue applied `inj`
// (the caller applies the hook itself otherwise); -1 if cstride > 1 and the shapes do not allow it.
int launch_update_with_chk(int64_t M, int64_t N, int64_t K, const double* A, int64_t lda, const double* B,
                           int64_t ldb, double* C, int64_t ldc, int64_t M2, const double* A2, double* C2,
                           int64_t ldc2, int64_t nb, const int32_t* abort_flag, cudaStream_t s,
                           abft::ColSumOut* cs, int64_t lda2 = 0, int64_t cstride = 1,
                           const abft::EpiInj* inj = nullptr, int nchk = 2, int64_t rstride = 1,
                           int64_t rfirst = 0);
