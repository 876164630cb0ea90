// gemm.cu — FP64 tensor-core (DMMA) GEMM for the trailing SYRK/GEMM update, the panel TRSM
// (as a product with the inverted diagonal block) and the recursive diagonal-block POTRF.
//
//   C[m,n] = beta * C[m,n] + alpha * sum_k A[m,k] * opB[k,n]
//   A : M x K column-major (lda);  opB = Bm^T with Bm N x K (TRANS_B, "NT") or Bm K x N ("NN").
//
// FP64 tensor work on sm_100a is warp-level DMMA (mma.sync.m8n8k4.f64 -> DMMA.8x8x4);
// tcgen05 has no kind::f64 (ptxas rejects it), so TMEM/UMMA do not apply to this path.
// Operands are staged global -> shared memory with a multi-stage cp.async (LDGSTS) pipeline;
// fragments are read with conflict-free 64-bit shared loads (row pitch = tile + 4 doubles,
// which is 4 mod 16 8-byte banks).
//
// Output masks:
//   MASK_NONE  : all of M x N
//   MASK_LOWER : only r >= c (SYRK of the trailing lower triangle; CTA tiles with tile-row <
//                tile-col are not launched). PAPER.md:137-153: A' = A - LC LC^T, B' = B - LD LC^T
//   MASK_CHK   : checksum rows: row q belongs to block I = q_tile0 + q/2, column c to block
//                J = c_tile0 + c/nb; written iff I >= J (chk(B') = chk(B) - chk(LD) LC^T)
// K-range restrictions exploit triangular operands (zeros are never multiplied):
//   KR_LE_N  : k < n0 + BN   (opB = inv(L)^T, lower inverse: TRSM)
//   KR_GE_N  : k >= n0       (opB = inv(L), NN)
//   KR_LE_M  : k < m0 + BM   (A = inv(L) lower, NN)
#include "common.cuh"

#include <algorithm>
#include <cstdlib>
#include <cstring>
#include <cstdio>

namespace abft {

enum { MASK_NONE = 0, MASK_LOWER = 1, MASK_CHK = 2 };
enum { KR_FULL = 0, KR_LE_N = 1, KR_GE_N = 2, KR_LE_M = 3 };

struct GemmArgs {
    int64_t M, N, K;
    const double* A; int64_t lda;
    const double* B; int64_t ldb;
    double* C; int64_t ldc;
    double alpha, beta;
    int32_t mask, krange;
    int64_t nb, q_tile0, c_tile0;   // MASK_CHK geometry
    int64_t tiles_n;                // number of column tiles (rect grid)
    const int32_t* abort;
    int32_t vecA, vecB;             // 16-byte cp.async allowed for A / B
    ColSumOut cs;                   // fused V5 partials (cs.p == nullptr: off)
    // optional second row segment (ws kernel only): the checksum rows appended to the update as
    // extra GEMM rows. Rows [0, M2) of A2 (lda) update C2 (ldc2) under MASK_CHK with
    // q_tile0 = c_tile0 = 0; their tiles follow the first segment's tiles.
    int64_t M2; const double* A2; double* C2; int64_t ldc2; int64_t lda2;
    // column-block stride (ws kernel, MASK_LOWER + checksum segment): column block t of C and of
    // the B operand's rows is global block t * cstride (1D block-cyclic local columns; 1 = dense)
    int64_t cstride;
    // data-row block filter (ws kernel, 2D block-cyclic NEXT-3; rstride = 1: every row): only the
    // nb-row blocks b = rfirst + u * rstride (relative to row 0 of A and C) are computed, the rest
    // belong to other ranks. Rows stay global (no remapping of A or C), requires nb % BM == 0 and
    // M % nb == 0 (the launchers fall back to rstride = 1, computing every row, otherwise)
    int64_t rstride, rfirst;
    // ws kernel: prefetch into L2 the C tile of tile index t + pf_ahead (0 = off; the launcher
    // sets it to the number of CTAs resident at once)
    int64_t pf_ahead;
    EpiInj inj;   // UPDATE_OUT hook in the epilogue (ws kernel; inj.n == 0: none)
    int32_t nchk; // MASK_CHK / checksum segment: checksum rows per block (row q is block q / nchk)
};

// block row of checksum row q (nchk = 2 or 3 rows per block): constant divisors, no runtime division
__host__ __device__ __forceinline__ int64_t chk_block(int64_t q, int32_t nchk) { return nchk == 3 ? q / 3 : q / 2; }

__device__ __forceinline__ void cp_async16(void* smem, const void* gmem, int src_bytes) {
    const unsigned s = (unsigned)__cvta_generic_to_shared(smem);
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;\n" ::"r"(s), "l"(gmem), "r"(src_bytes));
}
__device__ __forceinline__ void cp_async8(void* smem, const void* gmem, int src_bytes) {
    const unsigned s = (unsigned)__cvta_generic_to_shared(smem);
    asm volatile("cp.async.ca.shared.global [%0], [%1], 8, %2;\n" ::"r"(s), "l"(gmem), "r"(src_bytes));
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;\n" ::); }
template <int N>
__device__ __forceinline__ void cp_async_wait() { asm volatile("cp.async.wait_group %0;\n" ::"n"(N)); }


template <int BM, int BN, int BK, int WM, int WN, int STAGES, bool TB>
struct GemmCfg {
    static constexpr int WARPS_M = BM / WM, WARPS_N = BN / WN;
    static constexpr int THREADS = WARPS_M * WARPS_N * 32;
    static constexpr int PA = BM + 4;                    // sA[k][m], pitch PA
    static constexpr int PB_T = BN + 4;                  // TB: sB[k][n]
    static constexpr int PB_N = BK + 4;                  // NN: sB[n][k]
    static constexpr int SA = BK * PA;
    static constexpr int SB = TB ? BK * PB_T : BN * PB_N;
    static constexpr size_t SMEM = (size_t)STAGES * (SA + SB) * sizeof(double);
    static constexpr int FM = WM / 8, FN = WN / 8;
};

template <int BM, int BN, int BK, int WM, int WN, int STAGES, bool TB>
__global__ void __launch_bounds__(GemmCfg<BM, BN, BK, WM, WN, STAGES, TB>::THREADS, 1)
k_gemm_dmma(GemmArgs g) {
    using Cfg = GemmCfg<BM, BN, BK, WM, WN, STAGES, TB>;
    constexpr int T = Cfg::THREADS;
    if (cta_aborted(g.abort)) return;
    // ---- tile mapping ----
    int64_t tm, tn;
    if (g.mask == MASK_LOWER) {  // lower trapezoid (tile row >= tile col, col < tiles_n), row-major
        const int64_t idx = blockIdx.x, TN = g.tiles_n, tri = TN * (TN + 1) / 2;
        if (idx < tri) {
            int64_t a = (int64_t)((sqrt(8.0 * (double)idx + 1.0) - 1.0) * 0.5);
            while (a * (a + 1) / 2 > idx) --a;
            while ((a + 1) * (a + 2) / 2 <= idx) ++a;
            tm = a; tn = idx - a * (a + 1) / 2;
        } else {
            tm = TN + (idx - tri) / TN; tn = (idx - tri) % TN;
        }
    } else {
        tm = blockIdx.x / g.tiles_n; tn = blockIdx.x % g.tiles_n;
    }
    const int64_t m0 = tm * BM, n0 = tn * BN;
    if (g.mask == MASK_CHK) {  // skip tiles where no row reaches the column blocks
        const int64_t qmax = min(g.M, m0 + BM) - 1;
        const int64_t Imax = g.q_tile0 + chk_block(qmax, g.nchk), Jmin = g.c_tile0 + n0 / g.nb;
        if (Imax < Jmin) return;
    }
    int64_t kb = 0, ke = g.K;
    if (g.krange == KR_LE_N) ke = min(g.K, n0 + BN);
    else if (g.krange == KR_GE_N) kb = (n0 / BK) * BK;
    else if (g.krange == KR_LE_M) ke = min(g.K, m0 + BM);
    const int ktiles = (int)((ke - kb + BK - 1) / BK);

    extern __shared__ __align__(16) double smem[];
    double* sA = smem;
    double* sB = smem + STAGES * Cfg::SA;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int wm = warp / Cfg::WARPS_N, wn = warp % Cfg::WARPS_N;

    // ---- per-thread loader geometry (16-byte path): fixed row pair, k stepped by a constant ----
    static_assert(T % (BM / 2) == 0 && T % (BN / 2) == 0 && T % (BK / 2) == 0, "loader mapping");
    constexpr int A_KSTEP = T / (BM / 2), A_PER = BK / A_KSTEP;
    const int a_mm = (tid % (BM / 2)) * 2, a_kk = tid / (BM / 2);
    const int64_t a_gm = m0 + a_mm;
    const int a_bytes = (a_gm < g.M) ? ((a_gm + 1 < g.M) ? 16 : 8) : 0;
    const double* a_src = g.A + a_gm;                 // + k * lda
    constexpr int BT_KSTEP = T / (BN / 2), BT_PER = BK / BT_KSTEP;
    const int bt_nn = (tid % (BN / 2)) * 2, bt_kk = tid / (BN / 2);
    const int64_t bt_gn = n0 + bt_nn;
    const int bt_bytes = (bt_gn < g.N) ? ((bt_gn + 1 < g.N) ? 16 : 8) : 0;
    constexpr int BN_NSTEP = T / (BK / 2), BN_PER = BN / BN_NSTEP;
    const int bn_kk = (tid % (BK / 2)) * 2, bn_nn = tid / (BK / 2);

    auto load_stage = [&](int stage, int kt) {
        const int64_t k0 = kb + (int64_t)kt * BK;
        double* dA = sA + stage * Cfg::SA;
        double* dB = sB + stage * Cfg::SB;
        if (g.vecA) {
#pragma unroll
            for (int q = 0; q < A_PER; ++q) {
                const int kk = a_kk + q * A_KSTEP;
                const int64_t gk = k0 + kk;
                const int bytes = gk < ke ? a_bytes : 0;
                cp_async16(dA + kk * Cfg::PA + a_mm, bytes ? a_src + gk * g.lda : g.A, bytes);
            }
        } else {
            for (int i = tid; i < BK * BM; i += T) {
                const int kk = i / BM, mm = i % BM;
                const int64_t gm = m0 + mm, gk = k0 + kk;
                const bool ok = gk < ke && gm < g.M;
                cp_async8(dA + kk * Cfg::PA + mm, ok ? g.A + gk * g.lda + gm : g.A, ok ? 8 : 0);
            }
        }
        if (TB) {  // Bm is N x K: column k holds n contiguous
            if (g.vecB) {
#pragma unroll
                for (int q = 0; q < BT_PER; ++q) {
                    const int kk = bt_kk + q * BT_KSTEP;
                    const int64_t gk = k0 + kk;
                    const int bytes = gk < ke ? bt_bytes : 0;
                    cp_async16(dB + kk * Cfg::PB_T + bt_nn, bytes ? g.B + gk * g.ldb + bt_gn : g.B, bytes);
                }
            } else {
                for (int i = tid; i < BK * BN; i += T) {
                    const int kk = i / BN, nn = i % BN;
                    const int64_t gn = n0 + nn, gk = k0 + kk;
                    const bool ok = gk < ke && gn < g.N;
                    cp_async8(dB + kk * Cfg::PB_T + nn, ok ? g.B + gk * g.ldb + gn : g.B, ok ? 8 : 0);
                }
            }
        } else {   // Bm is K x N: column n holds k contiguous
            if (g.vecB) {
#pragma unroll
                for (int q = 0; q < BN_PER; ++q) {
                    const int nn = bn_nn + q * BN_NSTEP;
                    const int64_t gn = n0 + nn, gk = k0 + bn_kk;
                    int bytes = 0;
                    if (gn < g.N && gk < ke) bytes = (gk + 1 < ke) ? 16 : 8;
                    cp_async16(dB + nn * Cfg::PB_N + bn_kk, bytes ? g.B + gn * g.ldb + gk : g.B, bytes);
                }
            } else {
                for (int i = tid; i < BN * BK; i += T) {
                    const int nn = i / BK, kk = i % BK;
                    const int64_t gn = n0 + nn, gk = k0 + kk;
                    const bool ok = gn < g.N && gk < ke;
                    cp_async8(dB + nn * Cfg::PB_N + kk, ok ? g.B + gn * g.ldb + gk : g.B, ok ? 8 : 0);
                }
            }
        }
    };

    double acc[Cfg::FM][Cfg::FN][2];
#pragma unroll
    for (int i = 0; i < Cfg::FM; ++i)
#pragma unroll
        for (int j = 0; j < Cfg::FN; ++j) acc[i][j][0] = acc[i][j][1] = 0.0;

#pragma unroll
    for (int s = 0; s < STAGES - 1; ++s) {
        if (s < ktiles) load_stage(s, s);
        cp_async_commit();
    }
    const int fr = lane >> 2, fc = lane & 3;   // fragment row (groupID) / k (thread in group)
    for (int kt = 0; kt < ktiles; ++kt) {
        cp_async_wait<STAGES - 2>();
        __syncthreads();
        {   // prefetch stage kt + STAGES - 1 (its buffer was consumed at iteration kt - 1)
            const int nk = kt + STAGES - 1;
            if (nk < ktiles) load_stage(nk % STAGES, nk);
            cp_async_commit();
        }
        const double* cA = sA + (kt % STAGES) * Cfg::SA + wm * WM + fr;
        const double* cB = sB + (kt % STAGES) * Cfg::SB;
#pragma unroll
        for (int kk = 0; kk < BK; kk += 4) {
            double af[Cfg::FM], bf[Cfg::FN];
#pragma unroll
            for (int i = 0; i < Cfg::FM; ++i) af[i] = cA[(kk + fc) * Cfg::PA + i * 8];
#pragma unroll
            for (int j = 0; j < Cfg::FN; ++j) {
                const int nn = wn * WN + j * 8 + fr;
                bf[j] = TB ? cB[(kk + fc) * Cfg::PB_T + nn] : cB[nn * Cfg::PB_N + kk + fc];
            }
#pragma unroll
            for (int i = 0; i < Cfg::FM; ++i)
#pragma unroll
                for (int j = 0; j < Cfg::FN; ++j) dmma(acc[i][j][0], acc[i][j][1], af[i], bf[j]);
        }
    }
    cp_async_wait<0>();
    __syncthreads();

    // ---- epilogue: stage the tile in shared memory (column-major, pitch BM+2), then a coalesced
    // 16-byte read-modify-write of C, four independent column segments in flight per thread ----
    constexpr int PC = BM + 2;
    static_assert((size_t)BN * PC * sizeof(double) <= Cfg::SMEM, "epilogue staging fits");
    double* sC = smem;
#pragma unroll
    for (int i = 0; i < Cfg::FM; ++i)
#pragma unroll
        for (int j = 0; j < Cfg::FN; ++j)
#pragma unroll
            for (int h = 0; h < 2; ++h)
                sC[(wn * WN + j * 8 + fc * 2 + h) * PC + wm * WM + i * 8 + fr] = acc[i][j][h];
    __syncthreads();
    constexpr int RP = BM / 2;                 // row pairs per column
    constexpr int ITEMS = BN * RP;             // row pairs in the tile
    constexpr int BATCH = 4;
    static_assert(ITEMS % (T * BATCH) == 0, "epilogue batching");
    const bool vecC = ((((uintptr_t)g.C) & 15) == 0) && (g.ldc % 2 == 0);
    const double alpha = g.alpha, beta = g.beta;
    for (int base = tid; base < ITEMS; base += T * BATCH) {
        double2 old[BATCH];
        bool ok0[BATCH], ok1[BATCH];
        double* ptr[BATCH];
#pragma unroll
        for (int b = 0; b < BATCH; ++b) {
            const int idx = base + b * T;
            const int c = idx / RP, rp = (idx % RP) * 2;
            const int64_t gr = m0 + rp, gc = n0 + c;
            bool o0 = gr < g.M && gc < g.N, o1 = gr + 1 < g.M && gc < g.N;
            if (g.mask == MASK_LOWER) { o0 = o0 && gr >= gc; o1 = o1 && gr + 1 >= gc; }
            else if (g.mask == MASK_CHK) {
                const int64_t J = g.c_tile0 + gc / g.nb;
                o0 = o0 && (g.q_tile0 + chk_block(gr, g.nchk)) >= J;
                o1 = o1 && (g.q_tile0 + chk_block(gr + 1, g.nchk)) >= J;
            }
            ok0[b] = o0; ok1[b] = o1;
            ptr[b] = g.C + gc * g.ldc + gr;
            old[b] = make_double2(0.0, 0.0);
            if (beta != 0.0) {
                if (o0 && o1 && vecC) old[b] = *reinterpret_cast<const double2*>(ptr[b]);
                else { if (o0) old[b].x = ptr[b][0]; if (o1) old[b].y = ptr[b][1]; }
            }
        }
#pragma unroll
        for (int b = 0; b < BATCH; ++b) {
            const int idx = base + b * T;
            const int c = idx / RP, rp = (idx % RP) * 2;
            const double v0 = alpha * sC[c * PC + rp], v1 = alpha * sC[c * PC + rp + 1];
            const double r0 = beta == 0.0 ? v0 : fma(beta, old[b].x, v0);
            const double r1 = beta == 0.0 ? v1 : fma(beta, old[b].y, v1);
            if (ok0[b] && ok1[b] && vecC) *reinterpret_cast<double2*>(ptr[b]) = make_double2(r0, r1);
            else { if (ok0[b]) ptr[b][0] = r0; if (ok1[b]) ptr[b][1] = r1; }
        }
    }
}

template <int BM, int BN, int BK, int WM, int WN, int STAGES, bool TB>
static int run_cfg(GemmArgs g, cudaStream_t s) {
    using Cfg = GemmCfg<BM, BN, BK, WM, WN, STAGES, TB>;
    auto kern = k_gemm_dmma<BM, BN, BK, WM, WN, STAGES, TB>;
    static bool attr = false;
    if (!attr) {
        cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)Cfg::SMEM);
        attr = true;
    }
    const int64_t tm = (g.M + BM - 1) / BM, tn = (g.N + BN - 1) / BN;
    g.tiles_n = tn;
    int64_t grid;
    if (g.mask == MASK_LOWER) grid = tn * (tn + 1) / 2 + (tm - tn) * tn;   // requires N <= M
    else grid = tm * tn;
    if (grid <= 0) return 0;
    kern<<<(unsigned)grid, Cfg::THREADS, Cfg::SMEM, s>>>(g);
    abft_count_launch();
    return 0;
}

// ============================================================================================
// Warp-specialised persistent variant (the hot path: trailing update and panel TRSM).
//
// One CTA per SM loops over output tiles. Warp 8 is the producer: one elected lane arms an
// mbarrier with the stage's byte count, then the 32 lanes issue one cp.async.bulk per operand
// column (1 KB each, straight into the padded, conflict-free layout) that completes on that
// mbarrier; it also prefetches the next tile's C columns into L2. Warps 0-7 consume: wait on
// the stage's "full" barrier, run the DMMA k-steps, release the stage with one arrive per warp
// on its "empty" barrier. No CTA-wide barrier in the main loop. C is read into the
// accumulators at the start of a tile (acc = alpha*beta*C, alpha = +-1) so that the epilogue is
// a stream of fire-and-forget stores and never exposes load latency.
// ============================================================================================
__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;\n" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;\n" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];\n" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
    uint32_t done;
    do {
        asm volatile("{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n selp.u32 %0, 1, 0, p;\n}\n"
                     : "=r"(done) : "r"(smem_u32(bar)), "r"(parity) : "memory");
    } while (!done);
}
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];\n"
                 ::"r"(smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void prefetch_l2(const void* src, uint32_t bytes) {
    asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;\n" ::"l"(src), "r"(bytes) : "memory");
}

template <int BM_, int BN_, int BK_, int STAGES_, int WM_, int WN_, int REG_CONS_, int MINB_, bool LDG_ = false,
          bool IDLE_EXIT_ = false, bool CFENCE_ = true>
struct WsCfgT {
    static constexpr int BM = BM_, BN = BN_, BK = BK_, WM = WM_, WN = WN_, STAGES = STAGES_, MINB = MINB_;
    // LDG: the producer stages operands with per-lane 16-byte cp.async (LDGSTS) and signals the
    // "full" barrier with cp.async.mbarrier.arrive.noinc (32 arrivals) instead of bulk copies with
    // a transaction count (the bulk-copy pipeline picked up rare stale k-slices
    // under concurrent high-priority work; the LDGSTS one did not)
    static constexpr bool LDG = LDG_;
    // IDLE_EXIT (dev variant 2x, the round-2 kernel): with bulk copies the three idle producer warps
    // returned right after setmaxnreg.dec instead of waiting at the tail barrier
    static constexpr bool IDLE_EXIT = IDLE_EXIT_;
    // CFENCE (bulk copies): consumers issue fence.proxy.async before releasing a stage, ordering
    // their generic-proxy fragment loads (LDS) before the producer's next async-proxy (bulk) write
    // into that stage. Without it a delayed LDS could read the k-slice two stages later (a wrong
    // row of one warp tile, seen under concurrent high-priority work; profiles/r02/race_r02.md)
    static constexpr bool CFENCE = CFENCE_;
    static constexpr int WARPS_M = BM / WM, WARPS_N = BN / WN, CONSUMERS = WARPS_M * WARPS_N;
    static constexpr int THREADS = (CONSUMERS + 4) * 32;   // + one producer warpgroup (setmaxnreg)
    static constexpr int REG_CONS = REG_CONS_, REG_PROD = LDG_ ? 56 : 40;
    static constexpr int PA = BM + 4, PB = BN + 4;
    static constexpr int SA = BK * PA, SB = BK * PB;
    static constexpr size_t SMEM = (size_t)STAGES * (SA + SB) * sizeof(double) + 2 * STAGES * sizeof(uint64_t);
    static constexpr int FM = WM / 8, FN = WN / 8;
    // setmaxnreg moves registers inside the CTA's launch allocation (R0 per thread): what the
    // producer warpgroup releases must cover what the consumers add, or .inc blocks forever.
    static constexpr int R0 = (65536 / MINB / THREADS) / 8 * 8;
    static_assert(CONSUMERS * 32 * (REG_CONS - R0) <= 128 * (R0 - REG_PROD), "setmaxnreg budget");
    static_assert(SMEM * MINB <= 232448, "shared memory");
};
using WsCfg = WsCfgT<128, 128, 32, 3, 64, 32, 232, 1>;    // 8 consumer warps, 1 CTA/SM (default)
using WsCfg16 = WsCfgT<128, 128, 32, 3, 32, 32, 104, 1>;  // 16 consumer warps, 32x32 warp tiles
using WsCfg2a = WsCfgT<128, 64, 16, 4, 64, 32, 216, 2>;   // 2 CTAs/SM, 128x64 tiles, 4-stage BK=16
using WsCfg2b = WsCfgT<128, 64, 32, 2, 64, 32, 216, 2>;   // 2 CTAs/SM, 128x64 tiles, 2-stage BK=32
using WsCfg2nf = WsCfgT<128, 64, 32, 2, 64, 32, 216, 2, false, false, false>;  // dev: 2b without the consumer proxy fence
using WsCfg2l = WsCfgT<128, 64, 32, 2, 64, 32, 200, 2, true>;   // as 2b, LDGSTS producer warpgroup
using WsCfg2x = WsCfgT<128, 64, 32, 2, 64, 32, 216, 2, false, true, false>;   // dev: 2nf + idle producer warps exit (round-2 kernel)
using WsCfgNR = WsCfgT<128, 64, 32, 2, 64, 32, 128, 2>;   // dev: as 2b without setmaxnreg (spills)

// tile index -> (tm, tn) for the three masks; returns false for tiles with nothing to write
// Lower-trapezoid tile enumeration for BN = BM / R (R = 1 or 2): tile row tm holds the column
// tiles tn < min(R (tm + 1), TN); prefix(t) = tiles in rows < t.
template <int R>
__host__ __device__ __forceinline__ int64_t lower_prefix(int64_t t, int64_t TN) {
    const int64_t T0 = TN / R;   // rows whose count R(tm+1) <= TN
    if (t <= T0) return R * t * (t + 1) / 2;
    return R * T0 * (T0 + 1) / 2 + (t - T0) * TN;
}

// Column prefix inside a group of rows [a0, a0 + Gp) of the lower trapezoid: column u holds the
// rows a >= max(a0, floor(u / R)); P(u) = tiles in columns < u of the group.
template <int R>
__device__ __forceinline__ int64_t group_col_prefix(int64_t u, int64_t a0, int64_t Gp) {
    int64_t w = u - R * (a0 + 1);
    int64_t S = 0;
    if (w > 0) {
        const int64_t p = w / R, rem = w - p * R;
        S = R * p * (p + 1) / 2 + rem * (p + 1);
    }
    return u * Gp - S;
}

constexpr int kWsGroup = 8;   // tile rows per L2 group: A rows of a group stay in L2, W streams once per group

// One output tile of the warp-specialised kernel: which row segment, where its operands live.
struct WsTile {
    int64_t m0, n0;         // m0 relative to its segment
    bool seg2;              // checksum-row segment: A2 / C2 / ldc2 / M2, MASK_CHK with tile offsets 0
};

// Data-segment tile rows the ws kernel enumerates (the owned row blocks only when rstride > 1),
// and the global tile row of enumerated tile row tmL.
template <int BM>
__host__ __device__ __forceinline__ int64_t ws_tm(const GemmArgs& g) {
    const int64_t TM = (g.M + BM - 1) / BM;
    if (g.rstride <= 1) return TM;
    const int64_t nbt = g.nb / BM, NB = g.M / g.nb;
    return NB > g.rfirst ? ((NB - g.rfirst + g.rstride - 1) / g.rstride) * nbt : 0;
}
template <int BM>
__device__ __forceinline__ int64_t ws_row_of(const GemmArgs& g, int64_t tmL) {
    if (g.rstride <= 1) return tmL;
    const int64_t nbt = g.nb / BM;
    return (g.rfirst + (tmL / nbt) * g.rstride) * nbt + tmL % nbt;
}

// tile index -> tile; returns false for tiles with nothing to write. Segment-1 tiles are
// enumerated group by group (kWsGroup tile rows), column-major inside a group, so the CTAs
// running at the same time share operand tiles in L2; the checksum-row segment follows.
template <int BM, int BN>
__device__ __forceinline__ bool ws_tile(const GemmArgs& g, int64_t idx, int64_t n1tiles, WsTile& T) {
    constexpr int R = BM / BN;
    const int64_t TN = g.tiles_n, TM = ws_tm<BM>(g);
    int64_t tm, tn;
    if (idx >= n1tiles) {   // second segment: checksum rows, rectangular, row-major
        const int64_t e = idx - n1tiles;
        tm = e / TN; tn = e % TN;
        T.m0 = tm * BM; T.n0 = tn * BN; T.seg2 = true;
        const int64_t qmax = min(g.M2, T.m0 + BM) - 1;
        return chk_block(qmax, g.nchk) >= (T.n0 / g.nb) * g.cstride;
    }
    if (g.mask == MASK_LOWER && (g.cstride > 1 || g.rstride > 1)) {   // strided: grouped rectangle, skip tiles above
        const int64_t q = idx / (kWsGroup * TN), a0 = q * kWsGroup, Gp = ((TM - a0) < kWsGroup ? (TM - a0) : (int64_t)kWsGroup);
        const int64_t e = idx - a0 * TN;
        tn = e / Gp; tm = ws_row_of<BM>(g, a0 + e % Gp);
        T.m0 = tm * BM; T.n0 = tn * BN; T.seg2 = false;
        const int64_t rmax = min(g.M, T.m0 + BM) - 1;
        return rmax >= T.n0 + (T.n0 / g.nb) * g.nb * (g.cstride - 1);
    }
    if (g.mask == MASK_LOWER) {
        // group q: the last q with lower_prefix(q G) <= idx
        int64_t lo = 0, hi = (TM + kWsGroup - 1) / kWsGroup;
        while (hi - lo > 1) {
            const int64_t mid = (lo + hi) / 2;
            if (lower_prefix<R>(mid * kWsGroup, TN) <= idx) lo = mid; else hi = mid;
        }
        const int64_t a0 = lo * kWsGroup, Gp = ((TM - a0) < kWsGroup ? (TM - a0) : (int64_t)kWsGroup);
        const int64_t e = idx - lower_prefix<R>(a0, TN);
        const int64_t ncol = ((R * (a0 + Gp)) < TN ? (R * (a0 + Gp)) : TN);
        int64_t ul = 0, uh = ncol;   // column u: P(u) <= e < P(u + 1)
        while (uh - ul > 1) {
            const int64_t mid = (ul + uh) / 2;
            if (group_col_prefix<R>(mid, a0, Gp) <= e) ul = mid; else uh = mid;
        }
        tn = ul;
        const int64_t first = ((ul / R) > a0 ? (ul / R) : a0);
        tm = first + (e - group_col_prefix<R>(ul, a0, Gp));
    } else {
        const int64_t q = idx / (kWsGroup * TN), a0 = q * kWsGroup, Gp = ((TM - a0) < kWsGroup ? (TM - a0) : (int64_t)kWsGroup);
        const int64_t e = idx - a0 * TN;
        tn = e / Gp; tm = ws_row_of<BM>(g, a0 + e % Gp);
    }
    T.m0 = tm * BM; T.n0 = tn * BN; T.seg2 = false;
    if (g.mask == MASK_CHK) {
        const int64_t qmax = min(g.M, T.m0 + BM) - 1;
        if (g.q_tile0 + chk_block(qmax, g.nchk) < g.c_tile0 + T.n0 / g.nb) return false;
    }
    return true;
}

template <class C_, bool CS3 = false>
__device__ __forceinline__ void ws_body(const GemmArgs& g, int64_t ntiles, int64_t n1tiles) {
    constexpr int BM = C_::BM, BN = C_::BN, BK = C_::BK, WM = C_::WM, WN = C_::WN, STAGES = C_::STAGES;
    if (cta_aborted(g.abort)) return;
    extern __shared__ __align__(16) double smem[];
    double* sA = smem;
    double* sB = smem + STAGES * C_::SA;
    uint64_t* full = reinterpret_cast<uint64_t*>(smem + STAGES * (C_::SA + C_::SB));
    uint64_t* empty = full + STAGES;
    const int tid = threadIdx.x, lane = tid & 31, warp = __shfl_sync(0xffffffffu, tid >> 5, 0);   // warp-uniform
    if (tid == 0) {
        for (int i = 0; i < STAGES; ++i) { mbar_init(&full[i], C_::LDG ? 128 : 1); mbar_init(&empty[i], C_::CONSUMERS); }
        asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
    }
    __syncthreads();

    if (warp >= C_::CONSUMERS) {
        // ------------------------------- producer -------------------------------
        if constexpr (C_::REG_CONS != C_::R0)
            asm volatile("setmaxnreg.dec.sync.aligned.u32 %0;\n" ::"n"(C_::REG_PROD) : "memory");
        // bulk copies: one warp issues them; the other three warps of the producer warpgroup idle
        // at the tail barrier below instead of exiting (variant 2x restores the early exit for the
        // race matrix, profiles/r02/race_r02.md)
        if (!C_::LDG && warp != C_::CONSUMERS) {
            if constexpr (!C_::IDLE_EXIT) asm volatile("bar.sync 1, %0;\n" ::"n"((C_::CONSUMERS + 4) * 32) : "memory");
            return;
        }
        const int ptid = tid - C_::CONSUMERS * 32;       // 0..127 in the producer warpgroup
        const int64_t pf_ahead = (C_::LDG && warp != C_::CONSUMERS) ? 0 : g.pf_ahead;
        uint32_t it = 0;
        for (int64_t t = blockIdx.x; t < ntiles; t += gridDim.x) {
            WsTile T;
            if (!ws_tile<BM, BN>(g, t, n1tiles, T)) continue;
            const int64_t m0 = T.m0, n0 = T.n0;
            const int64_t ke = (g.krange == KR_LE_N) ? min(g.K, n0 + BN) : g.K;
            const int kt_n = (int)(ke / BK);
            const int64_t Ms = T.seg2 ? g.M2 : g.M;
            const double* Ap = T.seg2 ? g.A2 : g.A;
            const uint32_t rowsA = (uint32_t)(Ms - m0 < BM ? Ms - m0 : BM), rowsB = (uint32_t)(g.N - n0 < BN ? g.N - n0 : BN);
            const int64_t bn0 = n0 + (g.cstride > 1 ? (n0 / g.nb) * g.nb * (g.cstride - 1) : 0);   // B row of column n0
            for (int kt = 0; kt < kt_n; ++kt, ++it) {
                if (kt == 1 && g.beta != 0.0 && pf_ahead > 0) {
                    // warm L2 with the C tile of the CTA that will start about one residency wave
                    // later (tiles are dispatched in index order), so its accumulator preload
                    // hits L2 instead of HBM
                    WsTile Tn;
                    const int64_t tn = t + pf_ahead;
                    if (tn < ntiles && ws_tile<BM, BN>(g, tn, n1tiles, Tn)) {
                        const int64_t Msn = Tn.seg2 ? g.M2 : g.M;
                        double* Cn = Tn.seg2 ? g.C2 : g.C;
                        const int64_t ldn = Tn.seg2 ? g.ldc2 : g.ldc;
                        const uint32_t rA = (uint32_t)(Msn - Tn.m0 < BM ? Msn - Tn.m0 : BM);
                        const int cB = (int)(g.N - Tn.n0 < BN ? g.N - Tn.n0 : BN);
                        for (int c = lane; c < cB; c += 32) prefetch_l2(Cn + (Tn.n0 + c) * ldn + Tn.m0, rA * 8);
                    }
                }
                const int st = it % STAGES;
                const uint32_t ph = (it / STAGES) & 1;
                if constexpr (C_::LDG) {
                    if (lane == 0) mbar_wait(&empty[st], ph ^ 1);
                    __syncwarp();
                    // each of the 128 producer threads owns one 16-byte chunk column of A and of B and
                    // copies it for every RA-th (RB-th) k-row of the stage: a base pointer + constant
                    // strides, smem offsets are immediates (no per-copy index arithmetic)
                    constexpr int CA = BM / 2, CB = BN / 2;      // 16-byte chunks per k-row of A / B
                    constexpr int RA = 128 / CA, RB = 128 / CB;  // k-rows one pass of 128 threads covers
                    static_assert(BK % RA == 0 && BK % RB == 0, "LDGSTS producer mapping");
                    const int64_t ldA = T.seg2 ? g.lda2 : g.lda;
                    const int ra = ptid % CA, ka = ptid / CA, rb = ptid % CB, kb = ptid / CB;
                    const double* pa = Ap + ((int64_t)kt * BK + ka) * ldA + m0 + 2 * ra;
                    const double* pb = g.B + ((int64_t)kt * BK + kb) * g.ldb + bn0 + 2 * rb;
                    const uint32_t da = smem_u32(sA + st * C_::SA + ka * C_::PA + 2 * ra);
                    const uint32_t db = smem_u32(sB + st * C_::SB + kb * C_::PB + 2 * rb);
                    const int64_t sa_step = (int64_t)RA * ldA, sb_step = (int64_t)RB * g.ldb;
                    if (2 * ra < (int)rowsA) {
#pragma unroll 2
                        for (int u = 0; u < BK / RA; ++u)
                            asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"(da + u * RA * C_::PA * 8),
                                         "l"(pa + u * sa_step) : "memory");
                    }
                    if (2 * rb < (int)rowsB) {
#pragma unroll 2
                        for (int u = 0; u < BK / RB; ++u)
                            asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"(db + u * RB * C_::PB * 8),
                                         "l"(pb + u * sb_step) : "memory");
                    }
                    asm volatile("cp.async.mbarrier.arrive.noinc.shared::cta.b64 [%0];\n" ::"r"(smem_u32(&full[st])) : "memory");
                    continue;
                }
                if (lane == 0) {
                    mbar_wait(&empty[st], ph ^ 1);
                    mbar_expect_tx(&full[st], (uint32_t)BK * (rowsA + rowsB) * 8);
                }
                __syncwarp();
                const int64_t k0 = (int64_t)kt * BK;
                for (int kk = lane; kk < BK; kk += 32) {
                    bulk_g2s(sA + st * C_::SA + kk * C_::PA, Ap + (k0 + kk) * (T.seg2 ? g.lda2 : g.lda) + m0, rowsA * 8, &full[st]);
                    bulk_g2s(sB + st * C_::SB + kk * C_::PB, g.B + (k0 + kk) * g.ldb + bn0, rowsB * 8, &full[st]);
                }
            }
        }
        if constexpr (!C_::LDG) {
            // producer tail: the producer warps stay resident until the consumers have finished
            // (named barrier 1: these warps wait, the consumer warps arrive at their end), so no
            // warp of the CTA exits while bulk copies may still be in flight or while the
            // consumers run on registers the producer warpgroup released with setmaxnreg.dec
            if constexpr (C_::IDLE_EXIT) asm volatile("bar.sync 1, %0;\n" ::"n"((C_::CONSUMERS + 1) * 32) : "memory");
            else asm volatile("bar.sync 1, %0;\n" ::"n"((C_::CONSUMERS + 4) * 32) : "memory");
        }
        return;
    }
    // ------------------------------- consumers -------------------------------
    if constexpr (C_::REG_CONS != C_::R0)
        asm volatile("setmaxnreg.inc.sync.aligned.u32 %0;\n" ::"n"(C_::REG_CONS) : "memory");
    const int wm = warp / C_::WARPS_N, wn = warp % C_::WARPS_N;
    const int fr = lane >> 2, fc = lane & 3;
    const double ab = g.alpha * g.beta, alpha = g.alpha;
    uint32_t it = 0;
    for (int64_t t = blockIdx.x; t < ntiles; t += gridDim.x) {
        WsTile T;
        if (!ws_tile<BM, BN>(g, t, n1tiles, T)) continue;
        const int64_t m0 = T.m0, n0 = T.n0;
        const int64_t ke = (g.krange == KR_LE_N) ? min(g.K, n0 + BN) : g.K;
        const int kt_n = (int)(ke / BK);
        const bool seg2 = T.seg2;
        // ownership of element (r, c): r < Mlim and r >= rmin(c), rmin precomputed per owned column
        // (no per-element 64-bit division: the epilogue must stay short and I-cache friendly)
        const int64_t Mlim = seg2 ? g.M2 : g.M;
        const int64_t cshift = g.cstride > 1 ? (n0 / g.nb) * g.nb * (g.cstride - 1) : 0;   // global - local col
        int64_t rmin[C_::FN][2];
#pragma unroll
        for (int j = 0; j < C_::FN; ++j)
#pragma unroll
            for (int h = 0; h < 2; ++h) {
                const int64_t c = n0 + wn * WN + j * 8 + fc * 2 + h;
                int64_t v;
                if (c >= g.N) v = INT64_MAX;
                else if (seg2) v = g.nchk * (c / g.nb) * g.cstride;                  // q/nchk >= block of c
                else if (g.mask == MASK_LOWER) v = c + cshift;                        // r >= global c
                else if (g.mask == MASK_CHK) v = g.nchk * (g.c_tile0 + c / g.nb - g.q_tile0);
                else v = 0;
                rmin[j][h] = v;
            }
        auto owns = [&](int64_t r, int j, int h) { return r < Mlim && r >= rmin[j][h]; };
        double* Cp = seg2 ? g.C2 : g.C;
        const int64_t ldcp = seg2 ? g.ldc2 : g.ldc;
        double acc[C_::FM][C_::FN][2];
        // acc = alpha*beta*C on the elements this tile owns (masked / out-of-range: 0)
#pragma unroll
        for (int i = 0; i < C_::FM; ++i) {
            const int64_t r = m0 + wm * WM + i * 8 + fr;
#pragma unroll
            for (int j = 0; j < C_::FN; ++j)
#pragma unroll
                for (int h = 0; h < 2; ++h) {
                    const int64_t c = n0 + wn * WN + j * 8 + fc * 2 + h;
                    acc[i][j][h] = (owns(r, j, h) && ab != 0.0) ? ab * Cp[c * ldcp + r] : 0.0;
                }
        }
        for (int kt = 0; kt < kt_n; ++kt, ++it) {
            const int st = it % STAGES;
            mbar_wait(&full[st], (it / STAGES) & 1);
            const double* cA = sA + st * C_::SA + wm * WM + fr;
            const double* cB = sB + st * C_::SB + wn * WN + fr;
#pragma unroll
            for (int kk = 0; kk < BK; kk += 4) {
                double af[C_::FM], bf[C_::FN];
#pragma unroll
                for (int i = 0; i < C_::FM; ++i) af[i] = cA[(kk + fc) * C_::PA + i * 8];
#pragma unroll
                for (int j = 0; j < C_::FN; ++j) bf[j] = cB[(kk + fc) * C_::PB + j * 8];
#pragma unroll
                for (int i = 0; i < C_::FM; ++i)
#pragma unroll
                    for (int j = 0; j < C_::FN; ++j) dmma(acc[i][j][0], acc[i][j][1], af[i], bf[j]);
            }
            if constexpr (C_::CFENCE && !C_::LDG) asm volatile("fence.proxy.async.shared::cta;\n" ::: "memory");
            __syncwarp();
            if (lane == 0) mbar_arrive(&empty[st]);
        }
        // epilogue: C = alpha * acc, masked stores only
#pragma unroll
        for (int i = 0; i < C_::FM; ++i)
#pragma unroll
            for (int j = 0; j < C_::FN; ++j)
#pragma unroll
                for (int h = 0; h < 2; ++h) acc[i][j][h] = alpha * acc[i][j][h];
        // UPDATE_OUT hook (reading A21): XOR the injected bits into the updated value before it is
        // stored and before the fused V5 partials see it (warp-uniform test, off the common path)
        for (int q = 0; q < g.inj.n; ++q) {
            const EpiInjOp e = g.inj.op[q];
            const int64_t lr = e.r - (m0 + wm * WM), lc = e.c - (n0 + wn * WN);
            if (e.seg != (seg2 ? 1 : 0) || lr < 0 || lr >= WM || lc < 0 || lc >= WN) continue;
#pragma unroll
            for (int i = 0; i < C_::FM; ++i)
#pragma unroll
                for (int j = 0; j < C_::FN; ++j)
#pragma unroll
                    for (int h = 0; h < 2; ++h)
                        if (i * 8 + fr == lr && j * 8 + fc * 2 + h == lc)
                            acc[i][j][h] = __longlong_as_double(__double_as_longlong(acc[i][j][h]) ^ (long long)e.mask);
        }
#pragma unroll
        for (int i = 0; i < C_::FM; ++i) {
            const int64_t r = m0 + wm * WM + i * 8 + fr;
#pragma unroll
            for (int j = 0; j < C_::FN; ++j)
#pragma unroll
                for (int h = 0; h < 2; ++h) {
                    const int64_t c = n0 + wn * WN + j * 8 + fc * 2 + h;
                    if (owns(r, j, h)) Cp[c * ldcp + r] = acc[i][j][h];
                }
        }
        // fused V5 recalculation: per-column v1/v2 partial sums of the
        // updated values over each warp's 64 rows (slab = global_row / 64), for tiles off the
        // block diagonal (diagonal blocks are checked as sym(tril) by a re-read). Data rows only.
        if (g.cs.p != nullptr && t < n1tiles) {
            const int64_t gr0 = g.cs.row0 + m0 + wm * WM, gc0 = g.cs.col0 + n0;
            // warp-uniform; the shuffles below stay outside any branch so that they compile to
            // plain SHFLs (inside a possibly divergent branch they become WARPSYNC collectives)
            const bool offdiag = gr0 / g.cs.nb != (g.cs.colg0 + n0 + cshift) / g.cs.nb;
            const int64_t wbase = gr0 % g.cs.nb + fr + 1;   // weight (1-based) of row i = 0
            const int64_t slab = gr0 / g.cs.slab_rows;
            __syncwarp();
            // per-thread sums over its FM rows for its 8 columns (slot q = 2 j + h): v[2q] = v1
            // partial, v[2q + 1] = v2 partial; then a reduce-scatter butterfly over the 8 lanes
            // of equal fc (lane bits 2-4 = fr): each round halves the values a lane keeps, so 14
            // shuffles (not 48) leave lane fr holding the full sums of column slot fr
            static_assert(C_::FN == 4, "reduce-scatter assumes 8 column slots per thread");
            double v[16];
#pragma unroll
            for (int j = 0; j < C_::FN; ++j)
#pragma unroll
                for (int h = 0; h < 2; ++h) {
                    double s1 = 0.0, s2 = 0.0;
#pragma unroll
                    for (int i = 0; i < C_::FM; ++i) {
                        s1 += acc[i][j][h];
                        s2 = fma((double)(wbase + i * 8), acc[i][j][h], s2);
                    }
                    v[2 * (2 * j + h)] = s1;
                    v[2 * (2 * j + h) + 1] = s2;
                }
            {   // round 1: lane bit 4 (fr bit 2) picks the half of the 16 values it keeps
                const bool up = (fr & 4) != 0;
#pragma unroll
                for (int i = 0; i < 8; ++i) {
                    const double keep = up ? v[i + 8] : v[i], give = up ? v[i] : v[i + 8];
                    v[i] = keep + __shfl_xor_sync(0xffffffffu, give, 16);
                }
            }
            {   // round 2: fr bit 1
                const bool up = (fr & 2) != 0;
#pragma unroll
                for (int i = 0; i < 4; ++i) {
                    const double keep = up ? v[i + 4] : v[i], give = up ? v[i] : v[i + 4];
                    v[i] = keep + __shfl_xor_sync(0xffffffffu, give, 8);
                }
            }
            {   // round 3: fr bit 0
                const bool up = (fr & 1) != 0;
#pragma unroll
                for (int i = 0; i < 2; ++i) {
                    const double keep = up ? v[i + 2] : v[i], give = up ? v[i] : v[i + 2];
                    v[i] = keep + __shfl_xor_sync(0xffffffffu, give, 4);
                }
            }
            const int64_t gcs = gc0 + wn * WN + (fr >> 1) * 8 + fc * 2 + (fr & 1);   // column slot fr
            if (offdiag) {   // lane (fr, fc) holds column slot q = fr: j = fr / 2, h = fr % 2
                g.cs.p[slab * g.cs.ld + gcs] = v[0];
                g.cs.p[(g.cs.nslab + slab) * g.cs.ld + gcs] = v[1];
            }
            if (CS3) {   // third checksum (B10): weights (row + 1)^2, same butterfly on 8 values
                double u[8];
#pragma unroll
                for (int j = 0; j < C_::FN; ++j)
#pragma unroll
                    for (int h = 0; h < 2; ++h) {
                        double s3 = 0.0;
#pragma unroll
                        for (int i = 0; i < C_::FM; ++i) {
                            const double w = (double)(wbase + i * 8);
                            s3 = fma(w * w, acc[i][j][h], s3);
                        }
                        u[2 * j + h] = s3;
                    }
                {
                    const bool up = (fr & 4) != 0;
#pragma unroll
                    for (int i = 0; i < 4; ++i) {
                        const double keep = up ? u[i + 4] : u[i], give = up ? u[i] : u[i + 4];
                        u[i] = keep + __shfl_xor_sync(0xffffffffu, give, 16);
                    }
                }
                {
                    const bool up = (fr & 2) != 0;
#pragma unroll
                    for (int i = 0; i < 2; ++i) {
                        const double keep = up ? u[i + 2] : u[i], give = up ? u[i] : u[i + 2];
                        u[i] = keep + __shfl_xor_sync(0xffffffffu, give, 8);
                    }
                }
                {
                    const bool up = (fr & 1) != 0;
                    const double keep = up ? u[1] : u[0], give = up ? u[0] : u[1];
                    u[0] = keep + __shfl_xor_sync(0xffffffffu, give, 4);
                }
                if (offdiag) g.cs.p[(2 * g.cs.nslab + slab) * g.cs.ld + gcs] = u[0];
            }
        }
    }
    // release the copying producer warp (its tail waits on named barrier 1)
    if constexpr (!C_::LDG) {
        if constexpr (C_::IDLE_EXIT) asm volatile("bar.arrive 1, %0;\n" ::"n"((C_::CONSUMERS + 1) * 32) : "memory");
        else asm volatile("bar.arrive 1, %0;\n" ::"n"((C_::CONSUMERS + 4) * 32) : "memory");
    }
}

// Two entry points with one body, so that profiles attribute the trailing update (the dominant
// kernel of the factorisation) separately from the TRSM and the other products.
template <class C_>
__global__ void __launch_bounds__(C_::THREADS, C_::MINB) k_gemm_ws(GemmArgs g, int64_t ntiles, int64_t n1tiles) {
    ws_body<C_>(g, ntiles, n1tiles);
}
// CS3: the update also emits the third checksum's partials (nchk = 3, reading B10) — a separate
// instantiation so that the default two-checksum kernel keeps its register budget
template <class C_, bool CS3 = false>
__global__ void __launch_bounds__(C_::THREADS, C_::MINB) k_update_ws(GemmArgs g, int64_t ntiles, int64_t n1tiles) {
    ws_body<C_, CS3>(g, ntiles, n1tiles);
}

template <class C_>
static int run_ws(GemmArgs g, cudaStream_t s, bool update) {
    static bool attr = false;
    if (!attr) {
        cudaFuncSetAttribute(k_gemm_ws<C_>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)C_::SMEM);
        cudaFuncSetAttribute(k_update_ws<C_>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)C_::SMEM);
        cudaFuncSetAttribute(k_update_ws<C_, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)C_::SMEM);
        attr = true;
    }
    if (g.rstride > 1 && (g.nb % C_::BM != 0 || g.M % g.nb != 0)) { g.rstride = 1; g.rfirst = 0; }   // every row
    const int64_t tm = ws_tm<C_::BM>(g), tn = (g.N + C_::BN - 1) / C_::BN;
    g.tiles_n = tn;
    const int64_t n1 = (g.mask == MASK_LOWER && g.cstride <= 1 && g.rstride <= 1) ? lower_prefix<C_::BM / C_::BN>(tm, tn)
                                                                                  : tm * tn;
    const int64_t ntiles = n1 + (g.M2 > 0 ? ((g.M2 + C_::BM - 1) / C_::BM) * tn : 0);
    if (ntiles <= 0) return 0;
    // tiles per CTA: 1 lets the block scheduler interleave the high-priority look-ahead stream's
    // kernels as CTAs retire; a fully persistent grid would starve that stream.
    static int64_t tpc = -1;
    if (tpc < 0) { const char* e = getenv("ABFT_WS_TPC"); tpc = e ? std::max(1, atoi(e)) : 1; }
    const int64_t grid = std::max<int64_t>(1, (ntiles + tpc - 1) / tpc);
    static int64_t ahead = -1;
    if (ahead < 0) {
        int dev = 0, nsm = 148;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
        const char* e = getenv("ABFT_WS_PF");
        ahead = e ? atoi(e) : (int64_t)nsm * C_::MINB;
    }
    g.pf_ahead = (tpc == 1) ? ahead : 0;
    if (update && g.cs.p != nullptr && g.cs.nchk == 3)
        k_update_ws<C_, true><<<(unsigned)grid, C_::THREADS, C_::SMEM, s>>>(g, ntiles, n1);
    else if (update) k_update_ws<C_><<<(unsigned)grid, C_::THREADS, C_::SMEM, s>>>(g, ntiles, n1);
    else k_gemm_ws<C_><<<(unsigned)grid, C_::THREADS, C_::SMEM, s>>>(g, ntiles, n1);
    abft_count_launch();
    return 0;
}

// The trailing-update entry points (graph mode gives every other kernel node the panel stream's
// high priority, these keep the default one).
bool is_update_kernel(const void* f) {
    return f == (const void*)k_update_ws<WsCfg> || f == (const void*)k_update_ws<WsCfg16> ||
           f == (const void*)k_update_ws<WsCfg2a> || f == (const void*)k_update_ws<WsCfg2b> ||
           f == (const void*)k_update_ws<WsCfgNR> || f == (const void*)k_update_ws<WsCfg2l> ||
           f == (const void*)k_update_ws<WsCfg2b, true> || f == (const void*)k_update_ws<WsCfg2l, true> ||
           f == (const void*)k_update_ws<WsCfg2x> || f == (const void*)k_update_ws<WsCfg2x, true> ||
           f == (const void*)k_update_ws<WsCfg2nf> || f == (const void*)k_update_ws<WsCfg2nf, true>;
}

static int ws_variant() {   // dev knob ABFT_WS: 2b (default), 1 (one 128x128 CTA/SM), 16, 2a, 2l, 2nf, 2x, nr
    static int v = -1;
    if (v < 0) {
        const char* e = getenv("ABFT_WS");
        v = 22;
        if (e && !strcmp(e, "1")) v = 0;
        if (e && !strcmp(e, "16")) v = 16;
        if (e && !strcmp(e, "2a")) v = 21;
        if (e && !strcmp(e, "2b")) v = 22;
        if (e && !strcmp(e, "2l")) v = 25;
        if (e && !strcmp(e, "nr")) v = 24;
        if (e && !strcmp(e, "2x")) v = 26;
        if (e && !strcmp(e, "2nf")) v = 27;
    }
    return v;
}
static int ws_slab_rows() { return ws_variant() == 16 ? WsCfg16::WM : 64; }

static int run_ws_any(GemmArgs g, cudaStream_t s) {
    g.cs.slab_rows = ws_slab_rows();
    const bool upd = g.mask == MASK_LOWER && g.alpha == -1.0 && g.beta == 1.0;   // a trailing update
    switch (ws_variant()) {
        case 16: return run_ws<WsCfg16>(g, s, upd);
        case 21: return run_ws<WsCfg2a>(g, s, upd);
        case 22: return run_ws<WsCfg2b>(g, s, upd);
        case 26: return run_ws<WsCfg2x>(g, s, upd);
        case 27: return run_ws<WsCfg2nf>(g, s, upd);
        case 25: return run_ws<WsCfg2l>(g, s, upd);
        case 24: return run_ws<WsCfgNR>(g, s, upd);
        default: return run_ws<WsCfg>(g, s, upd);
    }
}

}  // namespace abft

using namespace abft;

static bool aligned16(const void* p) { return ((uintptr_t)p & 15) == 0; }

// Public-to-the-library launcher. Picks the CTA tile from the problem size so that small
// GEMMs inside the diagonal-block factorisation still spread over the SMs.
int launch_gemm(int64_t M, int64_t N, int64_t K, const double* A, int64_t lda, const double* B,
                int64_t ldb, double* C, int64_t ldc, double alpha, double beta, bool transB, int mask,
                int krange, int64_t nb, int64_t q_tile0, int64_t c_tile0, const int32_t* abort_flag,
                cudaStream_t s, int force_tile, ColSumOut* cs, int nchk) {
    if (M <= 0 || N <= 0) return 0;
    GemmArgs g;
    g.nchk = nchk;
    g.M = M; g.N = N; g.K = K; g.A = A; g.lda = lda; g.B = B; g.ldb = ldb; g.C = C; g.ldc = ldc;
    g.alpha = alpha; g.beta = beta; g.mask = mask; g.krange = krange; g.nb = nb;
    g.q_tile0 = q_tile0; g.c_tile0 = c_tile0; g.tiles_n = 1; g.abort = abort_flag;
    g.cs = cs ? *cs : ColSumOut{nullptr, 0, 0, 0, 0, 1, 64, 0, 2};
    g.M2 = 0; g.A2 = nullptr; g.C2 = nullptr; g.ldc2 = 1; g.lda2 = 1; g.cstride = 1;
    g.rstride = 1; g.rfirst = 0;
    g.inj.n = 0;
    g.vecA = aligned16(A) && (lda % 2 == 0);
    g.vecB = aligned16(B) && (ldb % 2 == 0);
    auto tiles = [&](int64_t t) {
        const int64_t tm = (M + t - 1) / t, tn = (N + t - 1) / t;
        return mask == MASK_LOWER ? tn * (tn + 1) / 2 + (tm - tn) * tn : tm * tn;
    };
    int tile = force_tile;
    if (!tile) {
        if (tiles(128) >= 148) tile = 128;
        else if (tiles(64) >= 148) tile = 64;
        else tile = 32;
    }
    static int variant = -1;
    if (variant < 0) { const char* e = getenv("ABFT_GEMM_VARIANT"); variant = e ? atoi(e) : 0; }
    // warp-specialised persistent fast path: NT, 16-byte aligned operands with even leading
    // dimensions, even M and N, alpha = +-1, whole BK-deep k-tiles (K % 32 == 0, k from 0)
    const bool ws_ok = transB && g.vecA && g.vecB && (M % 2 == 0) && (N % 2 == 0) && (K % WsCfg::BK == 0) &&
                       (krange == KR_FULL || krange == KR_LE_N) && (alpha == 1.0 || alpha == -1.0) &&
                       (mask != MASK_LOWER || N <= M);
    if (cs) {   // fused partials need the warp-specialised kernel with nb-aligned 128-row tiles
        if (!(ws_ok && variant != 2 && mask == MASK_LOWER && cs->nb % WsCfg::BM == 0 &&
              cs->row0 % WsCfg::BM == 0 && cs->colg0 % WsCfg::BN == 0 && M % WsCfg::BM == 0)) g.cs.p = nullptr;
        else { run_ws_any(g, s); cs->slab_rows = ws_slab_rows(); return 1; }
    }
    if (transB) {
        if (tile == 128 && ws_ok && variant != 2) return run_ws_any(g, s);
        if (tile == 128) return run_cfg<128, 128, 32, 64, 32, 3, true>(g, s);
        if (tile == 64) return run_cfg<64, 64, 16, 32, 32, 4, true>(g, s);
        return run_cfg<32, 32, 16, 16, 16, 4, true>(g, s);
    } else {
        if (tile == 128) return run_cfg<128, 128, 32, 64, 32, 3, false>(g, s);
        if (tile == 64) return run_cfg<64, 64, 16, 32, 32, 4, false>(g, s);
        return run_cfg<32, 32, 16, 16, 16, 4, false>(g, s);
    }
}

// Trailing update with the checksum rows appended as a second row segment of the same launch
// (chk(A') = chk(A) - chk(LC) LC^T as extra GEMM rows). Falls back to two
// launches when the warp-specialised kernel cannot take the shapes. Returns 1 if the fused V5
// partials were written.
int launch_update_with_chk(int64_t M, int64_t N, int64_t K, const double* A, int64_t lda, const double* B,
                           int64_t ldb, double* C, int64_t ldc, int64_t M2, const double* A2, double* C2,
                           int64_t ldc2, int64_t nb, const int32_t* abort_flag, cudaStream_t s, ColSumOut* cs,
                           int64_t lda2, int64_t cstride, const EpiInj* inj, int nchk, int64_t rstride,
                           int64_t rfirst) {
    if (lda2 <= 0) lda2 = lda;
    if (cstride < 1) cstride = 1;
    // the data segment's kernel must not depend on the checksum segment (same rounding with two or
    // three checksum rows): the checksum rows ride in the same launch when their shapes allow it,
    // else they get their own launch and the data rows still take the warp-specialised kernel
    const bool ok = M > 0 && N > 0 && (M % 2 == 0) && (N % 2 == 0) && (K % WsCfg::BK == 0) &&
                    aligned16(A) && aligned16(B) && lda % 2 == 0 && ldb % 2 == 0 && N <= M &&
                    M % WsCfg::BM == 0 && getenv("ABFT_GEMM_VARIANT") == nullptr &&
                    (cstride == 1 || nb % WsCfg::BN == 0);
    const bool chk_ok = M2 == 0 || ((M2 % 2 == 0) && aligned16(A2) && lda2 % 2 == 0);
    if (!ok && cstride > 1) return -1;   // strided columns need the warp-specialised kernel
    if (!ok) {   // fallback (two generic launches): the caller applies the hook, no fused partials
        const int f = launch_gemm(M, N, K, A, lda, B, ldb, C, ldc, -1.0, 1.0, true, MASK_LOWER, KR_FULL, 0, 0, 0,
                                  abort_flag, s, 0, (inj && inj->n > 0) ? nullptr : cs);
        if (M2 > 0)
            launch_gemm(M2, N, K, A2, lda2, B, ldb, C2, ldc2, -1.0, 1.0, true, MASK_CHK, KR_FULL, nb, 0, 0, abort_flag, s,
                        0, nullptr, nchk);
        return f == 1 ? 1 : 0;
    }
    const bool split = !chk_ok;
    if (split && cstride > 1) return -1;
    GemmArgs g;
    g.M = M; g.N = N; g.K = K; g.A = A; g.lda = lda; g.B = B; g.ldb = ldb; g.C = C; g.ldc = ldc;
    g.alpha = -1.0; g.beta = 1.0; g.mask = MASK_LOWER; g.krange = KR_FULL; g.nb = nb;
    g.q_tile0 = 0; g.c_tile0 = 0; g.tiles_n = 1; g.abort = abort_flag; g.vecA = 1; g.vecB = 1;
    g.cs = ColSumOut{nullptr, 0, 0, 0, 0, 1, 64, 0, 2};
    g.inj.n = 0;
    g.nchk = nchk;
    g.rstride = rstride > 1 ? rstride : 1; g.rfirst = rstride > 1 ? rfirst : 0;
    int ret = 0;
    bool inj_chk = false;   // a checksum-row target, which a split-off checksum launch cannot apply
    for (int q = 0; inj && q < inj->n && q < kMaxEpiInj; ++q) inj_chk |= inj->op[q].seg == 1;
    const bool inj_left = inj && (inj->n > kMaxEpiInj || (split && inj_chk));   // caller's hook
    if (inj && inj->n > 0 && !inj_left) { g.inj = *inj; ret |= 2; }
    if (cs && !inj_left && cs->nb % WsCfg::BM == 0 && cs->row0 % WsCfg::BM == 0 && cs->colg0 % WsCfg::BN == 0) {
        g.cs = *cs; ret |= 1;
    }
    if (split) {
        g.M2 = 0; g.A2 = nullptr; g.C2 = nullptr; g.ldc2 = 1; g.lda2 = 1; g.cstride = cstride;
        run_ws_any(g, s);
        if (M2 > 0)
            launch_gemm(M2, N, K, A2, lda2, B, ldb, C2, ldc2, -1.0, 1.0, true, MASK_CHK, KR_FULL, nb, 0, 0, abort_flag, s,
                        0, nullptr, nchk);
        if (ret & 1) cs->slab_rows = ws_slab_rows();
        return ret;
    }
    g.M2 = M2; g.A2 = A2; g.C2 = C2; g.ldc2 = ldc2; g.lda2 = lda2; g.cstride = cstride;
    run_ws_any(g, s);
    if (ret & 1) cs->slab_rows = ws_slab_rows();
    return ret;
}

// Panel TRSM with the checksum rows (Alg. 2 folded in, reading B1) as ONE
// launch: W[0:mB) = A_panel inv(L)^T (data rows, first row segment) and W[mB:mB+M2) =
// chk_rows inv(L)^T (second segment). Falls back to two launches when the warp-specialised kernel
// would not fill the GPU (small panels) or the shapes do not allow it.
int launch_trsm_with_chk(int64_t mB, int64_t B, const double* Ap, int64_t lda, const double* Li, double* W,
                         int64_t ldw, int64_t M2, const double* A2, int64_t lda2, const int32_t* abort_flag,
                         cudaStream_t s, int64_t rstride, int64_t rfirst) {
    const int64_t tiles = ((mB + WsCfg::BM - 1) / WsCfg::BM) * ((B + 63) / 64);
    const bool ok = mB > 0 && M2 > 0 && tiles >= 148 && (mB % 2 == 0) && (M2 % 2 == 0) && (B % WsCfg::BK == 0) &&
                    (B % 2 == 0) && aligned16(Ap) && aligned16(Li) && aligned16(A2) && aligned16(W) && aligned16(W + mB) &&
                    lda % 2 == 0 && lda2 % 2 == 0 && ldw % 2 == 0 && getenv("ABFT_GEMM_VARIANT") == nullptr;
    if (!ok) {
        launch_gemm(mB, B, B, Ap, lda, Li, B, W, ldw, 1.0, 0.0, true, MASK_NONE, KR_LE_N, 0, 0, 0, abort_flag, s);
        if (M2 > 0)
            launch_gemm(M2, B, B, A2, lda2, Li, B, W + mB, ldw, 1.0, 0.0, true, MASK_NONE, KR_LE_N, 0, 0, 0, abort_flag, s);
        return 0;
    }
    GemmArgs g;
    g.M = mB; g.N = B; g.K = B; g.A = Ap; g.lda = lda; g.B = Li; g.ldb = B; g.C = W; g.ldc = ldw;
    g.alpha = 1.0; g.beta = 0.0; g.mask = MASK_NONE; g.krange = KR_LE_N; g.nb = B;
    g.q_tile0 = 0; g.c_tile0 = 0; g.tiles_n = 1; g.abort = abort_flag; g.vecA = 1; g.vecB = 1;
    g.cs = ColSumOut{nullptr, 0, 0, 0, 0, 1, 64, 0, 2};
    g.inj.n = 0;
    g.nchk = 2;   // the TRSM's second segment covers every row (column block 0 only)
    g.M2 = M2; g.A2 = A2; g.C2 = W + mB; g.ldc2 = ldw; g.lda2 = lda2; g.cstride = 1;
    g.rstride = rstride > 1 ? rstride : 1; g.rfirst = rstride > 1 ? rfirst : 0;   // 2D: this rank's panel rows
    run_ws_any(g, s);
    return 1;
}
