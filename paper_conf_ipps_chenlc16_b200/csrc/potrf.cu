// potrf.cu — diagonal-block factorisation L_kk = chol(sym(T(k,k))) together with inv(L_kk).
//
// The paper runs POTF2 on the CPU (Alg. 1 line 5). On B200 the block
// stays on the GPU: a recursive split
//     [A11  .  ]   L11 = chol(A11),  L21 = A21 L11^-T,  A22 <- A22 - L21 L21^T,  L22 = chol(A22)
//     [A21 A22 ]   inv21 = -inv22 L21 inv11
// whose products run on the DMMA GEMM (gemm.cu) and whose leaves (<= 64 x 64) are factored and
// inverted by one CTA in shared memory. inv(L_kk) turns the panel TRSM and
// Alg. 2 (chk <- chk L^-T) into one tensor-core GEMM.
#include "common.cuh"

#include <vector>

#include <algorithm>
#include <cstdlib>
#include <cstring>
#include <cstdio>


namespace abft {

constexpr int kLeaf = 64;

// One CTA: Cholesky of the lower triangle of T (nl x nl, nl <= 64) and its inverse, in shared
// memory, with ONE barrier per column: each thread owns a fixed set of lower-triangle elements.
// Interval j runs Cholesky step j (A22 -= a_j a_j^T / d_j with the unscaled column a_j, which is
// l_j l_j^T) and forward-elimination step j of L X = I (Y(i,:) -= a_ij / d_j * Y(j,:), which is
// l_ij / l_jj); both only read column j, final since interval j-1. Columns and rows are scaled
// once at the end (l_j = a_j / sqrt(d_j), X(i,:) = Y(i,:) / sqrt(d_i)).
// Writes L (lower) into T and inv(L) (lower, upper zeroed) into Li. A non-positive pivot sets
// NOT_SPD with info = off + j + 1 and aborts.
constexpr int kLeafThreads = 512;
constexpr int kLeafOwn = (kLeaf * (kLeaf + 1) / 2 + kLeafThreads - 1) / kLeafThreads;   // 5

__global__ void __launch_bounds__(kLeafThreads) k_leaf_potrf_inv(double* T, int64_t ldt, double* Li, int64_t ldi,
                                                                 int nl, int64_t info_off, DevState* st) {
    if (cta_aborted(&st->abort)) return;
    extern __shared__ double leaf_smem[];
    constexpr int P = kLeaf + 1;
    double* L = leaf_smem;                 // L[c*P + r]: unscaled a, then l
    double* Y = leaf_smem + kLeaf * P;     // Y[c*P + i]: forward elimination of L X = I
    __shared__ double rdd[kLeaf];          // 1 / d_j
    const int tid = threadIdx.x;
    const int E = nl * (nl + 1) / 2;
    int own_r[kLeafOwn], own_c[kLeafOwn];
#pragma unroll
    for (int q = 0; q < kLeafOwn; ++q) {
        int e = tid + q * kLeafThreads, c = 0;
        if (e < E) {
            while (e >= nl - c) { e -= nl - c; ++c; }
            own_r[q] = c + e; own_c[q] = c;
        } else { own_r[q] = -1; own_c[q] = kLeaf; }
    }
#pragma unroll
    for (int q = 0; q < kLeafOwn; ++q)
        if (own_r[q] >= 0) {
            const int r = own_r[q], c = own_c[q];
            L[c * P + r] = T[c * ldt + r];
            Y[c * P + r] = (r == c) ? 1.0 : 0.0;
        }
    for (int j = 0; j < nl; ++j) {
        __syncthreads();
        const double d = L[j * P + j];
        if (!(d > 0.0)) {
            if (tid == 0 && atomicCAS(&st->abort, 0, 1) == 0) { st->status = ABFT_NOT_SPD; st->info = info_off + j + 1; }
            return;
        }
        const double inv_d = 1.0 / d;
        if (tid == 0) rdd[j] = inv_d;
        const double* colj = L + j * P;
        const double* rowj = Y + j;          // Y(j, c) at rowj[c * P]
#pragma unroll
        for (int q = 0; q < kLeafOwn; ++q) {
            const int r = own_r[q], c = own_c[q];
            if (c > j) L[c * P + r] -= colj[r] * (colj[c] * inv_d);             // Cholesky step j
            if (r > j && j >= c) Y[c * P + r] -= (colj[r] * inv_d) * rowj[c * P]; // elimination step j
        }
    }
    __syncthreads();
#pragma unroll
    for (int q = 0; q < kLeafOwn; ++q) {
        const int r = own_r[q], c = own_c[q];
        if (r >= 0) {
            const double sc = sqrt(rdd[c]);                 // 1 / sqrt(d_c)
            T[c * ldt + r] = (r == c) ? 1.0 / sc : L[c * P + r] * sc;
            Li[c * ldi + r] = Y[c * P + r] * sqrt(rdd[r]);
        }
    }
    for (int e = tid; e < nl * nl; e += kLeafThreads) {    // upper part of the inverse: zeros
        const int c = e / nl, i = e % nl;
        if (i < c) Li[c * ldi + i] = 0.0;
    }
}

// Column-major block copy (the W -> A / chk write-back, L21 in the recursion): blockIdx.y walks
// columns, threads walk rows two at a time (16-byte accesses when both sides allow), no division.
__global__ void k_copy_block(int64_t rows, int64_t cols, const double* src, int64_t lds, double* dst,
                             int64_t ldd, const int32_t* abort_flag, int vec) {
    if (*abort_flag) return;
    for (int64_t c = blockIdx.y; c < cols; c += gridDim.y) {
        const double* sc = src + c * lds;
        double* dc = dst + c * ldd;
        if (vec) {
            for (int64_t r = 2 * (blockIdx.x * (int64_t)blockDim.x + threadIdx.x); r < rows;
                 r += 2 * (int64_t)gridDim.x * blockDim.x) {
                if (r + 1 < rows) *reinterpret_cast<double2*>(dc + r) = *reinterpret_cast<const double2*>(sc + r);
                else dc[r] = sc[r];
            }
        } else {
            for (int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; r < rows; r += (int64_t)gridDim.x * blockDim.x)
                dc[r] = sc[r];
        }
    }
}

__global__ void k_zero_block(int64_t rows, int64_t cols, double* dst, int64_t ldd) {
    const int64_t total = rows * cols;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
        const int64_t c = i / rows, r = i % rows;
        dst[c * ldd + r] = 0.0;
    }
}

// ---------------------------------------------------------------------------------------------
// Task-graph diagonal block (nb % 64 == 0, nb >= 128): ONE launch factors the nb x nb block and
// inverts it. The block is cut into T x T tiles of 64; the tile algorithm is the paper's blocked
// POTRF/TRSM/SYRK recursion one level down plus a right-looking blocked
// inverse X = inv(L):
//   P(b)      [b >= 1: L_{b,b-1} = A_{b,b-1} inv(L_{b-1})^T, A_bb -= L_{b,b-1} L_{b,b-1}^T — the
//             critical path, fused into the CTA that then factors] L_bb = chol(A_bb), X_bb = inv(L_bb)
//   S(i,b)    L_ib = A_ib X_bb^T                                       i >= b + 2       (DMMA)
//   U(i,j,b)  A_ij -= L_ib L_jb^T  (lower half when i == j)           i >= j > b       (DMMA)
//   Z(i,j,b)  Y_ij (+)= L_ib X_bj  (Y_ij accumulates in X's tile)      i > b >= j       (DMMA)
//   F(i,j)    X_ij = -X_ii Y_ij  (= -inv(L_ii) sum_{c=j}^{i-1} L_ic X_cj), zero tile (j,i) i > j (DMMA)
// Tasks are numbered in a topological order (step b: P(b+1), S(., b), U(., ., b), F(b, .),
// Z(., ., b)); CTAs fetch them with an atomic counter and wait on per-tile completion flags
// (acquire/release at gpu scope), so no co-residency is needed: every dependency of a fetched
// task was fetched earlier by a running CTA. This replaces the ~50 dependent launches of the
// recursive path (each ~7 us of launch latency) on the look-ahead stream's critical path. The
// last CTA to exit zeroes the flags for the next launch (the sync area is zeroed once when it is
// allocated).
constexpr int kTT = 64;                 // tile
constexpr int kTP = kTT + 4;            // smem pitch: 4 mod 16 8-byte banks, conflict-free fragments
constexpr int kTaskThreads = 256;       // 8 warps: 2 x 4 grid of 32 x 16 warp tiles
constexpr size_t kTaskSmem = 3 * (size_t)kTT * kTP * sizeof(double);   // two operand tiles + leaf scratch
enum { TK_P = 0, TK_S = 1, TK_U = 2, TK_Z = 3, TK_F = 4 };

// tasks of step b (m = T - 1 - b tiles below the diagonal tile b)
__host__ __device__ __forceinline__ int task_step_count(int T, int b) {
    const int m = T - 1 - b;
    return (m >= 1 ? 1 : 0) + (m >= 2 ? m - 1 : 0) + m * (m + 1) / 2 - (m >= 1 ? 1 : 0) + b + m * (b + 1);
}
__host__ __device__ __forceinline__ int task_count(int T) {
    int s = 1;   // P(0)
    for (int b = 0; b < T; ++b) s += task_step_count(T, b);
    return s;
}
// [next task, exited CTAs, P flags (T), S flags (T x T), U flags (T x T), Z counts (T x T), F flags (T x T)]
__host__ __device__ __forceinline__ int task_sync_words(int T) { return 2 + T + 4 * T * T; }

__device__ __forceinline__ void decode_task(int T, int t, int& type, int& i, int& j, int& b) {
    if (t == 0) { type = TK_P; i = j = b = 0; return; }
    t -= 1;
    for (b = 0; b < T - 1; ++b) {
        const int cnt = task_step_count(T, b);
        if (t < cnt) break;
        t -= cnt;
    }
    const int m = T - 1 - b;
    if (m >= 1) {
        if (t == 0) { type = TK_P; i = j = b = b + 1; return; }
        t -= 1;
        if (t < m - 1) { type = TK_S; i = b + 2 + t; j = b; return; }
        t -= m - 1;
        const int nu = m * (m + 1) / 2 - 1;
        if (t < nu) {   // column-major over (j, i), b < j <= i, skipping (b+1, b+1)
            int e = t + 1, jj = b + 1;
            while (e >= T - jj) { e -= T - jj; ++jj; }
            type = TK_U; j = jj; i = jj + e; return;
        }
        t -= nu;
    }
    if (t < b) { type = TK_F; i = b; j = t; return; }
    t -= b;
    type = TK_Z; i = b + 1 + t / (b + 1); j = t % (b + 1);   // Z(i, j, b), i > b >= j
}

__device__ __forceinline__ void cpa16(double* smem, const double* gmem) {
    const unsigned s = (unsigned)__cvta_generic_to_shared(smem);
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"(s), "l"(gmem) : "memory");
}
__device__ __forceinline__ void cpa_wait_all() {
    asm volatile("cp.async.commit_group;\ncp.async.wait_group 0;\n" ::: "memory");
}
__device__ __forceinline__ uint32_t ld_acquire(const uint32_t* p) {
    uint32_t v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];\n" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_release(uint32_t* p, uint32_t v) {
    asm volatile("st.release.gpu.global.u32 [%0], %1;\n" ::"l"(p), "r"(v) : "memory");
}
// spin until *f >= v; false if the run aborted meanwhile
__device__ __forceinline__ bool wait_ge(const uint32_t* f, uint32_t v, const int32_t* abort) {
    if (gridDim.x == 1) return true;   // one CTA runs the tasks in order
    for (;;) {
        if (ld_acquire(f) >= v) return true;
        if (*(volatile const int32_t*)abort) return false;
        __nanosleep(32);
    }
}

// s[k][m] = X(m, k) of a 64 x 64 column-major tile (16-byte cp.async, L2 only)
__device__ __forceinline__ void tile_load_T(double* s, const double* X, int64_t ld) {
    for (int e = threadIdx.x; e < kTT * kTT / 2; e += kTaskThreads) {
        const int k = e >> 5, m2 = (e & 31) * 2;
        cpa16(s + k * kTP + m2, X + k * ld + m2);
    }
}
// s[k][n] = X(k, n) (the NN operand): 16-byte loads down a column, two 8-byte shared stores
__device__ __forceinline__ void tile_load_N(double* s, const double* X, int64_t ld) {
    for (int e = threadIdx.x; e < kTT * kTT / 2; e += kTaskThreads) {
        const int n = e & 63, k2 = (e >> 6) * 2;
        const double2 v = __ldcg(reinterpret_cast<const double2*>(X + n * ld + k2));
        s[k2 * kTP + n] = v.x;
        s[(k2 + 1) * kTP + n] = v.y;
    }
}
// acc (warp tile 32 x 16 at (wm, wn)) += A (64 x 64, staged s[k][m]) * op(B) (staged s[k][n])
__device__ __forceinline__ void tile_mma(double (&acc)[4][2][2], const double* sA, const double* sB, int wm, int wn,
                                         int fr, int fc) {
#pragma unroll 4
    for (int kk = 0; kk < kTT; kk += 4) {
        double af[4], bf[2];
#pragma unroll
        for (int i = 0; i < 4; ++i) af[i] = sA[(kk + fc) * kTP + wm * 32 + i * 8 + fr];
#pragma unroll
        for (int j = 0; j < 2; ++j) bf[j] = sB[(kk + fc) * kTP + wn * 16 + j * 8 + fr];
#pragma unroll
        for (int i = 0; i < 4; ++i)
#pragma unroll
            for (int j = 0; j < 2; ++j) dmma(acc[i][j][0], acc[i][j][1], af[i], bf[j]);
    }
}
__device__ __forceinline__ void zero_acc(double (&acc)[4][2][2]) {
#pragma unroll
    for (int x = 0; x < 4; ++x)
#pragma unroll
        for (int y = 0; y < 2; ++y) acc[x][y][0] = acc[x][y][1] = 0.0;
}
// fragment element (x, y, h) of warp (wm, wn), lane (fr, fc) -> tile row m, column n
#define ABFT_FRAG_MN const int m = wm * 32 + x * 8 + fr, n = wn * 16 + y * 8 + fc * 2 + h
#define ABFT_FRAG_LOOP _Pragma("unroll") for (int x = 0; x < 4; ++x) _Pragma("unroll") for (int y = 0; y < 2; ++y) \
    _Pragma("unroll") for (int h = 0; h < 2; ++h)

// P(b) leaf: Cholesky of the 64 x 64 lower tile held in shared memory Ls (column-major, pitch
// kTP) and its inverse, one CTA of 8 warps, in LDL^T form A = U D U^T (U unit lower, L = U D^1/2):
//  * 8 panels of 8 columns. Panel p is factored with scalar steps (one barrier per column: pivot
//    d_j, U_rj = f_r = a_rj / d_j into Qb, a_rc -= f_r a_cj inside the panel; Ls keeps the
//    unscaled columns), then the trailing lower part takes the rank-8 update
//    A22 -= U_p (D_p U_p^T) = Qb_p Ls_p^T on the tensor cores (DMMA 8x8x4 per 8 x 8 tile) — the
//    blocked right-looking step of PAPER.md:137-176 inside one tile.
//  * inv(U) by 8 x 8 blocks: the 8 diagonal blocks by warp-level forward substitution (shuffles),
//    then block row I = 1..7: Z_IJ = -Z_II sum_{C=J}^{I-1} U_IC Z_CJ (DMMA, one warp per J).
//  * out: inv(L) = D^-1/2 inv(U) -> Xb (zero above the diagonal); Ls keeps the unscaled factor and
//    the pivots' square roots stay in `ls` for leaf_store_L (L = a_rc / sqrt(d_c)), which runs
//    after the dependants have been released (nothing in the task graph reads L_bb).
// Us and Zs are scratch tiles (U, then Z = inv(U)). Returns false on a non-positive
// pivot (NOT_SPD raised with the LAPACK info of the first failing leading minor).
struct LeafSmem {
    double piv_s[kTT], piv_is[kTT];   // sqrt(d), 1 / sqrt(d)
    double tbuf[8][64];
};
__device__ bool leaf_tile(double* Ls, double* Us, double* Zs, LeafSmem& ls, double* Xb, int64_t ldi, int64_t info0,
                          DevState* st, long long* dbg) {
    double* piv_s = ls.piv_s;
    double* piv_is = ls.piv_is;
    const int tid = threadIdx.x, r = tid & 63, g = tid >> 6;
    const int lane = tid & 31, warp = tid >> 5, fr = lane >> 2, fc = lane & 3;
    if (dbg) dbg[0] = clock64();
    __shared__ int s_bad;   // first non-positive pivot + 1 (0: none)
    if (tid == 0) s_bad = 0;
    (void)r; (void)g;
    for (int p = 0; p < 8; ++p) {
        const int c0 = 8 * p;
        __syncthreads();
        // the 8-column panel, by warp 0 alone in registers (lane holds rows lane and lane + 32):
        // no CTA barrier per column step, the pivot and column j's panel rows by shuffles. Same
        // operations per element as a shared-memory step (f = a_rj * rcp(d), a_rc -= f a_cj).
        if (warp == 0) {
            const bool hi = p >= 4;          // rows c0..c0+7 are the lanes' second row (lane + 32)
            double a0[8], a1[8];
#pragma unroll
            for (int c = 0; c < 8; ++c) { a0[c] = Ls[(c0 + c) * kTP + lane]; a1[c] = Ls[(c0 + c) * kTP + lane + 32]; }
            int bad = 0;
#pragma unroll
            for (int j = 0; j < 8; ++j) {
                const int cj = c0 + j;
                const double d = __shfl_sync(0xffffffffu, hi ? a1[j] : a0[j], cj & 31);
                if (!(d > 0.0)) { bad = cj + 1; break; }   // warp-uniform
                const double rd = __drcp_rn(d);
                double acj[8];
#pragma unroll
                for (int c = 0; c < 8; ++c) acj[c] = __shfl_sync(0xffffffffu, hi ? a1[j] : a0[j], (c0 + c) & 31);
                if (lane > cj) {
                    const double f = a0[j] * rd;
                    Us[cj * kTP + lane] = f;
#pragma unroll
                    for (int c = j + 1; c < 8; ++c) a0[c] = fma(-f, acj[c], a0[c]);
                }
                if (lane + 32 > cj) {
                    const double f = a1[j] * rd;
                    Us[cj * kTP + lane + 32] = f;
#pragma unroll
                    for (int c = j + 1; c < 8; ++c) a1[c] = fma(-f, acj[c], a1[c]);
                }
                if (lane == 0) piv_s[cj] = d;
            }
#pragma unroll
            for (int c = 0; c < 8; ++c) { Ls[(c0 + c) * kTP + lane] = a0[c]; Ls[(c0 + c) * kTP + lane + 32] = a1[c]; }
            if (bad && lane == 0) {
                s_bad = bad;
                if (atomicCAS(&st->abort, 0, 1) == 0) { st->status = ABFT_NOT_SPD; st->info = info0 + bad; }
            }
        }
        __syncthreads();
        if (s_bad) return false;
        const int nt = 7 - p;            // trailing 8 x 8 tiles per side
        for (int e = warp; e < nt * (nt + 1) / 2; e += 8) {
            int tj = 0, rem = e;
            while (rem >= nt - tj) { rem -= nt - tj; ++tj; }
            const int m0 = c0 + 8 + 8 * (tj + rem), n0 = c0 + 8 + 8 * tj;
            double* c0p = Ls + (n0 + 2 * fc) * kTP + m0 + fr;
            double v0 = c0p[0], v1 = c0p[kTP];
#pragma unroll
            for (int kq = 0; kq < 8; kq += 4)
                dmma(v0, v1, -Us[(c0 + kq + fc) * kTP + m0 + fr], Ls[(c0 + kq + fc) * kTP + n0 + fr]);
            c0p[0] = v0; c0p[kTP] = v1;
        }
    }
    __syncthreads();
    if (tid < kTT) {
        const double sd = sqrt(piv_s[tid]);
        piv_is[tid] = 1.0 / sd;
        piv_s[tid] = sd;
    }
    if (dbg) dbg[1] = clock64();
    // inv(U): diagonal 8 x 8 blocks, warp w -> block w; lane (zr, cp) holds Z(zr, 2cp + {0,1}).
    {
        const int zr = lane >> 2, cp = lane & 3, b0 = 8 * warp;
        double z0 = (zr == 2 * cp) ? 1.0 : 0.0, z1 = (zr == 2 * cp + 1) ? 1.0 : 0.0;
#pragma unroll
        for (int j = 0; j < 7; ++j) {
            const double zj0 = __shfl_sync(0xffffffffu, z0, j * 4 + cp);
            const double zj1 = __shfl_sync(0xffffffffu, z1, j * 4 + cp);
            if (zr > j) {
                const double u = Us[(b0 + j) * kTP + b0 + zr];
                z0 = fma(-u, zj0, z0);
                z1 = fma(-u, zj1, z1);
            }
        }
        Zs[(b0 + 2 * cp) * kTP + b0 + zr] = z0;
        Zs[(b0 + 2 * cp + 1) * kTP + b0 + zr] = z1;
    }
    if (dbg) dbg[2] = clock64();
    for (int I = 1; I < 8; ++I) {        // block row I: Z_IJ = -Z_II sum_{C=J}^{I-1} U_IC Z_CJ
        __syncthreads();
        if (warp < I) {
            const int J = warp;
            double t0 = 0.0, t1 = 0.0;
            for (int C = J; C < I; ++C) {
#pragma unroll
                for (int kq = 0; kq < 8; kq += 4)
                    dmma(t0, t1, Us[(8 * C + kq + fc) * kTP + 8 * I + fr], Zs[(8 * J + fr) * kTP + 8 * C + kq + fc]);
            }
            double* tb = ls.tbuf[warp];    // T (8 x 8, column-major) as the B operand
            tb[(2 * fc) * 8 + fr] = t0;
            tb[(2 * fc + 1) * 8 + fr] = t1;
            __syncwarp();
            double x0 = 0.0, x1 = 0.0;
#pragma unroll
            for (int kq = 0; kq < 8; kq += 4)
                dmma(x0, x1, -Zs[(8 * I + kq + fc) * kTP + 8 * I + fr], tb[fr * 8 + kq + fc]);
            Zs[(8 * J + 2 * fc) * kTP + 8 * I + fr] = x0;
            Zs[(8 * J + 2 * fc + 1) * kTP + 8 * I + fr] = x1;
            __syncwarp();
        }
    }
    __syncthreads();
    for (int e = tid; e < kTT * kTT; e += kTaskThreads) {   // inv(L) = D^-1/2 inv(U), zero above
        const int c = e >> 6, rr = e & 63;
        Xb[c * ldi + rr] = (c <= rr) ? Zs[c * kTP + rr] * piv_is[rr] : 0.0;
    }
    if (dbg) {
        dbg[3] = clock64();
        if (tid == 0) printf("leaf %lld: factor %lld  inverse-diag %lld  inverse+X-out %lld cycles\n", info0,
                             dbg[1] - dbg[0], dbg[2] - dbg[1], dbg[3] - dbg[2]);
    }
    return true;
}

// L = a_rc / sqrt(d_c) (lower only) from the leaf's unscaled factor in Ls
__device__ __forceinline__ void leaf_store_L(const double* Ls, const LeafSmem& ls, double* Lb, int64_t lda) {
    for (int e = threadIdx.x; e < kTT * kTT; e += kTaskThreads) {
        const int c = e >> 6, rr = e & 63;
        if (c <= rr) Lb[c * lda + rr] = (c == rr) ? ls.piv_s[c] : Ls[c * kTP + rr] * ls.piv_is[c];
    }
}

// Tasks [t_begin, t_end) of the topological order (one launch = the whole graph, or one chunk of
// it: the chunked path splits the graph at step boundaries into short launches, see
// launch_chol_inv); reset_flags: the last chunk's last CTA clears the completion flags.
__global__ void __launch_bounds__(kTaskThreads) k_chol_inv_tasks(double* A, int64_t lda, double* Li, int64_t ldi, int T,
                                                                int t_begin, int t_end, int reset_flags, int64_t info_off,
                                                                uint32_t* sync, DevState* st, unsigned long long* trace) {
    extern __shared__ __align__(16) double tsm[];
    double* sA = tsm;
    double* sB = tsm + kTT * kTP;
    double* sC = tsm + 2 * kTT * kTP;
    __shared__ int s_task, s_go, s_go2;
    __shared__ LeafSmem lsm;
    const int32_t* abort_flag = &st->abort;
    if (cta_aborted(abort_flag)) return;
    uint32_t* next = sync;
    uint32_t* exited = sync + 1;
    uint32_t* fP = sync + 2;
    uint32_t* fS = fP + T;
    uint32_t* fU = fS + T * T;
    uint32_t* fZ = fU + T * T;
    uint32_t* fF = fZ + T * T;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int wm = warp >> 2, wn = warp & 3, fr = lane >> 2, fc = lane & 3;
    auto At = [&](int I, int J) { return A + (int64_t)J * kTT * lda + I * kTT; };     // tile (I, J) of the block
    auto Xt = [&](int I, int J) { return Li + (int64_t)J * kTT * ldi + I * kTT; };    // tile (I, J) of inv(L)
    for (;;) {
        __syncthreads();
        if (tid == 0) s_task = t_begin + (int)atomicAdd(next, 1u);
        __syncthreads();
        const int t = s_task;
        if (t >= t_end) break;
        int type, i, j, b;
        decode_task(T, t, type, i, j, b);
        unsigned long long t0 = 0, t1 = 0;
        if (trace && tid == 0) asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
        if (tid == 0) {
            bool ok = true;
            switch (type) {
                case TK_P:   // tiles (b, b-1), (b, b) updated through step b-2 (X_{b-1} is awaited below)
                    if (b > 1) ok = wait_ge(&fU[b * T + b - 1], (uint32_t)(b - 1), abort_flag) &&
                                    wait_ge(&fU[b * T + b], (uint32_t)(b - 1), abort_flag);
                    break;
                case TK_S:
                    ok = wait_ge(&fP[j], 1u, abort_flag);
                    if (ok && j > 0) ok = wait_ge(&fU[i * T + j], (uint32_t)j, abort_flag);
                    break;
                case TK_U:
                    ok = wait_ge(&fS[i * T + b], 1u, abort_flag) && wait_ge(&fS[j * T + b], 1u, abort_flag);
                    if (ok && b > 0) ok = wait_ge(&fU[i * T + j], (uint32_t)b, abort_flag);
                    break;
                case TK_Z:
                    ok = wait_ge(&fS[i * T + b], 1u, abort_flag) &&
                         wait_ge(b == j ? &fP[b] : &fF[b * T + j], 1u, abort_flag);
                    if (ok && b > j) ok = wait_ge(&fZ[i * T + j], (uint32_t)(b - j), abort_flag);
                    break;
                default:   // F(i, j)
                    ok = wait_ge(&fP[i], 1u, abort_flag) && wait_ge(&fZ[i * T + j], (uint32_t)(i - j), abort_flag);
                    break;
            }
            s_go = ok;
            if (trace) asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t1));
        }
        __syncthreads();
        if (!s_go) break;
        uint32_t* flag = nullptr;
        uint32_t fval = 1;
        double acc[4][2][2], cv[4][2][2];
        zero_acc(acc);
        if (type == TK_P) {
            if (b == 0) {   // the lower half of the first diagonal tile into shared memory
                const double* src = At(0, 0);
                for (int e = tid; e < kTT * kTT; e += kTaskThreads) {
                    const int c = e >> 6, rr = e & 63;
                    if (c <= rr) sB[c * kTP + rr] = src[(int64_t)c * lda + rr];
                }
            } else {
                // L_{b,b-1} = A_{b,b-1} X_{b-1,b-1}^T  (published for the other tasks of step b-1)
                // operands that are final already are fetched while the previous leaf finishes
                double* Cs = At(b, b - 1);
                tile_load_T(sA, Cs, lda);
                ABFT_FRAG_LOOP { ABFT_FRAG_MN; cv[x][y][h] = (m >= n) ? __ldcg(At(b, b) + (int64_t)n * lda + m) : 0.0; }
                if (tid == 0) s_go2 = wait_ge(&fP[b - 1], 1u, abort_flag);   // (s_go may still be read)
                __syncthreads();
                if (!s_go2) { cpa_wait_all(); break; }
                tile_load_T(sB, Xt(b - 1, b - 1), ldi);
                cpa_wait_all();
                __syncthreads();
                tile_mma(acc, sA, sB, wm, wn, fr, fc);
                __syncthreads();
                ABFT_FRAG_LOOP { ABFT_FRAG_MN; Cs[(int64_t)n * lda + m] = acc[x][y][h]; sA[n * kTP + m] = acc[x][y][h]; }
                __syncthreads();
                if (tid == 0 && gridDim.x > 1) { __threadfence(); st_release(&fS[b * T + b - 1], 1u); }
                // A_bb -= L_{b,b-1} L_{b,b-1}^T into shared memory (the leaf's input)
                zero_acc(acc);
                tile_mma(acc, sA, sA, wm, wn, fr, fc);
                ABFT_FRAG_LOOP { ABFT_FRAG_MN; sB[n * kTP + m] = cv[x][y][h] - acc[x][y][h]; }
            }
            __syncthreads();
            __shared__ long long dbg[4];
            if (!leaf_tile(sB, sA, sC, lsm, Xt(b, b), ldi, info_off + b * kTT, st, trace ? dbg : nullptr)) break;
            __syncthreads();   // X_bb is out: release the dependants, then store L_bb (nobody here reads it)
            if (tid == 0 && gridDim.x > 1) { __threadfence(); st_release(&fP[b], 1u); }
            leaf_store_L(sB, lsm, At(b, b), lda);
        } else if (type == TK_S || type == TK_U || type == TK_Z) {
            double* C;
            bool add = true, lower = false;
            if (type == TK_S) {          // L_ib = A_ib X_bb^T, in place (the tile is staged first)
                C = At(i, j);
                tile_load_T(sA, C, lda);
                tile_load_T(sB, Xt(j, j), ldi);
                flag = &fS[i * T + j];
                add = false;
            } else if (type == TK_U) {   // A_ij -= L_ib L_jb^T
                C = At(i, j);
                tile_load_T(sA, At(i, b), lda);
                tile_load_T(sB, At(j, b), lda);
                flag = &fU[i * T + j];
                fval = (uint32_t)(b + 1);
                lower = (i == j);
            } else {                     // Y_ij (+)= L_ib X_bj
                C = Xt(i, j);
                tile_load_T(sA, At(i, b), lda);
                tile_load_N(sB, Xt(b, j), ldi);
                flag = &fZ[i * T + j];
                fval = (uint32_t)(b - j + 1);
                add = (b > j);
            }
            const int64_t ldc = (type == TK_Z) ? ldi : lda;
            if (add) { ABFT_FRAG_LOOP { ABFT_FRAG_MN; cv[x][y][h] = (!lower || m >= n) ? __ldcg(C + (int64_t)n * ldc + m) : 0.0; } }
            cpa_wait_all();
            __syncthreads();
            tile_mma(acc, sA, sB, wm, wn, fr, fc);
            ABFT_FRAG_LOOP {
                ABFT_FRAG_MN;
                if (type == TK_U) { if (!lower || m >= n) C[(int64_t)n * ldc + m] = cv[x][y][h] - acc[x][y][h]; }
                else C[(int64_t)n * ldc + m] = add ? cv[x][y][h] + acc[x][y][h] : acc[x][y][h];
            }
        } else {   // F(i, j): X_ij = -X_ii Y_ij, and the zero tile (j, i) of inv(L)
            tile_load_T(sA, Xt(i, i), ldi);
            tile_load_N(sB, Xt(i, j), ldi);
            cpa_wait_all();
            __syncthreads();
            tile_mma(acc, sA, sB, wm, wn, fr, fc);
            double* Xij = Xt(i, j);
            double* Xji = Xt(j, i);
            ABFT_FRAG_LOOP { ABFT_FRAG_MN; Xij[(int64_t)n * ldi + m] = -acc[x][y][h]; Xji[(int64_t)n * ldi + m] = 0.0; }
            flag = &fF[i * T + j];
        }
        __syncthreads();
        if (tid == 0 && flag && gridDim.x > 1) { __threadfence(); st_release(flag, fval); }
        if (trace && tid == 0) {   // diagnostics (abft_dev_chol_trace): who ran what, when
            unsigned long long t2, smid;
            asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t2));
            asm volatile("{ .reg .u32 r; mov.u32 r, %%smid; cvt.u64.u32 %0, r; }" : "=l"(smid));
            trace[4 * t + 0] = (unsigned long long)type | ((unsigned long long)i << 8) | ((unsigned long long)j << 16) |
                               ((unsigned long long)b << 24) | (smid << 32) | ((unsigned long long)blockIdx.x << 48);
            trace[4 * t + 1] = t0; trace[4 * t + 2] = t1; trace[4 * t + 3] = t2;
        }
    }
    // exit: the last CTA out resets the sync area for the next launch
    __syncthreads();
    if (tid == 0) {
        __threadfence();
        s_go = (atomicAdd(exited, 1u) == gridDim.x - 1);
    }
    __syncthreads();
    if (s_go) {
        __threadfence();
        const int words = reset_flags ? task_sync_words(T) : 2;   // counters always, flags at the end
        for (int e = tid; e < words; e += kTaskThreads) sync[e] = 0u;
    }
}

// The recursive path's 64 x 64 leaf with the blocked DMMA leaf routine (one short launch, 8
// warps): lower half of T -> shared memory, factor + inverse (leaf_tile), L back into T.
__global__ void __launch_bounds__(kTaskThreads) k_leaf64_blocked(double* T, int64_t ldt, double* Li, int64_t ldi,
                                                                 int64_t info_off, DevState* st) {
    if (cta_aborted(&st->abort)) return;
    extern __shared__ __align__(16) double lsm_dyn[];
    double* Ls = lsm_dyn;
    double* Us = lsm_dyn + kTT * kTP;
    double* Zs = lsm_dyn + 2 * kTT * kTP;
    __shared__ LeafSmem lsm;
    for (int e = threadIdx.x; e < kTT * kTT; e += kTaskThreads) {
        const int c = e >> 6, rr = e & 63;
        if (c <= rr) Ls[c * kTP + rr] = T[(int64_t)c * ldt + rr];
    }
    __syncthreads();
    if (!leaf_tile(Ls, Us, Zs, lsm, Li, ldi, info_off, st, nullptr)) return;
    __syncthreads();
    leaf_store_L(Ls, lsm, T, ldt);
}

}  // namespace abft

using namespace abft;

size_t chol_sync_bytes(int64_t nb) {   // <= the scratch `tmp` callers allocate ((nb/2 + 64)^2 doubles)
    const int64_t T = std::max<int64_t>(1, std::min<int64_t>(nb / kTT, 32));
    return sizeof(uint32_t) * (size_t)task_sync_words((int)T);
}

static thread_local unsigned long long* g_chol_trace = nullptr;   // abft_dev_chol_trace only
void chol_set_trace(unsigned long long* t) { g_chol_trace = t; }
int chol_task_count(int64_t nb) { return (nb % kTT == 0 && nb / kTT <= 32) ? task_count((int)(nb / kTT)) : 0; }

// Path choice. Default: the one-launch task graph (nb % 64 == 0, nb >= 128, 16-byte aligned, even
// leading dimension; about 3x faster than the recursive path on its own). ABFT_CHOL=recursive
// selects the recursive multi-launch path. (Until the update kernel's consumer proxy fence, the
// task graph's long-lived high-priority CTAs exposed a stage-release race in the bulk-copy update
// pipeline, so it was opt-in: profiles/r02/race_r02.md.) Read per call (tests switch
// paths inside one process).
static bool use_tasks(const double* T, int64_t ldt, int64_t B) {
    const char* e = getenv("ABFT_CHOL");
    return (!(e && !strcmp(e, "recursive")) || g_chol_trace != nullptr) && B % kTT == 0 && B >= 2 * kTT && B / kTT <= 32 && ((uintptr_t)T & 15) == 0 && ldt % 2 == 0;
}

int launch_copy(int64_t rows, int64_t cols, const double* src, int64_t lds, double* dst, int64_t ldd,
                const int32_t* abort_flag, cudaStream_t s) {
    if (rows <= 0 || cols <= 0) return 0;
    const int vec = (((uintptr_t)src | (uintptr_t)dst) & 15) == 0 && lds % 2 == 0 && ldd % 2 == 0;
    const int64_t per = vec ? 512 : 256;                       // rows one CTA covers per pass
    const int64_t bx = std::min<int64_t>((rows + per - 1) / per, 64);
    const int64_t by = std::min<int64_t>(cols, std::max<int64_t>(1, 148 * 8 / bx));
    k_copy_block<<<dim3((unsigned)bx, (unsigned)by), 256, 0, s>>>(rows, cols, src, lds, dst, ldd, abort_flag, vec);
    abft_count_launch();
    return 0;
}

int launch_zero(int64_t rows, int64_t cols, double* dst, int64_t ldd, cudaStream_t s) {
    if (rows <= 0 || cols <= 0) return 0;
    const int64_t total = rows * cols;
    const int64_t blocks = std::min<int64_t>((total + 255) / 256, 148 * 16);
    k_zero_block<<<(unsigned)blocks, 256, 0, s>>>(rows, cols, dst, ldd);
    abft_count_launch();
    return 0;
}

// 64 x 64 leaves of the recursive path: the blocked DMMA leaf (default) or the one-barrier-per-
// column shared-memory leaf (ABFT_LEAF=scalar; also every leaf narrower than 64).
static bool blocked_leaf() {
    const char* e = getenv("ABFT_LEAF");
    return !(e && !strcmp(e, "scalar"));
}

// Recursive factorisation of the diagonal block [off, off+sz) of the B x B tile T (ldt) with
// its inverse into Li (ld = B). tmp: >= (B/2)^2 doubles of scratch.
static void chol_inv_rec(double* T, int64_t ldt, double* Li, int64_t ldi, int64_t off, int64_t sz,
                         int64_t info_off, double* tmp, DevState* st, cudaStream_t s) {
    const int32_t* ab = &st->abort;
    if (sz == kTT && blocked_leaf()) {
        static bool attr64 = false;
        if (!attr64) {
            cudaFuncSetAttribute(k_leaf64_blocked, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kTaskSmem);
            attr64 = true;
        }
        k_leaf64_blocked<<<1, kTaskThreads, kTaskSmem, s>>>(T + off * ldt + off, ldt, Li + off * ldi + off, ldi,
                                                          info_off + off, st);
        abft_count_launch();
        return;
    }
    if (sz <= kLeaf) {
        static bool attr = false;
        const int smem = 2 * kLeaf * (kLeaf + 1) * (int)sizeof(double);
        if (!attr) { cudaFuncSetAttribute(k_leaf_potrf_inv, cudaFuncAttributeMaxDynamicSharedMemorySize, smem); attr = true; }
        k_leaf_potrf_inv<<<1, kLeafThreads, smem, s>>>(T + off * ldt + off, ldt, Li + off * ldi + off, ldi, (int)sz,
                                           info_off + off, st);
        abft_count_launch();
        return;
    }
    // split at a multiple of the leaf size, first half >= second half
    int64_t s1 = ((sz / 2 + kLeaf - 1) / kLeaf) * kLeaf;
    if (s1 >= sz) s1 = sz - kLeaf;
    const int64_t s2 = sz - s1;
    double* A11 = T + off * ldt + off;
    double* A21 = A11 + s1;
    double* A22 = A21 + s1 * ldt;
    double* I11 = Li + off * ldi + off;
    double* I21 = I11 + s1;
    double* I22 = I21 + s1 * ldi;
    chol_inv_rec(T, ldt, Li, ldi, off, s1, info_off, tmp, st, s);
    // L21 = A21 inv11^T  (NT; inv11 lower -> k <= n)
    launch_gemm(s2, s1, s1, A21, ldt, I11, ldi, tmp, s2, 1.0, 0.0, true, 0, 1, 0, 0, 0, ab, s);
    launch_copy(s2, s1, tmp, s2, A21, ldt, ab, s);
    // A22 -= L21 L21^T  (lower)
    launch_gemm(s2, s2, s1, A21, ldt, A21, ldt, A22, ldt, -1.0, 1.0, true, 1, 0, 0, 0, 0, ab, s);
    chol_inv_rec(T, ldt, Li, ldi, off + s1, s2, info_off, tmp, st, s);
    // inv21 = -inv22 (L21 inv11)
    launch_gemm(s2, s1, s1, A21, ldt, I11, ldi, tmp, s2, 1.0, 0.0, false, 0, 2, 0, 0, 0, ab, s);
    launch_gemm(s2, s1, s2, I22, ldi, tmp, s2, I21, ldi, -1.0, 0.0, false, 0, 3, 0, 0, 0, ab, s);
}

// Factor the B x B diagonal tile at T and produce inv(L) in Li (B x B, ld B, upper zeroed).
int launch_chol_inv(double* T, int64_t ldt, double* Li, int64_t B, int64_t info_off, double* tmp,
                    DevState* st, cudaStream_t s) {
    if (use_tasks(T, ldt, B)) {
        static bool attr = false;
        if (!attr) {
            cudaFuncSetAttribute(k_chol_inv_tasks, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kTaskSmem);
            attr = true;
        }
        static int gmax = -1;
        if (gmax < 0) { const char* e = getenv("ABFT_CHOL_G"); gmax = e ? std::max(1, atoi(e)) : 10; }
        const int Tt = (int)(B / kTT), nt = task_count(Tt);
        // ABFT_CHOL_CHUNKS = c > 1: the graph split at step boundaries into c short launches
        // (long-lived high-priority CTAs are what the bulk-copy update pipeline does not survive,
        // profiles/r02/race_r02.md); 1 (default): one launch
        const char* ce = getenv("ABFT_CHOL_CHUNKS");
        const int chunks = std::max(1, std::min(ce ? atoi(ce) : 1, Tt));
        std::vector<int> cut(1, 0);
        {
            int t = 1;   // after P(0)
            for (int b = 0; b < Tt; ++b) {
                t += task_step_count(Tt, b);
                if ((int)cut.size() < chunks && (b + 1) * chunks / Tt >= (int)cut.size() && t < nt) cut.push_back(t);
            }
            cut.push_back(nt);
        }
        for (size_t c = 0; c + 1 < cut.size(); ++c) {
            const int cnt = cut[c + 1] - cut[c];
            if (cnt <= 0) continue;
            const int grid = std::min(cnt, gmax);
            k_chol_inv_tasks<<<grid, kTaskThreads, kTaskSmem, s>>>(T, ldt, Li, B, Tt, cut[c], cut[c + 1],
                                                                   c + 2 == cut.size() ? 1 : 0, info_off,
                                                                   reinterpret_cast<uint32_t*>(tmp), st, g_chol_trace);
            abft_count_launch();
        }
        return 0;
    }
    launch_zero(B, B, Li, B, s);
    chol_inv_rec(T, ldt, Li, B, 0, B, info_off, tmp, st, s);
    return 0;
}
