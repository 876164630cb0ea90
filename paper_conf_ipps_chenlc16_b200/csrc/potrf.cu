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

#include <algorithm>


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
    if (st->abort) return;
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

__global__ void k_copy_block(int64_t rows, int64_t cols, const double* src, int64_t lds, double* dst,
                             int64_t ldd, const int32_t* abort_flag) {
    if (*abort_flag) return;
    const int64_t total = rows * cols;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
        const int64_t c = i / rows, r = i % rows;
        dst[c * ldd + r] = src[c * lds + r];
    }
}

__global__ void k_zero_block(int64_t rows, int64_t cols, double* dst, int64_t ldd) {
    const int64_t total = rows * cols;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
        const int64_t c = i / rows, r = i % rows;
        dst[c * ldd + r] = 0.0;
    }
}

}  // namespace abft

using namespace abft;

int launch_copy(int64_t rows, int64_t cols, const double* src, int64_t lds, double* dst, int64_t ldd,
                const int32_t* abort_flag, cudaStream_t s) {
    if (rows <= 0 || cols <= 0) return 0;
    const int64_t total = rows * cols;
    const int64_t blocks = std::min<int64_t>((total + 255) / 256, 148 * 16);
    k_copy_block<<<(unsigned)blocks, 256, 0, s>>>(rows, cols, src, lds, dst, ldd, abort_flag);
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

// Recursive factorisation of the diagonal block [off, off+sz) of the B x B tile T (ldt) with
// its inverse into Li (ld = B). tmp: >= (B/2)^2 doubles of scratch.
static void chol_inv_rec(double* T, int64_t ldt, double* Li, int64_t ldi, int64_t off, int64_t sz,
                         int64_t info_off, double* tmp, DevState* st, cudaStream_t s) {
    const int32_t* ab = &st->abort;
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
    launch_zero(B, B, Li, B, s);
    chol_inv_rec(T, ldt, Li, B, 0, B, info_off, tmp, st, s);
    return 0;
}
