// util.cu — synthetic SPD generator (reading A15, the same counter-based generator as the
// Python module synthetic/, implemented independently here) and the fault-injection kernel.
#include "common.cuh"

#include <algorithm>

namespace abft {

__device__ __forceinline__ uint64_t splitmix64(uint64_t x) {
    uint64_t z = x + 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

// A[i,j] = A[j,i] = U(key(max, min)), A[i,i] += n; full matrix written, columns coalesced.
__global__ void k_gen_spd(int64_t n, uint64_t seed, double* A, int64_t lda) {
    const uint64_t nn = (uint64_t)n;
    const uint64_t base = seed * nn * nn;
    const int64_t total = n * n;
    for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < total; t += (int64_t)gridDim.x * blockDim.x) {
        const int64_t j = t / n, i = t % n;
        const uint64_t hi = (uint64_t)(i > j ? i : j), lo = (uint64_t)(i > j ? j : i);
        const uint64_t z = splitmix64(base + hi * nn + lo);
        double u = (double)(z >> 11) * 0x1p-53;
        if (i == j) u += (double)n;
        A[j * lda + i] = u;
    }
}

struct InjOp { double* p; uint64_t mask; };
struct InjBatch { int n; InjOp op[16]; };

// XOR masks into stored doubles (the harness of PAPER.md:383-385). Stream-ordered between
// the producing kernel and the next check; skipped after an abort.
__global__ void k_inject(InjBatch b, const int32_t* abort_flag) {
    if (*abort_flag) return;
    if (threadIdx.x != 0) return;
    for (int i = 0; i < b.n; ++i) {   // sequential: two specs may hit the same element
        unsigned long long* p = reinterpret_cast<unsigned long long*>(b.op[i].p);
        *p ^= (unsigned long long)b.op[i].mask;
    }
}

__global__ void k_axpy1(int64_t n, const double* x, double* y) {   // y += x
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        y[i] += x[i];
}
__global__ void k_abort_to_slot(const int32_t* abort_flag, double* slot) { *slot = (double)*abort_flag; }
__global__ void k_abort_from_slot(const double* slot, DevState* st) {
    if (*slot != 0.0 && st->abort == 0) st->abort = 1;   // the owner aborted: stop this rank too
}

// Fused write-back + push (NEXT-3): one read of W per element; local stores (A panel / chk) and
// one peer store per receiving rank (P2P over NVLink when the peer is another GPU). The abort slot
// `slot` after the panel travels with it. Column c of W is blockIdx.y; rows in 16-byte pairs.
// 2D block-cyclic (rmod > 1): only this rank's rows move — data row r (block r / B) iff
// (r / B) % rmod == dphase, checksum row q = r - mB (block q / 2) iff (q / 2) % rmod == cphase.
struct PeerList { double* p[16]; int n, pad; };
__global__ void k_panel_out(const double* W, int64_t ldw, int64_t mB, int64_t rows, int64_t B, double* Ap,
                            int64_t lda, double* ck, int64_t ldc, PeerList peers, int64_t rmod, int64_t dphase,
                            int64_t cphase, int slot, const int32_t* abort_flag) {
    const int64_t c = blockIdx.y;
    const double* col = W + c * ldw;
    // after an abort only the abort slot travels (the receivers stop on it)
    const int64_t rows_live = *(volatile const int32_t*)abort_flag ? 0 : rows;
    for (int64_t r = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) * 2; r < rows_live; r += (int64_t)gridDim.x * blockDim.x * 2) {
        if (rmod > 1 && (r < mB ? (r / B) % rmod != dphase : ((r - mB) / 2) % rmod != cphase)) continue;
        const double2 v = *reinterpret_cast<const double2*>(col + r);   // ldw, mB even: pairs never straddle
        for (int q = 0; q < peers.n; ++q) *reinterpret_cast<double2*>(peers.p[q] + c * ldw + r) = v;
        if (r < mB) { Ap[c * lda + r] = v.x; Ap[c * lda + r + 1] = v.y; }   // mB even
        else { ck[c * ldc + (r - mB)] = v.x; if (r + 1 < rows) ck[c * ldc + (r + 1 - mB)] = v.y; }
    }
    if (c == 0 && blockIdx.x == 0 && threadIdx.x == 0) {   // abort slot at W[ldw * B + slot]
        const double v = W[ldw * B + slot];
        for (int q = 0; q < peers.n; ++q) peers.p[q][ldw * B + slot] = v;
    }
}

}  // namespace abft

using namespace abft;

int launch_panel_out(const double* W, int64_t ldw, int64_t mB, int64_t ncrows, int64_t B, double* Apanel,
                     int64_t lda, double* chk, int64_t ldc, double* const* peers, int npeer, const int32_t* abort_flag,
                     cudaStream_t s, int64_t rmod, int64_t dphase, int64_t cphase, int slot) {
    PeerList pl;
    pl.n = 0;
    if (npeer > 16) return -1;
    for (int q = 0; q < npeer; ++q) pl.p[pl.n++] = peers[q];
    const int64_t rows = mB + ncrows;
    const int64_t bx = std::min<int64_t>(std::max<int64_t>((rows / 2 + 255) / 256, 1), 32);
    k_panel_out<<<dim3((unsigned)bx, (unsigned)B), 256, 0, s>>>(W, ldw, mB, rows, B, Apanel, lda, chk, ldc, pl,
                                                               rmod < 1 ? 1 : rmod, dphase, cphase, slot, abort_flag);
    abft_count_launch();
    return 0;
}

int launch_axpy(int64_t n, const double* x, double* y, cudaStream_t s) {
    if (n <= 0) return 0;
    k_axpy1<<<(unsigned)std::min<int64_t>((n + 255) / 256, 1024), 256, 0, s>>>(n, x, y);
    abft_count_launch();
    return 0;
}
int launch_abort_to_slot(const int32_t* abort_flag, double* slot, cudaStream_t s) {
    k_abort_to_slot<<<1, 1, 0, s>>>(abort_flag, slot); abft_count_launch(); return 0;
}
int launch_abort_from_slot(const double* slot, DevState* st, cudaStream_t s) {
    k_abort_from_slot<<<1, 1, 0, s>>>(slot, st); abft_count_launch(); return 0;
}

int launch_gen_spd(int64_t n, uint64_t seed, double* A, int64_t lda, cudaStream_t s) {
    if (n == 0) return 0;
    const int64_t total = n * n;
    const int64_t blocks = std::min<int64_t>((total + 255) / 256, 148 * 32);
    k_gen_spd<<<(unsigned)blocks, 256, 0, s>>>(n, seed, A, lda);
    abft_count_launch();
    return 0;
}

int launch_inject(int nops, double* const* ptrs, const uint64_t* masks, const int32_t* abort_flag,
                  cudaStream_t s) {
    for (int base = 0; base < nops; base += 16) {
        InjBatch b;
        b.n = std::min(16, nops - base);
        for (int i = 0; i < b.n; ++i) { b.op[i].p = ptrs[base + i]; b.op[i].mask = masks[base + i]; }
        k_inject<<<1, 32, 0, s>>>(b, abort_flag);
        abft_count_launch();
    }
    return 0;
}
