// check.cu — checksum encoding, recalculation (phase 1) and detect/locate/correct (phase 2).
//
// PAPER.md:121-129 (§IV.A encoding), :180-195 (§IV.C detection / location / correction),
// with the readings A4-A12 of DESIGN.md §3. The paper's checksum recalculation is a set of
// BLAS-2 dgemv calls spread over N CUDA streams (Opt. 1); here one
// bandwidth-bound launch covers every tile of a check stage: one warp per tile column,
// coalesced column loads and warp-shuffle reductions (the mirrored half of an unfactored
// diagonal tile is read row-wise, also coalesced).
#include <algorithm>
#include <cstdlib>

#include "common.cuh"

namespace abft {

constexpr int kChkThreads = 256;  // 8 warps
constexpr int kChkCols = 32;      // tile columns per CTA (4 per warp; the mirrored half of a diagonal tile: 8 row groups)

__device__ __forceinline__ double warp_sum(double v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    return v;
}

// Noise bookkeeping: the largest |d|/tau of a passing column (positive doubles order as their
// bit patterns, so an integer atomicMax keeps the maximum).
__device__ __forceinline__ void note_ratio(DevState* st, double q) {
    q = fmax(q, __shfl_xor_sync(0xffffffffu, q, 16));
    q = fmax(q, __shfl_xor_sync(0xffffffffu, q, 8));
    q = fmax(q, __shfl_xor_sync(0xffffffffu, q, 4));
    q = fmax(q, __shfl_xor_sync(0xffffffffu, q, 2));
    q = fmax(q, __shfl_xor_sync(0xffffffffu, q, 1));
    // one atomic per warp at most, and only when it raises the maximum (the common fault-free case
    // reads the current value and skips the atomic: thousands of warps per launch hit one address)
    if ((threadIdx.x & 31) == 0 && q > 0.0) {
        const unsigned long long b = (unsigned long long)__double_as_longlong(q);
        if (b > __ldcg(&st->max_ratio_bits)) atomicMax(&st->max_ratio_bits, b);
    }
}

// Compare a recalculated column with its stored checksums, flag it if |d| > tau or d is
// non-finite (P:195 + A5). Called by every thread of the CTA (inactive threads pass ok = false).
__device__ __forceinline__ void compare_column(const StageArgs& a, int part, const TileView& v, int64_t I, int64_t J,
                                               int64_t c, double r1, double r2, double r3, bool ok) {
    double q = 0.0;
    if (ok) {
        const double d1 = __dsub_rn(r1, v.c1[c * v.ldc]);
        const double d2 = __dsub_rn(r2, v.c2[c * v.ldc]);
        const double d3 = v.c3 ? __dsub_rn(r3, v.c3[c * v.ldc]) : 0.0;
        double tau1, tau2, tau3;
        thresholds(a, I, J * a.nb + c, v.factored, tau1, tau2, tau3);
        const bool f1 = !dfinite(d1) || fabs(d1) > tau1;
        const bool f2 = !dfinite(d2) || fabs(d2) > tau2;
        const bool f3 = v.c3 && (!dfinite(d3) || fabs(d3) > tau3);
        if (f1 || f2 || f3) {
            FlagList& FL = a.st->fl[a.flist];
            const int slot = atomicAdd(&FL.nflag, 1);
            if (slot >= kFlagCap) FL.overflow = 1;
            else {
                Flag& f = FL.flags[slot];
                f.I = (int32_t)I; f.J = (int32_t)J; f.c = (int32_t)c; f.part = part;
                f.d1 = d1; f.d2 = d2; f.r1 = r1; f.r2 = r2; f.d3 = d3; f.r3 = r3;
            }
        } else {
            q = fmax(fabs(d1) / tau1, fabs(d2) / tau2);
            if (v.c3) q = fmax(q, fabs(d3) / tau3);
        }
    }
    note_ratio(a.st, q);
}

// Phase 1, re-read: recompute r1 = v1^T X[:,c], r2 = v2^T X[:,c] for kChkCols columns of one tile
// of the stage (block `bid` of this part). encode = 1: store them as the checksums. One warp per
// column: coalesced loads (16-byte when the column is 16-byte aligned), shuffle reductions; the
// mirrored half of an unfactored diagonal tile is read row-wise (also coalesced).
__device__ void phase1_reread(const StageArgs& a, int part, int64_t bid) {
    const int64_t B = a.nb;
    const int64_t chunks = (B + kChkCols - 1) / kChkCols;
    const int64_t t = bid / chunks;
    const int64_t c0 = (bid % chunks) * kChkCols;
    int64_t I, J;
    stage_tile(a, t, I, J);
    const bool mine = tile_mine(a, I, J);   // dist: this rank's tile (CTA-uniform)
    const TileView v = stage_view(a, I, J);
    const int cw = (int)((B - c0) < kChkCols ? (B - c0) : kChkCols);
    __shared__ double s_r1[kChkCols], s_r2[kChkCols], s_r3[kChkCols];
    __shared__ double s_m1[kChkThreads], s_m2[kChkThreads], s_m3[kChkThreads];
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (mine) {
        for (int cc = warp; cc < cw; cc += kChkThreads / 32) {
            const int64_t c = c0 + cc;
            const double* col = v.T + c * v.ldt;
            const int64_t rbeg = v.diag ? c : 0;
            double r1 = 0.0, r2 = 0.0, r3 = 0.0;
            if (!v.diag && ((((uintptr_t)col) & 15) == 0) && (B % 2 == 0)) {
                const double2* col2 = reinterpret_cast<const double2*>(col);
#pragma unroll 4
                for (int64_t h = lane; h < B / 2; h += 32) {
                    const double2 x = col2[h];
                    const double w0 = (double)(2 * h + 1), w1 = (double)(2 * h + 2);
                    r1 += x.x; r1 += x.y;
                    r2 = fma(w0, x.x, r2);
                    r2 = fma(w1, x.y, r2);
                    if (v.c3) { r3 = fma(w0 * w0, x.x, r3); r3 = fma(w1 * w1, x.y, r3); }
                }
            } else {
#pragma unroll 4
                for (int64_t r = rbeg + lane; r < B; r += 32) {
                    const double x = col[r];
                    const double w = (double)(r + 1);
                    r1 += x;
                    r2 = fma(w, x, r2);
                    if (v.c3) r3 = fma(w * w, x, r3);
                }
            }
            r1 = warp_sum(r1);
            r2 = warp_sum(r2);
            if (v.c3) r3 = warp_sum(r3);
            if (lane == 0) { s_r1[cc] = r1; s_r2[cc] = r2; s_r3[cc] = r3; }
        }
    }
    // mirrored part of an unfactored diagonal tile: X[r,c] = T[c,r] for r < c (row c of T)
    if (mine && v.diag && !v.factored) {
        const int ngroups = kChkThreads / kChkCols;
        const int cc = threadIdx.x % kChkCols, grp = threadIdx.x / kChkCols;
        double m1 = 0.0, m2 = 0.0, m3 = 0.0;
        if (cc < cw) {
            const int64_t c = c0 + cc;
#pragma unroll 8
            for (int64_t r = grp; r < c; r += ngroups) {
                const double x = v.T[r * v.ldt + c];
                const double w = (double)(r + 1);
                m1 += x;
                m2 = fma(w, x, m2);
                if (v.c3) m3 = fma(w * w, x, m3);
            }
        }
        s_m1[threadIdx.x] = m1; s_m2[threadIdx.x] = m2; s_m3[threadIdx.x] = m3;
        __syncthreads();
        if (threadIdx.x < cw) {
            double a1 = 0.0, a2 = 0.0, a3 = 0.0;
            for (int g = 0; g < ngroups; ++g) {
                a1 += s_m1[g * kChkCols + threadIdx.x]; a2 += s_m2[g * kChkCols + threadIdx.x];
                a3 += s_m3[g * kChkCols + threadIdx.x];
            }
            s_r1[threadIdx.x] += a1; s_r2[threadIdx.x] += a2; s_r3[threadIdx.x] += a3;
        }
    }
    __syncthreads();
    if (!mine) return;   // CTA-uniform
    if (threadIdx.x == 0 && c0 == 0 && !a.encode) atomicAdd(&a.st->n_checks, 1ull);
    const bool act = threadIdx.x < cw;
    const int64_t c = c0 + threadIdx.x;
    const double r1 = act ? s_r1[threadIdx.x] : 0.0, r2 = act ? s_r2[threadIdx.x] : 0.0;
    const double r3 = act ? s_r3[threadIdx.x] : 0.0;
    if (a.encode) {
        if (act) { v.c1[c * v.ldc] = r1; v.c2[c * v.ldc] = r2; if (v.c3) v.c3[c * v.ldc] = r3; }
        return;
    }
    compare_column(a, part, v, I, J, c, r1, r2, r3, act);
}

// Phase 1 of V5 for off-diagonal trailing tiles from the partial sums the update GEMM left
// behind (SK_TRAIL_OFF): r1 = sum of the tile's slab partials, r2 likewise. One thread per column.
__device__ void phase1_fused(const StageArgs& a, int part, int64_t bid) {
    const int64_t B = a.nb;
    const int64_t chunks = (B + kChkThreads - 1) / kChkThreads;
    const int64_t t = bid / chunks;
    const int64_t c = (bid % chunks) * kChkThreads + threadIdx.x;
    int64_t I, J;
    stage_tile(a, t, I, J);
    if (!tile_mine(a, I, J)) return;   // CTA-uniform
    if (threadIdx.x == 0 && c == 0) atomicAdd(&a.st->n_checks, 1ull);
    const bool act = c < B;
    const TileView v = stage_view(a, I, J);
    double r1 = 0.0, r2 = 0.0, r3 = 0.0;
    if (act) {
        // the slab partials of the column are loaded 8 at a time before they are summed (in slab
        // order): the loads are independent, so a batch is in flight at once, not one per latency
        const int64_t g = local_col(a, J) + c, s0 = I * B / a.cs_slab_rows, ns = B / a.cs_slab_rows;
        const double* b1 = a.cs + s0 * a.cs_ld + g;
        const double* b2 = a.cs + (a.cs_nslab + s0) * a.cs_ld + g;
        const double* b3 = a.cs + (2 * a.cs_nslab + s0) * a.cs_ld + g;
        for (int64_t q0 = 0; q0 < ns; q0 += 8) {
            double p1[8], p2[8], p3[8];
#pragma unroll
            for (int q = 0; q < 8; ++q) {
                const bool in = q0 + q < ns;
                p1[q] = in ? b1[(q0 + q) * a.cs_ld] : 0.0;
                p2[q] = in ? b2[(q0 + q) * a.cs_ld] : 0.0;
                p3[q] = (in && v.c3) ? b3[(q0 + q) * a.cs_ld] : 0.0;
            }
#pragma unroll
            for (int q = 0; q < 8; ++q)
                if (q0 + q < ns) { r1 += p1[q]; r2 += p2[q]; r3 += p3[q]; }
        }
    }
    compare_column(a, part, v, I, J, c, r1, r2, r3, act);
}

// Block-wide reductions used by phase 2.
__device__ double block_sum(double v, double* red) {
    v = warp_sum(v);
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, nw = blockDim.x >> 5;
    __syncthreads();
    if (lane == 0) red[warp] = v;
    __syncthreads();
    double s = 0.0;
    for (int w = 0; w < nw; ++w) s += red[w];
    return s;
}

// argmax over r of (non-finite -> +inf, else |x|), lowest r on ties (reading A9)
__device__ int64_t block_argmax(const TileView& v, int64_t c, int64_t B, double* redv, long long* redi) {
    double best = -1.0; long long bi = 0x7fffffffffffffffll;
    for (int64_t r = threadIdx.x; r < B; r += blockDim.x) {
        const double x = view_x(v, r, c);
        const double m = dfinite(x) ? fabs(x) : INFINITY;
        if (m > best || (m == best && r < bi)) { best = m; bi = r; }
    }
    __syncthreads();
    redv[threadIdx.x] = best; redi[threadIdx.x] = bi;
    __syncthreads();
    if (threadIdx.x == 0) {
        double b = -1.0; long long i = 0x7fffffffffffffffll;
        for (int u = 0; u < (int)blockDim.x; ++u)
            if (redv[u] > b || (redv[u] == b && redi[u] < i)) { b = redv[u]; i = redi[u]; }
        redi[0] = i;
    }
    __syncthreads();
    const int64_t r = redi[0];
    __syncthreads();
    return r;
}


// Flags were written by other CTAs of this launch: read them from L2 (they are never in this
// SM's L1 for a reason this CTA could vouch for).
__device__ __forceinline__ Flag load_flag(const Flag* p) {
    Flag f;
    const int2 h0 = __ldcg(reinterpret_cast<const int2*>(p));       // Flag is 8-byte aligned
    const int2 h1 = __ldcg(reinterpret_cast<const int2*>(p) + 1);
    f.I = h0.x; f.J = h0.y; f.c = h1.x; f.part = h1.y;
    f.d1 = __ldcg(&p->d1); f.d2 = __ldcg(&p->d2); f.r1 = __ldcg(&p->r1); f.r2 = __ldcg(&p->r2);
    f.d3 = __ldcg(&p->d3); f.r3 = __ldcg(&p->r3);
    return f;
}

// Two errors in one column from three weighted sums (nchk = 3, reading B10): with
// Da at weight wa and Db at weight wb, d3 = S d2 - P d1 (S = wa + wb, P = wa wb). Scan S ascending,
// P = rint((S d2 - d3) / d1); accept integer roots 1 <= wa < wb <= B whose residual is within its
// rounding tolerance and whose two errors both exceed tau1; exactly one accepted pair locates them.
// Every operation is an explicit round-to-nearest one, in the oracle's order.
__device__ bool locate_two(double d1, double d2, double d3, double tau1, double tau2, double tau3, int64_t B,
                           int64_t& ra, int64_t& rb) {
    int found = 0;
    if (!(fabs(d1) > tau1)) return false;
    for (int64_t S = 3; S <= 2 * B - 1; ++S) {
        const double Sd = (double)S;
        const double Pd = rint(__ddiv_rn(__dsub_rn(__dmul_rn(Sd, d2), d3), d1));
        if (!(Pd >= 2.0) || Pd > __dmul_rn((double)B, (double)(B - 1))) continue;
        const int64_t P = (int64_t)Pd;
        const int64_t disc = S * S - 4 * P;
        if (disc <= 0) continue;
        int64_t q = (int64_t)sqrt((double)disc);
        while (q * q > disc) --q;
        while ((q + 1) * (q + 1) <= disc) ++q;
        if (q * q != disc || ((S - q) & 1)) continue;
        const int64_t wa = (S - q) / 2, wb = (S + q) / 2;
        if (wa < 1 || wb > B) continue;
        const double res = __dadd_rn(__dsub_rn(d3, __dmul_rn(Sd, d2)), __dmul_rn(Pd, d1));
        // 1/16 of the thresholds' combination (their full sum admits false pairs; the measured
        // noise is <= 2^-6 of tau, P9) + the relative slack ABFT_RHO2
        const double tol = __dadd_rn(__dmul_rn(__dadd_rn(__dadd_rn(tau3, __dmul_rn(Sd, tau2)), __dmul_rn(Pd, tau1)), 0.0625),
                                     __dmul_rn(ABFT_RHO2, __dadd_rn(__dadd_rn(fabs(d3), __dmul_rn(Sd, fabs(d2))),
                                                                   __dmul_rn(Pd, fabs(d1)))));
        if (!(fabs(res) <= tol)) continue;
        const double wad = (double)wa, wbd = (double)wb, den = (double)(wb - wa);
        const double Da = __ddiv_rn(__dsub_rn(__dmul_rn(wbd, d1), d2), den);
        const double Db = __ddiv_rn(__dsub_rn(d2, __dmul_rn(wad, d1)), den);
        if (!(fabs(Da) > tau1) || !(fabs(Db) > tau1)) continue;
        if (++found == 1) { ra = wa - 1; rb = wb - 1; }
    }
    return found == 1;
}

// Phase 2: resolve the flagged columns in the oracle's order (tile, then column): decide
// DATA / NONFINITE / CHK1 / CHK2 / UNCORRECTABLE, dedupe diagonal-tile mirrors, compute the
// corrections from the pre-correction tile, apply them per tile, log events. Run by one CTA: the
// last CTA of the check launch to finish its phase 1 (no separate launch).
__device__ void phase2_body(const StageArgs& a0, const StageArgs& a1, int flist) {
    DevState* st = a0.st;
    FlagList& FL = st->fl[flist];
    __shared__ int s_n;
    Fix* s_fix = FL.fix;   // global (block-visible after each __syncthreads)
    __shared__ int s_nfix, s_unc, s_stop;
    __shared__ double redv[kChkThreads];
    __shared__ long long redi[kChkThreads];
    __shared__ Flag s_flag;
    __shared__ long long s_rows[2];
    if (threadIdx.x == 0) {
        s_n = min(__ldcg(&FL.nflag), kFlagCap);
        if (__ldcg(&st->abort)) s_n = 0;
        if (__ldcg(&FL.overflow) && !__ldcg(&st->abort)) {   // more flagged columns than we can resolve
            st->status = ABFT_UNCORRECTABLE; st->abort = 1; s_n = 0;
            const long long e = (long long)atomicAdd(&st->nev, 1ull);
            if (e < a0.ev_cap) {
                abft_event_t& ev = a0.ev[e];
                ev.k = a0.k; ev.check = a0.V; ev.tile_i = -1; ev.tile_j = -1; ev.row = -3; ev.col = -1;
                ev.kind = ABFT_KIND_UNCORRECTABLE; ev.rank = a0.rank; ev.delta1 = 0; ev.delta2 = 0;
            }
            st->n_unc++;
        }
        // insertion sort by (J, I, c): the oracle's check order
        Flag* F = FL.flags;
        for (int i = 0; i < s_n; ++i) F[i] = load_flag(&F[i]);
        for (int i = 1; i < s_n; ++i) {
            Flag x = F[i]; int j = i - 1;
            auto key = [](const Flag& f) { return ((long long)f.J << 40) | ((long long)f.I << 20) | f.c; };
            while (j >= 0 && key(F[j]) > key(x)) { F[j + 1] = F[j]; --j; }
            F[j + 1] = x;
        }
        s_stop = 0;
    }
    __syncthreads();
    const int n = s_n;
    int i0 = 0;
    while (i0 < n && !s_stop) {
        // entries [i0, i1) belong to one tile (of one part)
        if (threadIdx.x == 0) s_flag = FL.flags[i0];
        __syncthreads();
        const Flag first = s_flag;
        const StageArgs& a = first.part ? a1 : a0;
        const int64_t B = a.nb;
        int i1 = i0;
        while (i1 < n && FL.flags[i1].I == first.I && FL.flags[i1].J == first.J && FL.flags[i1].part == first.part) ++i1;
        const TileView v = stage_view(a, first.I, first.J);
        if (threadIdx.x == 0) { s_nfix = 0; s_unc = 0; }
        __syncthreads();
        for (int e = i0; e < i1; ++e) {
            const Flag f = FL.flags[e];
            const int64_t c = f.c;
            double tau1, tau2, tau3;
            thresholds(a, f.I, (int64_t)f.J * B + c, v.factored, tau1, tau2, tau3);
            const bool has3 = v.c3 != nullptr;
            const bool f1 = !dfinite(f.d1) || fabs(f.d1) > tau1;
            const bool f2 = !dfinite(f.d2) || fabs(f.d2) > tau2;
            const bool f3 = has3 && (!dfinite(f.d3) || fabs(f.d3) > tau3);
            int kind = ABFT_KIND_UNCORRECTABLE; int64_t row = -1, row2 = -1;
            if (!dfinite(f.d1) || !dfinite(f.d2) || !dfinite(f.d3)) {
                kind = ABFT_KIND_NONFINITE;
                row = block_argmax(v, c, B, redv, redi);
            } else {
                bool done = false;
                if (f1) {
                    const double q = __ddiv_rn(f.d2, f.d1);
                    const double j = rint(q);                       // half-to-even
                    if (j >= 1.0 && j <= (double)B) {
                        const double jd1 = __dmul_rn(j, f.d1);
                        const double j2d1 = __dmul_rn(__dmul_rn(j, j), f.d1);
                        if (fabs(__dsub_rn(f.d2, jd1)) <= __dadd_rn(tau2, __dmul_rn(ABFT_RHO, fabs(jd1))) &&
                            (!has3 || fabs(__dsub_rn(f.d3, j2d1)) <= __dadd_rn(tau3, __dmul_rn(ABFT_RHO, fabs(j2d1))))) {
                            kind = ABFT_KIND_DATA; row = (int64_t)j - 1; done = true;
                        }
                    }
                }
                if (!done && (int)f1 + (int)f2 + (int)f3 == 1) {   // one checksum row corrupted (A10)
                    kind = f1 ? ABFT_KIND_CHK1 : f2 ? ABFT_KIND_CHK2 : ABFT_KIND_CHK3;
                    done = true;
                }
                if (!done && has3) {                                 // two data errors (B10)
                    if (threadIdx.x == 0) {
                        int64_t ra = -1, rb = -1;
                        if (!locate_two(f.d1, f.d2, f.d3, tau1, tau2, tau3, B, ra, rb)) ra = rb = -1;
                        s_rows[0] = ra; s_rows[1] = rb;
                    }
                    __syncthreads();
                    if (s_rows[0] >= 0) { kind = ABFT_KIND_DATA; row = s_rows[0]; row2 = s_rows[1]; }
                    __syncthreads();
                }
            }
            const int vcode = ((a.kind == SK_COLUMN || a.kind == SK_COL_DIAG) && f.I == a.k) ? ABFT_V1 : a.V;
            if (kind == ABFT_KIND_DATA && row2 >= 0) {
                // two errors (B10): x_a, x_b from chk1, chk2 and the other B-2 entries summed
                // directly (A8): R1 = x_a + x_b, R2 = wa x_a + wb x_b
                double p1 = 0.0, p2 = 0.0;
                for (int64_t r = threadIdx.x; r < B; r += blockDim.x)
                    if (r != row && r != row2) { const double x = view_x(v, r, c); p1 += x; p2 = fma((double)(r + 1), x, p2); }
                const double s1 = block_sum(p1, redv);
                const double s2 = block_sum(p2, redv);
                if (threadIdx.x == 0) {
                    const double wa = (double)(row + 1), wb = (double)(row2 + 1);
                    const double R1 = __dsub_rn(v.c1[c * v.ldc], s1), R2 = __dsub_rn(v.c2[c * v.ldc], s2);
                    const double xa = __ddiv_rn(__dsub_rn(__dmul_rn(wb, R1), R2), __dsub_rn(wb, wa));
                    const double xb = __ddiv_rn(__dsub_rn(R2, __dmul_rn(wa, R1)), __dsub_rn(wb, wa));
                    const int64_t rows[2] = {row, row2};
                    const double vals[2] = {xa, xb};
                    for (int h = 0; h < 2; ++h) {
                        double* p = view_store(v, rows[h], c);
                        bool dup = false;
                        for (int u = 0; u < s_nfix; ++u) dup |= (s_fix[u].p == p);
                        if (dup) continue;
                        if (s_nfix < kMaxFix) { s_fix[s_nfix].p = p; s_fix[s_nfix].p2 = nullptr; s_fix[s_nfix].val = vals[h]; s_nfix++; }
                        else s_unc = 1;
                        int64_t sr = rows[h], sc = c;
                        if (v.diag && !v.factored && sr < sc) { const int64_t t = sr; sr = sc; sc = t; }
                        const long long ev_i = (long long)atomicAdd(&st->nev, 1ull);
                        if (ev_i < a.ev_cap) {
                            abft_event_t& ev = a.ev[ev_i];
                            ev.k = a.k; ev.check = vcode; ev.tile_i = f.I; ev.tile_j = f.J;
                            ev.row = (int32_t)sr; ev.col = (int32_t)sc; ev.kind = ABFT_KIND_DATA; ev.rank = a.rank;
                            ev.delta1 = f.d1; ev.delta2 = f.d2;
                        }
                        st->n_detected++; st->n_data++;
                    }
                }
                __syncthreads();
            } else if (kind == ABFT_KIND_DATA || kind == ABFT_KIND_NONFINITE) {
                double* p = view_store(v, row, c);
                bool dup = false;
                for (int u = 0; u < s_nfix; ++u) dup |= (s_fix[u].p == p);
                if (dup) continue;                              // corrected once, logged once
                double part = 0.0;
                for (int64_t r = threadIdx.x; r < B; r += blockDim.x)
                    if (r != row) part += view_x(v, r, c);
                const double sum = block_sum(part, redv);
                if (threadIdx.x == 0) {
                    const double val = __dsub_rn(v.c1[c * v.ldc], sum);   // A8
                    if (s_nfix < kMaxFix) { s_fix[s_nfix].p = p; s_fix[s_nfix].p2 = nullptr; s_fix[s_nfix].val = val; s_nfix++; }
                    else s_unc = 1;
                    int64_t sr = row, sc = c;
                    if (v.diag && !v.factored && sr < sc) { const int64_t t = sr; sr = sc; sc = t; }
                    const long long ev_i = (long long)atomicAdd(&st->nev, 1ull);
                    if (ev_i < a.ev_cap) {
                        abft_event_t& ev = a.ev[ev_i];
                        ev.k = a.k; ev.check = vcode;
                        ev.tile_i = f.I; ev.tile_j = f.J;
                        ev.row = (int32_t)sr; ev.col = (int32_t)sc; ev.kind = kind; ev.rank = a.rank;
                        ev.delta1 = f.d1; ev.delta2 = f.d2;
                    }
                    st->n_detected++;
                    if (kind == ABFT_KIND_DATA) st->n_data++; else st->n_nonfinite++;
                }
                __syncthreads();
            } else if (threadIdx.x == 0) {
                const long long ev_i = (long long)atomicAdd(&st->nev, 1ull);
                if (ev_i < a.ev_cap) {
                    abft_event_t& ev = a.ev[ev_i];
                    ev.k = a.k; ev.check = vcode;
                    ev.tile_i = f.I; ev.tile_j = f.J;
                    ev.row = kind == ABFT_KIND_CHK1 ? -1 : kind == ABFT_KIND_CHK2 ? -2 : kind == ABFT_KIND_CHK3 ? -4 : -3;
                    ev.col = (int32_t)c; ev.kind = kind; ev.rank = a.rank;
                    ev.delta1 = f.d1; ev.delta2 = f.d2;
                }
                st->n_detected++;
                if (kind == ABFT_KIND_CHK1 || kind == ABFT_KIND_CHK2 || kind == ABFT_KIND_CHK3) {
                    if (kind == ABFT_KIND_CHK1) st->n_chk1++; else st->n_chk2++;
                    if (s_nfix < kMaxFix) {
                        s_fix[s_nfix].p = kind == ABFT_KIND_CHK1 ? &v.c1[c * v.ldc]
                                          : kind == ABFT_KIND_CHK2 ? &v.c2[c * v.ldc] : &v.c3[c * v.ldc];
                        s_fix[s_nfix].p2 = nullptr;
                        s_fix[s_nfix].val = kind == ABFT_KIND_CHK1 ? f.r1 : kind == ABFT_KIND_CHK2 ? f.r2 : f.r3;   // chk := v^T X
                        s_nfix++;
                    } else s_unc = 1;
                } else {
                    st->n_unc++;
                    s_unc = 1;
                }
            }
            __syncthreads();
        }
        __syncthreads();
        if (threadIdx.x == 0) {
            if (a.correct)
                for (int u = 0; u < s_nfix; ++u) *s_fix[u].p = s_fix[u].val;
            if (s_unc) { st->status = ABFT_UNCORRECTABLE; st->abort = 1; s_stop = 1; }
        }
        __syncthreads();
        i0 = i1;
    }
    if (threadIdx.x == 0) { FL.nflag = 0; FL.overflow = 0; }
}

// One check launch: phase 1 over the tiles of one or two stage parts (blocks [0, nblk0) run part
// 0, the rest part 1; kind SK_TRAIL_OFF reads the GEMM's fused partials, every other kind re-reads
// the tiles), then the last CTA to finish resolves the flags of both parts (phase 2) in the
// oracle's order. Every CTA reaches the completion counter (also when the run is aborted), and
// the last one resets it, so the counter is zero again for the next launch on this flag list.
// min 4 CTAs/SM: phase 1 is the hot part (bandwidth-bound); the rare phase 2 may spill instead
// The grid may be smaller than the work (launch_check caps it, ABFT_CHK_GRID): each CTA then takes
// work blocks blockIdx.x, + gridDim.x, ... so its fixed costs are paid once for several tiles.
__global__ void __launch_bounds__(kChkThreads, 4) k_check(StageArgs a0, StageArgs a1, int64_t nblk0, int64_t nblk) {
    __shared__ int s_last;
    // no abort test at entry (it would put a dependent global round trip in front of every check on
    // the panel chain): after an abort phase 1 only reads, and phase 2 resolves nothing
    {
        for (int64_t blk = blockIdx.x; blk < nblk; blk += gridDim.x) {
            const bool p1 = blk >= nblk0;
            const StageArgs& a = p1 ? a1 : a0;
            const int64_t bid = p1 ? blk - nblk0 : blk;
            if (a.kind == SK_TRAIL_OFF) phase1_fused(a, p1 ? 1 : 0, bid);
            else phase1_reread(a, p1 ? 1 : 0, bid);
            if (blk + gridDim.x < nblk) __syncthreads();   // shared sums are reused by the next block
        }
    }
    if (a0.encode) return;   // encode launches resolve nothing (no counter use)
    // the CTA's flags are ordered before its completion count by the barrier and thread 0's
    // (cumulative) gpu-scope fence: one fence per CTA, not one per thread
    __syncthreads();
    const int fl = a0.flist;
    if (threadIdx.x == 0) { __threadfence(); s_last = atomicAdd(&a0.st->done[fl], 1u) == gridDim.x - 1; }
    __syncthreads();
    if (!s_last) return;
    __threadfence();
    if (threadIdx.x == 0) a0.st->done[fl] = 0u;
    if (__ldcg(&a0.st->fl[fl].nflag) > 0 || __ldcg(&a0.st->fl[fl].overflow)) phase2_body(a0, a1, fl);
}

// Threshold scales of reading A4: s_i = sqrt(A_ii); S1_I = sum s_i, S2_I = sum (i+1) s_i over
// block I, summed sequentially in ascending order with explicit round-to-nearest operations.
__global__ void k_scales_diag(int64_t n, const double* A, int64_t lda, double* s) {
    const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (i < n) s[i] = __dsqrt_rn(A[i * lda + i]);
}
__global__ void k_scales_block(int64_t N, int64_t B, const double* s, double* S1, double* S2, double* S3) {
    const int64_t I = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (I >= N) return;
    double a = 0.0, b = 0.0, c = 0.0;
    for (int64_t r = 0; r < B; ++r) {
        a = __dadd_rn(a, s[I * B + r]);
        b = __dadd_rn(b, __dmul_rn((double)(r + 1), s[I * B + r]));
        c = __dadd_rn(c, __dmul_rn((double)((r + 1) * (r + 1)), s[I * B + r]));   // S3 (nchk = 3, B10)
    }
    S1[I] = a; S2[I] = b;
    if (S3) S3[I] = c;
}

}  // namespace abft

// ---- host launchers ---------------------------------------------------------------------
using namespace abft;

static int64_t check_blocks(const StageArgs& a) {
    const int64_t count = stage_count(a);
    if (count <= 0) return 0;
    const int64_t per = a.kind == SK_TRAIL_OFF ? kChkThreads : kChkCols;
    return count * ((a.nb + per - 1) / per);
}

// grid of a check launch: one CTA per work block, or at most ABFT_CHK_GRID CTAs (0: uncapped)
static int64_t check_grid(int64_t nblk) {
    static int64_t cap = -1;
    if (cap < 0) { const char* e = getenv("ABFT_CHK_GRID"); cap = e ? std::max(0, atoi(e)) : 0; }
    return cap > 0 && nblk > cap ? cap : nblk;
}

int launch_check(const StageArgs& a, cudaStream_t s) {
    const int64_t nb0 = check_blocks(a);
    if (nb0 <= 0) return 0;
    k_check<<<(unsigned)check_grid(nb0), kChkThreads, 0, s>>>(a, a, nb0, nb0);
    abft_count_launch();
    return 0;
}

// Two stages of one flag list in one launch, resolved together in the oracle's tile order
// (part 0's tiles precede part 1's in (J, I) order: V5 diagonal + off-diagonal tiles of the same
// block columns are interleaved by that sort; V3 (tile k,k) + V4 (tiles i>k, k)).
int launch_check2(const StageArgs& a0, const StageArgs& a1, cudaStream_t s) {
    const int64_t nb0 = check_blocks(a0), nb1 = check_blocks(a1);
    if (nb0 + nb1 <= 0) return 0;
    k_check<<<(unsigned)check_grid(nb0 + nb1), kChkThreads, 0, s>>>(a0, a1, nb0, nb0 + nb1);
    abft_count_launch();
    return 0;
}

// V5 with the fused recalculation: diagonal tiles re-read (sym), off-diagonal tiles from the
// update GEMM's partials; one launch, one flag list.
int launch_check_v5_fused(const StageArgs& diag, const StageArgs& off, cudaStream_t s) {
    return launch_check2(diag, off, s);
}

int launch_scales_diag(int64_t nrows, const double* Adiag, int64_t lda, double* s_out, cudaStream_t s) {
    if (nrows <= 0) return 0;
    k_scales_diag<<<(unsigned)((nrows + 255) / 256), 256, 0, s>>>(nrows, Adiag, lda, s_out);
    abft_count_launch();
    return 0;
}
int launch_scales_blocks(int64_t N, int64_t nb, const double* sv, double* S1, double* S2, cudaStream_t s) {
    if (N <= 0) return 0;
    k_scales_block<<<(unsigned)((N + 127) / 128), 128, 0, s>>>(N, nb, sv, S1, S2, nullptr);
    abft_count_launch();
    return 0;
}

int launch_scales(int64_t n, int64_t nb, const double* A, int64_t lda, double* scl, cudaStream_t s, int nchk) {
    const int64_t N = n / nb;
    if (n == 0) return 0;
    k_scales_diag<<<(unsigned)((n + 255) / 256), 256, 0, s>>>(n, A, lda, scl);
    k_scales_block<<<(unsigned)((N + 127) / 128), 128, 0, s>>>(N, nb, scl, scl + n, scl + n + N,
                                                               nchk == 3 ? scl + n + 2 * N : nullptr);
    abft_count_launch(2);
    return 0;
}
