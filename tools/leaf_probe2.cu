// leaf_probe2.cu — development tool: the 64 x 64 leaf step (factor + elimination) with NE
// elements per thread (64 * 16 / NE... threads = 64 * 64 / NE) and optionally the next pivot's
// reciprocal computed by its owner and published (PRE). Cycles per column step.
#include <cstdio>
constexpr int kTT = 64, kTP = 68;
template <int NE, bool PRE>
__global__ void leaf(double* out, long long* cyc) {
    extern __shared__ __align__(16) double dsm[];
    double* Ls = dsm;
    double* Ys = dsm + kTT * kTP;
    double* rcp = dsm + 2 * kTT * kTP;
    const int tid = threadIdx.x, me = tid & 63, g = tid >> 6, gb = NE * g;
    const int lo = tid & 32, hi = lo + 31;
    double a[NE], y[NE];
#pragma unroll
    for (int u = 0; u < NE; ++u) {
        const int r = gb + u;
        a[u] = (r >= me) ? (r == me ? 64.0 : 1.0 / (1.0 + r + me)) : 0.0;
        y[u] = (r == me) ? 1.0 : 0.0;
    }
    for (int e = tid; e < 2 * kTT * kTP + 64; e += blockDim.x) dsm[e] = (e < kTT * kTP && e % kTP == e / kTP) ? 64.0 : 0.01;
    __syncthreads();
    if (me == 0) for (int u = 0; u < NE; ++u) { Ls[gb + u] = a[u]; Ys[gb + u] = y[u]; }
    if (tid == 0) rcp[0] = 1.0 / 64.0;
    long long t0 = clock64();
    for (int jj = 0; jj < kTT; ++jj) {
        __syncthreads();
        const double* cj = Ls + jj * kTP;
        const double d = cj[jj];
        if (!(d > 0.0)) return;
        const double rd = PRE ? rcp[jj] : __drcp_rn(d);
        const double gm = cj[me] * rd;
        if (hi > jj && gb + NE - 1 > jj && gb + NE - 1 >= lo) {
            double rv[NE];
#pragma unroll
            for (int u = 0; u < NE; u += 2) {
                const double2 v = *reinterpret_cast<const double2*>(cj + gb + u);
                rv[u] = v.x; rv[u + 1] = v.y;
            }
#pragma unroll
            for (int u = 0; u < NE; ++u) a[u] = fma(-rv[u], gm, a[u]);
            if (me == jj + 1) {
#pragma unroll
                for (int u = 0; u < NE; u += 2)
                    *reinterpret_cast<double2*>(Ls + (jj + 1) * kTP + gb + u) = make_double2(a[u], a[u + 1]);
                if (PRE && gb <= jj + 1 && jj + 1 < gb + NE) {
#pragma unroll
                    for (int u = 0; u < NE; ++u) if (gb + u == jj + 1) rcp[jj + 1] = __drcp_rn(a[u]);
                }
            }
        }
        if (gb <= jj && hi > jj) {
            const double* yj = Ys + jj * kTP;
            double yv[NE];
#pragma unroll
            for (int u = 0; u < NE; u += 2) {
                const double2 v = *reinterpret_cast<const double2*>(yj + gb + u);
                yv[u] = v.x; yv[u + 1] = v.y;
            }
#pragma unroll
            for (int u = 0; u < NE; ++u) y[u] = fma(-gm, yv[u], y[u]);
        }
        if (me == jj + 1) {
#pragma unroll
            for (int u = 0; u < NE; u += 2)
                *reinterpret_cast<double2*>(Ys + me * kTP + gb + u) = make_double2(y[u], y[u + 1]);
        }
    }
    long long t1 = clock64();
    double s = 0;
    for (int u = 0; u < NE; ++u) s += a[u] + y[u];
    out[tid] = s;
    if (tid == 0) cyc[0] = (t1 - t0) / kTT;
}
template <int NE, bool PRE>
void run(double* out, long long* cyc) {
    const int sm = (2 * kTT * kTP + 64) * 8, threads = 64 * 64 / NE;
    cudaFuncSetAttribute(leaf<NE, PRE>, cudaFuncAttributeMaxDynamicSharedMemorySize, sm);
    leaf<NE, PRE><<<1, threads, sm>>>(out, cyc);
    leaf<NE, PRE><<<1, threads, sm>>>(out, cyc);
    long long h; cudaMemcpy(&h, cyc, 8, cudaMemcpyDeviceToHost);
    printf("NE %2d threads %4d pre-rcp %d: %lld cycles/step (%s)\n", NE, threads, (int)PRE, h,
           cudaGetErrorString(cudaGetLastError()));
}
int main() {
    double* out; long long* cyc;
    cudaMalloc(&out, 8 * 1024); cudaMalloc(&cyc, 8);
    run<16, false>(out, cyc); run<16, true>(out, cyc);
    run<8, false>(out, cyc);  run<8, true>(out, cyc);
    run<4, false>(out, cyc);  run<4, true>(out, cyc);
    return 0;
}
