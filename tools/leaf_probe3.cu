// leaf_probe3.cu — development tool: clock64 breakdown of the blocked 64 x 64 leaf (panel steps,
// rank-8 DMMA updates) on one CTA with the tile in shared memory.
#include <cstdio>
constexpr int kTT = 64, kTP = 68, kTaskThreads = 256;
__device__ __forceinline__ void dmma(double& c0, double& c1, double a, double b) {
    asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};\n"
                 : "+d"(c0), "+d"(c1) : "d"(a), "d"(b));
}
template <int MODE>   // 0: as in the library, 1: rcp once per thread via division, 2: no rcp (multiply)
__global__ void k(double* out, long long* cyc) {
    extern __shared__ __align__(16) double dsm[];
    double* Ls = dsm; double* Pb = dsm + kTT * kTP;
    __shared__ double piv[kTT];
    const int tid = threadIdx.x, r = tid & 63, g = tid >> 6;
    const int lane = tid & 31, warp = tid >> 5, fr = lane >> 2, fc = lane & 3;
    for (int e = tid; e < kTT * kTP; e += 256) { const int c = e / kTP, rr = e % kTP; Ls[e] = (rr == c) ? 64.0 : 1.0 / (1 + rr + c); }
    __syncthreads();
    long long tp = 0, tu = 0, t0, t1;
    for (int p = 0; p < 8; ++p) {
        const int c0 = 8 * p;
        t0 = clock64();
        for (int j = 0; j < 8; ++j) {
            const int cj = c0 + j;
            __syncthreads();
            const double d = Ls[cj * kTP + cj];
            if (!(d > 0.0)) return;
            if (r > cj) {
                const double rd = MODE == 0 ? __drcp_rn(d) : (MODE == 1 ? 1.0 / d : 0.015625);
                const double f = Ls[cj * kTP + r] * rd;
#pragma unroll
                for (int h = 0; h < 2; ++h) {
                    const int c = c0 + 2 * g + h;
                    if (c > cj) Ls[c * kTP + r] = fma(-f, Ls[cj * kTP + c], Ls[c * kTP + r]);
                }
            }
        }
        __syncthreads();
        t1 = clock64(); tp += t1 - t0; t0 = t1;
#pragma unroll
        for (int h = 0; h < 2; ++h) {
            const int c = c0 + 2 * g + h;
            if (r >= c) {
                const double v = Ls[c * kTP + r];
                Pb[(2 * g + h) * kTP + r] = v;
                if (r == c) piv[c] = v;
                else Ls[c * kTP + r] = v * __drcp_rn(Ls[c * kTP + c]);
            }
        }
        __syncthreads();
        const int nt = 7 - p;
        for (int e = warp; e < nt * (nt + 1) / 2; e += 8) {
            int tj = 0, rem = e;
            while (rem >= nt - tj) { rem -= nt - tj; ++tj; }
            const int m0 = c0 + 8 + 8 * (tj + rem), n0 = c0 + 8 + 8 * tj;
            double* c0p = Ls + (n0 + 2 * fc) * kTP + m0 + fr;
            double v0 = c0p[0], v1 = c0p[kTP];
#pragma unroll
            for (int kq = 0; kq < 8; kq += 4) dmma(v0, v1, -Ls[(c0 + kq + fc) * kTP + m0 + fr], Pb[(kq + fc) * kTP + n0 + fr]);
            c0p[0] = v0; c0p[kTP] = v1;
        }
        __syncthreads();
        t1 = clock64(); tu += t1 - t0;
    }
    out[tid] = Ls[tid];
    if (tid == 0) { cyc[0] = tp / 64; cyc[1] = tu / 8; }
}
template <int M> void run(double* out, long long* cyc) {
    const int sm = 2 * kTT * kTP * 8;
    cudaFuncSetAttribute(k<M>, cudaFuncAttributeMaxDynamicSharedMemorySize, sm);
    k<M><<<1, 256, sm>>>(out, cyc); k<M><<<1, 256, sm>>>(out, cyc);
    long long h[2]; cudaMemcpy(h, cyc, 16, cudaMemcpyDeviceToHost);
    printf("mode %d: panel step %lld cycles, per-panel finalize+DMMA update %lld cycles (%s)\n", M, h[0], h[1],
           cudaGetErrorString(cudaGetLastError()));
}
int main() {
    double* out; long long* cyc; cudaMalloc(&out, 8 * 256); cudaMalloc(&cyc, 16);
    run<0>(out, cyc); run<1>(out, cyc); run<2>(out, cyc);
}
