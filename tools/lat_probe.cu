// lat_probe.cu — dependent-chain latencies on this GPU (development tool):
// DFMA, DMUL, double division, double sqrt, LDS->DFMA->STS, __syncthreads (256 thr), cluster barrier.
#include <cstdio>
#include <cooperative_groups.h>
namespace cg = cooperative_groups;
__global__ void probe(double* out, long long* cyc, double seed, int n) {
    __shared__ double sm[1024];
    const int tid = threadIdx.x;
    sm[tid] = seed + tid;
    __syncthreads();
    double x = seed + tid * 1e-3, y = 1.0;
    long long t0, t1;
    // 1 DFMA chain
    t0 = clock64();
    for (int i = 0; i < n; ++i) x = fma(x, 0.999999, 1e-7);
    t1 = clock64(); if (tid == 0) cyc[0] = (t1 - t0) / n;
    // 2 division chain
    t0 = clock64();
    for (int i = 0; i < n; ++i) x = 1.0 / (x + 1.5);
    t1 = clock64(); if (tid == 0) cyc[1] = (t1 - t0) / n;
    // 3 sqrt chain
    t0 = clock64();
    for (int i = 0; i < n; ++i) x = sqrt(x + 2.0);
    t1 = clock64(); if (tid == 0) cyc[2] = (t1 - t0) / n;
    // 4 LDS -> DFMA -> STS chain (same thread)
    t0 = clock64();
    for (int i = 0; i < n; ++i) { double v = sm[(tid + i) & 1023]; sm[(tid + i + 1) & 1023] = v * 0.5 + x; }
    t1 = clock64(); if (tid == 0) cyc[3] = (t1 - t0) / n;
    // 5 __syncthreads
    t0 = clock64();
    for (int i = 0; i < n; ++i) { __syncthreads(); }
    t1 = clock64(); if (tid == 0) cyc[4] = (t1 - t0) / n;
    // 6 LDS-read then barrier then dependent (leaf-like step)
    t0 = clock64();
    for (int i = 0; i < n; ++i) {
        __syncthreads();
        double d = sm[i & 1023];
        double inv = 1.0 / d;
        sm[(i + 1) & 1023] = d + inv * 1e-9;
    }
    t1 = clock64(); if (tid == 0) cyc[5] = (t1 - t0) / n;
    out[tid] = x + y;
}
__global__ void __cluster_dims__(8, 1, 1) probe_cluster(long long* cyc, int n) {
    cg::cluster_group cl = cg::this_cluster();
    long long t0 = clock64();
    for (int i = 0; i < n; ++i) cl.sync();
    long long t1 = clock64();
    if (threadIdx.x == 0 && cl.block_rank() == 0) cyc[6] = (t1 - t0) / n;
    t0 = clock64();
    for (int i = 0; i < n; ++i) { __threadfence(); cl.sync(); }
    t1 = clock64();
    if (threadIdx.x == 0 && cl.block_rank() == 0) cyc[7] = (t1 - t0) / n;
}
int main() {
    double* out; long long* cyc;
    cudaMalloc(&out, 8 * 1024); cudaMalloc(&cyc, 8 * 16);
    const char* names[8] = {"DFMA chain", "double div chain", "double sqrt chain", "LDS->DFMA->STS chain",
                            "__syncthreads (256 thr)", "barrier+LDS+div+STS step", "cluster.sync (8 CTAs)",
                            "threadfence+cluster.sync"};
    for (int rep = 0; rep < 2; ++rep) {
        probe<<<1, 256>>>(out, cyc, 1.25, 1000);
        probe_cluster<<<8, 256>>>(cyc, 1000);
        cudaDeviceSynchronize();
    }
    long long h[8];
    cudaMemcpy(h, cyc, sizeof h, cudaMemcpyDeviceToHost);
    for (int i = 0; i < 8; ++i) printf("%-28s %lld cycles\n", names[i], h[i]);
    printf("%s\n", cudaGetErrorString(cudaGetLastError()));
}
