// coreside_probe.cu — development tool: is the warp-specialised update GEMM bit-reproducible when a
// long-running CTA of another kernel (another stream) shares its SMs? Runs C -= W W^T (lower) on
// the same inputs alone and next to a spinning "guest" kernel, and compares the results bitwise.
// Guest modes: 0 = spin only, 1 = spin + DMMA, 2 = spin + cp.async smem traffic, 3 = spin + nanosleep.
#include <cstdio>
#include <cstdint>
#include <cstring>
#include <vector>
#include <cuda_runtime.h>
#include <unistd.h>
#include <cstdlib>
extern "C" int abft_dev_chol_inv(int64_t, double*, int64_t, double*, void*);
extern "C" int abft_gen_spd(int64_t, uint64_t, double*, int64_t, void*);
extern "C" int abft_dev_gemm_nt(int64_t, int64_t, int64_t, const double*, int64_t, const double*, int64_t, double*,
                                int64_t, double, double, int, void*);
static int late_smem(int argc) { return argc > 1 ? 120 * 1024 : 104448; }
__global__ void guest(int mode, long long cycles, double* sink) {
    extern __shared__ double sm[];
    long long t0 = clock64();
    double acc0 = 0, acc1 = 0, a = threadIdx.x * 1e-3, b = 1.0;
    int it = 0;
    while (clock64() - t0 < cycles) {
        if (mode == 1) asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};\n"
                                    : "+d"(acc0), "+d"(acc1) : "d"(a), "d"(b));
        else if (mode == 2) { sm[(threadIdx.x + it * 256) % 13000] = acc0 + it; acc0 += sm[(threadIdx.x * 7 + it) % 13000]; __syncthreads(); }
        else if (mode == 3) __nanosleep(32);
        ++it;
    }
    if (acc0 == 12345.0) sink[0] = acc0 + acc1;
}
int main(int argc, char** argv) {
    const bool late = argc > 1;
    const int64_t M = argc > 2 ? atoll(argv[2]) : 16384, K = argc > 3 ? atoll(argv[3]) : 512;
    std::vector<double> hW(M * K), hC(M * M);
    uint64_t x = 12345;
    for (auto& v : hW) { x = x * 6364136223846793005ull + 1442695040888963407ull; v = (double)(x >> 11) * 0x1p-53 - 0.5; }
    for (auto& v : hC) { x = x * 6364136223846793005ull + 1442695040888963407ull; v = (double)(x >> 11) * 0x1p-53; }
    double *W, *C, *sink;
    cudaMalloc(&W, 8 * M * K); cudaMalloc(&C, 8 * M * M); cudaMalloc(&sink, 8);
    cudaMemcpy(W, hW.data(), 8 * M * K, cudaMemcpyHostToDevice);
    cudaStream_t s1, s2; cudaStreamCreateWithFlags(&s1, cudaStreamNonBlocking);
    int lo, hi; cudaDeviceGetStreamPriorityRange(&lo, &hi);
    cudaStreamCreateWithPriority(&s2, cudaStreamNonBlocking, hi);
    std::vector<double> ref(M * M), got(M * M);
    const int gsm = late_smem(argc);
    cudaFuncSetAttribute(guest, cudaFuncAttributeMaxDynamicSharedMemorySize, gsm);
    double *Ad, *Lid;
    const int64_t nbc = 1024;
    cudaMalloc(&Ad, 8 * nbc * nbc); cudaMalloc(&Lid, 8 * nbc * nbc);
    for (int mode = -1; mode < 5; ++mode) {
        for (int rep = 0; rep < 3; ++rep) {
            cudaMemcpy(C, hC.data(), 8 * M * M, cudaMemcpyHostToDevice);
            cudaDeviceSynchronize();
            if (mode >= 0 && mode < 4 && !late) guest<<<8, 256, gsm, s2>>>(mode, 40000000LL, sink);   // ~20 ms on 8 SMs
            abft_dev_gemm_nt(M, M, K, W, M, W, M, C, M, -1.0, 1.0, 1, s1);
            if (mode >= 0 && mode < 4 && late) {   // arrive while the GEMM fills the GPU (needs whole SMs)
                usleep(500);
                for (int q = 0; q < 20; ++q) guest<<<1, 256, gsm, s2>>>(mode, 400000LL, sink);
            }
            if (mode == 4)   // the task-graph diagonal block as the guest, repeatedly while the GEMM runs
                for (int q = 0; q < 6; ++q) { abft_gen_spd(nbc, 7 + q, Ad, nbc, s2); abft_dev_chol_inv(nbc, Ad, nbc, Lid, s2); }
            cudaDeviceSynchronize();
            cudaMemcpy(mode < 0 && rep == 0 ? ref.data() : got.data(), C, 8 * M * M, cudaMemcpyDeviceToHost);
            if (mode < 0 && rep == 0) continue;
            int64_t bad = 0, first = -1;
            for (int64_t c = 0; c < M; ++c)
                for (int64_t r = c; r < M; ++r)
                    if (memcmp(&ref[c * M + r], &got[c * M + r], 8)) { if (first < 0) first = c * M + r; ++bad; }
            printf("guest mode %d rep %d: %lld differing elements (first at r=%lld c=%lld) %s\n", mode, rep, (long long)bad,
                   first < 0 ? -1LL : (long long)(first % M), first < 0 ? -1LL : (long long)(first / M),
                   cudaGetErrorString(cudaGetLastError()));
        }
    }
    return 0;
}
