// FP64 peak probe for B200 (sm_100a): register-resident DMMA (mma.sync m8n8k4 f64) and
// DFMA loops. Used to derive the FP64 roofline denominator (MEASURED_PEAKS.json has none).
#include <cstdio>
#include <cuda_runtime.h>
#define CK(x) do{cudaError_t e=(x); if(e!=cudaSuccess){printf("CUDA %s @%d\n",cudaGetErrorString(e),__LINE__);return 1;}}while(0)

template<int NACC>
__global__ void dmma_loop(double* out, int iters) {
  double a = threadIdx.x * 1e-3, b = 1.0 + blockIdx.x * 1e-6;
  double c[NACC][2];
  #pragma unroll
  for (int i = 0; i < NACC; ++i) { c[i][0] = 0; c[i][1] = 0; }
  for (int it = 0; it < iters; ++it) {
    #pragma unroll
    for (int i = 0; i < NACC; ++i)
      asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};\n"
                   : "+d"(c[i][0]), "+d"(c[i][1]) : "d"(a), "d"(b));
  }
  double s = 0;
  #pragma unroll
  for (int i = 0; i < NACC; ++i) s += c[i][0] + c[i][1];
  if (s == 12345.678) out[0] = s;
}

template<int NACC>
__global__ void dfma_loop(double* out, int iters) {
  double a = threadIdx.x * 1e-3, b = 1.0 + blockIdx.x * 1e-6;
  double c[NACC];
  #pragma unroll
  for (int i = 0; i < NACC; ++i) c[i] = i;
  for (int it = 0; it < iters; ++it) {
    #pragma unroll
    for (int i = 0; i < NACC; ++i) c[i] = fma(a, c[i], b);
  }
  double s = 0;
  #pragma unroll
  for (int i = 0; i < NACC; ++i) s += c[i];
  if (s == 12345.678) out[0] = s;
}

int main() {
  double* d; CK(cudaMalloc(&d, 8));
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  int clk; cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  printf("SMs %d clock %d kHz\n", sms, clk);
  for (int warps : {4, 8, 16}) {
    for (int cpb : {1, 2}) {
      int grid = sms * cpb, iters = 20000;
      for (int rep = 0; rep < 2; ++rep) dmma_loop<8><<<grid, warps * 32>>>(d, 100);
      float best = 1e30;
      for (int rep = 0; rep < 5; ++rep) {
        cudaEventRecord(e0); dmma_loop<8><<<grid, warps * 32>>>(d, iters); cudaEventRecord(e1);
        CK(cudaEventSynchronize(e1)); float ms; cudaEventElapsedTime(&ms, e0, e1); if (ms < best) best = ms;
      }
      double flops = 2.0 * 256 * 8 * (double)iters * warps * grid;
      printf("DMMA m8n8k4 warps/CTA %d CTAs/SM %d : %.2f TFLOP/s\n", warps, cpb, flops / best / 1e9);
    }
  }
  for (int warps : {8, 16, 32}) {
    int grid = sms * 2, iters = 20000;
    for (int rep = 0; rep < 2; ++rep) dfma_loop<8><<<grid, warps * 32>>>(d, 100);
    float best = 1e30;
    for (int rep = 0; rep < 5; ++rep) {
      cudaEventRecord(e0); dfma_loop<8><<<grid, warps * 32>>>(d, iters); cudaEventRecord(e1);
      CK(cudaEventSynchronize(e1)); float ms; cudaEventElapsedTime(&ms, e0, e1); if (ms < best) best = ms;
    }
    double flops = 2.0 * 8 * (double)iters * warps * 32 * grid;
    printf("DFMA warps/CTA %d : %.2f TFLOP/s\n", warps, flops / best / 1e9);
  }
  // sustained DMMA: back to back for ~4 s
  {
    int grid = sms, warps = 8, iters = 200000;
    cudaEventRecord(e0);
    for (int rep = 0; rep < 10; ++rep) dmma_loop<8><<<grid, warps * 32>>>(d, iters);
    cudaEventRecord(e1); CK(cudaEventSynchronize(e1)); float ms; cudaEventElapsedTime(&ms, e0, e1);
    double flops = 10 * 2.0 * 256 * 8 * (double)iters * warps * grid;
    printf("DMMA sustained (%.1f s): %.2f TFLOP/s\n", ms / 1e3, flops / ms / 1e9);
  }
  return 0;
}
