// sanitize_driver.cu — development tool: a small, torch-free run of the library's hot path for
// compute-sanitizer (memcheck / racecheck / synccheck / initcheck): the update GEMM on its own
// (the warp-specialised bulk-copy kernel), then whole factorisations, fault-free and with
// injected storage + computing errors. Exit code 0 iff every call returned the expected status.
#include <cstdio>
#include <cstdint>
#include <cstdlib>
#include <vector>
#include <cuda_runtime.h>
#include "../include/abft.h"

int main(int argc, char** argv) {
    const int64_t n = argc > 1 ? atoll(argv[1]) : 1024, nb = argc > 2 ? atoll(argv[2]) : 256;
    double *A, *W, *C;
    cudaMalloc(&A, 8 * n * n);
    const int64_t M = n, K = nb;
    cudaMalloc(&W, 8 * M * K);
    cudaMalloc(&C, 8 * M * M);
    int bad = 0;
    // update GEMM alone: C -= W W^T (lower); W = the first K columns of a generated matrix
    abft_gen_spd(M, 5, C, M, nullptr);
    cudaMemcpy(W, C, 8 * M * K, cudaMemcpyDeviceToDevice);
    abft_gen_spd(M, 3, C, M, nullptr);
    int rc = abft_dev_gemm_nt(M, M, K, W, M, W, M, C, M, -1.0, 1.0, 1, nullptr);
    cudaDeviceSynchronize();
    printf("gemm_nt rc=%d (%s)\n", rc, cudaGetErrorString(cudaGetLastError()));
    bad |= rc != 0;
    if (argc > 3) { printf("%s\n", bad ? "FAIL" : "OK"); return bad; }   // GEMM only
    std::vector<abft_event_t> ev(64);
    for (int pass = 0; pass < 2; ++pass) {
        abft_gen_spd(n, n, A, n, nullptr);
        abft_report_t rep{};
        rep.cap = 64; rep.events = ev.data();
        abft_inject_spec_t inj[3] = {};
        inj[0] = {0, ABFT_HOOK_REST, ABFT_TGT_DATA, 0, 700, 300, 1ull << 52, 0, 0};
        inj[1] = {1, ABFT_HOOK_UPDATE_OUT, ABFT_TGT_DATA, 0, n - 5, 2 * nb + 17, 1ull << 51, 0, 0};
        inj[2].k = -1;
        rc = abft_potrf(n, nb, A, n, nullptr, pass ? inj : nullptr, &rep);
        printf("potrf pass %d rc=%d events=%lld checks=%lld (%s)\n", pass, rc, (long long)rep.n_events,
               (long long)rep.n_checks, cudaGetErrorString(cudaGetLastError()));
        bad |= rc != 0 || rep.n_events != (pass ? 2 : 0);
    }
    printf("%s\n", bad ? "FAIL" : "OK");
    return bad;
}
