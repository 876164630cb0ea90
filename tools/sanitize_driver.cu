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
    // multi-GPU driver in the one-device harness: 1D (4 ranks) and 2D block-cyclic (2 x 2 grid),
    // each rank's block columns (J mod Pc == rank mod Pc) full height, fault-free + one RECV error
    const int64_t N = n / nb;
    for (int prows = 1; prows <= 2; ++prows) {
        const int P = 4, Pc = P / prows;
        abft_gen_spd(n, n, A, n, nullptr);
        std::vector<double*> loc(P, nullptr);
        for (int r = 0; r < P; ++r) {
            const int64_t nbl = (N - r % Pc + Pc - 1) / Pc;
            if (nbl <= 0) continue;
            cudaMalloc(&loc[r], 8 * n * nbl * nb);
            for (int64_t t = 0; t < nbl; ++t)
                cudaMemcpy(loc[r] + t * nb * n, A + (t * Pc + r % Pc) * nb * n, 8 * n * nb, cudaMemcpyDeviceToDevice);
        }
        abft_options_t o{};
        o.abft_enabled = 1; o.K = 1; o.c_tau = 64.0; o.prows = prows;
        for (int pass = 0; pass < 2; ++pass) {
            abft_report_t rep{};
            rep.cap = 64; rep.events = ev.data();
            abft_inject_spec_t inj[2] = {};
            // RECV on a rank that does not own panel tile (2, 1) (owner: (2 mod Pr) * Pc + 1 mod Pc)
            const int owner = (int)((2 % prows) * Pc + 1 % Pc);
            inj[0] = {1, ABFT_HOOK_RECV, ABFT_TGT_DATA, 0, 2 * nb + 7, nb + 3, 1ull << 50, (owner + 1) % P, 0};
            inj[1].k = -1;
            if (pass == 1) {   // restore the inputs
                for (int r = 0; r < P; ++r) {
                    const int64_t nbl = (N - r % Pc + Pc - 1) / Pc;
                    for (int64_t t = 0; t < nbl; ++t)
                        cudaMemcpy(loc[r] + t * nb * n, A + (t * Pc + r % Pc) * nb * n, 8 * n * nb, cudaMemcpyDeviceToDevice);
                }
            }
            rc = abft_potrf_dist_sim(n, nb, P, loc.data(), n, nullptr, pass ? inj : nullptr, &rep, &o);
            printf("dist_sim prows %d pass %d rc=%d events=%lld checks=%lld (%s)\n", prows, pass, rc,
                   (long long)rep.n_events, (long long)rep.n_checks, cudaGetErrorString(cudaGetLastError()));
            bad |= rc != 0 || rep.n_events != (pass ? 1 : 0);
        }
        for (double* p : loc) if (p) cudaFree(p);
    }
    printf("%s\n", bad ? "FAIL" : "OK");
    return bad;
}
