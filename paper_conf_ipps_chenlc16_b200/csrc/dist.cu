// dist.cu — multi-GPU entry points (placeholder until the NCCL path lands).
#include "common.cuh"
extern "C" int abft_nccl_id(void* id128) { (void)id128; return ABFT_ERR_NCCL; }
extern "C" int abft_comm_init(void** comm, int nranks, const void* id128, int rank) {
    (void)comm; (void)nranks; (void)id128; (void)rank; return ABFT_ERR_NCCL; }
extern "C" int abft_comm_destroy(void* comm) { (void)comm; return ABFT_ERR_NCCL; }
extern "C" int abft_potrf_dist(int64_t, int64_t, double*, int64_t, void*, int, int, abft_stream_t,
                               const abft_inject_spec_t*, abft_report_t*, const abft_options_t*) {
    return ABFT_ERR_NCCL;
}
