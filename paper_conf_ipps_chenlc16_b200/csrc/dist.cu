// dist.cu — NCCL transport of the 1D block-cyclic multi-GPU path.
//
// One process per GPU; rank r owns block columns {J : J mod P = r}. Per iteration the owner of
// block column k broadcasts the packed panel W = [L(k+1:N,k); chk(k:N,k)] over NVLink/NVSwitch
// with ncclBroadcast (in place, on the caller's stream); the scales are all-reduced once at the
// start, the report's counters and events are all-reduced / all-gathered at the end. The
// factorisation itself is run_dist() in abft.cu (shared with the single-process simulation that
// replaces the broadcast by device copies, abft_potrf_dist_sim).
#include <nccl.h>

#include <cstring>

#include "common.cuh"

namespace {
struct NcclTransport : DistTransport {
    ncclComm_t comm;
    int bcast(void* buf, size_t bytes, int root, cudaStream_t s) override {
        return ncclBroadcast(buf, buf, bytes, ncclUint8, root, comm, s) == ncclSuccess ? 0 : 1;
    }
    int allreduce_sum(double* buf, size_t count, cudaStream_t s) override {
        return ncclAllReduce(buf, buf, count, ncclDouble, ncclSum, comm, s) == ncclSuccess ? 0 : 1;
    }
    int allreduce_max(double* buf, size_t count, cudaStream_t s) override {
        return ncclAllReduce(buf, buf, count, ncclDouble, ncclMax, comm, s) == ncclSuccess ? 0 : 1;
    }
    int allgather(const void* send, void* recv, size_t bytes, cudaStream_t s) override {
        return ncclAllGather(send, recv, bytes, ncclUint8, comm, s) == ncclSuccess ? 0 : 1;
    }
};
}  // namespace

extern "C" int abft_nccl_id(void* id128) {
    if (!id128) return -1;
    ncclUniqueId id;
    if (ncclGetUniqueId(&id) != ncclSuccess) return ABFT_ERR_NCCL;
    static_assert(sizeof(ncclUniqueId) == 128, "ncclUniqueId is 128 bytes");
    memcpy(id128, &id, sizeof id);
    return 0;
}

struct AbftComm;
AbftComm* abft_comm_cast(void* c);
void* abft_comm_wrap_nccl(void* nccl);
DistTransport* abft_comm_ipc_transport(AbftComm* a);
void* abft_comm_nccl(AbftComm* a);
int abft_comm_kind(AbftComm* a);
void abft_comm_free(AbftComm* a);

extern "C" int abft_comm_init(void** comm, int nranks, const void* id128, int rank) {
    if (!comm) return -1;
    if (nranks < 1) return -2;
    if (!id128) return -3;
    if (rank < 0 || rank >= nranks) return -4;
    ncclUniqueId id;
    memcpy(&id, id128, sizeof id);
    ncclComm_t c;
    if (ncclCommInitRank(&c, nranks, id, rank) != ncclSuccess) return ABFT_ERR_NCCL;
    *comm = abft_comm_wrap_nccl((void*)c);
    return 0;
}

extern "C" int abft_comm_destroy(void* comm) {
    AbftComm* a = abft_comm_cast(comm);
    if (!a) return -1;
    int rc = 0;
    if (abft_comm_kind(a) == 0 && ncclCommDestroy((ncclComm_t)abft_comm_nccl(a)) != ncclSuccess) rc = ABFT_ERR_NCCL;
    abft_comm_free(a);
    return rc;
}

extern "C" int abft_potrf_dist(int64_t n, int64_t nb, double* A_local, int64_t lda_local, void* comm, int rank,
                               int nranks, abft_stream_t stream, const abft_inject_spec_t* inj, abft_report_t* rep,
                               const abft_options_t* opt) {
    if (n < 0) return -1;
    if (nb < 1 || n % nb) return -2;
    const int64_t N = n / nb;
    if (nranks < 1) return -7;
    if (rank < 0 || rank >= nranks) return -6;
    if (!A_local && (N - rank + nranks - 1) / nranks > 0) return -3;
    if (lda_local < (n > 1 ? n : 1)) return -4;
    AbftComm* a = abft_comm_cast(comm);
    if (!a) return -5;
    DistLocal me{rank, A_local, lda_local};
    if (abft_comm_kind(a) == 1) {   // peer-memory (CUDA IPC) transport
        DistTransport* t = abft_comm_ipc_transport(a);
        if (t->rank != rank || t->nranks != nranks) return -5;
        return run_dist(n, nb, nranks, &me, 1, t, (cudaStream_t)stream, inj, rep, opt);
    }
    NcclTransport tp;
    tp.comm = (ncclComm_t)abft_comm_nccl(a);
    tp.rank = rank; tp.nranks = nranks;
    int cr = 0, cn = 0;
    if (ncclCommUserRank(tp.comm, &cr) != ncclSuccess || ncclCommCount(tp.comm, &cn) != ncclSuccess) return ABFT_ERR_NCCL;
    if (cr != rank || cn != nranks) return -5;
    return run_dist(n, nb, nranks, &me, 1, &tp, (cudaStream_t)stream, inj, rep, opt);
}
