// ipc.cu — peer-memory transport of the 1D block-cyclic multi-GPU path.
//
// One process per rank; every rank exports one device arena with cudaIpcGetMemHandle, the host
// exchanges the 64-byte handles out of band (torch.distributed in the Python binding), and every
// rank maps every peer's arena (cudaIpcOpenMemHandle: over NVLink/NVSwitch between GPUs, an alias of
// the same HBM when several ranks share one device, as the one-GPU test box does). The collectives
// run_dist needs are then plain peer loads and device-side flags, stream-ordered on the caller's
// stream, with no host round trip:
//   bcast       the root copies its panel into its arena and publishes a sequence number; every
//               receiver waits for it and pulls the panel straight out of the root's arena
//   allreduce   every rank publishes its vector, then reduces all arenas in rank order (the same
//               order on every rank, so every rank gets bit-identical sums)
//   allgather   every rank publishes its block, every rank pulls all blocks
// Arena reuse: before a rank overwrites its arena for collective s it waits until every peer has
// finished collective s-1 (each peer's `done` word). Flags use release/acquire at system scope.
#include <algorithm>
#include <cstring>
#include <vector>

#include "common.cuh"

namespace {

constexpr int kMaxRanks = 64;
constexpr size_t kCtlBytes = 256;   // flag words at the head of every arena

// posted/done: collective sequence numbers; panel: 1 + the last panel this rank pushed into its
// peers' receive buffers; freed: panels p < freed + 2 may be pushed into this rank's buffers
// (its update p - 2, the last reader of buffer p & 1, is complete)
// li: 1 + the last panel whose inv(L_kk) this rank (the diagonal block's owner, 2D) pushed
struct Ctl { unsigned long long posted, done, panel, freed, li; };

__device__ __forceinline__ unsigned long long ld_acquire_sys(const unsigned long long* p) {
    unsigned long long v;
    asm volatile("ld.acquire.sys.global.u64 %0, [%1];\n" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_release_sys(unsigned long long* p, unsigned long long v) {
    asm volatile("st.release.sys.global.u64 [%0], %1;\n" ::"l"(p), "l"(v) : "memory");
}

struct PeerTable { const Ctl* ctl[kMaxRanks]; const char* data[kMaxRanks]; };

// Wait until word `which` (0 posted, 1 done) of every rank in [0, np) except `skip` is >= v.
__global__ void k_ipc_wait(PeerTable t, int np, int skip, int which, unsigned long long v) {
    if (threadIdx.x != 0) return;
    for (int r = 0; r < np; ++r) {
        if (r == skip) continue;
        const unsigned long long* w = which == 0 ? &t.ctl[r]->posted : which == 1 ? &t.ctl[r]->done
                                    : which == 2 ? &t.ctl[r]->panel : which == 3 ? &t.ctl[r]->freed : &t.ctl[r]->li;
        while (ld_acquire_sys(w) < v) __nanosleep(256);
    }
}
__device__ __forceinline__ const unsigned long long* ctl_word(const Ctl* c, int which) {
    return which == 0 ? &c->posted : which == 1 ? &c->done : which == 2 ? &c->panel : which == 3 ? &c->freed : &c->li;
}
__global__ void k_ipc_wait_one(const Ctl* c, int which, unsigned long long v) {
    if (threadIdx.x != 0) return;
    const unsigned long long* w = ctl_word(c, which);
    while (ld_acquire_sys(w) < v) __nanosleep(256);
}
__global__ void k_ipc_set(Ctl* c, int which, unsigned long long v) {
    if (threadIdx.x == 0) {
        __threadfence_system();
        st_release_sys(const_cast<unsigned long long*>(ctl_word(c, which)), v);
    }
}
// buf[i] = op over ranks r = 0..np-1 (ascending) of data_r[i]; op 0 sum, 1 max
__global__ void k_ipc_reduce(PeerTable t, int np, double* buf, size_t count, int op) {
    for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < count; i += (size_t)gridDim.x * blockDim.x) {
        double a = reinterpret_cast<const double*>(t.data[0])[i];
        for (int r = 1; r < np; ++r) {
            const double b = __ldcg(reinterpret_cast<const double*>(t.data[r]) + i);
            a = op ? fmax(a, b) : a + b;
        }
        buf[i] = a;
    }
}

struct IpcTransport : DistTransport {
    char* mine = nullptr;                 // own arena (cudaMalloc, exported): [ctl | recv 0 | recv 1 | data]
    size_t cap = 0;                       // data bytes per arena (= bytes of each receive buffer)
    std::vector<char*> peer;              // mapped arenas (peer[rank] == mine)
    unsigned long long seq = 0;           // collectives issued (same sequence on every rank)
    // push-mode flag values of the current call are base + (panel index ...): every call moves base
    // past the previous call's range (same N and call sequence on every rank)
    unsigned long long base = 0, stride = 0;
    PeerTable table() const {
        PeerTable t;
        memset(&t, 0, sizeof t);
        for (int r = 0; r < nranks; ++r) { t.ctl[r] = reinterpret_cast<const Ctl*>(peer[r]); t.data[r] = data_of(r); }
        return t;
    }
    Ctl* my_ctl() const { return reinterpret_cast<Ctl*>(mine); }
    char* my_data() const { return mine + kCtlBytes + 2 * cap; }
    char* data_of(int r) const { return peer[r] + kCtlBytes + 2 * cap; }
    // push mode: receive buffer `slot` of rank r (mapped into this process)
    double* recv_buf(int r, int slot) override { return reinterpret_cast<double*>(peer[r] + kCtlBytes + slot * cap); }
    size_t recv_capacity() const override { return cap / sizeof(double); }
    int begin_call(int64_t N, cudaStream_t s) override {
        // the previous call on this comm finished on every rank (its closing collectives need every
        // rank's updates), so this rank's receive buffers are free: freed = the new base
        base += stride;
        stride = (unsigned long long)N + 4;
        k_ipc_set<<<1, 32, 0, s>>>(my_ctl(), 3, base);
        return cudaGetLastError() == cudaSuccess ? 0 : 1;
    }
    int wait_free(int64_t panel, cudaStream_t s) override {   // every peer finished update panel - 2
        const PeerTable t = table();
        k_ipc_wait<<<1, 32, 0, s>>>(t, nranks, rank, 3, base + (unsigned long long)(panel >= 1 ? panel - 1 : 0));
        return cudaGetLastError() == cudaSuccess ? 0 : 1;
    }
    int post_panel(int64_t panel, cudaStream_t s) override {
        k_ipc_set<<<1, 32, 0, s>>>(my_ctl(), 2, base + (unsigned long long)(panel + 1));
        return cudaGetLastError() == cudaSuccess ? 0 : 1;
    }
    int wait_panel(int root, int64_t panel, cudaStream_t s) override {
        k_ipc_wait_one<<<1, 32, 0, s>>>(reinterpret_cast<const Ctl*>(peer[root]), 2, base + (unsigned long long)(panel + 1));
        return cudaGetLastError() == cudaSuccess ? 0 : 1;
    }
    int post_li(int64_t panel, cudaStream_t s) override {
        k_ipc_set<<<1, 32, 0, s>>>(my_ctl(), 4, base + (unsigned long long)(panel + 1));
        return cudaGetLastError() == cudaSuccess ? 0 : 1;
    }
    int wait_li(int root, int64_t panel, cudaStream_t s) override {
        k_ipc_wait_one<<<1, 32, 0, s>>>(reinterpret_cast<const Ctl*>(peer[root]), 4, base + (unsigned long long)(panel + 1));
        return cudaGetLastError() == cudaSuccess ? 0 : 1;
    }
    int mark_free(int64_t value, cudaStream_t s) override {
        k_ipc_set<<<1, 32, 0, s>>>(my_ctl(), 3, base + (unsigned long long)value);
        return cudaGetLastError() == cudaSuccess ? 0 : 1;
    }
    // publish `bytes` from src into my arena as collective s (after every peer finished s-1)
    int publish(const void* src, size_t bytes, cudaStream_t s, const PeerTable& t) {
        if (bytes > cap) return 1;
        k_ipc_wait<<<1, 32, 0, s>>>(t, nranks, rank, 1, seq - 1);
        if (bytes && cudaMemcpyAsync(my_data(), src, bytes, cudaMemcpyDeviceToDevice, s) != cudaSuccess) return 1;
        k_ipc_set<<<1, 32, 0, s>>>(my_ctl(), 0, seq);
        return cudaGetLastError() == cudaSuccess ? 0 : 1;
    }
    int finish(cudaStream_t s) {
        k_ipc_set<<<1, 32, 0, s>>>(my_ctl(), 1, seq);
        return cudaGetLastError() == cudaSuccess ? 0 : 1;
    }
    int bcast(void* buf, size_t bytes, int root, cudaStream_t s) override {
        ++seq;
        const PeerTable t = table();
        if (rank == root) {
            if (publish(buf, bytes, s, t)) return 1;
        } else {
            if (bytes > cap) return 1;
            k_ipc_wait_one<<<1, 32, 0, s>>>(t.ctl[root], 0, seq);   // the root's panel of collective seq
            if (bytes && cudaMemcpyAsync(buf, data_of(root), bytes, cudaMemcpyDeviceToDevice, s) != cudaSuccess)
                return 1;
        }
        return finish(s);
    }
    int reduce(double* buf, size_t count, cudaStream_t s, int op) {
        ++seq;
        const PeerTable t = table();
        if (publish(buf, count * sizeof(double), s, t)) return 1;
        k_ipc_wait<<<1, 32, 0, s>>>(t, nranks, rank, 0, seq);
        k_ipc_reduce<<<(unsigned)std::min<size_t>((count + 255) / 256, 1024), 256, 0, s>>>(t, nranks, buf, count, op);
        return finish(s);
    }
    int allreduce_sum(double* buf, size_t count, cudaStream_t s) override { return reduce(buf, count, s, 0); }
    int allreduce_max(double* buf, size_t count, cudaStream_t s) override { return reduce(buf, count, s, 1); }
    int allgather(const void* send, void* recv, size_t bytes, cudaStream_t s) override {
        ++seq;
        const PeerTable t = table();
        if (publish(send, bytes, s, t)) return 1;
        k_ipc_wait<<<1, 32, 0, s>>>(t, nranks, rank, 0, seq);
        for (int r = 0; r < nranks; ++r)
            if (bytes && cudaMemcpyAsync((char*)recv + r * bytes, data_of(r), bytes, cudaMemcpyDeviceToDevice, s) !=
                             cudaSuccess)
                return 1;
        return finish(s);
    }
};

}  // namespace

// ---- the communicator object behind the C-ABI's void* comm (NCCL or peer-memory IPC) ----------
struct AbftComm {
    uint32_t magic;          // kCommMagic
    int kind;                // 0 NCCL, 1 IPC
    void* nccl;              // ncclComm_t
    IpcTransport* ipc;
};
static constexpr uint32_t kCommMagic = 0xABF7C033u;

AbftComm* abft_comm_cast(void* c) {
    AbftComm* a = reinterpret_cast<AbftComm*>(c);
    return (a && a->magic == kCommMagic) ? a : nullptr;
}
void* abft_comm_wrap_nccl(void* nccl) {
    AbftComm* a = new AbftComm{kCommMagic, 0, nccl, nullptr};
    return a;
}
DistTransport* abft_comm_ipc_transport(AbftComm* a) { return a ? a->ipc : nullptr; }
void* abft_comm_nccl(AbftComm* a) { return a ? a->nccl : nullptr; }
int abft_comm_kind(AbftComm* a) { return a ? a->kind : -1; }
void abft_comm_free(AbftComm* a) {
    if (!a) return;
    if (a->ipc) {
        for (int r = 0; r < a->ipc->nranks; ++r)
            if (a->ipc->peer[r] && a->ipc->peer[r] != a->ipc->mine) cudaIpcCloseMemHandle(a->ipc->peer[r]);
        if (a->ipc->mine) cudaFree(a->ipc->mine);
        delete a->ipc;
    }
    a->magic = 0;
    delete a;
}

extern "C" int abft_comm_init_ipc(void** comm, int nranks, int rank, int64_t cap_bytes, void* handle_out) {
    if (!comm) return -1;
    if (nranks < 1 || nranks > kMaxRanks) return -2;
    if (rank < 0 || rank >= nranks) return -3;
    if (cap_bytes < 0) return -4;
    if (!handle_out) return -5;
    IpcTransport* t = new IpcTransport;
    t->rank = rank; t->nranks = nranks; t->cap = (size_t)cap_bytes;
    if (cudaMalloc((void**)&t->mine, kCtlBytes + 3 * t->cap) != cudaSuccess) { delete t; return ABFT_ERR_CUDA; }
    cudaMemset(t->mine, 0, kCtlBytes);
    cudaDeviceSynchronize();
    cudaIpcMemHandle_t h;
    if (cudaIpcGetMemHandle(&h, t->mine) != cudaSuccess) { cudaFree(t->mine); delete t; return ABFT_ERR_CUDA; }
    static_assert(sizeof(cudaIpcMemHandle_t) == 64, "IPC handle is 64 bytes");
    memcpy(handle_out, &h, sizeof h);
    t->peer.assign(nranks, nullptr);
    t->peer[rank] = t->mine;
    *comm = new AbftComm{kCommMagic, 1, nullptr, t};
    return 0;
}

extern "C" int abft_comm_attach_ipc(void* comm, const void* handles) {
    AbftComm* a = abft_comm_cast(comm);
    if (!a || a->kind != 1) return -1;
    if (!handles) return -2;
    IpcTransport* t = a->ipc;
    for (int r = 0; r < t->nranks; ++r) {
        if (r == t->rank) continue;
        cudaIpcMemHandle_t h;
        memcpy(&h, (const char*)handles + 64 * r, sizeof h);
        void* p = nullptr;
        if (cudaIpcOpenMemHandle(&p, h, cudaIpcMemLazyEnablePeerAccess) != cudaSuccess) return ABFT_ERR_CUDA;
        t->peer[r] = (char*)p;
    }
    return 0;
}
