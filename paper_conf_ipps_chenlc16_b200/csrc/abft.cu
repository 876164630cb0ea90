// abft.cu — the C-ABI entry points and the single-GPU factorisation driver.
//
// Iteration k of the right-looking Enhanced Online-ABFT Cholesky (reading A1; the paper's
// Alg. 1 is left-looking), with verification before every read
// in the V1..V6 schedule of DESIGN.md §2:
//   REST(k) hook -> V1/V2 check of block column k (pre-read, unfactored)
//   POTRF + inv(L_kk)  (potrf.cu)
//   TRSM: W = [A(k+1:N,k); chk(k:N,k)] * inv(L_kk)^T  -- one DMMA GEMM that also performs Alg. 2
//         on the checksum rows of tile (k,k)
//   POTRF_OUT hook -> V3 (L_kk vs Alg.-2 checksums);  TRSM_OUT hook -> V4 (solved panel, in W)
//   write-back W -> A panel, chk
//   trailing SYRK/GEMM: A(trail) -= W_d W_d^T (lower), chk(trail) -= W_c W_d^T
//   UPDATE_OUT hook -> V5 (every trailing tile, every K-th iteration: Opt. 3)
// then REST(N) -> V6 over L. Everything is stream-ordered; the only host sync is the final
// report copy. An UNCORRECTABLE / NOT_SPD sets a device abort flag that every later kernel
// checks at entry.
#include <algorithm>
#include <cstdio>
#include <cstring>
#include <tuple>
#include <utility>
#include <vector>

#include "common.cuh"

using namespace abft;

int launch_check(const StageArgs& a, cudaStream_t s);
int launch_check_v5_fused(const StageArgs& diag, const StageArgs& off, cudaStream_t s);
int launch_check2(const StageArgs& a0, const StageArgs& a1, cudaStream_t s);

// Is there an injection at (k, hook)? (A hook between two checks keeps them in separate launches.)
static bool has_inj(const std::vector<abft_inject_spec_t>& list, int64_t k, int hook) {
    for (const auto& sp : list) if (sp.k == k && sp.hook == hook) return true;
    return false;
}
int launch_scales(int64_t n, int64_t nb, const double* A, int64_t lda, double* scl, cudaStream_t s, int nchk = 2);
int launch_copy(int64_t rows, int64_t cols, const double* src, int64_t lds, double* dst, int64_t ldd,
                const int32_t* abort_flag, cudaStream_t s);
int launch_zero(int64_t rows, int64_t cols, double* dst, int64_t ldd, cudaStream_t s);
size_t chol_sync_bytes(int64_t nb);
int launch_chol_inv(double* T, int64_t ldt, double* Li, int64_t B, int64_t info_off, double* tmp,
                    DevState* st, cudaStream_t s);
int launch_gen_spd(int64_t n, uint64_t seed, double* A, int64_t lda, cudaStream_t s);
int launch_inject(int nops, double* const* ptrs, const uint64_t* masks, const int32_t* abort_flag,
                  cudaStream_t s);
int launch_axpy(int64_t n, const double* x, double* y, cudaStream_t s);
int launch_abort_to_slot(const int32_t* abort_flag, double* slot, cudaStream_t s);
int launch_abort_from_slot(const double* slot, DevState* st, cudaStream_t s);
int launch_scales_diag(int64_t nrows, const double* Adiag, int64_t lda, double* s_out, cudaStream_t s);
int launch_scales_blocks(int64_t N, int64_t nb, const double* sv, double* S1, double* S2, cudaStream_t s);

// ---- diagnostics --------------------------------------------------------------------------
static thread_local int64_t g_launches = 0;
static thread_local char g_err[256] = {0};
void abft_count_launch(int n) { g_launches += n; }
void abft_set_error(cudaError_t e, const char* what) {
    snprintf(g_err, sizeof g_err, "%s: %s", what, cudaGetErrorString(e));
}
extern "C" int64_t abft_last_launch_count(void) { return g_launches; }
extern "C" const char* abft_version(void) {
    return "libabft 0.1 (sm_100a, DMMA f64; Enhanced Online-ABFT Cholesky, Chen-Liang-Chen IPDPS'16)";
}
extern "C" const char* abft_last_error(void) { return g_err; }

// ---- argument checking ----------------------------------------------------------------------
static int check_common(int64_t n, int64_t nb, const void* A, int64_t lda) {
    if (n < 0) return -1;
    if (nb < 1 || n % nb != 0) return -2;
    if (A == nullptr && n > 0) return -3;
    if (lda < std::max<int64_t>(1, n)) return -4;
    return 0;
}

// Injection specs: validated against the region their hook can touch.
static int collect_inj(const abft_inject_spec_t* inj, int64_t n, int64_t nb, std::vector<abft_inject_spec_t>& out,
                       int order = ABFT_ORDER_RIGHT, int nchk = 2) {
    out.clear();
    if (!inj) return 0;
    const int64_t N = n / nb;
    for (int t = 0; inj[t].k != -1; ++t) {
        const abft_inject_spec_t& s = inj[t];
        if (t > 1 << 20) return -1;
        if (s.hook < ABFT_HOOK_REST || s.hook > ABFT_HOOK_RECV) return -1;
        if (s.target != ABFT_TGT_DATA && s.target != ABFT_TGT_CHK) return -1;
        if (s.k < 0 || s.k > N || (s.hook != ABFT_HOOK_REST && s.k >= N)) return -1;
        int64_t I, J;
        if (s.target == ABFT_TGT_DATA) {
            if (s.col < 0 || s.row < s.col || s.row >= n) return -1;
            I = s.row / nb; J = s.col / nb;
        } else {
            if (s.row < 0 || s.row >= nchk * N || s.col < 0 || s.col >= n) return -1;
            I = s.row / nchk; J = s.col / nb;
            if (J > I) return -1;
        }
        const int64_t k = s.k;
        switch (s.hook) {
            case ABFT_HOOK_POTRF_OUT: if (!(I == k && J == k)) return -1; break;
            case ABFT_HOOK_TRSM_OUT: if (!(J == k && I > k)) return -1; break;
            case ABFT_HOOK_UPDATE_OUT:   // the block columns the update of iteration k writes
                if (order == ABFT_ORDER_LEFT ? !(J == k && k > 0) : !(J > k)) return -1;
                break;
            case ABFT_HOOK_RECV: if (!(J == k && I > k)) return -1; break;
            default: break;
        }
        out.push_back(s);
    }
    return 0;
}

namespace abft { bool is_update_kernel(const void* f); }

// ---- workspace -------------------------------------------------------------------------------
struct Work {
    int64_t n, nb, N;
    int nchk = 2;                                 // checksum rows per block (2, or 3: reading B10)
    double* chk = nullptr; int64_t ldc = 1;
    double* scl = nullptr;
    double* W = nullptr;
    double* Li = nullptr;
    double* tmp = nullptr;
    DevState* st = nullptr;
    abft_event_t* ev = nullptr; int64_t ev_cap = 0;
    double* cs = nullptr; int64_t cs_nslab = 0;   // fused-V5 partials (nb % 128 == 0)
};

static int work_alloc(Work& w, int64_t n, int64_t nb, int64_t ncols_local, int64_t ev_cap, bool abft, cudaStream_t s,
                      int nchk = 2) {
    w.n = n; w.nb = nb; w.N = n / nb; w.nchk = nchk;
    const int64_t N = w.N;
    w.ldc = std::max<int64_t>(1, nchk * N);
    if (abft) {
        ABFT_CUDA_TRY(cudaMallocAsync((void**)&w.chk, sizeof(double) * (size_t)(w.ldc * std::max<int64_t>(1, ncols_local)), s));
        ABFT_CUDA_TRY(cudaMallocAsync((void**)&w.scl, sizeof(double) * (size_t)(n + 3 * N + 1), s));
    }
    const int64_t wrows = (N - 1) * nb + nchk * N + nchk + 1;
    ABFT_CUDA_TRY(cudaMallocAsync((void**)&w.W, sizeof(double) * (size_t)(std::max<int64_t>(wrows, 1) * nb), s));
    ABFT_CUDA_TRY(cudaMallocAsync((void**)&w.Li, sizeof(double) * (size_t)(nb * nb), s));
    ABFT_CUDA_TRY(cudaMallocAsync((void**)&w.tmp, sizeof(double) * (size_t)(((nb + 1) / 2 + 64) * ((nb + 1) / 2 + 64)), s));
    ABFT_CUDA_TRY(cudaMemsetAsync(w.tmp, 0, chol_sync_bytes(nb), s));   // task-graph POTRF sync words
    ABFT_CUDA_TRY(cudaMallocAsync((void**)&w.st, sizeof(DevState), s));
    ABFT_CUDA_TRY(cudaMemsetAsync(w.st, 0, sizeof(DevState), s));
    w.ev_cap = std::max<int64_t>(ev_cap, 1);
    ABFT_CUDA_TRY(cudaMallocAsync((void**)&w.ev, sizeof(abft_event_t) * (size_t)w.ev_cap, s));
    return 0;
}

static void work_free(Work& w, cudaStream_t s) {
    if (w.chk) cudaFreeAsync(w.chk, s);
    if (w.scl) cudaFreeAsync(w.scl, s);
    if (w.W) cudaFreeAsync(w.W, s);
    if (w.Li) cudaFreeAsync(w.Li, s);
    if (w.tmp) cudaFreeAsync(w.tmp, s);
    if (w.st) cudaFreeAsync(w.st, s);
    if (w.ev) cudaFreeAsync(w.ev, s);
    if (w.cs) cudaFreeAsync(w.cs, s);
    w = Work();
}

static StageArgs stage_base(const Work& w, double* A, int64_t lda, double c_tau, int kind, int V, int k) {
    StageArgs a;
    memset(&a, 0, sizeof a);
    a.kind = kind; a.V = V; a.k = k; a.factored = 0; a.correct = 1; a.rank = 0; a.encode = 0;
    a.n = w.n; a.nb = w.nb; a.N = w.N;
    a.A = A; a.lda = lda; a.chk = w.chk; a.ldc = w.ldc; a.W = w.W; a.ldw = 1; a.mB = 0;
    a.s = w.scl; a.S1 = w.scl ? w.scl + w.n : nullptr; a.S2 = w.scl ? w.scl + w.n + w.N : nullptr;
    a.S3 = w.scl ? w.scl + w.n + 2 * w.N : nullptr; a.nchk = w.nchk;
    a.c_tau = c_tau; a.col_owner_mod = 1; a.col_owner_rank = 0;
    a.row_owner_mod = 1; a.row_owner_rank = 0; a.own_invert = 0;
    a.st = w.st; a.ev = w.ev; a.ev_cap = w.ev_cap;
    a.flist = 0; a.j_lo = k + 1; a.j_hi = w.N;
    return a;
}

// Fill the host report from the device state (the one synchronisation of a call).
static int finish_report(const Work& w, abft_report_t* rep, cudaStream_t s, int* status_out) {
    std::vector<char> hbuf(sizeof(DevState));
    DevState& hs = *reinterpret_cast<DevState*>(hbuf.data());
    ABFT_CUDA_TRY(cudaMemcpyAsync(&hs, w.st, offsetof(DevState, fl), cudaMemcpyDeviceToHost, s));
    ABFT_CUDA_TRY(cudaStreamSynchronize(s));
    const int64_t nev = (int64_t)hs.nev;
    if (rep) {
        rep->info = hs.info;
        rep->n_checks = (int64_t)hs.n_checks; rep->n_detected = hs.n_detected; rep->n_data = hs.n_data;
        rep->n_nonfinite = hs.n_nonfinite; rep->n_chk1 = hs.n_chk1; rep->n_chk2 = hs.n_chk2;
        rep->n_uncorrectable = hs.n_unc; rep->n_events = nev;
        { double q; memcpy(&q, &hs.max_ratio_bits, sizeof q); rep->max_noise_ratio = q; }
        const int64_t ncopy = std::min<int64_t>(std::min<int64_t>(nev, w.ev_cap), std::max<int64_t>(rep->cap, 0));
        if (ncopy > 0 && rep->events) {
            ABFT_CUDA_TRY(cudaMemcpy(rep->events, w.ev, sizeof(abft_event_t) * (size_t)ncopy, cudaMemcpyDeviceToHost));
            std::sort(rep->events, rep->events + ncopy, [](const abft_event_t& x, const abft_event_t& y) {
                if (x.k != y.k) return x.k < y.k;
                if (x.check != y.check) return x.check < y.check;
                if (x.tile_j != y.tile_j) return x.tile_j < y.tile_j;
                if (x.tile_i != y.tile_i) return x.tile_i < y.tile_i;
                if (x.col != y.col) return x.col < y.col;
                if (x.row != y.row) return x.row < y.row;
                return x.rank < y.rank;
            });
        }
    }
    *status_out = hs.status;
    return 0;
}

// Injection pointer at hook time (where the element lives at that moment).
struct Loc { double* A; int64_t lda; double* chk; int64_t ldc; double* W; int64_t ldw; int64_t mB; int nchk = 2; };

static double* inj_ptr(const abft_inject_spec_t& s, int64_t k, int64_t nb, const Loc& L) {
    const int hook = s.hook;
    if (hook == ABFT_HOOK_TRSM_OUT || hook == ABFT_HOOK_POTRF_OUT) {
        if (s.target == ABFT_TGT_DATA) {
            if (hook == ABFT_HOOK_TRSM_OUT)
                return L.W + (s.col - k * nb) * L.ldw + (s.row - (k + 1) * nb);
            return L.A + s.col * L.lda + s.row;
        }
        return L.W + (s.col - k * nb) * L.ldw + L.mB + (s.row - L.nchk * k);
    }
    if (s.target == ABFT_TGT_DATA) return L.A + s.col * L.lda + s.row;
    return L.chk + s.col * L.ldc + s.row;
}

static void do_inject(const std::vector<abft_inject_spec_t>& list, int64_t k, int hook, int64_t nb, const Loc& L,
                      const int32_t* ab, cudaStream_t s) {
    std::vector<double*> ptrs; std::vector<uint64_t> masks;
    for (const auto& sp : list)
        if (sp.k == k && sp.hook == hook) { ptrs.push_back(inj_ptr(sp, k, nb, L)); masks.push_back(sp.xor_mask); }
    if (!ptrs.empty()) launch_inject((int)ptrs.size(), ptrs.data(), masks.data(), ab, s);
}

// ---- per-thread caches: the look-ahead stream and CUDA events are created once and reused, so
// a call's host-side set-up / tear-down stays a few microseconds (it is inside the caller's timing)
struct EventPool {
    std::vector<cudaEvent_t> ev; size_t used = 0; unsigned flags;
    explicit EventPool(unsigned f) : flags(f) {}
    cudaEvent_t get() {
        if (used == ev.size()) { cudaEvent_t e; cudaEventCreateWithFlags(&e, flags); ev.push_back(e); }
        return ev[used++];
    }
    void reset() { used = 0; }
};
struct ThreadCache {
    int device = -1;
    cudaStream_t P = nullptr;
    cudaStream_t P2 = nullptr;   // panel side stream: V2 runs here while P factors the diagonal block
    cudaStream_t C = nullptr;    // copy stream of abft_potrf_host's overlapped write-back
    cudaStream_t Cin = nullptr;  // copy stream of abft_potrf_host's streamed input
    EventPool sync{cudaEventDisableTiming};
    EventPool timing{cudaEventDefault};
};
static thread_local ThreadCache g_tc;
static ThreadCache& thread_cache() {
    int dev = 0; cudaGetDevice(&dev);
    if (g_tc.device != dev) {   // first use on this device (events/streams belong to a device)
        g_tc.sync = EventPool(cudaEventDisableTiming);
        g_tc.timing = EventPool(cudaEventDefault);
        int lo = 0, hi = 0;
        cudaDeviceGetStreamPriorityRange(&lo, &hi);
        const char* pe = getenv("ABFT_P_PRIO");   // dev knob: 0 = default priority for the panel stream
        cudaStreamCreateWithPriority(&g_tc.P, cudaStreamNonBlocking, (pe && atoi(pe) == 0) ? lo : hi);
        cudaStreamCreateWithPriority(&g_tc.P2, cudaStreamNonBlocking, (pe && atoi(pe) == 0) ? lo : hi);
        // keep the workspace's pages mapped between calls: cudaMallocAsync / cudaFreeAsync then
        // cost microseconds instead of re-mapping ~n*nb*8*4 bytes at every call
        cudaMemPool_t pool;
        if (cudaDeviceGetDefaultMemPool(&pool, dev) == cudaSuccess) {
            uint64_t keep = UINT64_MAX;
            cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &keep);
        }
        g_tc.device = dev;
    }
    g_tc.sync.reset(); g_tc.timing.reset();
    return g_tc;
}

// ---- per-phase profiler (options.profile) ----------------------------------------------------
enum { PH_ENCODE, PH_V12, PH_POTRF, PH_TRSM, PH_V3, PH_V4, PH_WB, PH_UPD, PH_UPDC, PH_V5, PH_V6, PH_INJ, PH_WAIT };
static const char* kPhaseNames[ABFT_NPHASE] = {"encode", "v1v2", "potrf_inv", "trsm", "v3", "v4", "writeback",
                                               "update", "update_chk", "v5", "v6", "inject", "wait_panel"};
static thread_local abft_profile_t g_prof;

struct Profiler {
    bool on = false;
    EventPool* pool = nullptr;
    struct Rec { int ph; cudaEvent_t a, b; double flops, bytes; };
    std::vector<Rec> recs;
    // begin() returns a token; end() closes it (phases may be open on two streams at once)
    cudaEvent_t begin(cudaStream_t s) {
        if (!on) return nullptr;
        cudaEvent_t e = pool->get(); cudaEventRecord(e, s); return e;
    }
    void end(cudaEvent_t tok, int ph, cudaStream_t s, double flops = 0, double bytes = 0) {
        if (!on || !tok) return;
        cudaEvent_t e = pool->get(); cudaEventRecord(e, s);
        recs.push_back({ph, tok, e, flops, bytes});
    }
    void finish() {   // after a stream sync
        if (!on) return;
        memset(&g_prof, 0, sizeof g_prof);
        g_prof.nphase = ABFT_NPHASE;
        for (auto& r : recs) {
            float ms = 0; cudaEventElapsedTime(&ms, r.a, r.b);
            g_prof.ms[r.ph] += ms; g_prof.launches[r.ph] += 1;
            g_prof.flops[r.ph] += r.flops; g_prof.bytes[r.ph] += r.bytes;
        }
        recs.clear();
    }
};

extern "C" int abft_last_profile(abft_profile_t* out) {
    if (!out) return -1;
    *out = g_prof;
    return 0;
}
extern "C" const char* abft_phase_name(int phase) {
    return (phase >= 0 && phase < ABFT_NPHASE) ? kPhaseNames[phase] : "";
}

// Column-block filter for an injection (which block column J its target lives in).
static int64_t inj_col_block(const abft_inject_spec_t& sp, int64_t nb) { return sp.col / nb; }

static void do_inject_if(const std::vector<abft_inject_spec_t>& list, int64_t k, int hook, int64_t nb, const Loc& L,
                         const int32_t* ab, cudaStream_t s, int64_t jlo, int64_t jhi, bool inside) {
    std::vector<double*> ptrs; std::vector<uint64_t> masks;
    for (const auto& sp : list) {
        if (sp.k != k || sp.hook != hook) continue;
        const int64_t J = inj_col_block(sp, nb);
        const bool in = J >= jlo && J < jhi;
        if (in != inside) continue;
        ptrs.push_back(inj_ptr(sp, k, nb, L)); masks.push_back(sp.xor_mask);
    }
    if (!ptrs.empty()) launch_inject((int)ptrs.size(), ptrs.data(), masks.data(), ab, s);
}

// The single-GPU driver with depth-1 look-ahead: the panel of iteration k+1
// (V1/V2, POTRF + inverse, TRSM, V3, V4, write-back) runs on a high-priority stream P as soon
// as block column k+1 has received update k and its V5 check, while the main stream S applies
// the rest of update k and V5 to the trailing matrix. Hook timing and the set of events are
// those of the sequential schedule: injections and checks are split by block column exactly
// where the two streams split the work.
// abft_potrf_host's write-back of L overlapped with the factorisation: block column k of L is
// final once panel k is written back (only V6 can still correct it, which the host path checks),
// so it is copied to the host on a copy stream while the trailing updates continue.
struct HostSink {
    double* host = nullptr;
    int64_t ldh = 0;
    cudaStream_t cs = nullptr;
};
static thread_local HostSink g_sink;
// abft_potrf_host's input streamed in behind the factorisation's start: the block columns arrive
// on a copy stream (first every diagonal tile — the threshold scales need the whole diagonal —
// then each column below its diagonal tile, in order); ev[0] marks the diagonal tiles, ev[1 + k]
// block column k. The encode of later block columns and update 0 then run in column chunks as
// their data lands, overlapped with the transfer of the rest.
struct HostSource {
    bool active = false;
    std::vector<cudaEvent_t> ev;
};
static thread_local HostSource g_src;

// Buffers owned by a captured graph (graph mode, see run_graph): run_potrf then only enqueues the
// work (resets, kernels, cross-stream events) and leaves the report to the caller.
struct Persist {
    Work w;
    double* W1 = nullptr;
};

// Dev knob ABFT_DEV_ABLATE (bit mask; overhead attribution only — results are NOT protected and
// checks may flag stale checksums, so it is for timing fault-free runs): 1 no checksum rows in the
// TRSM / update / write-back, 2 no V5, 4 no V1-V4, 8 no fused V5 partials, 16 no encode / V6.
static int dev_ablate() {
    static int v = -1;
    if (v < 0) { const char* e = getenv("ABFT_DEV_ABLATE"); v = e ? atoi(e) : 0; }
    return v;
}

static int run_potrf(int64_t n, int64_t nb, double* A, int64_t lda, cudaStream_t s,
                     const std::vector<abft_inject_spec_t>& inj, abft_report_t* rep, const abft_options_t& o,
                     Persist* ps = nullptr) {
    const bool abft = o.abft_enabled != 0;
    const int abl = abft ? dev_ablate() : 0;
    const int K = std::max(1, o.K);
    Work w;
    int rc = 0;
    if (ps) {
        w = ps->w;
        ABFT_CUDA_TRY(cudaMemsetAsync(w.st, 0, sizeof(DevState), s));
        ABFT_CUDA_TRY(cudaMemsetAsync(w.tmp, 0, chol_sync_bytes(nb), s));
        rep = nullptr;
    } else {
        rc = work_alloc(w, n, nb, n, rep ? std::max<int64_t>(rep->cap, 1) : 1024, abft, s, o.nchk == 3 ? 3 : 2);
        if (rc) return rc;
    }
    const int64_t N = w.N, B = nb;
    const int64_t nc = w.nchk;                                   // checksum rows per block (2 or 3)
    const double Bd = (double)B;
    const int32_t* ab = &w.st->abort;
    // fused V5 partials: 64-row slabs x n columns x {v1, v2 (, v3)}
    const int mode = o.mode;
    const bool can_fuse = abft && mode != ABFT_MODE_OFFLINE && (nb % 128 == 0) && (lda % 2 == 0) &&
                          (((uintptr_t)A & 15) == 0) && !getenv("ABFT_NOFUSE") && !(abl & 8);   // dev knob: V5 re-reads
    if (can_fuse && !ps) {
        w.cs_nslab = n / 32;   // room for 32-row slabs (the smallest warp-tile height)
        ABFT_CUDA_TRY(cudaMallocAsync((void**)&w.cs, sizeof(double) * (size_t)(nc * w.cs_nslab * n), s));
    }
    if (ps && can_fuse && !w.cs) return ABFT_ERR_CUDA;
    // second panel buffer for the look-ahead
    double* Wbuf[2] = {w.W, ps ? ps->W1 : nullptr};
    const int64_t wrows = (N - 1) * nb + nc * N + nc + 1;
    if (!ps)
        ABFT_CUDA_TRY(cudaMallocAsync((void**)&Wbuf[1], sizeof(double) * (size_t)(std::max<int64_t>(wrows, 1) * nb), s));
    ThreadCache& tc = thread_cache();
    cudaStream_t P = tc.P;
    auto new_event = [&]() { return tc.sync.get(); };
    cudaEvent_t e0 = nullptr, e1 = nullptr;
    if (rep) { e0 = tc.timing.get(); e1 = tc.timing.get(); cudaEventRecord(e0, s); }
    Profiler prof; prof.on = o.profile != 0 && !ps; prof.pool = &tc.timing;
    const double lowerB = Bd * (Bd + 1) / 2;                 // elements of a tril tile
    launch_zero(B, B, w.Li, B, s);
    // encode: block column 0 first, then the panel stream may start (panel 0
    // reads only column 0's checksums), and the rest of the matrix is encoded on S concurrently
    // with panel 0 — before update 0, the first reader of those checksums (reading B9)
    cudaEvent_t t_enc = nullptr;
    // streamed input (abft_potrf_host): the diagonal tiles and block column 0 before anything reads
    // them; the other block columns are awaited chunk by chunk (ensure_chunk) before their encode
    const bool src = g_src.active && !ps && nc == 2 && N >= 2 && (int64_t)g_src.ev.size() >= N + 1;
    constexpr int64_t kSrcChunk = 8;   // block columns per chunk of the streamed input
    std::vector<char> chunk_done(src ? (size_t)((N + kSrcChunk - 1) / kSrcChunk) : 0, 0);
    if (src) { cudaStreamWaitEvent(s, g_src.ev[0], 0); cudaStreamWaitEvent(s, g_src.ev[1], 0); }
    else if (g_src.active && !ps && (int64_t)g_src.ev.size() >= N + 1) cudaStreamWaitEvent(s, g_src.ev[N], 0);   // all of it
    auto ensure_chunk = [&](int64_t c) {   // chunk c = block columns [c kSrcChunk, (c + 1) kSrcChunk)
        if (!src || chunk_done[(size_t)c]) return;
        const int64_t J0 = std::max<int64_t>(1, c * kSrcChunk), J1 = std::min<int64_t>(N, (c + 1) * kSrcChunk);
        chunk_done[(size_t)c] = 1;
        if (J0 >= J1) return;
        cudaStreamWaitEvent(s, g_src.ev[1 + J1 - 1], 0);   // in-order copies: the chunk's last column
        if (abft && !(abl & 16)) {
            StageArgs a = stage_base(w, A, lda, o.c_tau, SK_TRAIL, 0, 0);
            a.j_lo = J0; a.j_hi = J1; a.encode = 1;
            launch_check(a, s);
        }
    };
    if (abft && !(abl & 16)) {
        t_enc = prof.begin(s);
        launch_scales(n, nb, A, lda, w.scl, s, (int)nc);
        StageArgs a = stage_base(w, A, lda, o.c_tau, SK_COLUMN, 0, 0);
        a.encode = 1;
        launch_check(a, s);
    }
    {   // P starts after everything enqueued on S so far
        cudaEvent_t e = new_event(); cudaEventRecord(e, s); cudaStreamWaitEvent(P, e, 0);
    }
    if (abft && !(abl & 16)) {
        if (N > 1 && !src) {
            StageArgs a = stage_base(w, A, lda, o.c_tau, SK_TRAIL, 0, 0);
            a.j_lo = 1; a.j_hi = N; a.encode = 1;
            launch_check(a, s);
        }
        const double el = (double)(N * (N - 1) / 2) * Bd * Bd + (double)N * lowerB;
        prof.end(t_enc, PH_ENCODE, s, 4.0 * el, 8.0 * el);
    }

    // ABFT_WB_EARLY=1: the main stream starts update k+1 as soon as panel k passed V3/V4 and the
    // write-back of L(:,k) runs behind it (measured: -0.15 ms wait_panel but +1.2 ms of update at
    // C4 from the concurrent write-back, profiles/r02/ab_wb_early.txt; off by default)
    static const bool wb_early = [] { const char* e = getenv("ABFT_WB_EARLY"); return e && !strcmp(e, "1"); }();
    // ---- the panel of iteration k, on stream P ----
    auto panel = [&](int64_t k) {
        const int64_t m = N - k - 1, mB = m * B;
        const int64_t ldw = std::max<int64_t>(1, (mB + nc * m + nc + 1) / 2 * 2);   // even: 16-byte columns
        double* W = Wbuf[k & 1];
        double* Akk = A + k * B * lda + k * B;
        const Loc L{A, lda, w.chk, w.ldc, W, ldw, mB, (int)nc};
        const double md = (double)m, mBd = (double)mB;
        Work wk = w; wk.W = W;
        if (abft) do_inject_if(inj, k, ABFT_HOOK_REST, B, L, ab, P, k, k + 1, true);   // REST(k) into column k
        cudaEvent_t v2done = nullptr;
        if (abft && mode == ABFT_MODE_ENHANCED && !(abl & 4)) {
            // V1 (tile k,k) gates POTRF; V2 (the tiles below) only has to precede the TRSM, so it
            // runs on the side stream P2 while P factors the diagonal block (same checks, same
            // events: both are labelled V2 as one column stage; separate flag lists)
            StageArgs a1 = stage_base(wk, A, lda, o.c_tau, m > 0 ? SK_COL_DIAG : SK_COLUMN, ABFT_V2, (int)k);
            a1.flist = 1;
            cudaEvent_t t = prof.begin(P);
            launch_check(a1, P);                                                 // V1
            prof.end(t, PH_V12, P, 4.0 * lowerB, 8.0 * lowerB);
            if (m > 0) {
                cudaEvent_t f = new_event();
                cudaEventRecord(f, P);
                cudaStreamWaitEvent(tc.P2, f, 0);
                StageArgs a2 = stage_base(wk, A, lda, o.c_tau, SK_COL_BELOW, ABFT_V2, (int)k);
                a2.flist = 2;
                t = prof.begin(tc.P2);
                launch_check(a2, tc.P2);                                         // V2
                prof.end(t, PH_V12, tc.P2, 4.0 * mBd * Bd, 8.0 * mBd * Bd);
                v2done = new_event();
                cudaEventRecord(v2done, tc.P2);
            }
        }
        cudaEvent_t t = prof.begin(P);
        launch_chol_inv(Akk, lda, w.Li, B, k * B, w.tmp, w.st, P);
        prof.end(t, PH_POTRF, P, 2.0 * Bd * Bd * Bd / 3.0, 0);
        if (v2done) cudaStreamWaitEvent(P, v2done, 0);                          // V2 before the TRSM reads
        // TRSM (+ Alg. 2 on the checksum rows of tile (k,k)): one GEMM per row segment
        t = prof.begin(P);
        if (abft && !(abl & 1))
            launch_trsm_with_chk(mB, B, Akk + B, lda, w.Li, W, ldw, nc * m + nc, w.chk + k * B * w.ldc + nc * k, w.ldc,
                                 ab, P);
        else
            launch_gemm(mB, B, B, Akk + B, lda, w.Li, B, W, ldw, 1.0, 0.0, true, 0, 1, 0, 0, 0, ab, P);
        prof.end(t, PH_TRSM, P, (mBd + (abft ? (double)nc * (md + 1) : 0)) * Bd * Bd, 0);
        if (abft) {
            do_inject(inj, k, ABFT_HOOK_POTRF_OUT, B, L, ab, P);
            StageArgs a3 = stage_base(wk, A, lda, o.c_tau, SK_DIAG_FACT, ABFT_V3, (int)k);
            a3.ldw = ldw; a3.mB = mB; a3.flist = 1;
            StageArgs a4 = stage_base(wk, A, lda, o.c_tau, SK_PANEL, ABFT_V4, (int)k);
            a4.ldw = ldw; a4.mB = mB; a4.flist = 1;
            if (abl & 4) {
            } else if (mode != ABFT_MODE_OFFLINE && !has_inj(inj, k, ABFT_HOOK_TRSM_OUT)) {
                // V3 and V4 in one launch: V4 reads the solved panel and its checksum rows in W,
                // never L_kk, so V3's corrections need not precede it; phase 2 resolves tile (k,k)
                // first, as the sequential schedule does
                t = prof.begin(P);
                launch_check2(a3, a4, P);                                        // V3 + V4
                prof.end(t, PH_V4, P, 4.0 * (mBd * Bd + lowerB), 8.0 * (mBd * Bd + lowerB));
            } else {
                if (mode != ABFT_MODE_OFFLINE) {
                    t = prof.begin(P);
                    launch_check(a3, P);                                         // V3
                    prof.end(t, PH_V3, P, 4.0 * lowerB, 8.0 * lowerB);
                }
                do_inject(inj, k, ABFT_HOOK_TRSM_OUT, B, L, ab, P);
                if (mode != ABFT_MODE_OFFLINE) {
                    t = prof.begin(P);
                    launch_check(a4, P);                                         // V4
                    prof.end(t, PH_V4, P, 4.0 * mBd * Bd, 8.0 * mBd * Bd);
                }
            }
        }
        // the panel is final once V3/V4 passed: the trailing update reads W, not A's panel, so with
        // ABFT_WB_EARLY=1 the main stream may start while the write-back of L(:,k) runs behind it
        cudaEvent_t ready = nullptr;
        if (wb_early) { ready = new_event(); cudaEventRecord(ready, P); }
        t = prof.begin(P);
        if (abft && !(abl & 1) && mB % 2 == 0)   // L panel + its checksum rows: one pass over W, one launch
            launch_panel_out(W, ldw, mB, nc * m + nc, B, Akk + B, lda, w.chk + k * B * w.ldc + nc * k, w.ldc, nullptr, 0,
                             ab, P);
        else {
            launch_copy(mB, B, W, ldw, Akk + B, lda, ab, P);                    // L panel
            if (abft && !(abl & 1)) launch_copy(nc * m + nc, B, W + mB, ldw, w.chk + k * B * w.ldc + nc * k, w.ldc, ab, P);
        }
        prof.end(t, PH_WB, P, 0, 16.0 * (mBd + (abft ? (double)nc * (md + 1) : 0)) * Bd);
        cudaEvent_t e = new_event(); cudaEventRecord(e, P);
        return std::make_pair(ready ? ready : e, e);
    };

    int64_t slab_rows_used = 64;
    // ---- trailing update of iteration k restricted to block columns [jlo, jhi), on S ----
    // Returns a bit mask: 1 = the GEMM epilogue produced the fused V5 partials for these columns,
    // 2 = the epilogue applied the UPDATE_OUT injections of these columns (reading A21).
    auto update_cols = [&](int64_t k, int64_t jlo, int64_t jhi) -> int {
        const int64_t m = N - k - 1, mB = m * B;
        const int64_t ldw = std::max<int64_t>(1, (mB + nc * m + nc + 1) / 2 * 2);   // even: 16-byte columns
        double* W = Wbuf[k & 1];
        const int64_t c0 = (jlo - k - 1) * B, ncols = (jhi - jlo) * B;   // W row offset of column block jlo
        const int64_t rows = mB - c0;                                     // data rows from block jlo down
        double* C = A + jlo * B * lda + jlo * B;
        const double r = (double)rows, c = (double)ncols;
        cudaEvent_t t = prof.begin(s);
        // C[rows x nc] -= W[c0:, :] W[c0:c0+nc, :]^T, lower (r >= c)
        EpiInj ei; ei.n = 0;
        for (const auto& sp : inj)
            if (sp.k == k && sp.hook == ABFT_HOOK_UPDATE_OUT && sp.col / nb >= jlo && sp.col / nb < jhi) {
                if (ei.n < kMaxEpiInj) {
                    EpiInjOp& e = ei.op[ei.n];
                    e.seg = sp.target == ABFT_TGT_DATA ? 0 : 1;
                    e.r = sp.target == ABFT_TGT_DATA ? sp.row - jlo * B : sp.row - nc * jlo;
                    e.c = sp.col - jlo * B; e.mask = sp.xor_mask; e.pad = 0;
                }
                ei.n++;
            }
        ColSumOut cso{w.cs, n, w.cs_nslab, jlo * B, jlo * B, B, 64, jlo * B, nc};
        int fused;
        if (abft) {
            // checksum rows of tiles I >= jlo: chk[nc I + t, cols] -= W_chk(I) W[c0:c0+ncols]^T, I >= J,
            // appended to the same launch as a second row segment
            const int64_t q0 = nc * (jlo - k - 1);                      // first chk row of tile jlo in W
            const int64_t nq = (abl & 1) ? 0 : nc * (N - jlo);
            fused = launch_update_with_chk(rows, ncols, B, W + c0, ldw, W + c0, ldw, C, lda, nq, W + mB + nc + q0,
                                           w.chk + jlo * B * w.ldc + nc * jlo, w.ldc, B, ab, s,
                                           can_fuse ? &cso : nullptr, 0, 1, &ei, (int)nc);
            const double mm = (double)(N - jlo), jj = (double)(jhi - jlo);
            prof.end(t, PH_UPD, s, (c * (c + 1) / 2 + (r - c) * c) * 2.0 * Bd + 2.0 * nc * Bd * Bd * (jj * mm - jj * (jj - 1) / 2), 0);
        } else {
            fused = launch_gemm(rows, ncols, B, W + c0, ldw, W + c0, ldw, C, lda, -1.0, 1.0, true, 1, 0, 0, 0, 0, ab, s);
            fused = 0;
            prof.end(t, PH_UPD, s, (c * (c + 1) / 2 + (r - c) * c) * 2.0 * Bd, 0);
        }
        if (fused & 1) slab_rows_used = cso.slab_rows;
        return fused;
    };
    auto v5_cols = [&](int64_t k, int64_t jlo, int64_t jhi, bool fused, cudaStream_t vs = nullptr, int flist = 0) {
        if (!vs) vs = s;
        StageArgs a = stage_base(w, A, lda, o.c_tau, SK_TRAIL, ABFT_V5, (int)k);
        a.j_lo = jlo; a.j_hi = jhi; a.flist = flist;
        const double el = (double)stage_count(a) * Bd * Bd - (double)(jhi - jlo) * Bd * (Bd - 1) / 2;
        cudaEvent_t t = prof.begin(vs);
        if (fused) {
            StageArgs d = a; d.kind = SK_TRAIL_DIAG;
            StageArgs f = a; f.kind = SK_TRAIL_OFF;
            f.cs = w.cs; f.cs_ld = n; f.cs_nslab = w.cs_nslab; f.cs_slab_rows = slab_rows_used;
            launch_check_v5_fused(d, f, vs);
            const double rd = (double)(jhi - jlo) * lowerB, ro = (double)stage_count(f) * Bd * 2.0 * (Bd / (double)slab_rows_used);
            prof.end(t, PH_V5, vs, 4.0 * el, 8.0 * (rd + ro));   // bytes actually needed by the fused check
        } else {
            launch_check(a, vs);
            prof.end(t, PH_V5, vs, 4.0 * el, 8.0 * el);
        }
    };

    std::vector<cudaEvent_t> pan(N, nullptr), wbk(N, nullptr);   // panel k checked / written back
    if (abft) {   // REST(0) outside block column 0 (column 0 is handled by the panel stream)
        const Loc L0{A, lda, w.chk, w.ldc, Wbuf[0], 1, 0};
        do_inject_if(inj, 0, ABFT_HOOK_REST, B, L0, ab, s, 0, 1, false);
    }
    const bool sink = g_sink.host != nullptr && !ps;
    auto sink_col = [&](int64_t k) {   // L(kB:n, block column k) -> host, after panel k's write-back
        if (!sink) return;
        cudaStreamWaitEvent(g_sink.cs, wbk[k], 0);
        cudaMemcpy2DAsync(g_sink.host + k * B * g_sink.ldh + k * B, g_sink.ldh * sizeof(double), A + k * B * lda + k * B,
                          lda * sizeof(double), (size_t)(n - k * B) * sizeof(double), (size_t)B,
                          cudaMemcpyDeviceToHost, g_sink.cs);
    };
    std::tie(pan[0], wbk[0]) = panel(0);
    sink_col(0);
    for (int64_t k = 0; k < N; ++k) {
        {
            cudaEvent_t t = prof.begin(s);
            cudaStreamWaitEvent(s, pan[k], 0);
            prof.end(t, PH_WAIT, s);
        }
        const int64_t m = N - k - 1, mB = m * B;
        if (m == 0) break;
        const int64_t ldw = std::max<int64_t>(1, (mB + nc * m + nc + 1) / 2 * 2);   // even: 16-byte columns
        const Loc L{A, lda, w.chk, w.ldc, Wbuf[k & 1], ldw, mB, (int)nc};
        const bool gated = (((k + 1) % K == 0) || k == N - 2) && mode != ABFT_MODE_OFFLINE;
        // (a) block column k+1 first: update, UPDATE_OUT hook, V5 -> hand it to the panel stream
        if (k == 0) ensure_chunk(1 / kSrcChunk);
        const int fa = update_cols(k, k + 1, k + 2);
        if (abft) {
            if (!(fa & 2)) do_inject_if(inj, k, ABFT_HOOK_UPDATE_OUT, B, L, ab, s, k + 1, k + 2, true);
            if (gated && !(abl & 2)) v5_cols(k, k + 1, k + 2, (fa & 1) != 0);
        }
        cudaEvent_t ec = new_event(); cudaEventRecord(ec, s);
        cudaStreamWaitEvent(P, ec, 0);
        std::tie(pan[k + 1], wbk[k + 1]) = panel(k + 1);
        sink_col(k + 1);
        // (b) the rest of the trailing matrix (streamed input, k = 0: chunk by chunk as it lands)
        if (m > 1) {
            int fb;
            if (src && k == 0) {
                fb = 1 | 2;
                for (int64_t c = 2 / kSrcChunk; c * kSrcChunk < N; ++c) {
                    ensure_chunk(c);
                    const int64_t J0 = std::max<int64_t>(2, c * kSrcChunk), J1 = std::min<int64_t>(N, (c + 1) * kSrcChunk);
                    if (J0 < J1) fb &= update_cols(0, J0, J1);
                }
            } else {
                fb = update_cols(k, k + 2, N);
            }
            if (abft) {
                if (!(fb & 2)) do_inject_if(inj, k, ABFT_HOOK_UPDATE_OUT, B, L, ab, s, k + 2, N, true);
                if (gated && !(abl & 2)) v5_cols(k, k + 2, N, (fb & 1) != 0);
            }
        }
        if (abft) {   // REST(k+1) outside block column k+1 (that one was applied on P)
            // a target in a finished panel must follow its write-back (which runs behind S on P)
            if (has_inj(inj, k + 1, ABFT_HOOK_REST)) cudaStreamWaitEvent(s, wbk[k], 0);
            const Loc L1{A, lda, w.chk, w.ldc, Wbuf[(k + 1) & 1], 1, 0};
            do_inject_if(inj, k + 1, ABFT_HOOK_REST, B, L1, ab, s, k + 1, k + 2, false);
        }
    }
    if (N > 0) cudaStreamWaitEvent(s, wbk[N - 1], 0);   // every write-back (P is in order) before V6 / the end
    if (abft && !(abl & 16)) {
        const Loc L{A, lda, w.chk, w.ldc, w.W, 1, 0};
        do_inject(inj, N, ABFT_HOOK_REST, B, L, ab, s);
        StageArgs a6 = stage_base(w, A, lda, o.c_tau, SK_ALL, ABFT_V6, (int)N);
        a6.factored = 1;
        cudaEvent_t t = prof.begin(s);
        launch_check(a6, s);                                                              // V6
        const double el = (double)(N * (N - 1) / 2) * Bd * Bd + (double)N * lowerB;
        prof.end(t, PH_V6, s, 4.0 * el, 8.0 * el);
    }
    ABFT_CUDA_TRY(cudaGetLastError());
    if (ps) return 0;   // graph mode: the caller launches, reports and keeps the buffers
    int status = 0;
    if (rep) {
        cudaEventRecord(e1, s);
        rc = finish_report(w, rep, s, &status);
        float ms = 0; cudaEventElapsedTime(&ms, e0, e1);
        rep->seconds = ms * 1e-3;
    }
    if (prof.on) { cudaStreamSynchronize(s); prof.finish(); }
    cudaFreeAsync(Wbuf[1], s);
    work_free(w, s);
    if (rc) return rc;
    ABFT_CUDA_TRY(cudaGetLastError());
    return status;
}

static int run_potrf_direct(int64_t n, int64_t nb, double* A, int64_t lda, cudaStream_t s,
                            const std::vector<abft_inject_spec_t>& inj, abft_report_t* rep, const abft_options_t& o) {
    return run_potrf(n, nb, A, lda, s, inj, rep, o, nullptr);
}

// ---- graph mode ------------------------------------------------------------------------------
// The whole right-looking factorisation (both streams, ~12k kernels at n = 32768) captured once
// into a CUDA graph and replayed: no host launch overhead and shorter dependent-launch gaps on
// the look-ahead stream's panel chain. One cached graph per thread, keyed by every argument that
// shapes the work (device, n, nb, A, lda, options, event capacity); its workspace stays allocated
// until the key changes or abft_graph_release() is called. Used for fault-free calls only
// (injection lists change the hook sequence) and without the per-phase profiler.
struct GraphEntry {
    bool valid = false;
    int dev = -1;
    int64_t n = 0, nb = 0, lda = 0, cap = 0;
    double* A = nullptr;
    abft_options_t o{};
    cudaGraphExec_t exec = nullptr;
    cudaStream_t cs = nullptr;   // private capture / launch stream (the caller's may be the legacy one)
    Persist ps;
    int64_t launches = 0;
};
static thread_local GraphEntry g_graph;

static void graph_release(GraphEntry& g) {
    if (g.exec) cudaGraphExecDestroy(g.exec);
    Work& w = g.ps.w;
    for (void* p : {(void*)w.chk, (void*)w.scl, (void*)w.W, (void*)w.Li, (void*)w.tmp, (void*)w.st, (void*)w.ev,
                    (void*)w.cs, (void*)g.ps.W1})
        if (p) cudaFree(p);
    cudaStream_t cs = g.cs;
    g = GraphEntry();
    g.cs = cs;
}

// Default: graph mode for n <= 12288, where launch gaps are a visible share of the step (C2,
// n = 4096 nb = 256: 7.3 -> 6.2 ms; n = 8192 nb = 1024: 17.5 -> 16.5 ms). Above it the replayed
// graph was measured slower than direct launches (n = 16384: 59.9 vs 67.4 ms, n = 32768: 375.6 vs
// 397.9 ms, with or without per-node priorities), so large problems launch directly.
// ABFT_GRAPH=0 / 1 forces it off / on.
static bool graph_mode_enabled(int64_t n) {
    const char* e = getenv("ABFT_GRAPH");
    if (e) return atoi(e) != 0;
    return n <= 12288;
}

static int run_graph(int64_t n, int64_t nb, double* A, int64_t lda, cudaStream_t s, abft_report_t* rep,
                     const abft_options_t& o) {
    int dev = 0;
    cudaGetDevice(&dev);
    GraphEntry& g = g_graph;
    const int64_t cap = rep ? std::max<int64_t>(rep->cap, 1) : 1024;
    const bool hit = g.valid && g.dev == dev && g.n == n && g.nb == nb && g.A == A && g.lda == lda && g.cap == cap &&
                     !memcmp(&g.o, &o, sizeof o);
    if (!hit) {
        if (g.valid || g.exec) { cudaStreamSynchronize(g.cs); graph_release(g); }
        if (!g.cs || g.dev != dev) ABFT_CUDA_TRY(cudaStreamCreateWithFlags(&g.cs, cudaStreamNonBlocking));
        const int64_t N = n / nb;
        Work& w = g.ps.w;
        const int nchk = o.nchk == 3 ? 3 : 2;
        w.n = n; w.nb = nb; w.N = N; w.nchk = nchk; w.ldc = std::max<int64_t>(1, nchk * N);
        const bool abft = o.abft_enabled != 0;
        const int64_t wrows = std::max<int64_t>((N - 1) * nb + nchk * N + nchk + 1, 1);
        const size_t tmpn = (size_t)(((nb + 1) / 2 + 64) * ((nb + 1) / 2 + 64));
        if (abft) {
            ABFT_CUDA_TRY(cudaMalloc((void**)&w.chk, sizeof(double) * (size_t)(w.ldc * n)));
            ABFT_CUDA_TRY(cudaMalloc((void**)&w.scl, sizeof(double) * (size_t)(n + 3 * N + 1)));
            w.cs_nslab = n / 32;
            ABFT_CUDA_TRY(cudaMalloc((void**)&w.cs, sizeof(double) * (size_t)(nchk * w.cs_nslab * n)));
        }
        ABFT_CUDA_TRY(cudaMalloc((void**)&w.W, sizeof(double) * (size_t)(wrows * nb)));
        ABFT_CUDA_TRY(cudaMalloc((void**)&g.ps.W1, sizeof(double) * (size_t)(wrows * nb)));
        ABFT_CUDA_TRY(cudaMalloc((void**)&w.Li, sizeof(double) * (size_t)(nb * nb)));
        ABFT_CUDA_TRY(cudaMalloc((void**)&w.tmp, sizeof(double) * tmpn));
        ABFT_CUDA_TRY(cudaMalloc((void**)&w.st, sizeof(DevState)));
        w.ev_cap = cap;
        ABFT_CUDA_TRY(cudaMalloc((void**)&w.ev, sizeof(abft_event_t) * (size_t)cap));
        g.dev = dev;
        // capture: everything run_potrf enqueues on cs and on the look-ahead stream it forks
        const std::vector<abft_inject_spec_t> none;
        ABFT_CUDA_TRY(cudaStreamBeginCapture(g.cs, cudaStreamCaptureModeRelaxed));
        g_launches = 0;
        const int rc = run_potrf(n, nb, A, lda, g.cs, none, nullptr, o, &g.ps);
        cudaGraph_t graph = nullptr;
        const cudaError_t ce = cudaStreamEndCapture(g.cs, &graph);
        if (rc || ce != cudaSuccess || !graph) {
            if (graph) cudaGraphDestroy(graph);
            cudaGetLastError();
            graph_release(g);
            return rc ? rc : ABFT_ERR_CUDA;
        }
        {   // stream priorities are not kept by capture: restore the panel chain's precedence by
            // giving every kernel node except the trailing updates the high priority
            size_t nn = 0;
            cudaGraphGetNodes(graph, nullptr, &nn);
            std::vector<cudaGraphNode_t> nodes(nn);
            if (nn) cudaGraphGetNodes(graph, nodes.data(), &nn);
            int lo = 0, hi = 0;
            cudaDeviceGetStreamPriorityRange(&lo, &hi);
            for (cudaGraphNode_t nd : nodes) {
                cudaGraphNodeType t;
                if (cudaGraphNodeGetType(nd, &t) != cudaSuccess || t != cudaGraphNodeTypeKernel) continue;
                cudaKernelNodeParams kp;
                if (cudaGraphKernelNodeGetParams(nd, &kp) != cudaSuccess) continue;
                if (abft::is_update_kernel(kp.func)) continue;
                cudaKernelNodeAttrValue v;
                memset(&v, 0, sizeof v);
                v.priority = hi;
                cudaGraphKernelNodeSetAttribute(nd, cudaLaunchAttributePriority, &v);
            }
            cudaGetLastError();
        }
        const cudaError_t ie = cudaGraphInstantiate(&g.exec, graph, 0);
        cudaGraphDestroy(graph);
        if (ie != cudaSuccess) { cudaGetLastError(); graph_release(g); return ABFT_ERR_CUDA; }
        g.launches = g_launches;
        g.n = n; g.nb = nb; g.A = A; g.lda = lda; g.cap = cap; g.o = o; g.valid = true;
    }
    // stream semantics of the caller's s: cs waits for s, s waits for the graph
    ThreadCache& tc = thread_cache();
    cudaEvent_t fork = tc.sync.get(), join = tc.sync.get();
    cudaEvent_t e0 = tc.timing.get(), e1 = tc.timing.get();
    cudaEventRecord(fork, s);
    cudaStreamWaitEvent(g.cs, fork, 0);
    cudaEventRecord(e0, g.cs);
    ABFT_CUDA_TRY(cudaGraphLaunch(g.exec, g.cs));
    cudaEventRecord(e1, g.cs);
    cudaEventRecord(join, g.cs);
    cudaStreamWaitEvent(s, join, 0);
    g_launches = g.launches;
    int status = 0;
    ABFT_CUDA_TRY(cudaGetLastError());
    if (!rep) return 0;   // fully asynchronous without a report (abft.h): no stream synchronisation
    const int rc = finish_report(g.ps.w, rep, g.cs, &status);
    if (rc) return rc;
    float ms = 0; cudaEventElapsedTime(&ms, e0, e1); rep->seconds = ms * 1e-3;
    return status;
}

extern "C" int abft_graph_release(void) {
    if (g_graph.valid || g_graph.exec) {
        if (g_graph.cs) cudaStreamSynchronize(g_graph.cs);
        graph_release(g_graph);
    }
    return 0;
}


// =============================================================================================
// 1D block-cyclic multi-GPU driver. Rank r owns block columns {J : J mod P = r},
// stored contiguously (local block t = global block t*P + r). Per iteration k the owner of block
// column k runs V1/V2, POTRF + inverse, TRSM (+ Alg. 2 rows), V3, V4 and the write-back exactly as
// on one GPU, then broadcasts the packed panel W = [L(k+1:N,k); chk rows 2k..2N-1] (plus one
// slot carrying its abort flag); every receiver re-checks its copy (RECV hook -> V4R, rank r)
// and all ranks apply the trailing update to their own block columns, checksum rows included,
// followed by V5 on their own tiles. Decisions are owner-local, so the event multiset is the
// single-GPU one plus V4R events (the oracle's P-rank simulation reproduces it).
// =============================================================================================
namespace {
struct RankState {
    int r, pr, pc;            // rank, its process-grid row and column (2D block-cyclic; pr = 0 in 1D)
    double* A; int64_t lda;
    int64_t nblk, ncl;        // local block columns, local columns
    Work w;
    double* Wb[2] = {nullptr, nullptr};   // double-buffered panel (look-ahead)
    double* Wt = nullptr;     // 2D: this rank's TRSM output (its own panel rows), pushed from here into
                              // every rank's Wb (its own included), which the other owners fill too
};
// Process grid of the dist driver: P = Pr x Pc ranks, rank r = pr * Pc + pc; tile (I, J) is owned by
// rank (I mod Pr) * Pc + (J mod Pc) (Pr = 1: the 1D column-cyclic distribution). Every rank stores
// its block columns {J : J mod Pc = pc} contiguously and full height (global rows); it maintains
// only its own tiles.
struct Grid {
    int P, Pr, Pc;
    int owner(int64_t I, int64_t J) const { return (int)((I % Pr) * Pc + (J % Pc)); }
};
}

static int64_t dist_lc(int64_t J, int Pc, int64_t nb) { return (J / Pc) * nb; }   // local column of block J

// block row of an injection's target (data row / nb, or checksum row / 2)
static int64_t inj_row_block(const abft_inject_spec_t& sp, int64_t nb) {
    return sp.target == ABFT_TGT_DATA ? sp.row / nb : sp.row / 2;
}

static double* dist_inj_ptr(const abft_inject_spec_t& sp, int64_t k, int64_t nb, const Grid& G, const RankState& R,
                            int64_t ldw, int64_t mB) {
    const int hook = sp.hook;
    const int64_t Jc = sp.col / nb, lcol = dist_lc(Jc, G.Pc, nb) + sp.col % nb;
    if (hook == ABFT_HOOK_TRSM_OUT || hook == ABFT_HOOK_RECV) {
        if (sp.target == ABFT_TGT_DATA) return R.w.W + (sp.col - k * nb) * ldw + (sp.row - (k + 1) * nb);
        return R.w.W + (sp.col - k * nb) * ldw + mB + (sp.row - 2 * k);
    }
    if (hook == ABFT_HOOK_POTRF_OUT && sp.target == ABFT_TGT_CHK)
        return R.w.W + (sp.col - k * nb) * ldw + mB + (sp.row - 2 * k);
    if (sp.target == ABFT_TGT_DATA) return R.A + lcol * R.lda + sp.row;
    return R.w.chk + lcol * R.w.ldc + sp.row;
}

// Apply rank R's share of the injections at (k, hook): targets in the tiles it owns, or for RECV
// the ones addressed to it that land in a panel tile it received (not one it owns).
static void dist_inject(const std::vector<abft_inject_spec_t>& list, int64_t k, int hook, int64_t nb, const Grid& G,
                        const RankState& R, int64_t ldw, int64_t mB, cudaStream_t s) {
    std::vector<double*> ptrs; std::vector<uint64_t> masks;
    for (const auto& sp : list) {
        if (sp.k != k || sp.hook != hook) continue;
        const int own = G.owner(inj_row_block(sp, nb), sp.col / nb);
        if (hook == ABFT_HOOK_RECV) { if (sp.rank != R.r || own == R.r) continue; }
        else if (own != R.r) continue;       // the owner of the target's tile
        ptrs.push_back(dist_inj_ptr(sp, k, nb, G, R, ldw, mB)); masks.push_back(sp.xor_mask);
    }
    if (!ptrs.empty()) launch_inject((int)ptrs.size(), ptrs.data(), masks.data(), &R.w.st->abort, s);
}

int run_dist(int64_t n, int64_t nb, int P, const DistLocal* locals, int nlocal, DistTransport* tp,
             cudaStream_t s, const abft_inject_spec_t* inj_c, abft_report_t* rep, const abft_options_t* opt) {
    abft_options_t o = opt ? *opt : abft_options_t{1, 1, 64.0, 0, 0, ABFT_MODE_ENHANCED, 0, 0, 0};
    const int Pr = o.prows > 0 ? o.prows : 1;
    if (o.K < 1 || !(o.c_tau > 0) || o.mode != ABFT_MODE_ENHANCED || o.order != ABFT_ORDER_RIGHT ||
        (o.nchk != 0 && o.nchk != 2) || P % Pr != 0 || Pr > 15)
        return -11;   // dist: Enhanced scheme, right-looking order, two checksum rows, Pr | P
    const Grid G{P, Pr, P / Pr};
    const int Pc = G.Pc;
    std::vector<abft_inject_spec_t> inj;
    if (collect_inj(inj_c, n, nb, inj)) return -9;
    if (rep) { rep->info = 0; rep->n_events = 0; rep->n_checks = 0; }
    if (n == 0) return 0;
    const bool abft = o.abft_enabled != 0;
    const int K = std::max(1, o.K);
    const int64_t N = n / nb, B = nb;
    std::vector<RankState> R(nlocal);
    const int64_t evcap = rep ? std::max<int64_t>(rep->cap, 1) : 1024;
    // W layout: packed panel (ldw x B) + 16 abort slots (one per contributing process row); 2D also
    // keeps the received inv(L_kk) (+ its abort slot) behind them
    const int64_t wrows_max = (N - 1) * nb + 2 * N + 2;
    const size_t wcap = (size_t)(std::max<int64_t>(wrows_max, 1) * nb) + 16;
    const size_t wbuf = wcap + (Pr > 1 ? (size_t)(B * B) + 2 : 0);
    // push mode (NEXT-3): a peer-memory transport owns every rank's two receive buffers; the owner's
    // write-back kernel stores the panel straight into them (launch_panel_out)
    const bool push = tp && tp->recv_buf(tp->rank, 0) != nullptr && tp->recv_capacity() >= wbuf &&
                      tp->nranks <= 16 && nb % 2 == 0 && getenv("ABFT_DIST_PULL") == nullptr;
    // 2D needs peer memory (IPC transport) or the one-device harness; the row-filtered push moves
    // 16-byte row pairs
    if (Pr > 1 && ((tp && !push) || nb % 2)) return -11;
    if (tp && tp->begin_call(N, s)) return ABFT_ERR_NCCL;   // fresh flag range for this call (IPC)
    for (int i = 0; i < nlocal; ++i) {
        RankState& q = R[i];
        q.r = locals[i].rank; q.pr = q.r / Pc; q.pc = q.r % Pc; q.A = locals[i].A; q.lda = locals[i].lda;
        q.nblk = (N - q.pc + Pc - 1) / Pc; q.ncl = q.nblk * B;
        int rc = work_alloc(q.w, n, nb, std::max<int64_t>(q.ncl, 1), evcap, abft, s);
        if (rc) return rc;
        cudaFreeAsync(q.w.W, s);
        if (push) q.w.W = tp->recv_buf(q.r, 0);
        else ABFT_CUDA_TRY(cudaMallocAsync((void**)&q.w.W, sizeof(double) * wbuf, s));
        if (abft && nb % 128 == 0 && q.lda % 2 == 0 && ((uintptr_t)q.A & 15) == 0) {
            q.w.cs_nslab = n / 32;
            ABFT_CUDA_TRY(cudaMallocAsync((void**)&q.w.cs, sizeof(double) * (size_t)(2 * q.w.cs_nslab * std::max<int64_t>(q.ncl, 1)), s));
        }
        launch_zero(B, B, q.w.Li, B, s);
    }
    auto stage = [&](RankState& q, int kind, int V, int k) {
        StageArgs a = stage_base(q.w, q.A, q.lda, o.c_tau, kind, V, k);
        a.col_owner_mod = Pc; a.col_owner_rank = q.pc; a.row_owner_mod = Pr; a.row_owner_rank = q.pr; a.rank = q.r;
        return a;
    };
    cudaEvent_t e0 = nullptr, e1 = nullptr;
    if (rep) { cudaEventCreate(&e0); cudaEventCreate(&e1); cudaEventRecord(e0, s); }
    // ---- encode: scales need every diagonal block -> all-reduce of the owner-local parts ----
    if (abft) {
        for (auto& q : R) {
            cudaMemsetAsync(q.w.scl, 0, sizeof(double) * (size_t)(n + 2 * N), s);
            for (int64_t J = q.pc; J < N; J += Pc)
                if (G.owner(J, J) == q.r)
                    launch_scales_diag(B, q.A + dist_lc(J, Pc, B) * q.lda + J * B, q.lda, q.w.scl + J * B, s);
        }
        if (tp) {
            if (tp->allreduce_sum(R[0].w.scl, (size_t)n, s)) return ABFT_ERR_NCCL;
        } else {
            for (int i = 1; i < nlocal; ++i) launch_axpy(n, R[i].w.scl, R[0].w.scl, s);
            for (int i = 1; i < nlocal; ++i)
                cudaMemcpyAsync(R[i].w.scl, R[0].w.scl, sizeof(double) * (size_t)n, cudaMemcpyDeviceToDevice, s);
        }
        for (auto& q : R) {
            launch_scales_blocks(N, B, q.w.scl, q.w.scl + n, q.w.scl + n + N, s);
            StageArgs a = stage(q, SK_ALL, 0, -1);
            a.encode = 1;
            launch_check(a, s);
        }
    }
    // ---- look-ahead across ranks: the owners of block column k+1 update that
    // column with panel k first, then factor it and broadcast panel k+1 on their panel stream while
    // every rank applies the rest of update k on its main stream. Panel + broadcast + V4R run on the
    // panel stream PS (high priority), updates + V5 on the main stream (the caller's).
    // Single-process simulation: every rank shares the two streams; the broadcast is a device copy
    // (1D) or the owners' push into the other ranks' panel buffers (2D), issued on PS.
    ThreadCache& tc = thread_cache();
    cudaStream_t PS = tc.P;
    // The transport's waiting kernels (NCCL collectives, IPC flag waits) are long-lived CTAs; they
    // run on a NORMAL-priority comm stream joined to PS by events
    if (tp && !tc.C) ABFT_CUDA_TRY(cudaStreamCreateWithFlags(&tc.C, cudaStreamNonBlocking));
    cudaStream_t CS = tp ? tc.C : PS;
    auto hop = [&](cudaStream_t from, cudaStream_t to) {   // `to` waits for everything enqueued on `from`
        if (from == to) return;
        cudaEvent_t e = tc.sync.get(); cudaEventRecord(e, from); cudaStreamWaitEvent(to, e, 0);
    };
    auto new_event = [&]() { return tc.sync.get(); };
    {   // panel stream starts after the encode
        cudaEvent_t e = new_event(); cudaEventRecord(e, s); cudaStreamWaitEvent(PS, e, 0);
    }
    for (auto& q : R) {   // second panel buffer per rank (W of iteration k lives in Wb[k & 1])
        q.Wb[0] = q.w.W;
        if (push) q.Wb[1] = tp->recv_buf(q.r, 1);
        else ABFT_CUDA_TRY(cudaMallocAsync((void**)&q.Wb[1], sizeof(double) * wbuf, s));
        if (Pr > 1) ABFT_CUDA_TRY(cudaMallocAsync((void**)&q.Wt, sizeof(double) * wcap, s));
    }
    {   // Wb[1] allocated on s: the panel stream must see it
        cudaEvent_t e = new_event(); cudaEventRecord(e, s); cudaStreamWaitEvent(PS, e, 0);
    }
    auto geom = [&](int64_t k, int64_t& m, int64_t& mB, int64_t& ldw) {
        m = N - k - 1; mB = m * B; ldw = std::max<int64_t>(1, mB + 2 * m + 2);
    };
    // injections of hook REST(k) split by block column: inside [jlo, jhi) or outside it
    auto rest_inject = [&](RankState& q, int64_t k, int64_t jlo, int64_t jhi, bool inside, cudaStream_t st) {
        std::vector<abft_inject_spec_t> sub;
        for (const auto& sp : inj) {
            if (sp.k != k || sp.hook != ABFT_HOOK_REST) continue;
            const int64_t J = sp.col / nb;
            if ((J >= jlo && J < jhi) == inside) sub.push_back(sp);
        }
        if (!sub.empty()) dist_inject(sub, k, ABFT_HOOK_REST, B, G, q, 1, 0, st);
    };
    // the other ranks' panel buffers Wb[slot] (peer stores of the push)
    auto peer_bufs = [&](const RankState& q, int slot) {
        std::vector<double*> peers;
        if (push) { for (int r = 0; r < P; ++r) if (r != q.r) peers.push_back(tp->recv_buf(r, slot)); }
        else for (auto& p : R) if (p.r != q.r) peers.push_back(p.Wb[slot]);
        return peers;
    };
    // the panel of iteration k, on the panel stream of the ranks of process column k mod Pc: V1/V2
    // of their tiles of block column k, POTRF + inverse on the diagonal block's owner (2D: inv(L_kk)
    // pushed to the column's other ranks), TRSM of each rank's own panel rows (+ Alg. 2 rows), V3,
    // V4, write-back, abort slot; 2D / peer memory: each rank's rows pushed into every other rank's
    // panel buffer Wb[k & 1]
    auto panel = [&](int64_t k) -> int {
        int64_t m, mB, ldw; geom(k, m, mB, ldw);
        const int kc = (int)(k % Pc), d = G.owner(k, k);
        const size_t wcount = (size_t)(ldw * B);
        std::vector<RankState*> col;
        for (auto& q : R) if (q.pc == kc) col.push_back(&q);
        if (col.empty()) return 0;
        for (RankState* qp : col) {                                                    // REST(k), V1, V2
            RankState& q = *qp;
            q.w.W = q.Wb[k & 1];
            if (abft) {
                rest_inject(q, k, k, k + 1, true, PS);
                StageArgs a = stage(q, SK_COLUMN, ABFT_V2, (int)k); a.flist = 1;
                launch_check(a, PS);
            }
        }
        for (RankState* qp : col) {                                                    // POTRF + inverse
            RankState& q = *qp;
            if (q.r != d) continue;
            double* Akk = q.A + dist_lc(k, Pc, B) * q.lda + k * B;
            launch_chol_inv(Akk, q.lda, q.w.Li, B, k * B, q.w.tmp, q.w.st, PS);
            if (Pr > 1 && m > 0) {   // inv(L_kk) + abort flag to the column's other ranks (their Wb + wcap)
                for (int pr = 0; pr < Pr; ++pr) {
                    const int r = pr * Pc + kc;
                    if (r == d) continue;
                    double* dst = nullptr;
                    if (push) dst = tp->recv_buf(r, (int)(k & 1)) + wcap;
                    else for (auto& p : R) if (p.r == r) dst = p.Wb[k & 1] + wcap;
                    if (!dst) continue;
                    cudaMemcpyAsync(dst, q.w.Li, sizeof(double) * (size_t)(B * B), cudaMemcpyDeviceToDevice, PS);
                    launch_abort_to_slot(&q.w.st->abort, dst + B * B, PS);
                }
                if (push && tp->post_li(k, PS)) return ABFT_ERR_NCCL;
            }
        }
        for (RankState* qp : col) {
            RankState& q = *qp;
            const int32_t* ab = &q.w.st->abort;
            double* Akk = q.A + dist_lc(k, Pc, B) * q.lda + k * B;
            double* ckk = q.w.chk + dist_lc(k, Pc, B) * q.w.ldc;
            if (m == 0 && q.r != d) continue;                     // last panel: the diagonal block only
            if (Pr > 1) q.w.W = q.Wt;   // 2D: solve into the private buffer (Wb[k & 1] receives the other owners' rows)
            const double* Li = q.w.Li;
            if (q.r != d) {                                       // 2D: the column's other ranks
                double* li_in = q.Wb[k & 1] + wcap;
                if (push) { hop(PS, CS); if (tp->wait_li(d, k, CS)) return ABFT_ERR_NCCL; hop(CS, PS); }
                launch_abort_from_slot(li_in + B * B, q.w.st, PS);
                Li = li_in;
            }
            // this rank's panel rows: data blocks k+1+b with (k+1+b) mod Pr = pr
            const int64_t rfirst = ((q.pr - (k + 1) % Pr) % Pr + Pr) % Pr;
            if (abft)
                launch_trsm_with_chk(mB, B, Akk + B, q.lda, Li, q.w.W, ldw, 2 * m + 2, ckk + 2 * k, q.w.ldc, ab, PS, Pr,
                                     rfirst);
            else
                launch_gemm(mB, B, B, Akk + B, q.lda, Li, B, q.w.W, ldw, 1.0, 0.0, true, 0, 1, 0, 0, 0, ab, PS);
            if (abft) {
                StageArgs a3 = stage(q, SK_DIAG_FACT, ABFT_V3, (int)k);
                a3.ldw = ldw; a3.mB = mB; a3.flist = 1;
                StageArgs a4 = stage(q, SK_PANEL, ABFT_V4, (int)k);
                a4.ldw = ldw; a4.mB = mB; a4.flist = 1;
                dist_inject(inj, k, ABFT_HOOK_POTRF_OUT, B, G, q, ldw, mB, PS);
                if (q.r == d && !has_inj(inj, k, ABFT_HOOK_TRSM_OUT)) {
                    launch_check2(a3, a4, PS);                                         // V3 + V4
                } else {
                    if (q.r == d) launch_check(a3, PS);                                // V3
                    dist_inject(inj, k, ABFT_HOOK_TRSM_OUT, B, G, q, ldw, mB, PS);
                    launch_check(a4, PS);                                              // V4
                }
            }
            launch_abort_to_slot(ab, q.w.W + wcount + q.pr, PS);
            const int64_t ncr = abft ? 2 * m + 2 : 0;
            if ((push || Pr > 1) && k + 1 < N) {
                // write-back fused with the broadcast: one pass over this rank's rows of W stores them
                // locally (L panel, checksum rows) and into every other rank's panel buffer (peer
                // stores), once every peer released that buffer
                if (push) { hop(PS, CS); if (tp->wait_free(k, CS)) return ABFT_ERR_NCCL; hop(CS, PS); }
                std::vector<double*> peers = peer_bufs(q, (int)(k & 1));
                if (Pr > 1) peers.push_back(q.Wb[k & 1]);   // and its own receive buffer
                if (launch_panel_out(q.w.W, ldw, mB, ncr, B, Akk + B, q.lda, ckk + 2 * k, q.w.ldc, peers.data(),
                                     (int)peers.size(), ab, PS, Pr, rfirst, ((q.pr - k % Pr) % Pr + Pr) % Pr, q.pr))
                    return -11;
                if (push && tp->post_panel(k, PS)) return ABFT_ERR_NCCL;
                q.w.W = q.Wb[k & 1];
                continue;
            }
            if (abft && mB % 2 == 0 && ldw % 2 == 0)
                launch_panel_out(q.w.W, ldw, mB, ncr, B, Akk + B, q.lda, ckk + 2 * k, q.w.ldc, nullptr, 0, ab, PS);
            else {
                launch_copy(mB, B, q.w.W, ldw, Akk + B, q.lda, ab, PS);
                if (abft) launch_copy(ncr, B, q.w.W + mB, ldw, ckk + 2 * k, q.w.ldc, ab, PS);
            }
            q.w.W = q.Wb[k & 1];
        }
        return 0;
    };
    // broadcast of panel k (+ abort slots) from its owners, then every receiver's RECV hook and V4R
    // on the tiles it received; afterwards evB[rank] marks "panel k usable on this rank"
    std::vector<cudaEvent_t> evU(nlocal, nullptr), evUprev(nlocal, nullptr);   // after update k / k-1
    std::vector<cudaEvent_t> evB(nlocal, nullptr);
    auto bcast = [&](int64_t k) -> int {
        int64_t m, mB, ldw; geom(k, m, mB, ldw);
        const size_t wcount = (size_t)(ldw * B);
        const int kc = (int)(k % Pc), owner = G.owner(k, k);
        for (int i = 0; i < nlocal; ++i)   // the receive buffer Wb[k & 1] was last read by update k-2
            if (evUprev[i]) cudaStreamWaitEvent(PS, evUprev[i], 0);
        if (tp && push) {
            hop(PS, CS);
            for (int pr = 0; pr < Pr; ++pr) {   // pushed by the panel's owners (the ranks of column kc)
                const int c = pr * Pc + kc;
                if (c != R[0].r && tp->wait_panel(c, k, CS)) return ABFT_ERR_NCCL;
            }
            hop(CS, PS);
        } else if (tp) {
            hop(PS, CS);
            if (tp->bcast(R[0].Wb[k & 1], (wcount + 1) * sizeof(double), owner, CS)) return ABFT_ERR_NCCL;
            hop(CS, PS);
        } else if (Pr == 1) {
            const RankState* src = nullptr;
            for (auto& q : R) if (q.r == owner) src = &q;
            for (auto& q : R)
                if (q.r != owner)
                    cudaMemcpyAsync(q.Wb[k & 1], src->Wb[k & 1], (wcount + 1) * sizeof(double), cudaMemcpyDeviceToDevice, PS);
        }   // 2D one-device harness: the owners' pushes on PS already filled every buffer
        for (int i = 0; i < nlocal; ++i) {
            RankState& q = R[i];
            q.w.W = q.Wb[k & 1];
            bool received = false;
            for (int64_t I = k + 1; I < N; ++I) received = received || G.owner(I, k) != q.r;
            if (received) {
                for (int pr = 0; pr < Pr; ++pr)
                    if (pr * Pc + kc != q.r) launch_abort_from_slot(q.w.W + wcount + pr, q.w.st, PS);
                if (abft) {
                    dist_inject(inj, k, ABFT_HOOK_RECV, B, G, q, ldw, mB, PS);
                    StageArgs a = stage(q, SK_PANEL, ABFT_V4R, (int)k);               // V4R
                    a.ldw = ldw; a.mB = mB; a.own_invert = 1; a.flist = 1;
                    launch_check(a, PS);
                }
            }
            evB[i] = new_event(); cudaEventRecord(evB[i], PS);
        }
        return 0;
    };
    int64_t dist_slab_rows = 64;
    // trailing update of iteration k on rank q's tiles in block columns [jlo, jhi) (main stream),
    // UPDATE_OUT hook and V5 of those tiles
    auto update = [&](RankState& q, int64_t k, int64_t jlo, int64_t jhi) {
        int64_t m, mB, ldw; geom(k, m, mB, ldw);
        double* W = q.Wb[k & 1];
        const int32_t* ab = &q.w.st->abort;
        bool any = false;
        for (int64_t J = jlo; J < jhi; ++J) any = any || (J % Pc == q.pc);
        if (!any) return;
        bool all_fused = q.w.cs != nullptr;
        // the owned block columns J in [jlo, jhi) are J0, J0 + Pc, ...: one launch whose column
        // block t is global block J0 + t Pc (cstride), checksum rows appended as its second segment;
        // 2D: only the row blocks I = J0 + rfirst + u Pr (this rank's tiles) are computed
        int64_t J0 = jlo;
        while (J0 % Pc != q.pc) ++J0;
        const int64_t nt = (jhi - 1 - J0) / Pc + 1, t0 = J0 / Pc;
        const int64_t rfirst = ((q.pr - J0 % Pr) % Pr + Pr) % Pr;
        double* W0 = W + (J0 - k - 1) * B;
        double* C = q.A + t0 * B * q.lda + J0 * B;
        // this rank's UPDATE_OUT injections in [jlo, jhi), in the launch's local coordinates
        EpiInj ei; ei.n = 0;
        for (const auto& sp : inj)
            if (sp.k == k && sp.hook == ABFT_HOOK_UPDATE_OUT && G.owner(inj_row_block(sp, B), sp.col / B) == q.r &&
                sp.col / B >= jlo && sp.col / B < jhi) {
                if (ei.n < kMaxEpiInj) {
                    EpiInjOp& e = ei.op[ei.n];
                    e.seg = sp.target == ABFT_TGT_DATA ? 0 : 1;
                    e.r = sp.target == ABFT_TGT_DATA ? sp.row - J0 * B : sp.row - 2 * J0;
                    e.c = ((sp.col / B) / Pc - t0) * B + sp.col % B; e.mask = sp.xor_mask; e.pad = 0;
                }
                ei.n++;
            }
        bool applied = false;
        ColSumOut cso{q.w.cs, q.ncl, q.w.cs_nslab, J0 * B, t0 * B, B, 64, J0 * B};
        const int f = abft ? launch_update_with_chk((N - J0) * B, nt * B, B, W0, ldw, W0, ldw, C, q.lda, 2 * (N - J0),
                                                    W + mB + 2 + 2 * (J0 - k - 1), q.w.chk + t0 * B * q.w.ldc + 2 * J0,
                                                    q.w.ldc, B, ab, s, all_fused ? &cso : nullptr, 0, Pc, &ei, 2, Pr,
                                                    rfirst)
                           : launch_update_with_chk((N - J0) * B, nt * B, B, W0, ldw, W0, ldw, C, q.lda, 0, W0, C,
                                                    q.lda, B, ab, s, nullptr, 0, Pc, nullptr, 2, Pr, rfirst);
        if (f < 0) {   // shapes the strided launch cannot take (or ABFT off): one launch per block column
            if (ei.n > 0) all_fused = false;   // the hook is applied after the launches
            for (int64_t J = J0; J < jhi; J += Pc) {
                const int64_t t = J / Pc;
                double* Wj = W + (J - k - 1) * B;
                double* Cj = q.A + t * B * q.lda + J * B;
                ColSumOut csj{q.w.cs, q.ncl, q.w.cs_nslab, J * B, t * B, B, 64, J * B};
                int fj;
                if (abft)
                    fj = launch_update_with_chk((N - J) * B, B, B, Wj, ldw, Wj, ldw, Cj, q.lda, 2 * (N - J),
                                                W + mB + 2 + 2 * (J - k - 1), q.w.chk + t * B * q.w.ldc + 2 * J,
                                                q.w.ldc, B, ab, s, all_fused ? &csj : nullptr, 0, 1, nullptr, 2, Pr,
                                                ((q.pr - J % Pr) % Pr + Pr) % Pr);
                else
                    fj = launch_gemm((N - J) * B, B, B, Wj, ldw, Wj, ldw, Cj, q.lda, -1.0, 1.0, true, 1, 0, 0, 0, 0, ab, s);
                if (!(fj & 1)) all_fused = false;
                if (fj & 1) dist_slab_rows = csj.slab_rows;
            }
        } else {
            applied = (f & 2) != 0;
            if (!(f & 1)) all_fused = false;
            if (f & 1) dist_slab_rows = cso.slab_rows;
        }
        if (!abft) return;
        if (!applied) {   // UPDATE_OUT injections of this rank inside [jlo, jhi)
            std::vector<abft_inject_spec_t> sub;
            for (const auto& sp : inj)
                if (sp.k == k && sp.hook == ABFT_HOOK_UPDATE_OUT && sp.col / B >= jlo && sp.col / B < jhi) sub.push_back(sp);
            if (!sub.empty()) dist_inject(sub, k, ABFT_HOOK_UPDATE_OUT, B, G, q, ldw, mB, s);
        }
        const bool gated = ((k + 1) % K == 0) || k == N - 2;
        if (!gated) return;
        StageArgs a = stage(q, SK_TRAIL, ABFT_V5, (int)k);
        a.j_lo = jlo; a.j_hi = jhi; a.flist = 0;
        if (all_fused) {
            StageArgs d = a; d.kind = SK_TRAIL_DIAG;
            StageArgs f = a; f.kind = SK_TRAIL_OFF;
            f.cs = q.w.cs; f.cs_ld = q.ncl; f.cs_nslab = q.w.cs_nslab; f.cs_slab_rows = dist_slab_rows;
            launch_check_v5_fused(d, f, s);                                            // V5 (fused)
        } else {
            launch_check(a, s);                                                        // V5
        }
    };

    if (abft) for (auto& q : R) rest_inject(q, 0, 0, 1, false, s);   // REST(0) outside column 0
    {   // P streams see those injections before the first panel
        cudaEvent_t e = new_event(); cudaEventRecord(e, s); cudaStreamWaitEvent(PS, e, 0);
    }
    { const int rcp = panel(0); if (rcp) return rcp; }
    if (N > 1) { int rc2 = bcast(0); if (rc2) return rc2; }
    for (int64_t k = 0; k + 1 < N; ++k) {
        for (int i = 0; i < nlocal; ++i) cudaStreamWaitEvent(s, evB[i], 0);      // panel k usable
        const int c1 = (int)((k + 1) % Pc);
        // (a) block column k+1 on its owners: update, UPDATE_OUT, V5 -> panel k+1 on PS
        bool mine = false;
        for (auto& q : R) if (q.pc == c1) { update(q, k, k + 1, k + 2); mine = true; }
        if (mine) {
            cudaEvent_t ec = new_event(); cudaEventRecord(ec, s); cudaStreamWaitEvent(PS, ec, 0);
            const int rcp = panel(k + 1); if (rcp) return rcp;
        }
        // (b) the rest of update k on every rank (the owners of k+1 included)
        for (auto& q : R) update(q, k, k + 2, N);
        for (int i = 0; i < nlocal; ++i) { evUprev[i] = evU[i]; evU[i] = new_event(); cudaEventRecord(evU[i], s); }
        if (push && tp->mark_free(k + 1, s)) return ABFT_ERR_NCCL;   // buffer (k & 1) read for the last time
        // (c) REST(k+1) outside block column k+1 (column k+1's share was applied on PS)
        if (abft) for (auto& q : R) rest_inject(q, k + 1, k + 1, k + 2, false, s);
        // (d) broadcast panel k+1 (receivers wait for their update k-1 ... k to release the buffer)
        if (k + 2 < N) {   // Wb[(k+1) & 1] was last read by update k-1 (evUprev)
            int rc2 = bcast(k + 1); if (rc2) return rc2;
        } else {
            for (int i = 0; i < nlocal; ++i) { evB[i] = new_event(); cudaEventRecord(evB[i], PS); }
        }
    }
    {   // main stream waits for the last panel
        cudaEvent_t e = new_event(); cudaEventRecord(e, PS); cudaStreamWaitEvent(s, e, 0);
    }
    for (auto& q : R) {
        if (q.Wt) cudaFreeAsync(q.Wt, s);
        q.Wt = nullptr;
        if (q.Wb[1] && !push) cudaFreeAsync(q.Wb[1], s);
        q.Wb[1] = nullptr; q.w.W = push ? nullptr : q.Wb[0];   // push mode: the transport owns them
    }
    if (abft) {
        for (auto& q : R) {
            dist_inject(inj, N, ABFT_HOOK_REST, B, G, q, 1, 0, s);
            StageArgs a6 = stage(q, SK_ALL, ABFT_V6, (int)N);
            a6.factored = 1;
            launch_check(a6, s);                                                       // V6
        }
    }
    ABFT_CUDA_TRY(cudaGetLastError());
    // ---- report: counters summed, status/info maxed, events of every rank merged ----
    int status = 0;
    {
        const int nc = 8;
        std::vector<double> cnt(nc * nlocal, 0.0), mx(2 * nlocal, 0.0);
        std::vector<abft_event_t> evs;
        double* dbuf = nullptr;     // device staging for the collectives
        abft_event_t* evg = nullptr;
        const int nr = tp ? tp->nranks : 1;
        if (tp) ABFT_CUDA_TRY(cudaMallocAsync((void**)&dbuf, sizeof(double) * 16, s));
        std::vector<char> hbuf(sizeof(DevState));
        DevState& hs = *reinterpret_cast<DevState*>(hbuf.data());
        double tot[8] = {0}, smax[4] = {0, 0, 0, 0};   // status, info, noise ratio, local event count
        for (auto& q : R) {
            ABFT_CUDA_TRY(cudaMemcpyAsync(&hs, q.w.st, offsetof(DevState, fl), cudaMemcpyDeviceToHost, s));
            ABFT_CUDA_TRY(cudaStreamSynchronize(s));
            const double v[8] = {(double)hs.n_checks, (double)hs.n_detected, (double)hs.n_data, (double)hs.n_nonfinite,
                                 (double)hs.n_chk1, (double)hs.n_chk2, (double)hs.n_unc, (double)hs.nev};
            for (int i = 0; i < 8; ++i) tot[i] += v[i];
            double q_ratio; memcpy(&q_ratio, &hs.max_ratio_bits, sizeof q_ratio);
            smax[0] = std::max(smax[0], (double)hs.status); smax[1] = std::max(smax[1], (double)hs.info);
            smax[2] = std::max(smax[2], q_ratio);
            const int64_t ne = std::min<int64_t>((int64_t)hs.nev, q.w.ev_cap);
            std::vector<abft_event_t> tmp(ne);
            if (ne > 0) ABFT_CUDA_TRY(cudaMemcpy(tmp.data(), q.w.ev, sizeof(abft_event_t) * (size_t)ne, cudaMemcpyDeviceToHost));
            evs.insert(evs.end(), tmp.begin(), tmp.end());
        }
        smax[3] = (double)evs.size();
        if (tp) {
            double hb[16] = {0};
            for (int i = 0; i < 8; ++i) hb[i] = tot[i];
            ABFT_CUDA_TRY(cudaMemcpyAsync(dbuf, hb, sizeof(double) * 8, cudaMemcpyHostToDevice, s));
            if (tp->allreduce_sum(dbuf, 8, s)) return ABFT_ERR_NCCL;
            ABFT_CUDA_TRY(cudaMemcpyAsync(hb, dbuf, sizeof(double) * 8, cudaMemcpyDeviceToHost, s));
            double hm[4] = {smax[0], smax[1], smax[2], smax[3]};
            ABFT_CUDA_TRY(cudaMemcpyAsync(dbuf + 8, hm, sizeof(double) * 4, cudaMemcpyHostToDevice, s));
            if (tp->allreduce_max(dbuf + 8, 4, s)) return ABFT_ERR_NCCL;
            ABFT_CUDA_TRY(cudaMemcpyAsync(hm, dbuf + 8, sizeof(double) * 4, cudaMemcpyDeviceToHost, s));
            ABFT_CUDA_TRY(cudaStreamSynchronize(s));
            // events: every rank contributes a block as large as the largest rank's list (no cap)
            const int64_t capg = std::max<int64_t>(1, (int64_t)hm[3]);
            ABFT_CUDA_TRY(cudaMallocAsync((void**)&evg, sizeof(abft_event_t) * (size_t)(capg * (nr + 1)), s));
            std::vector<abft_event_t> mine((size_t)capg);
            memset(mine.data(), 0, sizeof(abft_event_t) * (size_t)capg);
            for (size_t i = 0; i < evs.size(); ++i) mine[i] = evs[i];
            for (int64_t i = (int64_t)evs.size(); i < capg; ++i) mine[i].k = -2;   // padding marker
            ABFT_CUDA_TRY(cudaMemcpyAsync(evg + capg * nr, mine.data(), sizeof(abft_event_t) * (size_t)capg, cudaMemcpyHostToDevice, s));
            if (tp->allgather(evg + capg * nr, evg, sizeof(abft_event_t) * (size_t)capg, s)) return ABFT_ERR_NCCL;
            std::vector<abft_event_t> all((size_t)(capg * nr));
            ABFT_CUDA_TRY(cudaMemcpyAsync(all.data(), evg, sizeof(abft_event_t) * (size_t)(capg * nr), cudaMemcpyDeviceToHost, s));
            ABFT_CUDA_TRY(cudaStreamSynchronize(s));
            evs.clear();
            for (auto& e : all) if (e.k != -2) evs.push_back(e);
            for (int i = 0; i < 8; ++i) tot[i] = hb[i];
            for (int i = 0; i < 4; ++i) smax[i] = hm[i];
            cudaFreeAsync(dbuf, s); cudaFreeAsync(evg, s);
        }
        status = (int)smax[0];
        if (rep) {
            rep->info = (int64_t)smax[1];
            rep->n_checks = (int64_t)tot[0]; rep->n_detected = (int64_t)tot[1]; rep->n_data = (int64_t)tot[2];
            rep->n_nonfinite = (int64_t)tot[3]; rep->n_chk1 = (int64_t)tot[4]; rep->n_chk2 = (int64_t)tot[5];
            rep->n_uncorrectable = (int64_t)tot[6]; rep->n_events = (int64_t)tot[7];
            rep->max_noise_ratio = smax[2];
            std::sort(evs.begin(), evs.end(), [](const abft_event_t& x, const abft_event_t& y) {
                if (x.k != y.k) return x.k < y.k;
                if (x.check != y.check) return x.check < y.check;
                if (x.tile_j != y.tile_j) return x.tile_j < y.tile_j;
                if (x.tile_i != y.tile_i) return x.tile_i < y.tile_i;
                if (x.col != y.col) return x.col < y.col;
                if (x.row != y.row) return x.row < y.row;
                return x.rank < y.rank;
            });
            const int64_t nc2 = std::min<int64_t>((int64_t)evs.size(), std::max<int64_t>(rep->cap, 0));
            if (rep->events) for (int64_t i = 0; i < nc2; ++i) rep->events[i] = evs[i];
            cudaEventRecord(e1, s);
            cudaEventSynchronize(e1);
            float ms = 0; cudaEventElapsedTime(&ms, e0, e1);
            rep->seconds = ms * 1e-3;
            cudaEventDestroy(e0); cudaEventDestroy(e1);
        }
        (void)cnt; (void)mx;
    }
    for (auto& q : R) work_free(q.w, s);
    ABFT_CUDA_TRY(cudaStreamSynchronize(s));
    return status;
}

extern "C" int abft_potrf_dist_sim(int64_t n, int64_t nb, int nranks, double* const* A_locals, int64_t lda_local,
                                   abft_stream_t stream, const abft_inject_spec_t* inj, abft_report_t* rep,
                                   const abft_options_t* opt) {
    g_launches = 0;
    if (n < 0) return -1;
    if (nb < 1 || n % nb) return -2;
    if (nranks < 1) return -3;
    if (!A_locals) return -4;
    if (lda_local < std::max<int64_t>(1, n)) return -5;
    std::vector<DistLocal> L(nranks);
    const int Pc = (opt && opt->prows > 1 && nranks % opt->prows == 0) ? nranks / opt->prows : nranks;
    for (int r = 0; r < nranks; ++r) {
        if (!A_locals[r] && (n / nb - r % Pc + Pc - 1) / Pc > 0) return -4;
        L[r] = DistLocal{r, A_locals[r], lda_local};
    }
    return run_dist(n, nb, nranks, L.data(), nranks, nullptr, (cudaStream_t)stream, inj, rep, opt);
}


// ---- left-looking order (NEXT-1): MAGMA's Alg. 1 with Table I's verification ----
// Iteration j: V7 re-verifies the L blocks the SYRK/GEMM will read (C = L[j,0:j] always, D =
// L[j+1:,0:j] every K-th iteration: Opt. 3), V1/V2 the column to update; one launch updates block
// column j with its checksum rows appended (A[j:N,j] -= L[j:N,0:j] L[j,0:j]^T, K = j*nb), V5
// checks the updated column (fused partials), then POTRF + inverse, TRSM, V3 (and V4 for the
// Online scheme), write-back. Single stream: the next column's update needs this panel.
static int run_potrf_left(int64_t n, int64_t nb, double* A, int64_t lda, cudaStream_t s,
                          const std::vector<abft_inject_spec_t>& inj, abft_report_t* rep, const abft_options_t& o) {
    const bool abft = o.abft_enabled != 0;
    const int K = std::max(1, o.K);
    const int mode = o.mode;
    Work w;
    int rc = work_alloc(w, n, nb, n, rep ? std::max<int64_t>(rep->cap, 1) : 1024, abft, s);
    if (rc) return rc;
    const int64_t N = w.N, B = nb;
    const int32_t* ab = &w.st->abort;
    const bool can_fuse = abft && mode != ABFT_MODE_OFFLINE && (nb % 128 == 0) && (lda % 2 == 0) &&
                          (((uintptr_t)A & 15) == 0) && !getenv("ABFT_NOFUSE");   // dev knob: V5 re-reads
    if (can_fuse) {
        w.cs_nslab = n / 32;
        ABFT_CUDA_TRY(cudaMallocAsync((void**)&w.cs, sizeof(double) * (size_t)(2 * w.cs_nslab * n), s));
    }
    ThreadCache& tc = thread_cache();
    cudaEvent_t e0 = nullptr, e1 = nullptr;
    if (rep) { e0 = tc.timing.get(); e1 = tc.timing.get(); cudaEventRecord(e0, s); }
    launch_zero(B, B, w.Li, B, s);
    if (abft) {
        launch_scales(n, nb, A, lda, w.scl, s);
        StageArgs a = stage_base(w, A, lda, o.c_tau, SK_ALL, 0, -1);
        a.encode = 1;
        launch_check(a, s);
    }
    for (int64_t j = 0; j < N; ++j) {
        const int64_t m = N - j - 1, mB = m * B;
        const int64_t ldw = std::max<int64_t>(1, mB + 2 * m + 2);
        double* Ajj = A + j * B * lda + j * B;
        const Loc L{A, lda, w.chk, w.ldc, w.W, ldw, mB};
        if (abft) do_inject(inj, j, ABFT_HOOK_REST, B, L, ab, s);
        if (abft && mode == ABFT_MODE_ENHANCED && j > 0) {                       // V7: C, D
            StageArgs a = stage_base(w, A, lda, o.c_tau, SK_LEFT_L, ABFT_V7, (int)j);
            a.factored = 1;
            a.j_hi = (j % K == 0) ? N - j : 1;
            launch_check(a, s);
        }
        if (abft && mode == ABFT_MODE_ENHANCED)
            launch_check(stage_base(w, A, lda, o.c_tau, SK_COLUMN, ABFT_V2, (int)j), s);   // V1, V2
        bool fused = false;
        if (j > 0) {   // SYRK + GEMM of block column j, checksum rows as a second row segment
            EpiInj ei; ei.n = 0;
            for (const auto& sp : inj)
                if (sp.k == j && sp.hook == ABFT_HOOK_UPDATE_OUT) {
                    if (ei.n < kMaxEpiInj) {
                        EpiInjOp& e = ei.op[ei.n];
                        e.seg = sp.target == ABFT_TGT_DATA ? 0 : 1;
                        e.r = sp.target == ABFT_TGT_DATA ? sp.row - j * B : sp.row - 2 * j;
                        e.c = sp.col - j * B; e.mask = sp.xor_mask; e.pad = 0;
                    }
                    ei.n++;
                }
            ColSumOut cso{w.cs, n, w.cs_nslab, j * B, j * B, B, 64, j * B};
            int f = 0;
            if (abft)
                f = launch_update_with_chk((N - j) * B, B, j * B, A + j * B, lda, A + j * B, lda, Ajj, lda,
                                           2 * (N - j), w.chk + 2 * j, w.chk + j * B * w.ldc + 2 * j, w.ldc, B,
                                           ab, s, can_fuse ? &cso : nullptr, w.ldc, 1, &ei);
            else
                launch_gemm((N - j) * B, B, j * B, A + j * B, lda, A + j * B, lda, Ajj, lda, -1.0, 1.0, true, 1, 0,
                            0, 0, 0, ab, s);
            fused = (f & 1) != 0;
            if (abft && !(f & 2)) do_inject(inj, j, ABFT_HOOK_UPDATE_OUT, B, L, ab, s);
            if (abft && mode != ABFT_MODE_OFFLINE) {                              // V5: column j
                StageArgs a = stage_base(w, A, lda, o.c_tau, SK_TRAIL, ABFT_V5, (int)j);
                a.j_lo = j; a.j_hi = j + 1;
                if (fused) {
                    StageArgs d = a; d.kind = SK_TRAIL_DIAG;
                    StageArgs f = a; f.kind = SK_TRAIL_OFF;
                    f.cs = w.cs; f.cs_ld = n; f.cs_nslab = w.cs_nslab; f.cs_slab_rows = cso.slab_rows;
                    launch_check_v5_fused(d, f, s);
                } else {
                    launch_check(a, s);
                }
            }
        }
        launch_chol_inv(Ajj, lda, w.Li, B, j * B, w.tmp, w.st, s);
        launch_gemm(mB, B, B, Ajj + B, lda, w.Li, B, w.W, ldw, 1.0, 0.0, true, 0, 1, 0, 0, 0, ab, s);
        if (abft) {
            launch_gemm(2 * m + 2, B, B, w.chk + j * B * w.ldc + 2 * j, w.ldc, w.Li, B, w.W + mB, ldw, 1.0, 0.0,
                        true, 0, 1, 0, 0, 0, ab, s);
            do_inject(inj, j, ABFT_HOOK_POTRF_OUT, B, L, ab, s);
            if (mode != ABFT_MODE_OFFLINE) {
                StageArgs a3 = stage_base(w, A, lda, o.c_tau, SK_DIAG_FACT, ABFT_V3, (int)j);
                a3.ldw = ldw; a3.mB = mB;
                launch_check(a3, s);                                              // V3
            }
            do_inject(inj, j, ABFT_HOOK_TRSM_OUT, B, L, ab, s);
            if (mode == ABFT_MODE_ONLINE) {
                StageArgs a4 = stage_base(w, A, lda, o.c_tau, SK_PANEL, ABFT_V4, (int)j);
                a4.ldw = ldw; a4.mB = mB;
                launch_check(a4, s);                                              // V4 (Online)
            }
        }
        launch_copy(mB, B, w.W, ldw, Ajj + B, lda, ab, s);
        if (abft) launch_copy(2 * m + 2, B, w.W + mB, ldw, w.chk + j * B * w.ldc + 2 * j, w.ldc, ab, s);
    }
    if (abft) {
        const Loc L{A, lda, w.chk, w.ldc, w.W, 1, 0};
        do_inject(inj, N, ABFT_HOOK_REST, B, L, ab, s);
        StageArgs a6 = stage_base(w, A, lda, o.c_tau, SK_ALL, ABFT_V6, (int)N);
        a6.factored = 1;
        launch_check(a6, s);                                                      // V6
    }
    ABFT_CUDA_TRY(cudaGetLastError());
    int status = 0;
    if (rep) {
        cudaEventRecord(e1, s);
        rc = finish_report(w, rep, s, &status);
        float ms = 0; cudaEventElapsedTime(&ms, e0, e1);
        rep->seconds = ms * 1e-3;
    }
    work_free(w, s);
    if (rc) return rc;
    ABFT_CUDA_TRY(cudaGetLastError());
    return status;
}

using RunFn = int (*)(int64_t, int64_t, double*, int64_t, cudaStream_t, const std::vector<abft_inject_spec_t>&,
                      abft_report_t*, const abft_options_t&);

static abft_options_t default_options() {
    abft_options_t o;
    memset(&o, 0, sizeof o);
    o.abft_enabled = 1; o.K = 1; o.c_tau = 64.0; o.lookahead = 0; o.profile = 0; o.mode = ABFT_MODE_ENHANCED;
    o.order = ABFT_ORDER_RIGHT;
    return o;
}

extern "C" int abft_potrf_ex(int64_t n, int64_t nb, double* A, int64_t lda, abft_stream_t stream,
                             const abft_inject_spec_t* inj, abft_report_t* rep, const abft_options_t* opt) {
    g_launches = 0;
    int rc = check_common(n, nb, A, lda);
    if (rc) return rc;
    abft_options_t o = opt ? *opt : default_options();
    if (o.K < 1 || !(o.c_tau > 0)) return -8;
    if (o.nchk != 0 && o.nchk != 2 && o.nchk != 3) return -8;
    if (o.nchk == 3 && o.order != ABFT_ORDER_RIGHT) return -8;   // NEXT-4: right-looking driver
    std::vector<abft_inject_spec_t> list;
    if (collect_inj(inj, n, nb, list, o.order, o.nchk == 3 ? 3 : 2)) return -6;
    if (o.mode < ABFT_MODE_ENHANCED || o.mode > ABFT_MODE_ENHANCED_REDO) return -8;
    const bool redo = o.mode == ABFT_MODE_ENHANCED_REDO;   // NEXT-4: Enhanced + re-do on UNCORRECTABLE
    if (redo) o.mode = ABFT_MODE_ENHANCED;
    if (o.order != ABFT_ORDER_RIGHT && o.order != ABFT_ORDER_LEFT) return -8;
    const RunFn run = o.order == ABFT_ORDER_LEFT ? run_potrf_left : run_potrf_direct;
    if (rep) { rep->info = 0; rep->n_events = 0; rep->n_checks = 0; rep->reruns = 0; }
    if (n == 0) return 0;
    cudaStream_t s = (cudaStream_t)stream;
    if (((o.mode == ABFT_MODE_ENHANCED && !redo) || !o.abft_enabled) && o.order == ABFT_ORDER_RIGHT && list.empty() &&
        !o.profile && graph_mode_enabled(n))
        return run_graph(n, nb, A, lda, s, rep, o);
    if ((o.mode == ABFT_MODE_ENHANCED && !redo) || !o.abft_enabled) return run(n, nb, A, lda, s, list, rep, o);
    // Online / Offline: keep the input; an uncorrectable outcome or a detection by the final
    // sweep means an error propagated -> re-do the factorisation once, without the faults.
    // Enhanced + re-do: only an UNCORRECTABLE outcome (> 1 error in a block column) re-runs.
    double* A0 = nullptr;
    ABFT_CUDA_TRY(cudaMallocAsync((void**)&A0, sizeof(double) * (size_t)(n * n), s));
    ABFT_CUDA_TRY(cudaMemcpy2DAsync(A0, n * sizeof(double), A, lda * sizeof(double), n * sizeof(double), n,
                                    cudaMemcpyDeviceToDevice, s));
    abft_report_t r1;
    memset(&r1, 0, sizeof r1);
    std::vector<abft_event_t> ev1(rep ? std::max<int64_t>(rep->cap, 4096) : 4096);
    r1.cap = (int64_t)ev1.size(); r1.events = ev1.data();
    int st = run(n, nb, A, lda, s, list, &r1, o);
    bool v6 = false;
    for (int64_t e = 0; e < std::min<int64_t>(r1.n_events, r1.cap); ++e) v6 |= (ev1[e].check == ABFT_V6);
    abft_report_t r2;
    memset(&r2, 0, sizeof r2);
    std::vector<abft_event_t> ev2(rep ? std::max<int64_t>(rep->cap, 16) : 16);
    r2.cap = (int64_t)ev2.size(); r2.events = ev2.data();
    int reruns = 0;
    if (redo ? st == ABFT_UNCORRECTABLE : (st == ABFT_UNCORRECTABLE || st == ABFT_NOT_SPD || v6)) {
        ABFT_CUDA_TRY(cudaMemcpy2DAsync(A, lda * sizeof(double), A0, n * sizeof(double), n * sizeof(double), n,
                                        cudaMemcpyDeviceToDevice, s));
        const std::vector<abft_inject_spec_t> none;
        st = run(n, nb, A, lda, s, none, &r2, o);
        reruns = 1;
    }
    cudaFreeAsync(A0, s);
    ABFT_CUDA_TRY(cudaStreamSynchronize(s));
    if (rep) {
        rep->info = reruns ? r2.info : r1.info;
        rep->n_checks = r1.n_checks + r2.n_checks; rep->n_detected = r1.n_detected + r2.n_detected;
        rep->n_data = r1.n_data + r2.n_data; rep->n_nonfinite = r1.n_nonfinite + r2.n_nonfinite;
        rep->n_chk1 = r1.n_chk1 + r2.n_chk1; rep->n_chk2 = r1.n_chk2 + r2.n_chk2;
        rep->n_uncorrectable = r1.n_uncorrectable + r2.n_uncorrectable;
        rep->n_events = r1.n_events + r2.n_events;
        rep->seconds = r1.seconds + r2.seconds;
        rep->reruns = reruns;
        rep->max_noise_ratio = std::max(r1.max_noise_ratio, r2.max_noise_ratio);
        int64_t w = 0;
        for (int64_t e = 0; e < std::min<int64_t>(r1.n_events, r1.cap) && w < rep->cap; ++e) rep->events[w++] = ev1[e];
        for (int64_t e = 0; e < std::min<int64_t>(r2.n_events, r2.cap) && w < rep->cap; ++e) rep->events[w++] = ev2[e];
    }
    return st;
}

extern "C" int abft_potrf(int64_t n, int64_t nb, double* A, int64_t lda, abft_stream_t stream,
                          const abft_inject_spec_t* inj, abft_report_t* rep) {
    return abft_potrf_ex(n, nb, A, lda, stream, inj, rep, nullptr);
}

extern "C" int abft_potrf_host(int64_t n, int64_t nb, double* A_host, int64_t lda, abft_stream_t stream,
                               const abft_inject_spec_t* inj, abft_report_t* rep, const abft_options_t* opt) {
    int rc = check_common(n, nb, A_host, lda);
    if (rc) return rc;
    if (n == 0) return 0;
    cudaStream_t s = (cudaStream_t)stream;
    double* dA = nullptr;
    ABFT_CUDA_TRY(cudaMallocAsync((void**)&dA, sizeof(double) * (size_t)(n * n), s));
    // Overlapped write-back (HostSink) on the direct right-looking Enhanced / ABFT-off path without
    // injections; anything else (or a V6 event, i.e. a correction of finished L) copies L back
    // after the factorisation as before.
    const abft_options_t o = opt ? *opt : default_options();
    bool has_inj = false;
    for (const abft_inject_spec_t* q = inj; q && q->k >= 0; ++q) has_inj = true;
    // the overlapped write-back needs page-locked host memory: a copy from pageable memory is
    // synchronous to the host and would serialise the enqueue loop behind each block column
    cudaPointerAttributes pa;
    memset(&pa, 0, sizeof pa);
    const bool pinned = cudaPointerGetAttributes(&pa, A_host) == cudaSuccess &&
                        (pa.type == cudaMemoryTypeHost || pa.type == cudaMemoryTypeManaged);
    cudaGetLastError();
    const bool overlap = pinned && !has_inj && o.order == ABFT_ORDER_RIGHT &&
                         (o.mode == ABFT_MODE_ENHANCED || !o.abft_enabled) && !graph_mode_enabled(n) &&
                         getenv("ABFT_HOST_OVERLAP") == nullptr;
    const int64_t N = n / nb;
    const bool stream_in = overlap && N >= 2 && (!opt || opt->nchk == 0 || opt->nchk == 2) &&
                           getenv("ABFT_HOST_STREAM_IN") == nullptr;   // dev knob: set = copy all first
    if (stream_in) {
        // only what the factorisation reads goes over PCIe, and it streams in behind the start of
        // the factorisation on its own copy stream (HostSource): every diagonal tile first (the
        // threshold scales need the whole diagonal), then each block column below its diagonal
        // tile, in order, one event each
        ThreadCache& tc = thread_cache();
        if (!tc.Cin) ABFT_CUDA_TRY(cudaStreamCreateWithFlags(&tc.Cin, cudaStreamNonBlocking));
        while ((int64_t)g_src.ev.size() < N + 2) {
            cudaEvent_t e;
            ABFT_CUDA_TRY(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
            g_src.ev.push_back(e);
        }
        cudaEvent_t alloc = g_src.ev[N + 1];   // dA allocated on s
        ABFT_CUDA_TRY(cudaEventRecord(alloc, s));
        ABFT_CUDA_TRY(cudaStreamWaitEvent(tc.Cin, alloc, 0));
        for (int64_t k = 0; k < N; ++k)
            ABFT_CUDA_TRY(cudaMemcpy2DAsync(dA + k * nb * n + k * nb, n * sizeof(double), A_host + k * nb * lda + k * nb,
                                            lda * sizeof(double), (size_t)nb * sizeof(double), (size_t)nb,
                                            cudaMemcpyHostToDevice, tc.Cin));
        ABFT_CUDA_TRY(cudaEventRecord(g_src.ev[0], tc.Cin));
        for (int64_t k = 0; k < N; ++k) {
            if (k + 1 < N)
                ABFT_CUDA_TRY(cudaMemcpy2DAsync(dA + k * nb * n + (k + 1) * nb, n * sizeof(double),
                                                A_host + k * nb * lda + (k + 1) * nb, lda * sizeof(double),
                                                (size_t)(n - (k + 1) * nb) * sizeof(double), (size_t)nb,
                                                cudaMemcpyHostToDevice, tc.Cin));
            ABFT_CUDA_TRY(cudaEventRecord(g_src.ev[1 + k], tc.Cin));
        }
        g_src.active = true;
    } else if (overlap) {
        // only what the factorisation reads goes over PCIe: each block column from its diagonal
        // block down (the strict upper triangle outside the diagonal blocks is never read)
        for (int64_t k = 0; k < n / nb; ++k)
            ABFT_CUDA_TRY(cudaMemcpy2DAsync(dA + k * nb * n + k * nb, n * sizeof(double), A_host + k * nb * lda + k * nb,
                                            lda * sizeof(double), (size_t)(n - k * nb) * sizeof(double), (size_t)nb,
                                            cudaMemcpyHostToDevice, s));
    } else {
        ABFT_CUDA_TRY(cudaMemcpy2DAsync(dA, n * sizeof(double), A_host, lda * sizeof(double), n * sizeof(double), n,
                                        cudaMemcpyHostToDevice, s));
    }
    abft_report_t lrep;
    std::vector<abft_event_t> lev;
    abft_report_t* r = rep;
    if (overlap && !r) {   // the V6 test needs the events
        memset(&lrep, 0, sizeof lrep);
        lev.resize(4096); lrep.cap = (int64_t)lev.size(); lrep.events = lev.data();
        r = &lrep;
    }
    if (overlap) {
        ThreadCache& tc = thread_cache();
        if (!tc.C) ABFT_CUDA_TRY(cudaStreamCreateWithFlags(&tc.C, cudaStreamNonBlocking));
        g_sink.host = A_host; g_sink.ldh = lda; g_sink.cs = tc.C;
    }
    rc = abft_potrf_ex(n, nb, dA, n, stream, inj, r, opt);
    if (stream_in) {   // s has consumed every column unless the call failed early: join the copies anyway
        g_src.active = false;
        ABFT_CUDA_TRY(cudaStreamWaitEvent(s, g_src.ev[N], 0));
    }
    bool recopy = !overlap;
    if (overlap) {
        g_sink = HostSink();
        ABFT_CUDA_TRY(cudaStreamSynchronize(thread_cache().C));
        for (int64_t e = 0; e < std::min<int64_t>(r->n_events, r->cap); ++e) recopy |= (r->events[e].check == ABFT_V6);
        recopy |= r->n_events > r->cap || rc != 0;
    }
    if (recopy && rc >= 0 && rc != ABFT_ERR_CUDA) {
        if (overlap) {   // the device holds only the block columns from their diagonal blocks down
            for (int64_t k = 0; k < n / nb; ++k)
                ABFT_CUDA_TRY(cudaMemcpy2DAsync(A_host + k * nb * lda + k * nb, lda * sizeof(double), dA + k * nb * n + k * nb,
                                                n * sizeof(double), (size_t)(n - k * nb) * sizeof(double), (size_t)nb,
                                                cudaMemcpyDeviceToHost, s));
        } else {
            ABFT_CUDA_TRY(cudaMemcpy2DAsync(A_host, lda * sizeof(double), dA, n * sizeof(double), n * sizeof(double), n,
                                            cudaMemcpyDeviceToHost, s));
        }
    }
    cudaFreeAsync(dA, s);
    ABFT_CUDA_TRY(cudaStreamSynchronize(s));
    return rc;
}

extern "C" int abft_encode(int64_t n, int64_t nb, const double* A, int64_t lda, double* chk, int64_t ldchk,
                           double* scales, abft_stream_t stream) {
    g_launches = 0;
    int rc = check_common(n, nb, A, lda);
    if (rc) return rc;
    if (!chk && n > 0) return -5;
    const int64_t N = n / nb;
    if (ldchk < std::max<int64_t>(1, 2 * N)) return -6;
    if (!scales && n > 0) return -7;
    if (n == 0) return 0;
    cudaStream_t s = (cudaStream_t)stream;
    DevState* st = nullptr;
    ABFT_CUDA_TRY(cudaMallocAsync((void**)&st, sizeof(DevState), s));
    ABFT_CUDA_TRY(cudaMemsetAsync(st, 0, sizeof(DevState), s));
    launch_scales(n, nb, A, lda, scales, s);
    Work w; w.n = n; w.nb = nb; w.N = N; w.chk = chk; w.ldc = ldchk; w.scl = scales; w.st = st;
    StageArgs a = stage_base(w, (double*)A, lda, 64.0, SK_ALL, 0, -1);
    a.encode = 1;
    launch_check(a, s);
    cudaFreeAsync(st, s);
    ABFT_CUDA_TRY(cudaGetLastError());
    return 0;
}

extern "C" int abft_verify(int64_t n, int64_t nb, double* A, int64_t lda, double* chk, int64_t ldchk,
                           const double* scales, int factored, int correct, abft_stream_t stream,
                           abft_report_t* rep) {
    g_launches = 0;
    int rc = check_common(n, nb, A, lda);
    if (rc) return rc;
    if (!chk && n > 0) return -5;
    const int64_t N = n / nb;
    if (ldchk < std::max<int64_t>(1, 2 * N)) return -6;
    if (!scales && n > 0) return -7;
    if (factored != 0 && factored != 1) return -8;
    if (correct != 0 && correct != 1) return -9;
    if (rep) { rep->info = 0; rep->n_events = 0; rep->n_checks = 0; }
    if (n == 0) return 0;
    cudaStream_t s = (cudaStream_t)stream;
    Work w; w.n = n; w.nb = nb; w.N = N;
    w.ldc = ldchk; w.chk = chk; w.scl = (double*)scales;
    ABFT_CUDA_TRY(cudaMallocAsync((void**)&w.st, sizeof(DevState), s));
    ABFT_CUDA_TRY(cudaMemsetAsync(w.st, 0, sizeof(DevState), s));
    w.ev_cap = rep ? std::max<int64_t>(rep->cap, 1) : 1;
    ABFT_CUDA_TRY(cudaMallocAsync((void**)&w.ev, sizeof(abft_event_t) * (size_t)w.ev_cap, s));
    StageArgs a = stage_base(w, A, lda, 64.0, SK_ALL, factored ? ABFT_V6 : ABFT_V5, -1);
    a.factored = factored; a.correct = correct;
    launch_check(a, s);
    int status = 0;
    if (rep) rc = finish_report(w, rep, s, &status);
    cudaFreeAsync(w.st, s); cudaFreeAsync(w.ev, s);
    if (rc) return rc;
    ABFT_CUDA_TRY(cudaGetLastError());
    return status;
}

extern "C" int abft_dev_gemm_nt(int64_t M, int64_t N, int64_t K, const double* A, int64_t lda, const double* B,
                                int64_t ldb, double* C, int64_t ldc, double alpha, double beta, int lower,
                                abft_stream_t stream) {
    g_launches = 0;
    if (M < 0 || N < 0 || K < 0 || (lower && N > M) || lda < std::max<int64_t>(1, M) ||
        ldb < std::max<int64_t>(1, N) || ldc < std::max<int64_t>(1, M)) return -1;
    static int32_t* zero_flag = nullptr;
    if (!zero_flag) { ABFT_CUDA_TRY(cudaMalloc((void**)&zero_flag, sizeof(int32_t))); ABFT_CUDA_TRY(cudaMemset(zero_flag, 0, 4)); }
    launch_gemm(M, N, K, A, lda, B, ldb, C, ldc, alpha, beta, true, lower ? 1 : 0, 0, 0, 0, 0, zero_flag,
                (cudaStream_t)stream);
    ABFT_CUDA_TRY(cudaGetLastError());
    return 0;
}

extern "C" int abft_dev_chol_inv(int64_t nb, double* A, int64_t lda, double* Li, abft_stream_t stream) {
    g_launches = 0;
    if (nb < 1 || !A || !Li || lda < nb) return -1;
    cudaStream_t s = (cudaStream_t)stream;
    DevState* st = nullptr;
    double* tmp = nullptr;
    ABFT_CUDA_TRY(cudaMallocAsync((void**)&st, sizeof(DevState), s));
    ABFT_CUDA_TRY(cudaMemsetAsync(st, 0, offsetof(DevState, fl), s));
    ABFT_CUDA_TRY(cudaMallocAsync((void**)&tmp, sizeof(double) * (size_t)(((nb + 1) / 2 + 64) * ((nb + 1) / 2 + 64)), s));
    ABFT_CUDA_TRY(cudaMemsetAsync(tmp, 0, chol_sync_bytes(nb), s));
    launch_chol_inv(A, lda, Li, nb, 0, tmp, st, s);
    int32_t status = 0;
    ABFT_CUDA_TRY(cudaMemcpyAsync(&status, &st->status, sizeof status, cudaMemcpyDeviceToHost, s));
    cudaFreeAsync(tmp, s); cudaFreeAsync(st, s);
    ABFT_CUDA_TRY(cudaStreamSynchronize(s));
    return status;
}

void chol_set_trace(unsigned long long* t);
int chol_task_count(int64_t nb);
extern "C" int abft_dev_chol_trace(int64_t nb, double* A, int64_t lda, double* Li, uint64_t* trace_host, int64_t cap,
                                   abft_stream_t stream) {
    const int nt = chol_task_count(nb);
    if (nt <= 0 || cap < 4 * (int64_t)nt) return -1;
    unsigned long long* d = nullptr;
    ABFT_CUDA_TRY(cudaMalloc((void**)&d, sizeof(uint64_t) * 4 * (size_t)nt));
    ABFT_CUDA_TRY(cudaMemset(d, 0, sizeof(uint64_t) * 4 * (size_t)nt));
    chol_set_trace(d);
    const int st = abft_dev_chol_inv(nb, A, lda, Li, stream);
    chol_set_trace(nullptr);
    ABFT_CUDA_TRY(cudaMemcpy(trace_host, d, sizeof(uint64_t) * 4 * (size_t)nt, cudaMemcpyDeviceToHost));
    cudaFree(d);
    return st == 0 ? nt : -2;
}

extern "C" int abft_gen_spd(int64_t n, uint64_t seed, double* A, int64_t lda, abft_stream_t stream) {
    g_launches = 0;
    if (n < 0) return -1;
    if (!A && n > 0) return -3;
    if (lda < std::max<int64_t>(1, n)) return -4;
    launch_gen_spd(n, seed, A, lda, (cudaStream_t)stream);
    ABFT_CUDA_TRY(cudaGetLastError());
    return 0;
}
