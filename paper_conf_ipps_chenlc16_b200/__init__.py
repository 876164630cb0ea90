"""Thin ctypes binding of libabft.so (include/abft.h) — argument marshalling only.

Every step of the factorisation runs in the CUDA kernels of csrc/; this module never computes
anything itself and has no CPU fallback: importing it on a machine where libabft.so is missing
raises, and calling into it without a CUDA device fails inside the library.

Names follow the C-ABI: abft_potrf, abft_potrf_ex, abft_potrf_host, abft_encode, abft_verify,
abft_gen_spd, abft_nccl_id, abft_comm_init, abft_comm_destroy, abft_potrf_dist.
Device buffers are passed as torch CUDA tensors (float64, column-major = a transposed view of a
contiguous row-major tensor, or any tensor whose column stride is 1) or as raw integer device
pointers; streams default to torch's current stream.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
# ABFT_LIB_NAME: another in-tree build of the same library (development A/B timing on one box)
LIB_PATH = os.path.join(_HERE, os.environ.get("ABFT_LIB_NAME", "libabft.so"))

# Codes restated from include/abft.h
OK, UNCORRECTABLE, NOT_SPD, ERR_CUDA, ERR_NCCL = 0, 1, 2, 3, 4
HOOK = {"REST": 0, "POTRF_OUT": 1, "TRSM_OUT": 2, "UPDATE_OUT": 3, "RECV": 4}
CHECK = {1: "V1", 2: "V2", 3: "V3", 4: "V4", 5: "V5", 6: "V6", 7: "V4R", 8: "V7"}
KIND = {1: "DATA", 2: "NONFINITE", 3: "CHK1", 4: "CHK2", 5: "UNCORRECTABLE", 6: "CHK3"}

EVENT_DTYPE = np.dtype([
    ("k", "<i4"), ("check", "<i4"), ("tile_i", "<i4"), ("tile_j", "<i4"),
    ("row", "<i4"), ("col", "<i4"), ("kind", "<i4"), ("rank", "<i4"),
    ("delta1", "<f8"), ("delta2", "<f8"),
])
INJ_DTYPE = np.dtype([
    ("k", "<i4"), ("hook", "<i4"), ("target", "<i4"), ("pad0", "<i4"),
    ("row", "<i8"), ("col", "<i8"), ("xor_mask", "<u8"), ("rank", "<i4"), ("pad1", "<i4"),
])


class Event(ctypes.Structure):
    _fields_ = [(n, ctypes.c_int32) for n in ("k", "check", "tile_i", "tile_j", "row", "col", "kind", "rank")] + \
               [("delta1", ctypes.c_double), ("delta2", ctypes.c_double)]


class Report(ctypes.Structure):
    _fields_ = [("info", ctypes.c_int64), ("n_checks", ctypes.c_int64), ("n_detected", ctypes.c_int64),
                ("n_data", ctypes.c_int64), ("n_nonfinite", ctypes.c_int64), ("n_chk1", ctypes.c_int64),
                ("n_chk2", ctypes.c_int64), ("n_uncorrectable", ctypes.c_int64), ("n_events", ctypes.c_int64),
                ("cap", ctypes.c_int64), ("events", ctypes.c_void_p), ("seconds", ctypes.c_double),
                ("reruns", ctypes.c_int64), ("max_noise_ratio", ctypes.c_double)]


class Options(ctypes.Structure):
    _fields_ = [("abft_enabled", ctypes.c_int32), ("K", ctypes.c_int32), ("c_tau", ctypes.c_double),
                ("lookahead", ctypes.c_int32), ("profile", ctypes.c_int32), ("mode", ctypes.c_int32),
                ("order", ctypes.c_int32), ("nchk", ctypes.c_int32), ("prows", ctypes.c_int32)]


class Profile(ctypes.Structure):
    _fields_ = [("nphase", ctypes.c_int32), ("pad", ctypes.c_int32), ("ms", ctypes.c_double * 16),
                ("launches", ctypes.c_int64 * 16), ("flops", ctypes.c_double * 16), ("bytes", ctypes.c_double * 16)]


if not os.path.exists(LIB_PATH):
    raise ImportError(f"libabft.so not built ({LIB_PATH}); run `python paper_conf_ipps_chenlc16_b200/build.py` "
                      "(there is no CPU fallback)")
_lib = ctypes.CDLL(LIB_PATH)
_i64, _i32, _vp, _dbl = ctypes.c_int64, ctypes.c_int, ctypes.c_void_p, ctypes.c_double
_lib.abft_encode.argtypes = [_i64, _i64, _vp, _i64, _vp, _i64, _vp, _vp]
_lib.abft_verify.argtypes = [_i64, _i64, _vp, _i64, _vp, _i64, _vp, _i32, _i32, _vp, _vp]
_lib.abft_potrf.argtypes = [_i64, _i64, _vp, _i64, _vp, _vp, _vp]
_lib.abft_potrf_ex.argtypes = [_i64, _i64, _vp, _i64, _vp, _vp, _vp, _vp]
_lib.abft_potrf_host.argtypes = [_i64, _i64, _vp, _i64, _vp, _vp, _vp, _vp]
_lib.abft_gen_spd.argtypes = [_i64, ctypes.c_uint64, _vp, _i64, _vp]
_lib.abft_nccl_id.argtypes = [_vp]
_lib.abft_comm_init.argtypes = [ctypes.POINTER(_vp), _i32, _vp, _i32]
_lib.abft_comm_destroy.argtypes = [_vp]
_lib.abft_comm_init_ipc.argtypes = [ctypes.POINTER(_vp), _i32, _i32, _i64, _vp]
_lib.abft_comm_attach_ipc.argtypes = [_vp, _vp]
_lib.abft_potrf_dist.argtypes = [_i64, _i64, _vp, _i64, _vp, _i32, _i32, _vp, _vp, _vp, _vp]
_lib.abft_potrf_dist_sim.argtypes = [_i64, _i64, _i32, _vp, _i64, _vp, _vp, _vp, _vp]
_lib.abft_potrf_dist_sim.restype = _i32
_lib.abft_dev_chol_inv.argtypes = [_i64, _vp, _i64, _vp, _vp]
_lib.abft_dev_chol_inv.restype = _i32
_lib.abft_dev_chol_trace.argtypes = [_i64, _vp, _i64, _vp, _vp, _i64, _vp]
_lib.abft_dev_chol_trace.restype = _i32
_lib.abft_dev_gemm_nt.argtypes = [_i64, _i64, _i64, _vp, _i64, _vp, _i64, _vp, _i64, _dbl, _dbl, _i32, _vp]
_lib.abft_dev_gemm_nt.restype = _i32
_lib.abft_last_launch_count.restype = _i64
_lib.abft_version.restype = ctypes.c_char_p
_lib.abft_last_error.restype = ctypes.c_char_p
_lib.abft_phase_name.restype = ctypes.c_char_p
_lib.abft_phase_name.argtypes = [_i32]
_lib.abft_last_profile.argtypes = [_vp]
for _f in ("abft_encode", "abft_verify", "abft_potrf", "abft_potrf_ex", "abft_potrf_host", "abft_gen_spd",
           "abft_nccl_id", "abft_comm_init", "abft_comm_destroy", "abft_potrf_dist", "abft_comm_init_ipc",
           "abft_comm_attach_ipc"):
    getattr(_lib, _f).restype = _i32

EXPORTS = ["abft_encode", "abft_verify", "abft_potrf", "abft_potrf_ex", "abft_potrf_host", "abft_gen_spd",
           "abft_nccl_id", "abft_comm_init", "abft_comm_destroy", "abft_potrf_dist",
           "abft_last_launch_count", "abft_version", "abft_last_error", "abft_last_profile", "abft_dev_gemm_nt", "abft_dev_chol_inv",
           "abft_dev_chol_trace", "abft_potrf_dist_sim", "abft_graph_release",
           "abft_phase_name", "abft_comm_init_ipc", "abft_comm_attach_ipc"]


def lib():
    return _lib


# ---- marshalling helpers ---------------------------------------------------------------------
def _dev(x):
    """(pointer, leading dimension) of a column-major float64 CUDA tensor, or (int, None)."""
    if x is None:
        return None, None
    if isinstance(x, int):
        return x, None
    import torch
    assert x.is_cuda and x.dtype == torch.float64, "expected a float64 CUDA tensor"
    if x.dim() == 1:
        return x.data_ptr(), None
    assert x.stride(0) == 1, "expected column-major storage (stride(0) == 1)"
    return x.data_ptr(), x.stride(1)


def _stream(stream):
    if stream is None:
        import torch
        return torch.cuda.current_stream().cuda_stream
    return getattr(stream, "cuda_stream", stream)


def _inj(inj):
    if inj is None:
        return None, None
    arr = np.ascontiguousarray(inj, dtype=INJ_DTYPE)
    if len(arr) == 0 or arr[-1]["k"] != -1:
        arr = np.concatenate([arr, np.zeros(1, INJ_DTYPE)])
        arr[-1]["k"] = -1
    return arr, arr.ctypes.data


def _new_report(cap):
    ev = np.zeros(max(cap, 1), dtype=EVENT_DTYPE)
    rep = Report()
    rep.cap = cap
    rep.events = ev.ctypes.data
    return rep, ev


def _report_dict(rep, ev):
    n = min(rep.n_events, rep.cap)
    return dict(info=rep.info, n_checks=rep.n_checks, n_detected=rep.n_detected, n_data=rep.n_data,
                n_nonfinite=rep.n_nonfinite, n_chk1=rep.n_chk1, n_chk2=rep.n_chk2,
                n_uncorrectable=rep.n_uncorrectable, n_events=rep.n_events, events=ev[:n].copy(),
                seconds=rep.seconds, reruns=rep.reruns, max_noise_ratio=rep.max_noise_ratio)


MODE = {"enhanced": 0, "online": 1, "offline": 2, "enhanced_redo": 3}


def options(abft_enabled=True, K=1, c_tau=64.0, lookahead=0, profile=False, mode="enhanced", order="right", nchk=2,
            prows=1):
    """nchk: checksum rows per block, 2 (the paper's choice) or 3 (up to two errors per column).
    prows: multi-GPU process-grid rows (2D block-cyclic when > 1; 1 = column-cyclic)."""
    return Options(int(bool(abft_enabled)), int(K), float(c_tau), int(lookahead), int(bool(profile)),
                   MODE[mode] if isinstance(mode, str) else int(mode), {"right": 0, "left": 1}[order], int(nchk),
                   int(prows))


def abft_last_profile():
    """{phase name: dict(ms, launches, flops, bytes)} of the last profiled call on this thread."""
    pr = Profile()
    _lib.abft_last_profile(ctypes.byref(pr))
    out = {}
    for i in range(pr.nphase):
        out[_lib.abft_phase_name(i).decode()] = dict(ms=pr.ms[i], launches=int(pr.launches[i]),
                                                      flops=pr.flops[i], bytes=pr.bytes[i])
    return out


# ---- entry points (same names as the C-ABI) --------------------------------------------------
def abft_potrf_ex(n, nb, A, lda=None, stream=None, inj=None, report=True, cap=1 << 16, opt=None):
    """Factor A (n x n float64 CUDA, column-major) in place. Returns (status, report|None)."""
    p, ld = _dev(A)
    lda = lda if lda is not None else (ld if ld is not None else n)
    arr, pinj = _inj(inj)
    rep, ev = _new_report(cap) if report else (None, None)
    o = opt if opt is not None else options()
    st = _lib.abft_potrf_ex(n, nb, p, lda, _stream(stream), pinj, ctypes.byref(rep) if rep else None,
                            ctypes.byref(o))
    return st, (_report_dict(rep, ev) if rep else None)


def abft_potrf(n, nb, A, lda=None, stream=None, inj=None, report=True, cap=1 << 16):
    return abft_potrf_ex(n, nb, A, lda, stream, inj, report, cap, None)


def abft_potrf_host(n, nb, A_host, lda=None, stream=None, inj=None, report=True, cap=1 << 16, opt=None):
    """A_host: numpy float64 array, Fortran order (or a raw pointer + lda). Pinned memory is the
    caller's choice (e.g. a torch pinned tensor's .numpy() view)."""
    if isinstance(A_host, np.ndarray):
        assert A_host.dtype == np.float64 and A_host.flags.f_contiguous
        p, lda = A_host.ctypes.data, (lda or A_host.shape[0])
    else:
        p = A_host
    arr, pinj = _inj(inj)
    rep, ev = _new_report(cap) if report else (None, None)
    o = opt if opt is not None else options()
    st = _lib.abft_potrf_host(n, nb, p, lda, _stream(stream), pinj, ctypes.byref(rep) if rep else None,
                              ctypes.byref(o))
    return st, (_report_dict(rep, ev) if rep else None)


def abft_encode(n, nb, A, chk, scales, lda=None, ldchk=None, stream=None):
    pa, la = _dev(A)
    pc, lc = _dev(chk)
    ps, _ = _dev(scales)
    return _lib.abft_encode(n, nb, pa, lda or la or n, pc, ldchk or lc or max(1, 2 * (n // nb)), ps,
                            _stream(stream))


def abft_verify(n, nb, A, chk, scales, factored=False, correct=True, lda=None, ldchk=None, stream=None,
                report=True, cap=1 << 16):
    pa, la = _dev(A)
    pc, lc = _dev(chk)
    ps, _ = _dev(scales)
    rep, ev = _new_report(cap) if report else (None, None)
    st = _lib.abft_verify(n, nb, pa, lda or la or n, pc, ldchk or lc or max(1, 2 * (n // nb)), ps,
                          int(factored), int(correct), _stream(stream), ctypes.byref(rep) if rep else None)
    return st, (_report_dict(rep, ev) if rep else None)


def abft_gen_spd(n, A, seed=None, lda=None, stream=None):
    p, ld = _dev(A)
    return _lib.abft_gen_spd(n, n if seed is None else seed, p, lda or ld or n, _stream(stream))


def abft_nccl_id():
    buf = ctypes.create_string_buffer(128)
    st = _lib.abft_nccl_id(buf)
    return st, bytes(buf.raw)


def abft_comm_init(nranks, id128, rank):
    comm = ctypes.c_void_p()
    buf = ctypes.create_string_buffer(bytes(id128), 128)
    st = _lib.abft_comm_init(ctypes.byref(comm), nranks, buf, rank)
    return st, comm.value


def abft_comm_init_ipc(nranks, rank, cap_bytes):
    """Peer-memory (CUDA IPC) communicator: returns (status, comm, 64-byte handle of this rank)."""
    comm = ctypes.c_void_p()
    h = ctypes.create_string_buffer(64)
    st = _lib.abft_comm_init_ipc(ctypes.byref(comm), nranks, rank, int(cap_bytes), h)
    return st, comm.value, bytes(h.raw)


def abft_comm_attach_ipc(comm, handles):
    """handles: the nranks 64-byte handles in rank order."""
    buf = ctypes.create_string_buffer(b"".join(handles), 64 * len(handles))
    return _lib.abft_comm_attach_ipc(comm, buf)


def ipc_comm(n, nb, group=None):
    """Host plumbing of the peer-memory transport: every rank of the torch.distributed group
    exports its arena (sized for the largest message of an n x n factorisation with block nb)
    and maps every peer's. Returns the comm for abft_potrf_dist."""
    import torch.distributed as dist
    rank, world = dist.get_rank(group), dist.get_world_size(group)
    # packed panel + 16 abort slots + a received inv(L_kk) (2D) + its slot; event gather (8192)
    cap = 8 * ((n - nb) * nb + 2 * n + 2 * nb + 16 + nb * nb + 2) + 48 * 8192
    st, comm, h = abft_comm_init_ipc(world, rank, cap)
    assert st == 0, f"abft_comm_init_ipc: {st} {abft_last_error()}"
    hs = [None] * world
    dist.all_gather_object(hs, h, group=group)
    st = abft_comm_attach_ipc(comm, hs)
    assert st == 0, f"abft_comm_attach_ipc: {st} {abft_last_error()}"
    return comm


def abft_last_error():
    return _lib.abft_last_error().decode()


def abft_comm_destroy(comm):
    return _lib.abft_comm_destroy(comm)


def abft_potrf_dist(n, nb, A_local, comm, rank, nranks, lda=None, stream=None, inj=None, report=True,
                    cap=1 << 16, opt=None):
    p, ld = _dev(A_local)
    arr, pinj = _inj(inj)
    rep, ev = _new_report(cap) if report else (None, None)
    o = opt if opt is not None else options()
    st = _lib.abft_potrf_dist(n, nb, p, lda or ld or n, comm, rank, nranks, _stream(stream), pinj,
                              ctypes.byref(rep) if rep else None, ctypes.byref(o))
    return st, (_report_dict(rep, ev) if rep else None)


def abft_dev_gemm_nt(M, N, K, A, B, C, alpha=-1.0, beta=1.0, lower=True, stream=None):
    """Diagnostics: the update GEMM alone (C = beta C + alpha A B^T, lower triangle)."""
    pa, la = _dev(A)
    pb, lb = _dev(B)
    pc, lc = _dev(C)
    return _lib.abft_dev_gemm_nt(M, N, K, pa, la or M, pb, lb or N, pc, lc or M, alpha, beta, int(lower),
                                 _stream(stream))


def abft_potrf_dist_sim(n, nb, A_locals, lda=None, stream=None, inj=None, report=True, cap=1 << 16, opt=None):
    """Multi-GPU algorithm with nranks = len(A_locals) simulated ranks on one device (tests)."""
    ptrs = [(_dev(a)[0] if a is not None else None) or 0 for a in A_locals]
    lds = [_dev(a)[1] for a in A_locals if a is not None and _dev(a)[1] is not None]
    arrp = (ctypes.c_void_p * len(ptrs))(*ptrs)
    arr, pinj = _inj(inj)
    rep, ev = _new_report(cap) if report else (None, None)
    o = opt if opt is not None else options()
    st = _lib.abft_potrf_dist_sim(n, nb, len(ptrs), arrp, lda or (lds[0] if lds else n), _stream(stream), pinj,
                                  ctypes.byref(rep) if rep else None, ctypes.byref(o))
    return st, (_report_dict(rep, ev) if rep else None)


def owned_blocks(N, rank, nranks):
    """Block columns rank `rank` owns in the 1D block-cyclic layout (J mod nranks == rank)."""
    return list(range(rank, N, nranks))


def nccl_id_exchange(group=None):
    """Host plumbing of the multi-GPU path: rank 0 creates the NCCL unique id through the C-ABI
    and every rank of the torch.distributed group receives the same 128 bytes."""
    import torch.distributed as dist
    obj = [None]
    if dist.get_rank(group) == 0:
        st, nid = abft_nccl_id()
        assert st == 0, "abft_nccl_id failed"
        obj[0] = nid
    dist.broadcast_object_list(obj, src=0, group=group)
    return obj[0]


def block_cyclic_split(A, nb, nranks):
    """Global column-major matrix (numpy, n x n) -> per-rank local block columns (F-order arrays)."""
    n = A.shape[0]
    N = n // nb
    out = []
    for r in range(nranks):
        cols = [np.arange(J * nb, (J + 1) * nb) for J in range(r, N, nranks)]
        idx = np.concatenate(cols) if cols else np.zeros(0, dtype=np.int64)
        out.append(np.asfortranarray(A[:, idx]))
    return out


def grid_owner(I, J, nranks, prows=1):
    """Rank owning tile (I, J) on the prows x (nranks / prows) process grid (2D block-cyclic)."""
    pc = nranks // prows
    return (I % prows) * pc + J % pc


def block_cyclic_split_2d(A, nb, nranks, prows):
    """Per-rank local arrays of the 2D layout: rank r = pr * Pc + pc holds the block columns
    J = pc (mod Pc), full height (its own tiles are the rows I = pr (mod Pr); the rest is workspace)."""
    pc_n = nranks // prows
    cols = block_cyclic_split(A, nb, pc_n)
    return [cols[r % pc_n].copy(order="F") for r in range(nranks)]


def block_cyclic_join_2d(locals_, nb, n, prows):
    """Inverse of block_cyclic_split_2d: tile (I, J) from its owner's local array."""
    P = len(locals_)
    pc_n = P // prows
    A = np.zeros((n, n), order="F")
    N = n // nb
    for J in range(N):
        t = J // pc_n
        for I in range(N):
            L = locals_[grid_owner(I, J, P, prows)]
            A[I * nb:(I + 1) * nb, J * nb:(J + 1) * nb] = L[I * nb:(I + 1) * nb, t * nb:(t + 1) * nb]
    return A


def block_cyclic_join(locals_, nb, n):
    """Inverse of block_cyclic_split."""
    P = len(locals_)
    A = np.zeros((n, n), order="F")
    for r, L in enumerate(locals_):
        for t, J in enumerate(range(r, n // nb, P)):
            A[:, J * nb:(J + 1) * nb] = L[:, t * nb:(t + 1) * nb]
    return A


def abft_dev_chol_inv(nb, A, Li, stream=None):
    """Diagnostics: POTRF + inverse of one nb x nb block (A lower -> L, Li <- inv(L))."""
    pa, la = _dev(A)
    pl, _ = _dev(Li)
    return _lib.abft_dev_chol_inv(nb, pa, la or nb, pl, _stream(stream))


def abft_dev_chol_trace(nb, A, Li, stream=None):
    """Diagnostics: the task-graph diagonal block with a per-task trace; returns (ntasks, rows) with
    rows = (type, i, j, b, smid, cta, fetch_ns, start_ns, end_ns), or (status, [])."""
    import numpy as np
    pa, la = _dev(A)
    pl, _ = _dev(Li)
    cap = 4 * 4096
    buf = np.zeros(cap, dtype=np.uint64)
    nt = _lib.abft_dev_chol_trace(nb, pa, la or nb, pl, buf.ctypes.data, cap, _stream(stream))
    if nt <= 0:
        return nt, []
    rows = []
    for t in range(nt):
        w = int(buf[4 * t])
        rows.append((w & 255, (w >> 8) & 255, (w >> 16) & 255, (w >> 24) & 255, (w >> 32) & 0xFFFF, w >> 48,
                     int(buf[4 * t + 1]), int(buf[4 * t + 2]), int(buf[4 * t + 3])))
    return nt, rows


def abft_graph_release():
    """Free the cached graph-mode factorisation (graph + workspace) of this thread."""
    return int(_lib.abft_graph_release())


def abft_last_launch_count():
    return int(_lib.abft_last_launch_count())


def abft_version():
    return _lib.abft_version().decode()


def sorted_event_tuples(events):
    """(k, V, J, I, col, row, kind, rank) — the parity key shared with the oracle's tests."""
    return sorted((int(e["k"]), int(e["check"]), int(e["tile_j"]), int(e["tile_i"]), int(e["col"]),
                   int(e["row"]), int(e["kind"]), int(e["rank"])) for e in events)


def colmajor(A_np, device="cuda"):
    """Upload a numpy (any order) n x n matrix as a column-major float64 CUDA tensor view."""
    import torch
    t = torch.from_numpy(np.ascontiguousarray(np.asarray(A_np, dtype=np.float64).T)).to(device)
    return t.T   # stride(0) == 1


def to_numpy_colmajor(At):
    """Download a column-major CUDA tensor view into a Fortran-ordered numpy array."""
    return np.asfortranarray(At.T.contiguous().cpu().numpy().T)
