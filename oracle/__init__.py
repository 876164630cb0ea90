"""CPU oracle for the Enhanced Online-ABFT Cholesky — TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference legs may
import this package. The product path (paper_conf_ipps_chenlc16_b200/) never does, and this
package never imports the product path: they share no code.

The arithmetic lives in oracle/abft_oracle.c (plain C, FP64, OpenMP over independent tiles,
no BLAS, -ffp-contract=off); this module only marshals arguments through ctypes.
Functions and the paper passages they follow:
  potrf(...)   the whole Enhanced Online-ABFT factorisation, PAPER.md:100-195 (§III-IV),
               schedule V1..V6 of SURVEY.md §8c (readings A1-A22)
  encode(...)  checksum encoding, §IV.A
  verify(...)  one detect/locate/correct sweep over every lower tile, §IV.C
Parity pins: tests/test_oracle_pins.py (P1-P9 of SURVEY.md §8c). The threshold constants
C_tau = 64 and rho = 2^-30 are "parity unpinned" by the paper (pinned only by measured noise).
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "abft_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")

EVENT_DTYPE = np.dtype([
    ("k", "<i4"), ("check", "<i4"), ("tile_i", "<i4"), ("tile_j", "<i4"),
    ("row", "<i4"), ("col", "<i4"), ("kind", "<i4"), ("rank", "<i4"),
    ("delta1", "<f8"), ("delta2", "<f8"),
])
COUNT_DTYPE = np.dtype([
    ("n_checks", "<i8"), ("n_detected", "<i8"), ("n_data", "<i8"), ("n_nonfinite", "<i8"),
    ("n_chk1", "<i8"), ("n_chk2", "<i8"), ("n_uncorrectable", "<i8"),
    ("flops_factor", "<f8"), ("flops_chkupd", "<f8"), ("flops_check", "<f8"),
    ("flops_encode", "<f8"), ("bytes_check", "<f8"), ("max_ratio", "<f8"),
])
CHECK = {1: "V1", 2: "V2", 3: "V3", 4: "V4", 5: "V5", 6: "V6", 7: "V4R", 8: "V7"}
KIND = {1: "DATA", 2: "NONFINITE", 3: "CHK1", 4: "CHK2", 5: "UNCORRECTABLE", 6: "CHK3"}
STATUS = {0: "OK", 1: "UNCORRECTABLE", 2: "NOT_SPD"}


def build(force: bool = False) -> str:
    """Compile liboracle.so with gcc (plain C, OpenMP, strict FP)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        cmd = ["gcc", "-O3", "-std=c11", "-fopenmp", "-ffp-contract=off", "-fno-fast-math",
               "-fPIC", "-shared", "-o", _LIB, _SRC, "-lm"]
        subprocess.run(cmd, check=True)
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        _lib = ctypes.CDLL(build())
        i64, i32, dp, vp = ctypes.c_int64, ctypes.c_int, ctypes.POINTER(ctypes.c_double), ctypes.c_void_p
        _lib.oracle_potrf.argtypes = [i64, i64, vp, i64, vp, i64, i32, i32, ctypes.c_double, i32,
                                      vp, i64, ctypes.POINTER(i64), ctypes.POINTER(i64), vp, vp, vp]
        _lib.oracle_potrf.restype = i32
        _lib.oracle_potrf_mode.argtypes = [i64, i64, vp, i64, vp, i64, i32, i32, ctypes.c_double, i32, i32, i32,
                                           vp, i64, ctypes.POINTER(i64), ctypes.POINTER(i64), vp, vp, vp,
                                           ctypes.POINTER(i32)]
        _lib.oracle_potrf_mode.restype = i32
        _lib.oracle_potrf_nchk.argtypes = [i64, i64, vp, i64, vp, i64, i32, i32, ctypes.c_double, i32, i32, i32,
                                           vp, i64, ctypes.POINTER(i64), ctypes.POINTER(i64), vp, vp, vp,
                                           ctypes.POINTER(i32), i32]
        _lib.oracle_potrf_nchk.restype = i32
        _lib.oracle_potrf_grid.argtypes = [i64, i64, vp, i64, vp, i64, i32, i32, i32, ctypes.c_double, i32, i32,
                                           i32, vp, i64, ctypes.POINTER(i64), ctypes.POINTER(i64), vp, vp, vp,
                                           ctypes.POINTER(i32), i32]
        _lib.oracle_potrf_grid.restype = i32
        _lib.oracle_encode.argtypes = [i64, i64, vp, i64, vp, i64, vp]
        _lib.oracle_encode.restype = i32
        _lib.oracle_verify.argtypes = [i64, i64, vp, i64, vp, i64, vp, i32, i32, ctypes.c_double,
                                       vp, i64, ctypes.POINTER(i64), vp]
        _lib.oracle_verify.restype = i32
        _lib.oracle_num_threads.restype = i32
        _lib.oracle_potrf_prefix.argtypes = [i64, i64, vp, i64, i64, vp]
        _lib.oracle_potrf_prefix.restype = i32
    return _lib


def _ptr(a):
    return ctypes.c_void_p(a.ctypes.data) if a is not None else None


def _as_f(A):
    A = np.asarray(A, dtype=np.float64)
    return A if A.flags.f_contiguous else np.asfortranarray(A)


class Result:
    def __init__(self, L, status, info, events, counts, chk=None, scales=None):
        self.L, self.status, self.info, self.events, self.counts = L, status, info, events, counts
        self.chk, self.scales = chk, scales

    def event_tuples(self):
        """Events as sortable tuples (k, V, J, I, col, row, kind, rank) — the parity key."""
        return sorted_events(self.events)


def sorted_events(ev):
    keys = [(int(e["k"]), int(e["check"]), int(e["tile_j"]), int(e["tile_i"]), int(e["col"]),
             int(e["row"]), int(e["kind"]), int(e["rank"])) for e in ev]
    return sorted(keys)


MODE = {"enhanced": 0, "online": 1, "offline": 2, "enhanced_redo": 3}


def potrf(A, nb, inj=None, nranks=1, K=1, c_tau=64.0, abft=True, cap=1 << 16, inplace=False, mode="enhanced",
          order="right", nchk=2, prows=1):
    """ABFT Cholesky of A (lower), n % nb == 0. mode: "enhanced" (the paper's scheme, default),
    "online" or "offline" (its comparison schemes, which re-run once on an uncorrectable error).
    nchk: checksum rows per block, 2 (the paper's choice) or 3 (m+1 = 3 checksums locate and
    correct up to m = 2 errors per column; reading B10). Checksum-row injection targets are
    rows nchk*I + t of the checksum matrix.
    Returns Result with L in the lower triangle (upper triangle untouched), status (0/1/2),
    LAPACK info, sorted events, reruns.
    nranks > 1 simulates the multi-GPU path: process grid prows x (nranks / prows), tile (I, J) owned
    by rank (I % prows) * (nranks / prows) + J % (nranks / prows) (prows = 1: 1D column-cyclic;
    prows > 1: 2D block-cyclic); events carry the checking rank, every rank
    re-checks the panel tiles it receives (V4R) after its RECV hook."""
    L = _as_f(A)
    if not inplace:
        L = L.copy(order="F")
    n = L.shape[0]
    ev = np.zeros(cap, dtype=EVENT_DTYPE)
    cnt = np.zeros(1, dtype=COUNT_DTYPE)
    nev, info = ctypes.c_int64(0), ctypes.c_int64(0)
    if inj is None:
        inj_arr, ninj = None, 0
    else:
        inj_arr = np.ascontiguousarray(inj)
        ninj = int(np.argmax(inj_arr["k"] == -1)) if (inj_arr["k"] == -1).any() else len(inj_arr)
    N = n // nb if nb > 0 else 0
    chk = np.zeros((max(nchk * N, 1), n), dtype=np.float64, order="F")
    scl = np.zeros(n + 3 * N, dtype=np.float64)
    reruns = ctypes.c_int(0)
    st = lib().oracle_potrf_grid(n, nb, _ptr(L), max(n, 1), _ptr(inj_arr), ninj, nranks, prows, K, c_tau, int(abft),
                                 MODE[mode] if isinstance(mode, str) else int(mode),
                                 {"right": 0, "left": 1}[order], _ptr(ev), cap,
                                 ctypes.byref(nev), ctypes.byref(info), _ptr(cnt), _ptr(chk), _ptr(scl),
                                 ctypes.byref(reruns), int(nchk))
    if st < 0:
        raise ValueError(f"oracle_potrf: invalid argument {-st}")
    ev = ev[: min(nev.value, cap)]
    order = np.lexsort((ev["row"], ev["col"], ev["tile_i"], ev["tile_j"], ev["check"], ev["k"]))
    res = Result(L, st, info.value, ev[order], cnt[0], chk, scl)
    res.reruns = reruns.value
    return res


def encode(A, nb):
    """Returns (chk (2N x n, F-order), scales = [s (n) | S1 (N) | S2 (N)])."""
    A = _as_f(A)
    n = A.shape[0]
    N = n // nb
    chk = np.zeros((max(2 * N, 1), n), dtype=np.float64, order="F")
    scl = np.zeros(n + 2 * N, dtype=np.float64)
    st = lib().oracle_encode(n, nb, _ptr(A), max(n, 1), _ptr(chk), max(2 * N, 1), _ptr(scl))
    if st < 0:
        raise ValueError(f"oracle_encode: invalid argument {-st}")
    return chk, scl


def verify(A, nb, chk, scl, factored=False, correct=True, c_tau=64.0, cap=1 << 16):
    """One check of every lower tile. A and chk are modified in place when correct=True.
    Returns (status, events, counts)."""
    assert A.flags.f_contiguous and chk.flags.f_contiguous
    n = A.shape[0]
    ev = np.zeros(cap, dtype=EVENT_DTYPE)
    cnt = np.zeros(1, dtype=COUNT_DTYPE)
    nev = ctypes.c_int64(0)
    st = lib().oracle_verify(n, nb, _ptr(A), max(n, 1), _ptr(chk), chk.shape[0], _ptr(scl), int(factored),
                             int(correct), c_tau, _ptr(ev), cap, ctypes.byref(nev), _ptr(cnt))
    if st < 0:
        raise ValueError(f"oracle_verify: invalid argument {-st}")
    return st, ev[: min(nev.value, cap)], cnt[0]


def potrf_prefix(A, nb, kstop):
    """Timing sample (bench.py only): the Enhanced factorisation of A (modified in place, must be
    Fortran-ordered float64) stopped after kstop iterations. Returns (status, counts); counts'
    flops_* fields are the work those iterations did."""
    assert A.flags.f_contiguous and A.dtype == np.float64
    cnt = np.zeros(1, dtype=COUNT_DTYPE)
    st = lib().oracle_potrf_prefix(A.shape[0], nb, _ptr(A), max(A.shape[0], 1), int(kstop), _ptr(cnt))
    if st < 0:
        raise ValueError(f"oracle_potrf_prefix: invalid argument {-st}")
    return st, cnt[0]


def num_threads() -> int:
    return int(lib().oracle_num_threads())
