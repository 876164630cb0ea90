"""Seeded synthetic inputs shared by the oracle tests, the GPU tests and bench.py.

This module holds NONE of the method's arithmetic (no checksums, no factorisation, no
thresholds). It only produces input matrices and fault-injection lists, so that the CPU
oracle (`oracle/`) and the CUDA path (`paper_conf_ipps_chenlc16_b200/`) can be fed the
same bytes without sharing any code.  The CUDA library implements the same counter-based
generator on the device (`abft_gen_spd`), which the GPU tests compare bit-for-bit against
`spd_matrix` below.

Generator (reading A15; the paper does not specify its test matrices,
PAPER.md:381 only gives the sizes):
    U(i, j)  = top 53 bits of splitmix64(seed*n^2 + max(i,j)*n + min(i,j)) * 2^-53
    A[i, j]  = A[j, i] = U(i, j)            (i != j)
    A[i, i]  = U(i, i) + n                  (diagonally dominant => SPD, MAGMA style)
All arithmetic on the keys is modulo 2^64.

Matrices are returned column-major (numpy order='F'), the layout the C-ABI takes.
"""
from __future__ import annotations

import numpy as np

__all__ = [
    "splitmix64", "spd_matrix", "spd_diag", "pascal_mod2", "pascal", "HOOK", "TARGET",
    "inj_array", "INJ_DTYPE", "bit_mask", "c1_injections", "per_iteration_injections",
    "mixed_injections", "next4_injections",
]

_GOLDEN = np.uint64(0x9E3779B97F4A7C15)
_M1 = np.uint64(0xBF58476D1CE4E5B9)
_M2 = np.uint64(0x94D049BB133111EB)


def splitmix64(x):
    """splitmix64 finaliser of (x + golden gamma), vectorised over uint64 arrays."""
    with np.errstate(over="ignore"):
        z = np.asarray(x, dtype=np.uint64) + _GOLDEN
        z = (z ^ (z >> np.uint64(30))) * _M1
        z = (z ^ (z >> np.uint64(27))) * _M2
        return z ^ (z >> np.uint64(31))


def _u01(keys):
    return (splitmix64(keys) >> np.uint64(11)).astype(np.float64) * (2.0 ** -53)


def spd_matrix(n: int, seed: int | None = None, dtype=np.float64) -> np.ndarray:
    """Random SPD matrix of the A15 recipe, full symmetric, column-major (n x n)."""
    if seed is None:
        seed = n
    A = np.empty((n, n), dtype=dtype, order="F")
    if n == 0:
        return A
    nn = np.uint64(n)
    base = np.uint64(seed % (1 << 64)) * nn * nn if n else np.uint64(0)
    rows = np.arange(n, dtype=np.uint64)
    step = max(1, (1 << 23) // n)
    with np.errstate(over="ignore"):
        for c0 in range(0, n, step):
            c1 = min(n, c0 + step)
            cols = np.arange(c0, c1, dtype=np.uint64)
            hi = np.maximum(rows[:, None], cols[None, :])
            lo = np.minimum(rows[:, None], cols[None, :])
            A[:, c0:c1] = _u01(base + hi * nn + lo)
    A[np.arange(n), np.arange(n)] += float(n)
    return A


def spd_diag(n: int, seed: int | None = None) -> np.ndarray:
    """The diagonal of spd_matrix(n, seed) without forming the matrix (for full-size checks)."""
    if seed is None:
        seed = n
    nn = np.uint64(n)
    i = np.arange(n, dtype=np.uint64)
    with np.errstate(over="ignore"):
        return _u01(np.uint64(seed % (1 << 64)) * nn * nn + i * nn + i) + float(n)


def pascal_mod2(n: int) -> np.ndarray:
    """'Pascal-type' matrix of config C1: A_ij = 2^popcount(i & j) (0-based).

    Its Cholesky factor is L_ij = C(i, j) mod 2 = [(i & j) == j] (Lucas), so every
    intermediate of the factorisation is an integer below 2^53.
    """
    i = np.arange(n, dtype=np.int64)
    pc = np.vectorize(lambda v: bin(int(v)).count("1"))(i[:, None] & i[None, :]) if n else np.zeros((0, 0))
    return np.asfortranarray(np.power(2.0, pc).astype(np.float64))


def pascal(n: int) -> np.ndarray:
    """Symmetric Pascal matrix P_ij = C(i+j, i) (exact in FP64 for n <= 29)."""
    from math import comb
    P = np.empty((n, n), dtype=np.float64, order="F")
    for i in range(n):
        for j in range(n):
            P[i, j] = float(comb(i + j, i))
    return P


# ---- fault-injection lists -------------------------------------------------------------
# Hook points and targets. Codes are part of the C-ABI contract
# (include/abft.h) and are restated there; this module only builds lists of them.
HOOK = {"REST": 0, "POTRF_OUT": 1, "TRSM_OUT": 2, "UPDATE_OUT": 3, "RECV": 4}
TARGET = {"DATA": 0, "CHK": 1}

INJ_DTYPE = np.dtype([
    ("k", "<i4"), ("hook", "<i4"), ("target", "<i4"), ("pad0", "<i4"),
    ("row", "<i8"), ("col", "<i8"), ("xor_mask", "<u8"), ("rank", "<i4"), ("pad1", "<i4"),
])


def bit_mask(bit: int) -> int:
    return 1 << int(bit)


def inj_array(specs) -> np.ndarray:
    """List of dicts {k, hook, target, row, col, bit|xor_mask, rank} -> packed struct array
    terminated by k = -1 (the C-ABI list terminator)."""
    arr = np.zeros(len(specs) + 1, dtype=INJ_DTYPE)
    for t, s in enumerate(specs):
        arr[t]["k"] = s["k"]
        arr[t]["hook"] = HOOK[s["hook"]] if isinstance(s["hook"], str) else s["hook"]
        arr[t]["target"] = TARGET[s.get("target", "DATA")] if isinstance(s.get("target", "DATA"), str) else s["target"]
        arr[t]["row"] = s["row"]
        arr[t]["col"] = s["col"]
        arr[t]["xor_mask"] = s["xor_mask"] if "xor_mask" in s else bit_mask(s["bit"])
        arr[t]["rank"] = s.get("rank", 0)
    arr[-1]["k"] = -1
    return arr


def c1_injections():
    """Config C1: one storage error and one computing error."""
    return [
        dict(k=2, hook="REST", target="DATA", row=200, col=100, bit=52),
        dict(k=4, hook="UPDATE_OUT", target="DATA", row=230, col=170, bit=51),
    ]


def _rng(seed, k, salt):
    return int(splitmix64(np.uint64((seed * 1000003 + k * 7919 + salt) % (1 << 64))))


def per_iteration_injections(n: int, nb: int, seed: int | None = None, bits=(41, 62), kmax=None):
    """Config C2 (ii): one injection per iteration k, hook cycling REST / POTRF_OUT /
    TRSM_OUT / UPDATE_OUT, target element drawn from splitmix64(seed, k) inside the region
    that hook can touch at iteration k. Data targets only."""
    if seed is None:
        seed = n
    N = n // nb
    kmax = N - 1 if kmax is None else kmax
    hooks = ["REST", "POTRF_OUT", "TRSM_OUT", "UPDATE_OUT"]
    out = []
    for k in range(kmax):
        h = hooks[k % 4]
        r = _rng(seed, k, 1)
        bit = bits[0] + (r >> 40) % (bits[1] - bits[0] + 1)
        if h == "POTRF_OUT":           # inside L_kk (lower, incl. diagonal)
            a, b = (r % nb), ((r >> 20) % nb)
            row, col = k * nb + max(a, b), k * nb + min(a, b)
        elif h == "TRSM_OUT":          # inside the solved panel L(k+1:N, k)
            row = (k + 1) * nb + r % ((N - k - 1) * nb)
            col = k * nb + (r >> 24) % nb
        else:                          # REST / UPDATE_OUT: inside the trailing matrix
            lo = (k + 1) * nb if h == "UPDATE_OUT" else k * nb
            span = n - lo
            a, b = lo + r % span, lo + (r >> 24) % span
            row, col = max(a, b), min(a, b)
        out.append(dict(k=k, hook=h, target="DATA", row=int(row), col=int(col), bit=int(bit)))
    return out


def mixed_injections(n: int, nb: int, seed: int | None = None, kmax=None):
    """Config C3 style: per iteration one REST storage error (10% into checksum rows, 10% into
    finished L, else trailing data) plus one computing error (round-robin POTRF_OUT / TRSM_OUT
    / UPDATE_OUT). Bits 41..62. At most one pending error per (tile, column) is NOT enforced
    here; tests filter with the oracle's ground truth."""
    if seed is None:
        seed = n
    N = n // nb
    kmax = N - 1 if kmax is None else kmax
    out = []
    comp = ["POTRF_OUT", "TRSM_OUT", "UPDATE_OUT"]
    for k in range(kmax):
        r = _rng(seed, k, 11)
        bit = 41 + (r >> 50) % 22
        sel = r % 10
        if sel == 0 and k < N:        # checksum row of a trailing tile
            I = k + (r >> 8) % (N - k)
            J = k + (r >> 16) % (I - k + 1)
            out.append(dict(k=k, hook="REST", target="CHK", row=2 * I + ((r >> 24) & 1),
                            col=J * nb + (r >> 28) % nb, bit=int(bit)))
        elif sel == 1 and k > 0:      # finished L (caught by V6)
            a, b = (r >> 8) % n, (r >> 32) % (k * nb)
            row, col = max(a, b), b
            out.append(dict(k=k, hook="REST", target="DATA", row=int(row), col=int(col), bit=int(bit)))
        else:
            lo = k * nb
            a, b = lo + (r >> 8) % (n - lo), lo + (r >> 32) % (n - lo)
            out.append(dict(k=k, hook="REST", target="DATA", row=int(max(a, b)), col=int(min(a, b)),
                            bit=int(bit)))
        r2 = _rng(seed, k, 23)
        sub = dict(k=k, hook=comp[k % 3], target="DATA", bit=int(41 + (r2 >> 52) % 22))
        if sub["hook"] == "POTRF_OUT":
            a, b = r2 % nb, (r2 >> 20) % nb
            sub["row"], sub["col"] = k * nb + max(a, b), k * nb + min(a, b)
        elif sub["hook"] == "TRSM_OUT":
            if k == N - 1:
                continue
            sub["row"] = (k + 1) * nb + r2 % ((N - k - 1) * nb)
            sub["col"] = k * nb + (r2 >> 24) % nb
        else:
            if k == N - 1:
                continue
            lo = (k + 1) * nb
            a, b = lo + r2 % (n - lo), lo + (r2 >> 24) % (n - lo)
            sub["row"], sub["col"] = int(max(a, b)), int(min(a, b))
        out.append(sub)
    return out


def next4_injections(n: int, nb: int, seed: int | None = None):
    """NEXT-4 recipe (three checksum rows per block): the mixed_injections list with its
    checksum-row targets renumbered for three rows per block (row 2I+t -> 3I+t), plus a second
    error next to every tenth data error of hook UPDATE_OUT / REST whose bit is <= 58 (no
    overflow: a non-finite error would mask its partner), 97 rows further down the same block
    column of the same tile — two errors in one column of a block."""
    specs = []
    for sp in mixed_injections(n, nb, seed):
        if sp.get("target", "DATA") == "CHK":
            sp = dict(sp, row=3 * (sp["row"] // 2) + sp["row"] % 2)
        specs.append(sp)
    for sp in list(specs)[1::10]:
        if sp.get("target", "DATA") == "DATA" and sp["hook"] in ("UPDATE_OUT", "REST") and sp["bit"] <= 58:
            r2 = (sp["row"] // nb) * nb + (sp["row"] % nb + 97) % nb
            if r2 >= sp["col"] and r2 != sp["row"]:
                specs.append(dict(sp, row=r2, bit=53))
    return specs
