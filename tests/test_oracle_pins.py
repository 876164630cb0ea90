"""Pins of the CPU oracle against what the paper and mathematics fix.

None of these compare the oracle with itself: each checks a closed form, an invariant of the
paper's checksum relations, a textbook/library special case, brute force on tiny inputs, or
injection ground truth derived from the schedule (tests/_predict.py).
"""
import math
import os

import numpy as np
import pytest
import scipy.linalg

import oracle
import synthetic as syn
from tests._predict import predict, V, KIND

EPS = 2.0 ** -52
GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def lucas_L(n):
    i = np.arange(n)
    return ((i[:, None] & i[None, :]) == i[None, :]).astype(np.float64)


def floor_rel(L, Lref, A):
    """|dL_ij| / max(|L_ij|, 1e-3 sqrt(A_ii))  (reading A18)."""
    s = np.sqrt(np.diag(A))[:, None]
    return np.max(np.abs(np.tril(L) - np.tril(Lref)) / np.maximum(np.abs(np.tril(Lref)), 1e-3 * s))


# ---- P1: true Pascal, L_ij = C(i, j) exactly (closed form) --------------------------------
@pytest.mark.parametrize("n,nb", [(8, 8), (16, 8), (24, 8), (29, 29)])
def test_p1_pascal_binomial_factor(n, nb):
    A = syn.pascal(n)
    # At n = 29 (cond ~ 1e25) Alg. 2's triangular solve amplifies the rounding of the
    # (> 2^53) checksums far beyond the Cauchy-Schwarz threshold of reading A4, so V3 raises
    # false CHK2 alarms there: the factor arithmetic is pinned with the checks off, and the
    # checked path on the n <= 24 cases (A4 limitation).
    r = oracle.potrf(A, nb, abft=(n <= 24))
    assert r.status == 0 and len(r.events) == 0
    Lx = np.array([[float(math.comb(i, j)) if i >= j else 0.0 for j in range(n)] for i in range(n)])
    assert np.array_equal(np.tril(r.L), Lx)
    assert np.array_equal(np.triu(r.L, 1), np.triu(A, 1)), "strict upper triangle must be untouched"


# ---- P2: Pascal mod 2 (config C1), L = Lucas, with the C1 injections (golden) -------------
def _golden_c1():
    rows = []
    for line in open(os.path.join(GOLDEN, "c1_events.txt")):
        line = line.strip()
        if line and not line.startswith("#"):
            k, v, ti, tj, row, col, kind, rank = map(int, line.split())
            rows.append((k, v, tj, ti, col, row, kind, rank))
    return sorted(rows)


def test_p2_pascal_mod2_fault_free():
    A = syn.pascal_mod2(256)
    r = oracle.potrf(A, 32)
    assert r.status == 0 and len(r.events) == 0
    assert np.array_equal(np.tril(r.L), lucas_L(256))


def test_p2_c1_injections_golden_events_and_exact_factor():
    A = syn.pascal_mod2(256)
    r = oracle.potrf(A, 32, inj=syn.inj_array(syn.c1_injections()))
    assert r.status == 0
    assert r.event_tuples() == _golden_c1()
    assert np.array_equal(np.tril(r.L), lucas_L(256))      # P7: bit-exact after correction
    # the schedule predictor agrees with the hand-derived golden file
    assert sorted(predict(s, 256, 32) for s in syn.c1_injections()) == _golden_c1()


def test_p2_four_injections_bits_51_52_55_63():
    A = syn.pascal_mod2(256)
    specs = [dict(k=1, hook="REST", row=100, col=70, bit=52),
             dict(k=3, hook="UPDATE_OUT", row=250, col=140, bit=51),
             dict(k=2, hook="TRSM_OUT", row=200, col=72, bit=55),
             dict(k=5, hook="POTRF_OUT", row=170, col=165, bit=63)]
    r = oracle.potrf(A, 32, inj=syn.inj_array(specs))
    # an exact-zero element flipped in its sign bit (bit 63) is masked: -0.0 == 0.0
    live = [s for s in specs if not (s["bit"] == 63 and lucas_L(256)[s["row"], s["col"]] == 0)]
    assert r.status == 0
    assert r.event_tuples() == sorted(predict(s, 256, 32) for s in live)
    assert np.array_equal(np.tril(r.L), lucas_L(256))


# ---- P3: brute force vs textbook unblocked Cholesky-Banachiewicz (separate code) ---------
def banachiewicz(A):
    n = A.shape[0]
    L = [[0.0] * n for _ in range(n)]
    for i in range(n):
        for j in range(i + 1):
            s = sum(L[i][p] * L[j][p] for p in range(j))
            L[i][j] = math.sqrt(A[i, i] - s) if i == j else (A[i, j] - s) / L[j][j]
    return np.array(L)


@pytest.mark.parametrize("n,nb,seed", [(8, 4, 1), (24, 8, 2), (32, 8, 3), (48, 16, 4), (64, 16, 5),
                                       (64, 32, 6), (60, 12, 7), (9, 3, 8)])
def test_p3_blocked_vs_unblocked_textbook(n, nb, seed):
    A = syn.spd_matrix(n, seed=seed)
    r = oracle.potrf(A, nb)
    assert r.status == 0 and len(r.events) == 0
    Lt = banachiewicz(A)
    s = np.sqrt(np.diag(A))[:, None]
    assert np.max(np.abs(np.tril(r.L) - Lt) / s) <= 8 * EPS


# ---- P4: LAPACK dpotrf at scale; backward error --------------------------------------------
@pytest.mark.parametrize("n,nb", [(512, 64), (1024, 128), (1536, 256)])
def test_p4_lapack_and_backward_error(n, nb):
    A = syn.spd_matrix(n)
    r = oracle.potrf(A, nb)
    assert r.status == 0 and len(r.events) == 0
    Lref = scipy.linalg.cholesky(A, lower=True)
    assert floor_rel(r.L, Lref, A) <= 1e-11
    L = np.tril(r.L)
    be = np.linalg.norm(A - L @ L.T) / np.linalg.norm(A)
    assert be <= 10 * n * EPS


def test_p4_not_spd_info_matches_lapack():
    n, nb = 96, 16
    A = syn.spd_matrix(n, seed=3)
    A[70, 70] = -5.0                       # leading minor of order 71 is not positive
    r = oracle.potrf(A, nb)
    _, info = scipy.linalg.lapack.dpotrf(A, lower=1)
    assert r.status == 2 and r.info == info == 71


# ---- P5: checksum maintenance invariants ---------------------
@pytest.mark.parametrize("n,nb", [(512, 64), (1024, 256)])
def test_p5_checksums_carried_to_v_tril_L(n, nb):
    A = syn.spd_matrix(n)
    r = oracle.potrf(A, nb)
    N = n // nb
    L = np.tril(r.L)
    w = np.arange(1, nb + 1, dtype=np.float64)
    S1 = r.scales[n:n + N]
    for I in range(N):
        for J in range(I + 1):
            T = L[I * nb:(I + 1) * nb, J * nb:(J + 1) * nb]
            c1 = r.chk[2 * I, J * nb:(J + 1) * nb]
            c2 = r.chk[2 * I + 1, J * nb:(J + 1) * nb]
            tau = 64 * EPS * S1[I]
            assert np.max(np.abs(T.sum(0) - c1)) <= tau / 64
            assert np.max(np.abs(w @ T - c2)) <= tau * nb / 64
    # and every check in the run passed with a wide margin
    assert r.counts["max_ratio"] <= 2.0 ** -6


def test_p5_encode_is_column_sums_of_symmetric_tiles():
    n, nb = 96, 32
    A = syn.spd_matrix(n, seed=9)
    Al = np.tril(A)
    Asym = Al + np.tril(Al, -1).T
    chk, scl = oracle.encode(np.asfortranarray(Al + np.triu(np.full((n, n), 7.0), 1)), nb)  # upper is junk
    w = np.arange(1, nb + 1)
    for I in range(n // nb):
        for J in range(I + 1):
            T = Asym[I * nb:(I + 1) * nb, J * nb:(J + 1) * nb]
            assert np.allclose(chk[2 * I, J * nb:(J + 1) * nb], T.sum(0), rtol=0, atol=1e-12 * n)
            assert np.allclose(chk[2 * I + 1, J * nb:(J + 1) * nb], w @ T, rtol=0, atol=1e-12 * n * nb)
    s = np.sqrt(np.diag(A))
    assert np.array_equal(scl[:n], s)
    assert np.allclose(scl[n:n + 3], s.reshape(3, nb).sum(1), rtol=1e-15)
    assert np.allclose(scl[n + 3:], (s.reshape(3, nb) * w).sum(1), rtol=1e-15)


# ---- P6/P7: injection ground truth ------------------------------------------------------------
def test_p6_exhaustive_rest0_every_lower_element():
    """Brute force: every lower element of a small matrix, storage error at REST(0), bit 60."""
    n, nb = 24, 8
    A = syn.spd_matrix(n, seed=11)
    ref = oracle.potrf(A, nb)
    for r_ in range(n):
        for c_ in range(r_ + 1):
            spec = dict(k=0, hook="REST", row=r_, col=c_, bit=60)
            res = oracle.potrf(A, nb, inj=syn.inj_array([spec]))
            assert res.status == 0
            assert res.event_tuples() == [predict(spec, n, nb)], (r_, c_)
            assert floor_rel(res.L, ref.L, A) <= 1e-12


@pytest.mark.parametrize("hook", ["REST", "POTRF_OUT", "TRSM_OUT", "UPDATE_OUT"])
def test_p6_per_iteration_injections(hook):
    n, nb = 1024, 128
    A = syn.spd_matrix(n)
    specs = [s for s in syn.per_iteration_injections(n, nb, bits=(45, 61)) if s["hook"] == hook]
    ref = oracle.potrf(A, nb)
    r = oracle.potrf(A, nb, inj=syn.inj_array(specs))
    assert r.status == 0
    assert r.event_tuples() == sorted(predict(s, n, nb) for s in specs)
    assert floor_rel(r.L, ref.L, A) <= 1e-11


def test_p6_c2_schedule_all_hooks():
    n, nb = 4096, 256
    A = syn.spd_matrix(n)
    specs = syn.per_iteration_injections(n, nb)
    r = oracle.potrf(A, nb, inj=syn.inj_array(specs))
    assert r.status == 0
    pred = sorted(predict(s, n, nb) for s in specs)
    assert r.event_tuples() == pred
    Lref = scipy.linalg.cholesky(A, lower=True)
    assert floor_rel(r.L, Lref, A) <= 1e-11


@pytest.mark.parametrize("cr_off", [0, 1])
def test_p6_checksum_row_errors_leave_L_bit_identical(cr_off):
    n, nb = 512, 64
    A = syn.spd_matrix(n)
    specs = [dict(k=1, hook="REST", target="CHK", row=2 * 5 + cr_off, col=3 * nb + 7, bit=55),
             dict(k=2, hook="REST", target="CHK", row=2 * 2 + cr_off, col=2 * nb + 9, bit=50),
             dict(k=4, hook="REST", target="CHK", row=2 * 1 + cr_off, col=0 * nb + 3, bit=49)]
    ref = oracle.potrf(A, nb)
    r = oracle.potrf(A, nb, inj=syn.inj_array(specs))
    assert r.status == 0
    assert r.event_tuples() == sorted(predict(s, n, nb) for s in specs)
    assert np.array_equal(r.L, ref.L)


def test_p6_diagonal_tile_symmetric_dedupe():
    """An error in the stored lower half of an unfactored diagonal tile appears twice in
    sym(tril(T)) (row r of column c and row c of column r): exactly one event (reading A12)."""
    n, nb = 256, 32
    A = syn.spd_matrix(n, seed=5)
    ref = oracle.potrf(A, nb)
    for (row, col) in [(100, 97), (127, 96), (200, 200), (230, 224)]:
        spec = dict(k=2, hook="REST", row=row, col=col, bit=57)
        r = oracle.potrf(A, nb, inj=syn.inj_array([spec]))
        assert r.event_tuples() == [predict(spec, n, nb)]
        assert floor_rel(r.L, ref.L, A) <= 1e-12


def test_p6_nonfinite_rule():
    n, nb = 256, 64
    A = syn.spd_matrix(n, seed=2)
    ref = oracle.potrf(A, nb)
    # bit 62 of an input value in [0.25, 1): exponent 0x3FD/0x3FE -> 0x7FD/0x7FE, |x| >= 4e307;
    # with row weight >= 41 the weighted recalculation overflows -> non-finite delta ->
    # NONFINITE, located by argmax |X|. REST(0) reads the input value itself.
    row = next(r_ for r_ in range(192 + 40, 256) if A[r_, 150] >= 0.25)
    spec = dict(k=0, hook="REST", row=row, col=150, bit=62)
    r = oracle.potrf(A, nb, inj=syn.inj_array([spec]))
    e = predict(spec, n, nb)
    assert r.event_tuples() == [e[:6] + (KIND["NONFINITE"], 0)]
    assert floor_rel(r.L, ref.L, A) <= 1e-12
    # a mask that turns the stored value into a NaN (exponent all ones, mantissa != 0)
    nanmask = int(np.float64(A[200, 150]).view(np.uint64)) ^ 0x7FF8000000000001
    spec = dict(k=0, hook="REST", row=200, col=150, xor_mask=nanmask)
    r = oracle.potrf(A, nb, inj=syn.inj_array([spec]))
    assert [t[6] for t in r.event_tuples()] == [KIND["NONFINITE"]]
    assert floor_rel(r.L, ref.L, A) <= 1e-12


def test_p6_two_errors_one_column_is_uncorrectable():
    n, nb = 256, 64
    A = syn.spd_matrix(n, seed=2)
    specs = [dict(k=1, hook="REST", row=200, col=150, bit=55),
             dict(k=1, hook="REST", row=220, col=150, bit=56)]
    r = oracle.potrf(A, nb, inj=syn.inj_array(specs))
    assert r.status == 1
    assert [t[6] for t in r.event_tuples()] == [KIND["UNCORRECTABLE"]]
    assert r.event_tuples()[0][:5] == (1, V["V5"], 2, 3, 150 - 128)


def test_p6_masked_small_injection_produces_no_event():
    n, nb = 512, 64
    A = syn.spd_matrix(n)
    spec = dict(k=1, hook="REST", row=300, col=200, bit=2)   # |Delta| ~ 1e-16 << tau
    r = oracle.potrf(A, nb, inj=syn.inj_array([spec]))
    assert r.status == 0 and len(r.events) == 0


def test_p6_factored_L_storage_error_caught_by_v6():
    n, nb = 512, 64
    A = syn.spd_matrix(n)
    ref = oracle.potrf(A, nb)
    specs = [dict(k=5, hook="REST", row=300, col=20, bit=50),     # finished panel 0
             dict(k=8, hook="REST", row=70, col=70, bit=50)]      # finished diagonal L_11 (k = N)
    r = oracle.potrf(A, nb, inj=syn.inj_array(specs))
    assert r.event_tuples() == sorted(predict(s, n, nb) for s in specs)
    assert floor_rel(r.L, ref.L, A) <= 1e-12


# ---- multi-rank simulation and Opt. 3 --------------------------------------------------------
@pytest.mark.parametrize("P", [2, 3, 4])
def test_nranks_simulation_matches_single_rank(P):
    n, nb = 1024, 128
    A = syn.spd_matrix(n)
    specs = syn.per_iteration_injections(n, nb, bits=(45, 61))
    r1 = oracle.potrf(A, nb, inj=syn.inj_array(specs))
    rP = oracle.potrf(A, nb, inj=syn.inj_array(specs), nranks=P)
    assert np.array_equal(r1.L, rP.L)
    # same decisions; the rank field names the owner of the block column that ran the check
    assert [e[:7] for e in r1.event_tuples()] == [e[:7] for e in rP.event_tuples() if e[1] != V["V4R"]]
    assert all(e[7] == e[2] % P for e in rP.event_tuples() if e[1] != V["V4R"])


def test_recv_injection_caught_by_receiver():
    n, nb, P = 1024, 128, 4
    A = syn.spd_matrix(n)
    ref = oracle.potrf(A, nb)
    specs = [dict(k=1, hook="RECV", row=700, col=150, bit=50, rank=3),
             dict(k=2, hook="RECV", target="CHK", row=2 * 6 + 1, col=2 * nb + 5, bit=50, rank=0)]
    r = oracle.potrf(A, nb, inj=syn.inj_array(specs), nranks=P)
    assert r.event_tuples() == sorted(predict(s, n, nb) for s in specs)
    assert floor_rel(r.L, ref.L, A) <= 1e-12


def _grid_owner(I, J, P, prows):
    pc = P // prows
    return (I % prows) * pc + J % pc


@pytest.mark.parametrize("P,prows", [(2, 2), (4, 2), (6, 2), (6, 3), (8, 4)])
def test_grid_simulation_matches_single_rank(P, prows):
    """2D block-cyclic simulation: the arithmetic of every tile is the one-process
    arithmetic, so L is bit-identical and every decision is the same; the rank field names the
    owner of the tile that was checked, (I mod prows) * pcols + J mod pcols."""
    n, nb = 1024, 128
    A = syn.spd_matrix(n)
    specs = syn.per_iteration_injections(n, nb, bits=(45, 61))
    r1 = oracle.potrf(A, nb, inj=syn.inj_array(specs))
    rP = oracle.potrf(A, nb, inj=syn.inj_array(specs), nranks=P, prows=prows)
    assert rP.status == 0 and np.array_equal(r1.L, rP.L)
    assert [e[:7] for e in r1.event_tuples()] == [e[:7] for e in rP.event_tuples() if e[1] != V["V4R"]]
    assert all(e[7] == _grid_owner(e[3], e[2], P, prows) for e in rP.event_tuples() if e[1] != V["V4R"])
    # fault-free: the tile checks are the one-rank ones plus one V4R per (rank, received panel tile)
    f1, fP = oracle.potrf(A, nb), oracle.potrf(A, nb, nranks=P, prows=prows)
    N = n // nb
    v4r = sum(1 for k in range(N - 1) for r in range(P) for i in range(k + 1, N) if _grid_owner(i, k, P, prows) != r)
    assert fP.counts["n_checks"] - f1.counts["n_checks"] == v4r
    assert np.array_equal(f1.L, fP.L) and len(fP.events) == 0


def test_grid_recv_injection_caught_by_receiver_only():
    """A RECV error lands in the receiving rank's copy of a panel tile it does not own and is
    corrected there by V4R (event on that rank); a RECV target inside a tile the rank owns is not
    received by it and has no effect."""
    n, nb, P, prows = 1024, 128, 4, 2
    A = syn.spd_matrix(n)
    ref = oracle.potrf(A, nb)
    # k = 1: panel tiles (i, 1), owners (i % 2) * 2 + 1 -> tile 5 (rows 640..767) belongs to rank 3
    assert _grid_owner(5, 1, P, prows) == 3 and _grid_owner(6, 2, P, prows) == 0
    specs = [dict(k=1, hook="RECV", row=700, col=150, bit=50, rank=0),
             dict(k=2, hook="RECV", target="CHK", row=2 * 6 + 1, col=2 * nb + 5, bit=50, rank=3)]
    r = oracle.potrf(A, nb, inj=syn.inj_array(specs), nranks=P, prows=prows)
    assert r.event_tuples() == sorted(predict(s, n, nb) for s in specs)
    assert floor_rel(r.L, ref.L, A) <= 1e-12
    owned = [dict(k=1, hook="RECV", row=700, col=150, bit=50, rank=3)]   # rank 3 owns tile (5, 1)
    r2 = oracle.potrf(A, nb, inj=syn.inj_array(owned), nranks=P, prows=prows)
    assert len(r2.events) == 0 and np.array_equal(r2.L, ref.L)


@pytest.mark.parametrize("K", [3, 5])
def test_opt3_verify_every_K(K):
    n, nb = 1024, 64
    A = syn.spd_matrix(n)
    ref = oracle.potrf(A, nb)
    rK = oracle.potrf(A, nb, K=K)
    assert np.array_equal(rK.L, ref.L) and len(rK.events) == 0
    specs = [dict(k=2, hook="REST", row=900, col=700, bit=50),
             dict(k=4, hook="UPDATE_OUT", row=600, col=330, bit=52)]
    r = oracle.potrf(A, nb, inj=syn.inj_array(specs), K=K)
    assert r.event_tuples() == sorted(predict(s, n, nb, K=K) for s in specs)
    assert rK.counts["flops_check"] < ref.counts["flops_check"]


# ---- P8: overhead bookkeeping vs the paper's closed forms (Tables III, V) ----------
def test_p8_counters_leading_terms():
    n, nb = 2048, 128
    A = syn.spd_matrix(n)
    r = oracle.potrf(A, nb)
    c = r.counts
    assert abs(c["flops_factor"] / (n ** 3 / 3) - 1) < 3 * nb / n        # N_Cho = n^3/3
    assert abs(c["flops_chkupd"] / (2 * n ** 3 / (3 * nb)) - 1) < 6 * nb / n  # GEMM row, Table III
    assert abs(c["flops_encode"] / (2 * n ** 2) - 1) < 2 * nb / n
    # V5 recalculation ~ 2n^3/(3B) (Table V GEMM, K=1) + O(n^2) for V1-V4, V6
    assert abs(c["flops_check"] / (2 * n ** 3 / (3 * nb)) - 1) < 12 * nb / n


# ---- P9: threshold margin (C_tau = 64 is parity-unpinned by the paper) --------------------
@pytest.mark.parametrize("n,nb", [(1024, 64), (2048, 512), (2048, 1024), (4096, 256)])
def test_p9_noise_margin(n, nb):
    """Fault-free rounding noise, normalised by the threshold, stays below 2^-6 (SURVEY SX2:
    <= 0.064 eps*scale for n <= 8192, i.e. >= 640x margin to C_tau = 64)."""
    A = syn.spd_matrix(n)
    r = oracle.potrf(A, nb)
    assert r.status == 0 and len(r.events) == 0
    assert r.counts["max_ratio"] <= 2.0 ** -6


def test_verify_entry_detects_and_corrects():
    n, nb = 256, 64
    A = np.asfortranarray(np.tril(syn.spd_matrix(n, seed=4)))
    chk, scl = oracle.encode(A, nb)
    st, ev, _ = oracle.verify(A.copy(order="F"), nb, chk.copy(order="F"), scl)
    assert st == 0 and len(ev) == 0
    B = A.copy(order="F")
    B[150, 70] += 3.0
    st, ev, _ = oracle.verify(B, nb, chk.copy(order="F"), scl)
    assert st == 0 and len(ev) == 1
    assert (ev[0]["tile_i"], ev[0]["tile_j"], ev[0]["row"], ev[0]["col"]) == (2, 1, 150 - 128, 70 - 64)
    assert abs(ev[0]["delta1"] - 3.0) < 1e-9 and abs(ev[0]["delta2"] - 3.0 * (150 - 128 + 1)) < 1e-8
    assert abs(B[150, 70] - A[150, 70]) < 1e-13


# ---- comparison schemes (NEXT-2): Tables VII/VIII ---------------------------
SCHEME_FAULTS = {
    "none": [],
    # computation error: corrupt the output of the trailing update
    "computation": [dict(k=2, hook="UPDATE_OUT", row=800, col=500, bit=50)],
    # memory error "between checksum verification and data access": the diagonal block of
    # column 3 after its last verification (V5 of iteration 2) and before POTRF(3) reads it
    "memory": [dict(k=3, hook="REST", row=3 * 128 + 100, col=3 * 128 + 50, bit=50)],
}
# Enhanced corrects both kinds; Online corrects computing errors but must re-do the
# decomposition for a memory error; Offline must re-do it for both.
SCHEME_RERUNS = {("enhanced", "none"): 0, ("enhanced", "computation"): 0, ("enhanced", "memory"): 0,
                 ("online", "none"): 0, ("online", "computation"): 0, ("online", "memory"): 1,
                 ("offline", "none"): 0, ("offline", "computation"): 1, ("offline", "memory"): 1}


@pytest.mark.parametrize("mode", ["enhanced", "online", "offline"])
@pytest.mark.parametrize("fault", ["none", "computation", "memory"])
def test_schemes_table_vii_capability(mode, fault):
    n, nb = 1024, 128
    A = syn.spd_matrix(n)
    ref = oracle.potrf(A, nb)
    specs = SCHEME_FAULTS[fault]
    r = oracle.potrf(A, nb, inj=syn.inj_array(specs) if specs else None, mode=mode)
    assert r.status == 0
    assert r.reruns == SCHEME_RERUNS[(mode, fault)]
    assert floor_rel(r.L, ref.L, A) <= 1e-11          # every scheme ends with the right factor
    if mode == "enhanced" and specs:
        assert r.event_tuples() == [predict(s, n, nb) for s in specs]


# ---- NEXT-1: the paper's own (left-looking, MAGMA Alg. 1) order with Table I's checks ------
from tests._predict import predict_left


@pytest.mark.parametrize("n,nb", [(512, 64), (1024, 128), (96, 24)])
def test_left_looking_factor_matches_lapack(n, nb):
    A = syn.spd_matrix(n)
    r = oracle.potrf(A, nb, order="left")
    assert r.status == 0 and len(r.events) == 0
    assert floor_rel(r.L, scipy.linalg.cholesky(A, lower=True), A) <= 1e-11
    assert r.counts["max_ratio"] <= 2.0 ** -6


def test_left_looking_pascal_mod2_c1_exact():
    A = syn.pascal_mod2(256)
    specs = [dict(k=2, hook="REST", row=232, col=40, bit=52),      # finished L block (value 1), read by V7
             dict(k=4, hook="UPDATE_OUT", row=230, col=130, bit=51)]
    r = oracle.potrf(A, 32, inj=syn.inj_array(specs), order="left")
    i = np.arange(256)
    assert np.array_equal(np.tril(r.L), ((i[:, None] & i[None, :]) == i[None, :]).astype(float))
    assert r.event_tuples() == sorted(predict_left(s, 256, 32) for s in specs)


@pytest.mark.parametrize("K", [1, 3])
def test_left_looking_injection_ground_truth(K):
    """K = 1: each error is reported once, at its first read. K = 3 (Opt. 3): a D block is not
    re-verified at every read, so an error there is used by the GEMM first and shows up again in
    the updated column (caught by V5, one element per column) before V7 repairs the source."""
    n, nb = 1024, 128
    A = syn.spd_matrix(n)
    ref = oracle.potrf(A, nb, order="left")
    specs = [dict(k=2, hook="REST", row=900, col=130, bit=50),
             dict(k=3, hook="TRSM_OUT", row=700, col=3 * nb + 5, bit=50),
             dict(k=4, hook="UPDATE_OUT", row=800, col=4 * nb + 9, bit=52),
             dict(k=5, hook="POTRF_OUT", row=5 * nb + 9, col=5 * nb + 2, bit=52),
             dict(k=1, hook="REST", row=1000, col=7 * nb + 3, bit=50),
             dict(k=8, hook="REST", row=600, col=300, bit=50)]
    r = oracle.potrf(A, nb, inj=syn.inj_array(specs), order="left", K=K)
    assert r.status == 0
    if K == 1:
        assert r.event_tuples() == sorted(predict_left(s, n, nb, K=K) for s in specs)
    else:
        assert set(predict_left(s, n, nb, K=K) for s in specs) <= set(r.event_tuples())
    assert floor_rel(r.L, ref.L, A) <= 1e-11


def test_left_looking_verifies_more_than_right_looking():
    """Table I / P:255: the Enhanced scheme re-verifies L blocks at every read in the left-looking
    order (O(n) verifications per block), so its check volume exceeds the right-looking one."""
    n, nb = 1024, 64
    A = syn.spd_matrix(n)
    rl = oracle.potrf(A, nb)
    ll = oracle.potrf(A, nb, order="left")
    assert ll.counts["bytes_check"] > rl.counts["bytes_check"]
    ll3 = oracle.potrf(A, nb, order="left", K=3)
    assert ll3.counts["bytes_check"] < ll.counts["bytes_check"]


# ---- NEXT-4: more errors in a block column than two checksums locate ("m+1 checksums
# ... up to m errors per column"; reading A11) -> Enhanced + re-do (the paper's re-do) ----
TWO_IN_A_COLUMN = [dict(k=1, hook="REST", row=300, col=150, bit=55),
                   dict(k=1, hook="REST", row=310, col=150, bit=56)]   # same tile (2,1), same column


def test_enhanced_two_errors_in_a_column_uncorrectable_without_redo():
    n, nb = 512, 64
    A = syn.spd_matrix(n, seed=2)
    r = oracle.potrf(A, nb, inj=syn.inj_array(TWO_IN_A_COLUMN))
    assert r.status == 1 and r.reruns == 0
    assert any(e[6] == KIND["UNCORRECTABLE"] for e in r.event_tuples())


def test_enhanced_redo_recovers_and_matches_lapack():
    """With re-do the call ends with status 0, one re-run, the UNCORRECTABLE event of the first
    run in the report, and the factor of the fault-free run (bit-identical: the re-run starts
    from the saved input without faults) = LAPACK within P4 tolerances."""
    n, nb = 512, 64
    A = syn.spd_matrix(n, seed=2)
    r = oracle.potrf(A, nb, inj=syn.inj_array(TWO_IN_A_COLUMN), mode="enhanced_redo")
    clean = oracle.potrf(A, nb)
    assert r.status == 0 and r.reruns == 1
    assert any(e[6] == KIND["UNCORRECTABLE"] for e in r.event_tuples())
    assert np.array_equal(np.tril(r.L), np.tril(clean.L))
    assert floor_rel(r.L, scipy.linalg.cholesky(A, lower=True), A) <= 1e-11
    # single errors are corrected in place: no re-run
    one = oracle.potrf(A, nb, inj=syn.inj_array(TWO_IN_A_COLUMN[:1]), mode="enhanced_redo")
    assert one.status == 0 and one.reruns == 0 and len(one.events) == 1


# ---- NEXT-4: m+1 = 3 checksums locate and correct up to m = 2 errors per column -----
# Reading B10: v3 = [1, 4, ..., B^2]; two errors Da (weight wa), Db (weight wb) give
# d1 = Da + Db, d2 = wa Da + wb Db, d3 = wa^2 Da + wb^2 Db, hence d3 = (wa + wb) d2 - wa wb d1; the
# integers wa < wb are found by scanning S = wa + wb; corrections from the first two checksum rows.

def test_next4_three_checksums_same_factor_and_checksum_invariant():
    """nchk = 3 changes no data arithmetic: L bit-identical to nchk = 2, no event; the carried
    third checksum row equals v3^T tril(L) (the P5 invariant with weights r^2)."""
    n, nb = 512, 64
    A = syn.spd_matrix(n)
    r2 = oracle.potrf(A, nb)
    r3 = oracle.potrf(A, nb, nchk=3)
    assert r3.status == 0 and len(r3.events) == 0
    assert np.array_equal(np.tril(r2.L), np.tril(r3.L))
    L = np.tril(r3.L)
    N = n // nb
    w3 = (np.arange(1, nb + 1, dtype=np.float64)) ** 2
    for I in range(N):
        for J in range(I + 1):
            T = L[I * nb:(I + 1) * nb, J * nb:(J + 1) * nb]
            ref = w3 @ T
            got = r3.chk[3 * I + 2, J * nb:(J + 1) * nb]
            assert np.max(np.abs(got - ref)) <= 1e-9 * max(1.0, np.max(np.abs(ref)))


def test_next4_pascal_mod2_two_errors_ambiguity_of_three_sums():
    """The limit of m+1 = 3 sums for m = 2 (reading B10): they fix the pair only up to the line
    d3 = S d2 - P d1 in (S = wa + wb, P = wa wb). With P2's integer data both d2/d1 = 15 and
    d3/d1 = 249 are integers, so EVERY S gives an integer P and five row pairs inside the block fit
    exactly (wa, wb) = (3, 17), (7, 18), (9, 19) (the true one), (11, 21), (12, 23): ambiguous ->
    UNCORRECTABLE (never a mis-correction); two checksums mis-correct this case."""
    n, nb = 256, 32
    A = syn.pascal_mod2(n)
    # both targets hold 1.0 at k = 2: bit 52 -> 0.5 (Delta -0.5), bit 53 -> 0.25 (Delta -0.75)
    specs = [dict(k=2, hook="REST", row=200, col=100, bit=52),
             dict(k=2, hook="REST", row=210, col=100, bit=53)]
    inj = syn.inj_array(specs)
    two = oracle.potrf(A, nb, inj=inj)
    assert two.status != 0                 # two checksums: UNCORRECTABLE or a mis-correction
    r = oracle.potrf(A, nb, inj=inj, nchk=3)
    assert r.status == 1
    ev = r.event_tuples()
    assert len(ev) == 1 and ev[0][6] == KIND["UNCORRECTABLE"] and ev[0][:5] == (2, V["V5"], 3, 6, 4)


def test_next4_two_errors_in_one_column_generic_values():
    """Two storage errors in ONE column of one tile of a random SPD matrix (real, generic values):
    with three checksums both are located where the schedule predicts and corrected (L within
    the P4 tolerance of the fault-free factor); with two checksums the run cannot complete."""
    n, nb = 512, 64
    A = syn.spd_matrix(n, seed=9)
    specs = [dict(k=2, hook="REST", row=400, col=200, bit=52),
             dict(k=2, hook="REST", row=430, col=200, bit=55)]
    inj = syn.inj_array(specs)
    assert oracle.potrf(A, nb, inj=inj).status != 0
    r = oracle.potrf(A, nb, inj=inj, nchk=3)
    assert r.status == 0
    assert r.event_tuples() == sorted(predict(s, n, nb, nchk=3) for s in specs)
    assert floor_rel(r.L, oracle.potrf(A, nb, nchk=3).L, A) <= 1e-11


@pytest.mark.parametrize("hook", ["REST", "UPDATE_OUT"])
def test_next4_brute_force_every_row_pair_of_a_column(hook):
    """Brute force on a tiny case: two errors at EVERY pair of rows (a < b) of one tile column
    (nb = 16: 120 pairs), each located at the predicted check and corrected: L equal to the
    fault-free factor within the P4 tolerance."""
    n, nb = 64, 16
    A = syn.spd_matrix(n, seed=21)
    ref = oracle.potrf(A, nb, nchk=3)
    k, J, I, c = 1, 2, 3, 5
    for a in range(nb):
        for b in range(a + 1, nb):
            specs = [dict(k=k, hook=hook, row=I * nb + a, col=J * nb + c, bit=55),
                     dict(k=k, hook=hook, row=I * nb + b, col=J * nb + c, bit=54)]
            r = oracle.potrf(A, nb, inj=syn.inj_array(specs), nchk=3)
            assert r.status == 0, (a, b)
            assert r.event_tuples() == sorted(predict(s, n, nb, nchk=3) for s in specs), (a, b)
            assert floor_rel(r.L, ref.L, A) <= 1e-11, (a, b)


def test_next4_single_errors_unchanged_and_chk3_repair():
    """Single errors are located exactly as with two checksums (C2 schedule), and a corrupted
    third checksum row is repaired from the data (CHK3) leaving L bit-identical."""
    n, nb = 1024, 128
    A = syn.spd_matrix(n)
    specs = syn.per_iteration_injections(n, nb, bits=(45, 61))
    inj = syn.inj_array(specs)
    r2 = oracle.potrf(A, nb, inj=inj)
    r3 = oracle.potrf(A, nb, inj=inj, nchk=3)
    assert r3.status == r2.status == 0
    assert r3.event_tuples() == r2.event_tuples()
    c3 = [dict(k=1, hook="REST", target="CHK", row=3 * 5 + 2, col=2 * nb + 9, bit=50)]
    r = oracle.potrf(A, nb, inj=syn.inj_array(c3), nchk=3)
    clean = oracle.potrf(A, nb, nchk=3)
    assert r.status == 0 and r.event_tuples() == [predict(c3[0], n, nb, nchk=3)]
    assert np.array_equal(np.tril(r.L), np.tril(clean.L))


def test_next4_equal_and_opposite_pair_is_uncorrectable():
    """Da = -Db: d1 = 0 leaves P undetermined (no set of m+1 sums locates it) -> UNCORRECTABLE."""
    n, nb = 256, 32
    A = syn.pascal_mod2(n)
    specs = [dict(k=2, hook="REST", row=200, col=100, bit=52),    # 1.0 -> 0.5
             dict(k=2, hook="REST", row=210, col=100, bit=51)]    # 1.0 -> 1.5: d1 = 0
    r = oracle.potrf(A, nb, inj=syn.inj_array(specs), nchk=3)
    assert r.status == 1


def test_next4_three_errors_in_a_column_uncorrectable():
    n, nb = 256, 32
    A = syn.spd_matrix(n, seed=5)
    specs = [dict(k=1, hook="REST", row=100 + 7 * t, col=70, bit=52 - t) for t in range(3)]
    r = oracle.potrf(A, nb, inj=syn.inj_array(specs), nchk=3)
    assert r.status == 1
    assert any(e[6] == KIND["UNCORRECTABLE"] for e in r.event_tuples())
