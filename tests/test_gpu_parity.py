"""GPU parity: the CUDA path (through the C-ABI) against the CPU oracle on the same seeded
inputs. Decisions (events: k, check, tile, row, col, kind) must be identical; L within the
floor-relative 1e-11 of reading A18 (BASELINE.json north_star: 1e-11 max relative elementwise,
with the 1e-3 sqrt(A_ii) floor that the literal form needs); backward error
||A - L L^T||_F / ||A||_F <= 10 n eps."""
import numpy as np
import pytest

import oracle
import synthetic as syn
from tests._predict import predict, KIND

pytestmark = pytest.mark.gpu
EPS = 2.0 ** -52


@pytest.fixture(scope="module")
def P():
    import torch
    import paper_conf_ipps_chenlc16_b200 as p
    assert torch.cuda.is_available()
    return p


def floor_rel(L, Lref, A):
    s = np.sqrt(np.diag(A))[:, None]
    return float(np.max(np.abs(np.tril(L) - np.tril(Lref)) / np.maximum(np.abs(np.tril(Lref)), 1e-3 * s)))


def backward_error(A, L):
    L = np.tril(L)
    return float(np.linalg.norm(A - L @ L.T) / np.linalg.norm(A))


def run_gpu(P, A, nb, inj=None, opt=None):
    import torch
    n = A.shape[0]
    At = P.colmajor(A)
    st, rep = P.abft_potrf_ex(n, nb, At, inj=inj, opt=opt)
    torch.cuda.synchronize()
    return st, rep, P.to_numpy_colmajor(At)


# ---- generator and the bandwidth kernels --------------------------------------------------
@pytest.mark.parametrize("n,seed", [(1, 1), (300, 300), (1024, 1024), (777, 5)])
def test_gen_spd_bit_identical_to_synthetic(P, n, seed):
    import torch
    A = torch.empty(n, n, dtype=torch.float64, device="cuda").T
    assert P.abft_gen_spd(n, A, seed=seed) == 0
    torch.cuda.synchronize()
    assert np.array_equal(P.to_numpy_colmajor(A), syn.spd_matrix(n, seed=seed))


@pytest.mark.parametrize("n,nb", [(256, 32), (1024, 128), (1536, 512), (96, 24), (87, 29)])
def test_encode_matches_oracle(P, n, nb):
    import torch
    A = syn.spd_matrix(n, seed=3)
    N = n // nb
    chk_o, scl_o = oracle.encode(A, nb)
    At = P.colmajor(A)
    chk = torch.zeros(n, 2 * N, dtype=torch.float64, device="cuda").T
    scl = torch.zeros(n + 2 * N, dtype=torch.float64, device="cuda")
    assert P.abft_encode(n, nb, At, chk, scl) == 0
    torch.cuda.synchronize()
    scl_g = scl.cpu().numpy()
    assert np.array_equal(scl_g[:n], scl_o[:n])                    # sqrt is correctly rounded
    assert np.array_equal(scl_g[n:], scl_o[n:])                    # same sequential order
    chk_g = P.to_numpy_colmajor(chk)
    for I in range(N):
        for J in range(I + 1):
            sl = slice(J * nb, (J + 1) * nb)
            tol = 64 * EPS * scl_o[n + I] * np.max(scl_o[:n]) / 64
            assert np.max(np.abs(chk_g[2 * I, sl] - chk_o[2 * I, sl])) <= tol
            assert np.max(np.abs(chk_g[2 * I + 1, sl] - chk_o[2 * I + 1, sl])) <= tol * nb


def test_verify_matches_oracle_with_injected_errors(P):
    import torch
    n, nb = 1024, 128
    A = np.asfortranarray(np.tril(syn.spd_matrix(n, seed=8)))
    chk, scl = oracle.encode(A, nb)
    B = A.copy(order="F")
    chkB = chk.copy(order="F")
    B[700, 130] += 5.0                    # data error off-diagonal tile
    B[300, 260] *= -3.0                   # diagonal tile (2,2): mirrored twice -> one event
    chkB[2 * 5 + 1, 5 * nb + 17] += 1e3   # checksum row 2 of tile (5,5)
    ref_B, ref_c = B.copy(order="F"), chkB.copy(order="F")
    st_o, ev_o, _ = oracle.verify(ref_B, nb, ref_c, scl, factored=False)
    Bt, ct = P.colmajor(B), P.colmajor(chkB)
    sc = torch.from_numpy(scl).cuda()
    st, rep = P.abft_verify(n, nb, Bt, ct, sc, factored=False)
    torch.cuda.synchronize()
    assert st == st_o == 0
    assert P.sorted_event_tuples(rep["events"]) == oracle.sorted_events(ev_o)
    assert len(ev_o) == 3
    Bg = P.to_numpy_colmajor(Bt)
    assert np.max(np.abs(np.tril(Bg) - np.tril(A))) < 1e-12 * n


# ---- whole factorisation ------------------------------------------------------------------
def test_c1_pascal_mod2_golden_bit_exact(P):
    A = syn.pascal_mod2(256)
    inj = syn.inj_array(syn.c1_injections())
    st, rep, L = run_gpu(P, A, 32, inj=inj)
    ref = oracle.potrf(A, 32, inj=inj)
    assert st == 0 == ref.status
    assert P.sorted_event_tuples(rep["events"]) == ref.event_tuples()
    i = np.arange(256)
    assert np.array_equal(np.tril(L), ((i[:, None] & i[None, :]) == i[None, :]).astype(float))
    assert np.array_equal(np.triu(L, 1), np.triu(A, 1)), "upper triangle must be untouched"


@pytest.mark.parametrize("n,nb", [(64, 64), (256, 32), (512, 128), (1024, 128), (1024, 256), (2048, 512),
                                  (96, 24), (87, 29), (4096, 256)])
def test_fault_free_factor_matches_oracle(P, n, nb):
    A = syn.spd_matrix(n)
    st, rep, L = run_gpu(P, A, nb)
    ref = oracle.potrf(A, nb)
    assert st == 0 and rep["n_events"] == 0
    assert floor_rel(L, ref.L, A) <= 1e-11
    assert backward_error(A, L) <= 10 * n * EPS
    assert np.array_equal(np.triu(L, 1), np.triu(A, 1))
    N = n // nb
    assert rep["n_checks"] == ref.counts["n_checks"]


def test_c2_one_injection_per_iteration_events_identical(P):
    n, nb = 4096, 256
    A = syn.spd_matrix(n)
    inj = syn.inj_array(syn.per_iteration_injections(n, nb))
    st, rep, L = run_gpu(P, A, nb, inj=inj)
    ref = oracle.potrf(A, nb, inj=inj)
    assert st == 0 == ref.status
    assert P.sorted_event_tuples(rep["events"]) == ref.event_tuples()
    assert floor_rel(L, ref.L, A) <= 1e-11
    assert backward_error(A, L) <= 10 * n * EPS


@pytest.mark.parametrize("n,nb", [(2048, 256), (1024, 128)])
def test_mixed_storage_and_computing_errors(P, n, nb):
    A = syn.spd_matrix(n)
    specs = syn.mixed_injections(n, nb)
    inj = syn.inj_array(specs)
    ref = oracle.potrf(A, nb, inj=inj)
    st, rep, L = run_gpu(P, A, nb, inj=inj)
    assert st == ref.status
    assert P.sorted_event_tuples(rep["events"]) == ref.event_tuples()
    if ref.status == 0:
        assert floor_rel(L, ref.L, A) <= 1e-11


def test_exhaustive_small_every_element_every_hook(P):
    """Brute force on a small case: a bit-55 error at every lower element of tile column 1 at each
    hook that can reach it; GPU events equal the oracle's and the schedule prediction."""
    n, nb = 128, 32
    A = syn.spd_matrix(n, seed=12)
    specs = []
    for r in range(32, n):
        for c in range(32, 64):
            if r < c:
                continue
            specs.append(dict(k=1, hook="REST", row=r, col=c, bit=55))
            specs.append(dict(k=1, hook="POTRF_OUT" if r < 64 else "TRSM_OUT", row=r, col=c, bit=55))
    for s in specs[::7]:
        inj = syn.inj_array([s])
        ref = oracle.potrf(A, nb, inj=inj)
        st, rep, L = run_gpu(P, A, nb, inj=inj)
        assert P.sorted_event_tuples(rep["events"]) == ref.event_tuples() == [predict(s, n, nb)], s


def test_nonfinite_and_checksum_row_errors(P):
    n, nb = 512, 64
    A = syn.spd_matrix(n)
    row = next(r for r in range(192 + 40, 256) if A[r, 150] >= 0.25)
    nanmask = int(np.float64(A[400, 300]).view(np.uint64)) ^ 0x7FF8000000000001
    specs = [dict(k=0, hook="REST", row=row, col=150, bit=62),
             dict(k=0, hook="REST", row=400, col=300, xor_mask=nanmask),
             dict(k=2, hook="REST", target="CHK", row=2 * 6, col=3 * nb + 5, bit=50),
             dict(k=3, hook="REST", target="CHK", row=2 * 7 + 1, col=3 * nb + 9, bit=50),
             dict(k=4, hook="POTRF_OUT", target="CHK", row=2 * 4 + 1, col=4 * nb + 9, bit=53),
             dict(k=5, hook="TRSM_OUT", target="CHK", row=2 * 7, col=5 * nb + 1, bit=53)]
    inj = syn.inj_array(specs)
    ref = oracle.potrf(A, nb, inj=inj)
    st, rep, L = run_gpu(P, A, nb, inj=inj)
    assert st == 0 == ref.status
    got = P.sorted_event_tuples(rep["events"])
    assert got == ref.event_tuples()
    assert sorted(e[6] for e in got) == sorted([KIND["NONFINITE"]] * 2 + [KIND["CHK1"], KIND["CHK2"], KIND["CHK2"],
                                                KIND["CHK1"]])
    assert floor_rel(L, ref.L, A) <= 1e-11


def test_uncorrectable_aborts_like_oracle(P):
    n, nb = 512, 64
    A = syn.spd_matrix(n, seed=2)
    specs = [dict(k=1, hook="REST", row=300, col=150, bit=55),     # both in tile (4, 2), column 22
             dict(k=1, hook="REST", row=310, col=150, bit=56)]
    inj = syn.inj_array(specs)
    ref = oracle.potrf(A, nb, inj=inj)
    st, rep, _ = run_gpu(P, A, nb, inj=inj)
    assert ref.status == 1 and st == 1
    assert P.sorted_event_tuples(rep["events"]) == ref.event_tuples()


def test_not_spd_info(P):
    n, nb = 512, 64
    A = syn.spd_matrix(n, seed=3)
    A[333, 333] = -1.0
    ref = oracle.potrf(A, nb)
    st, rep, _ = run_gpu(P, A, nb)
    assert st == 2 == ref.status
    assert rep["info"] == ref.info == 334


def test_abft_disabled_same_factor(P):
    n, nb = 2048, 256
    A = syn.spd_matrix(n)
    st, rep, L = run_gpu(P, A, nb, opt=P.options(abft_enabled=False))
    ref = oracle.potrf(A, nb, abft=False)
    assert st == 0 and rep["n_checks"] == 0
    assert floor_rel(L, ref.L, A) <= 1e-11


@pytest.mark.parametrize("K", [3, 5])
def test_opt3_K(P, K):
    n, nb = 1024, 64
    A = syn.spd_matrix(n)
    specs = [dict(k=2, hook="REST", row=900, col=700, bit=50),
             dict(k=4, hook="UPDATE_OUT", row=600, col=330, bit=52)]
    inj = syn.inj_array(specs)
    ref = oracle.potrf(A, nb, inj=inj, K=K)
    st, rep, L = run_gpu(P, A, nb, inj=inj, opt=P.options(K=K))
    assert P.sorted_event_tuples(rep["events"]) == ref.event_tuples() == sorted(predict(s, n, nb, K=K) for s in specs)
    assert floor_rel(L, ref.L, A) <= 1e-11


def test_host_entry_point(P):
    n, nb = 1024, 128
    A = syn.spd_matrix(n)
    Ah = A.copy(order="F")
    inj = syn.inj_array([dict(k=1, hook="REST", row=900, col=200, bit=51)])
    st, rep = P.abft_potrf_host(n, nb, Ah, inj=inj)
    ref = oracle.potrf(A, nb, inj=inj)
    assert st == 0
    assert P.sorted_event_tuples(rep["events"]) == ref.event_tuples()
    assert floor_rel(Ah, ref.L, A) <= 1e-11


# ---- full-size configurations: sampled / property parity ----------------------------------
@pytest.mark.parametrize("n,nb,lead", [(16384, 512, 2048)])
def test_c3_full_size_sampled(P, n, nb, lead):
    """C3 at full size. The oracle computes the leading lead x lead block of L (which depends only
    on the leading block of A) and the injections there; the rest is checked by properties:
    backward error by random probes, every injection located as the schedule predicts."""
    import torch
    At = torch.empty(n, n, dtype=torch.float64, device="cuda").T
    P.abft_gen_spd(n, At)
    A0 = At.clone()       # column-major clone keeps stride(0) == 1
    specs = [s for s in syn.per_iteration_injections(n, nb) if s["row"] < lead]
    specs += [dict(k=10, hook="REST", row=15000, col=9000, bit=50),
              dict(k=20, hook="UPDATE_OUT", row=16000, col=12000, bit=48),
              dict(k=25, hook="TRSM_OUT", row=14000, col=25 * nb + 3, bit=55)]
    inj = syn.inj_array(specs)
    st, rep = P.abft_potrf_ex(n, nb, At, inj=inj)
    torch.cuda.synchronize()
    assert st == 0
    assert P.sorted_event_tuples(rep["events"]) == sorted(predict(s, n, nb) for s in specs)
    Al = syn.spd_matrix(n)[:lead, :lead]
    ref = oracle.potrf(Al, nb, inj=syn.inj_array([s for s in specs if s["row"] < lead]))
    Lg = At[:lead, :lead].cpu().numpy()
    assert floor_rel(Lg, ref.L, Al) <= 1e-11
    g = torch.Generator(device="cuda").manual_seed(0)
    X = torch.randn(n, 16, dtype=torch.float64, device="cuda", generator=g)
    Lt = torch.tril(At)
    Asym = torch.tril(A0) + torch.tril(A0, -1).T
    R = Asym @ X - Lt @ (Lt.T @ X)
    be = (R.norm() / (Asym @ X).norm()).item()
    assert be <= 10 * n * EPS


@pytest.mark.parametrize("mode", ["enhanced", "online", "offline"])
@pytest.mark.parametrize("fault", ["none", "computation", "memory"])
def test_schemes_match_oracle(P, mode, fault):
    """The comparison schemes of Tables VII/VIII (NEXT-2): same events, same re-runs, same factor."""
    from tests.test_oracle_pins import SCHEME_FAULTS
    n, nb = 1024, 128
    A = syn.spd_matrix(n)
    specs = SCHEME_FAULTS[fault]
    inj = syn.inj_array(specs) if specs else None
    ref = oracle.potrf(A, nb, inj=inj, mode=mode)
    st, rep, L = run_gpu(P, A, nb, inj=inj, opt=P.options(mode=mode))
    assert st == ref.status == 0
    assert rep["reruns"] == ref.reruns
    if ref.reruns == 0:
        assert P.sorted_event_tuples(rep["events"]) == ref.event_tuples()
    else:   # after propagation the first run's event list depends on rounding; the decision does not
        assert rep["n_events"] > 0
    assert floor_rel(L, ref.L, A) <= 1e-11


# ---- NEXT-1: left-looking order (MAGMA Alg. 1) with Table I's verification --------------------
@pytest.mark.parametrize("n,nb", [(1024, 128), (2048, 256), (512, 64), (96, 24)])
def test_left_looking_fault_free(P, n, nb):
    A = syn.spd_matrix(n)
    ref = oracle.potrf(A, nb, order="left")
    st, rep, L = run_gpu(P, A, nb, opt=P.options(order="left"))
    assert st == 0 and rep["n_events"] == 0
    assert rep["n_checks"] == ref.counts["n_checks"]
    assert floor_rel(L, ref.L, A) <= 1e-11
    assert backward_error(A, L) <= 10 * n * EPS


@pytest.mark.parametrize("K", [1, 3])
def test_left_looking_injections(P, K):
    n, nb = 1024, 128
    A = syn.spd_matrix(n)
    specs = [dict(k=2, hook="REST", row=900, col=130, bit=50),
             dict(k=3, hook="TRSM_OUT", row=700, col=3 * nb + 5, bit=50),
             dict(k=4, hook="UPDATE_OUT", row=800, col=4 * nb + 9, bit=52),
             dict(k=5, hook="POTRF_OUT", row=5 * nb + 9, col=5 * nb + 2, bit=52),
             dict(k=1, hook="REST", row=1000, col=7 * nb + 3, bit=50),
             dict(k=8, hook="REST", row=600, col=300, bit=50)]
    inj = syn.inj_array(specs)
    ref = oracle.potrf(A, nb, inj=inj, order="left", K=K)
    st, rep, L = run_gpu(P, A, nb, inj=inj, opt=P.options(order="left", K=K))
    assert st == ref.status == 0
    assert P.sorted_event_tuples(rep["events"]) == ref.event_tuples()
    assert floor_rel(L, ref.L, A) <= 1e-11


def test_left_looking_c1_golden_exact(P):
    A = syn.pascal_mod2(256)
    specs = [dict(k=2, hook="REST", row=232, col=40, bit=52), dict(k=4, hook="UPDATE_OUT", row=230, col=130, bit=51)]
    inj = syn.inj_array(specs)
    ref = oracle.potrf(A, 32, inj=inj, order="left")
    st, rep, L = run_gpu(P, A, 32, inj=inj, opt=P.options(order="left"))
    assert P.sorted_event_tuples(rep["events"]) == ref.event_tuples()
    i = np.arange(256)
    assert np.array_equal(np.tril(L), ((i[:, None] & i[None, :]) == i[None, :]).astype(float))


@pytest.mark.parametrize("mode", ["online", "offline"])
def test_left_looking_schemes(P, mode):
    from tests.test_oracle_pins import SCHEME_FAULTS
    n, nb = 1024, 128
    A = syn.spd_matrix(n)
    # left-looking: the update of iteration k writes block column k
    faults = {"computation": [dict(k=2, hook="UPDATE_OUT", row=800, col=2 * nb + 10, bit=50)],
              "memory": SCHEME_FAULTS["memory"]}
    for fault in ("computation", "memory"):
        inj = syn.inj_array(faults[fault])
        ref = oracle.potrf(A, nb, inj=inj, mode=mode, order="left")
        st, rep, L = run_gpu(P, A, nb, inj=inj, opt=P.options(mode=mode, order="left"))
        assert st == ref.status == 0 and rep["reruns"] == ref.reruns
        assert floor_rel(L, ref.L, A) <= 1e-11


@pytest.mark.parametrize("mode", ["enhanced", "enhanced_redo"])
def test_two_errors_in_a_column_redo_matches_oracle(P, mode):
    """NEXT-4: two errors in one column of a block (beyond what two checksums locate):
    plain Enhanced aborts with UNCORRECTABLE; with re-do it re-runs once from the saved input.
    Same status, re-runs and events as the oracle; the re-run's factor within 1e-11."""
    from tests.test_oracle_pins import TWO_IN_A_COLUMN
    n, nb = 512, 64
    A = syn.spd_matrix(n, seed=2)
    inj = syn.inj_array(TWO_IN_A_COLUMN)
    ref = oracle.potrf(A, nb, inj=inj, mode=mode)
    st, rep, L = run_gpu(P, A, nb, inj=inj, opt=P.options(mode=mode))
    assert st == ref.status
    assert rep["reruns"] == ref.reruns
    assert P.sorted_event_tuples(rep["events"]) == ref.event_tuples()
    if mode == "enhanced_redo":
        assert st == 0 and rep["reruns"] == 1
        assert floor_rel(L, ref.L, A) <= 1e-11


@pytest.mark.parametrize("pinned", [True, False])
@pytest.mark.parametrize("n,nb", [(2048, 256), (3072, 512)])
def test_host_entry_overlapped_writeback(P, n, nb, pinned, monkeypatch):
    """abft_potrf_host copies each finished block column of L to the host while the factorisation
    continues (fault-free direct path on page-locked memory — a torch pinned tensor's column-major
    numpy view; ABFT_GRAPH=0 forces direct launches at this size), or takes the plain
    copy-factor-copy path on pageable memory: either way the host result equals the device path
    bit for bit and the strict upper triangle keeps the input."""
    import torch
    monkeypatch.setenv("ABFT_GRAPH", "0")
    A = syn.spd_matrix(n)
    if pinned:
        buf = torch.empty((n, n), dtype=torch.float64, pin_memory=True)
        Ah = buf.T.numpy()                      # F-contiguous view of page-locked memory
        Ah[:, :] = A
    else:
        Ah = A.copy(order="F")
    st, rep = P.abft_potrf_host(n, nb, Ah)
    assert st == 0 and rep["n_events"] == 0
    Ad = P.colmajor(A)
    st2, _ = P.abft_potrf(n, nb, Ad)
    torch.cuda.synchronize()
    Ld = P.to_numpy_colmajor(Ad)
    assert np.array_equal(np.tril(Ah), np.tril(Ld))
    assert np.array_equal(np.triu(Ah, 1), np.triu(A, 1))
