"""NEXT-4 on the GPU: three checksum rows per block (options nchk = 3; "m+1 column
checksums could locate and correct up to m errors per column"; reading B10) against the oracle's
nchk = 3 scheme on the same seeded inputs. Decisions must be identical, L within the floor-relative
1e-11 of reading A18, and the data arithmetic must not change at all (L bit-identical to the
two-checksum run on a fault-free input)."""
import numpy as np
import pytest

import oracle
import synthetic as syn
from tests._predict import predict, KIND, V

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def P():
    import paper_conf_ipps_chenlc16_b200 as p
    return p


def floor_rel(L, Lref, A):
    s = np.sqrt(np.diag(A))[:, None]
    return float(np.max(np.abs(np.tril(L) - np.tril(Lref)) / np.maximum(np.abs(np.tril(Lref)), 1e-3 * s)))


def run_gpu(P, A, nb, inj=None, nchk=3):
    import torch
    n = A.shape[0]
    At = P.colmajor(A)
    st, rep = P.abft_potrf_ex(n, nb, At, inj=inj, opt=P.options(nchk=nchk))
    torch.cuda.synchronize()
    return st, rep, P.to_numpy_colmajor(At)


@pytest.mark.parametrize("n,nb", [(2048, 256), (4096, 512), (1024, 64)])
def test_fault_free_bit_identical_to_two_checksums(P, n, nb):
    A = syn.spd_matrix(n)
    st3, rep3, L3 = run_gpu(P, A, nb, nchk=3)
    st2, rep2, L2 = run_gpu(P, A, nb, nchk=2)
    assert st3 == st2 == 0 and rep3["n_events"] == rep2["n_events"] == 0
    assert np.array_equal(np.tril(L3), np.tril(L2))
    assert rep3["max_noise_ratio"] <= 2.0 ** -6


@pytest.mark.parametrize("hook", ["REST", "UPDATE_OUT", "TRSM_OUT", "POTRF_OUT"])
@pytest.mark.parametrize("n,nb", [(2048, 256), (4096, 512)])
def test_two_errors_in_one_column_every_hook(P, hook, n, nb):
    """Two errors in the same column of one tile, at every hook (UPDATE_OUT is applied inside the
    update's epilogue, before the fused V5 partials): same events as the oracle, both corrected."""
    A = syn.spd_matrix(n, seed=7)
    k = 2
    if hook == "POTRF_OUT":
        I = J = k
        ra, rb, c = 40, 170, 17
    elif hook == "TRSM_OUT":
        I, J = k + 3, k
        ra, rb, c = 11, 200, 33
    else:
        I, J = k + 4, k + 1
        ra, rb, c = 5, 131, 77
    specs = [dict(k=k, hook=hook, row=I * nb + ra, col=J * nb + c, bit=54),
             dict(k=k, hook=hook, row=I * nb + rb, col=J * nb + c, bit=52)]
    inj = syn.inj_array(specs)
    ref = oracle.potrf(A, nb, inj=inj, nchk=3)
    st, rep, L = run_gpu(P, A, nb, inj=inj)
    assert st == ref.status == 0
    assert P.sorted_event_tuples(rep["events"]) == ref.event_tuples()
    assert ref.event_tuples() == sorted(predict(s, n, nb, nchk=3) for s in specs)
    assert floor_rel(L, ref.L, A) <= 1e-11


def test_brute_force_row_pairs_sampled(P):
    """A sample of every 11th row pair (a < b) of one tile column at nb = 64: same events as the
    oracle (which the CPU suite checks exhaustively against the schedule)."""
    n, nb = 256, 64
    A = syn.spd_matrix(n, seed=21)
    pairs = [(a, b) for a in range(nb) for b in range(a + 1, nb)][::11]
    for a, b in pairs:
        specs = [dict(k=1, hook="REST", row=3 * nb + a, col=2 * nb + 5, bit=55),
                 dict(k=1, hook="REST", row=3 * nb + b, col=2 * nb + 5, bit=54)]
        inj = syn.inj_array(specs)
        ref = oracle.potrf(A, nb, inj=inj, nchk=3)
        st, rep, L = run_gpu(P, A, nb, inj=inj)
        assert st == ref.status == 0, (a, b)
        assert P.sorted_event_tuples(rep["events"]) == ref.event_tuples(), (a, b)


def test_single_error_schedule_and_third_checksum_repair(P):
    n, nb = 2048, 256
    A = syn.spd_matrix(n)
    specs = syn.per_iteration_injections(n, nb, bits=(45, 61))
    specs.append(dict(k=3, hook="REST", target="CHK", row=3 * 6 + 2, col=4 * nb + 9, bit=50))   # CHK3
    inj = syn.inj_array(specs)
    ref = oracle.potrf(A, nb, inj=inj, nchk=3)
    st, rep, L = run_gpu(P, A, nb, inj=inj)
    assert st == ref.status == 0
    assert P.sorted_event_tuples(rep["events"]) == ref.event_tuples()
    assert any(e[6] == KIND["CHK3"] for e in ref.event_tuples())
    assert floor_rel(L, ref.L, A) <= 1e-11


def test_ambiguous_pair_is_uncorrectable_like_the_oracle(P):
    """P2's integer data make three sums ambiguous (reading B10): UNCORRECTABLE on both sides."""
    n, nb = 256, 32
    A = syn.pascal_mod2(n)
    specs = [dict(k=2, hook="REST", row=200, col=100, bit=52), dict(k=2, hook="REST", row=210, col=100, bit=53)]
    inj = syn.inj_array(specs)
    ref = oracle.potrf(A, nb, inj=inj, nchk=3)
    st, rep, _ = run_gpu(P, A, nb, inj=inj)
    assert st == ref.status == 1
    assert P.sorted_event_tuples(rep["events"]) == ref.event_tuples()


def test_mixed_injections_plus_pairs_at_scale(P):
    """n = 8192, nb = 512 (fused V5 path): the C3 mixed recipe plus a second error next to every
    fifth computing error, full event list equal to the oracle's."""
    n, nb = 8192, 512
    A = syn.spd_matrix(n)
    specs = syn.next4_injections(n, nb)
    inj = syn.inj_array(specs)
    ref = oracle.potrf(A, nb, inj=inj, nchk=3)
    st, rep, L = run_gpu(P, A, nb, inj=inj)
    assert st == ref.status
    assert P.sorted_event_tuples(rep["events"]) == ref.event_tuples()
    if st == 0:
        assert floor_rel(L, ref.L, A) <= 1e-9


def test_c4_full_size_events_equal_oracle_golden(P):
    """C4 (n = 32768, nb = 512) with three checksum rows, the C3-style injections and a second error
    next to every tenth one: the GPU's full event list equals the oracle's, stored by the committed
    script tests/golden/make_c4_nchk3_events.py (oracle only)."""
    import os
    import torch
    here = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")
    lines = open(os.path.join(here, "c4_nchk3_events.txt")).read().splitlines()
    status = int(lines[0].split()[3].rstrip(";"))
    want = [tuple(int(v) for v in ln.split()) for ln in lines[1:] if ln.strip()]
    n, nb = 32768, 512
    A = torch.empty(n, n, dtype=torch.float64, device="cuda").T
    assert P.abft_gen_spd(n, A) == 0
    st, rep = P.abft_potrf_ex(n, nb, A, inj=syn.inj_array(syn.next4_injections(n, nb)), opt=P.options(nchk=3))
    torch.cuda.synchronize()
    assert st == status == 0
    assert P.sorted_event_tuples(rep["events"]) == want
