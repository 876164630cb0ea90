"""GPU parity of the multi-GPU algorithm (1D block-cyclic, panel broadcast, V4R) against the
oracle's P-rank simulation: the single-process harness abft_potrf_dist_sim runs all P ranks on
one device (broadcast = device copy), and the real NCCL path runs with world size 1."""
import numpy as np
import pytest

import oracle
import synthetic as syn
from tests._predict import predict

pytestmark = pytest.mark.gpu
EPS = 2.0 ** -52


def floor_rel(L, Lref, A):
    s = np.sqrt(np.diag(A))[:, None]
    return float(np.max(np.abs(np.tril(L) - np.tril(Lref)) / np.maximum(np.abs(np.tril(Lref)), 1e-3 * s)))


def run_sim(P, A, nb, Pn, inj=None, opt=None):
    import torch
    n = A.shape[0]
    locs = P.block_cyclic_split(A, nb, Pn)
    dev = [P.colmajor(L) if L.shape[1] else None for L in locs]
    st, rep = P.abft_potrf_dist_sim(n, nb, dev, lda=n, inj=inj, opt=opt)
    torch.cuda.synchronize()
    out = [P.to_numpy_colmajor(d) if d is not None else np.zeros((n, 0), order="F") for d in dev]
    return st, rep, P.block_cyclic_join(out, nb, n)


@pytest.fixture(scope="module")
def P():
    import paper_conf_ipps_chenlc16_b200 as p
    return p


@pytest.mark.parametrize("Pn", [1, 2, 3, 4])
@pytest.mark.parametrize("n,nb", [(1024, 128), (512, 64), (768, 256)])
def test_sim_fault_free(P, Pn, n, nb):
    A = syn.spd_matrix(n)
    ref = oracle.potrf(A, nb, nranks=Pn)
    st, rep, L = run_sim(P, A, nb, Pn)
    assert st == 0 and rep["n_events"] == 0
    assert floor_rel(L, ref.L, A) <= 1e-11
    assert rep["n_checks"] == ref.counts["n_checks"]


@pytest.mark.parametrize("Pn", [2, 3, 4])
def test_sim_injections_including_recv(P, Pn):
    n, nb = 1024, 128
    A = syn.spd_matrix(n)
    specs = syn.per_iteration_injections(n, nb, bits=(45, 61))
    specs += [dict(k=1, hook="RECV", row=700, col=150, bit=50, rank=(1 + 1) % Pn),
              dict(k=2, hook="RECV", target="CHK", row=2 * 6 + 1, col=2 * nb + 5, bit=50, rank=(2 + 1) % Pn)]
    inj = syn.inj_array(specs)
    ref = oracle.potrf(A, nb, inj=inj, nranks=Pn)
    st, rep, L = run_sim(P, A, nb, Pn, inj=inj)
    assert st == ref.status == 0
    assert P.sorted_event_tuples(rep["events"]) == ref.event_tuples()
    assert floor_rel(L, ref.L, A) <= 1e-11


@pytest.mark.parametrize("diag", ["default", "recursive"])
def test_sim_four_ranks_c4_block_size(P, diag, monkeypatch):
    """P = 4 at the C4 block size: run_dist selects the task-graph diagonal block + LDGSTS update
    producer for P >= 4 (DESIGN.md §5 P-model); ABFT_DIST_DIAG=recursive restores the single-GPU
    configuration. Both: same events as the oracle's 4-rank simulation, factor within 1e-11."""
    if diag != "default":
        monkeypatch.setenv("ABFT_DIST_DIAG", diag)
    n, nb = 4096, 512
    A = syn.spd_matrix(n, seed=5)
    specs = syn.per_iteration_injections(n, nb, bits=(45, 61))
    specs.append(dict(k=2, hook="RECV", row=3000, col=1100, bit=51, rank=3))
    inj = syn.inj_array(specs)
    ref = oracle.potrf(A, nb, inj=inj, nranks=4)
    st, rep, L = run_sim(P, A, nb, 4, inj=inj)
    assert st == ref.status == 0
    assert P.sorted_event_tuples(rep["events"]) == ref.event_tuples()
    assert floor_rel(L, ref.L, A) <= 1e-11


def test_sim_c1_golden(P):
    A = syn.pascal_mod2(256)
    inj = syn.inj_array(syn.c1_injections())
    ref = oracle.potrf(A, 32, inj=inj, nranks=3)
    st, rep, L = run_sim(P, A, 32, 3, inj=inj)
    assert P.sorted_event_tuples(rep["events"]) == ref.event_tuples()
    i = np.arange(256)
    assert np.array_equal(np.tril(L), ((i[:, None] & i[None, :]) == i[None, :]).astype(float))


def test_sim_uncorrectable_propagates(P):
    n, nb = 512, 64
    A = syn.spd_matrix(n, seed=2)
    specs = [dict(k=1, hook="REST", row=300, col=150, bit=55), dict(k=1, hook="REST", row=310, col=150, bit=56)]
    inj = syn.inj_array(specs)
    ref = oracle.potrf(A, nb, inj=inj, nranks=2)
    st, rep, _ = run_sim(P, A, nb, 2, inj=inj)
    assert st == 1 == ref.status


def test_nccl_world_size_one(P):
    """The real NCCL path (ncclBroadcast etc.) with one rank on this GPU."""
    import torch
    n, nb = 1024, 128
    A = syn.spd_matrix(n)
    st, nid = P.abft_nccl_id()
    assert st == 0
    st, comm = P.abft_comm_init(1, nid, 0)
    assert st == 0
    inj = syn.inj_array(syn.per_iteration_injections(n, nb, bits=(45, 61)))
    At = P.colmajor(A)
    st, rep = P.abft_potrf_dist(n, nb, At, comm, 0, 1, inj=inj)
    torch.cuda.synchronize()
    ref = oracle.potrf(A, nb, inj=inj)
    assert st == 0
    assert P.sorted_event_tuples(rep["events"]) == ref.event_tuples()
    assert floor_rel(P.to_numpy_colmajor(At), ref.L, A) <= 1e-11
    assert P.abft_comm_destroy(comm) == 0
