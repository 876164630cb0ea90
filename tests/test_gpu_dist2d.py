"""GPU parity of the 2D block-cyclic multi-GPU path against the oracle's 2D P-rank
simulation (oracle.potrf(..., nranks=P, prows=Pr)): tile (I, J) on rank (I mod Pr) * Pc + J mod Pc,
the diagonal block's owner pushes inv(L_kk) to its process column, every rank of that column solves
and checks its own panel tiles (V4) and pushes them to every rank, every rank re-checks the tiles
it received (V4R) and updates only its own tiles. Run (a) as the one-device harness
abft_potrf_dist_sim (all ranks in one process) and (b) as separate processes on the one GPU through
the peer-memory (CUDA IPC) transport. Events must equal the oracle's, the factor within 1e-11."""
import os
import socket

import numpy as np
import pytest

import oracle
import synthetic as syn

pytestmark = pytest.mark.gpu


def floor_rel(L, Lref, A):
    s = np.sqrt(np.diag(A))[:, None]
    return float(np.max(np.abs(np.tril(L) - np.tril(Lref)) / np.maximum(np.abs(np.tril(Lref)), 1e-3 * s)))


@pytest.fixture(scope="module")
def P():
    import paper_conf_ipps_chenlc16_b200 as p
    return p


def run_sim2d(P, A, nb, Pn, prows, inj=None, abft=True):
    import torch
    n = A.shape[0]
    locs = P.block_cyclic_split_2d(A, nb, Pn, prows)
    dev = [P.colmajor(L) if L.shape[1] else None for L in locs]
    st, rep = P.abft_potrf_dist_sim(n, nb, dev, lda=n, inj=inj, opt=P.options(abft_enabled=abft, prows=prows))
    torch.cuda.synchronize()
    out = [P.to_numpy_colmajor(d) if d is not None else np.zeros((n, 0), order="F") for d in dev]
    return st, rep, P.block_cyclic_join_2d(out, nb, n, prows)


GRIDS = [(2, 2), (4, 2), (6, 2), (6, 3), (4, 4)]


@pytest.mark.parametrize("Pn,prows", GRIDS)
@pytest.mark.parametrize("n,nb", [(1024, 128), (768, 256), (640, 128)])
def test_sim2d_fault_free(P, Pn, prows, n, nb):
    A = syn.spd_matrix(n)
    ref = oracle.potrf(A, nb, nranks=Pn, prows=prows)
    st, rep, L = run_sim2d(P, A, nb, Pn, prows)
    assert st == 0 and rep["n_events"] == 0
    assert floor_rel(L, ref.L, A) <= 1e-11
    assert rep["n_checks"] == ref.counts["n_checks"]


@pytest.mark.parametrize("Pn,prows", [(4, 2), (6, 3), (2, 2)])
def test_sim2d_injections_including_recv(P, Pn, prows):
    n, nb = 1024, 128
    A = syn.spd_matrix(n)
    specs = syn.per_iteration_injections(n, nb, bits=(45, 61))
    pc = Pn // prows
    # RECV into a panel tile the receiving rank does not own (data and checksum-row targets)
    r1 = next(r for r in range(Pn) if P.grid_owner(5, 1, Pn, prows) != r)
    r2 = next(r for r in reversed(range(Pn)) if P.grid_owner(6, 2, Pn, prows) != r)
    specs += [dict(k=1, hook="RECV", row=700, col=150, bit=50, rank=r1),
              dict(k=2, hook="RECV", target="CHK", row=2 * 6 + 1, col=2 * nb + 5, bit=50, rank=r2)]
    inj = syn.inj_array(specs)
    ref = oracle.potrf(A, nb, inj=inj, nranks=Pn, prows=prows)
    st, rep, L = run_sim2d(P, A, nb, Pn, prows, inj=inj)
    assert st == ref.status == 0
    got = P.sorted_event_tuples(rep["events"])
    assert got == ref.event_tuples()
    assert {e[7] for e in got if e[1] != 7} <= set(range(Pn)) and pc >= 1
    assert floor_rel(L, ref.L, A) <= 1e-11


def test_sim2d_c4_block_size(P):
    """nb = 512 (the C4 block size) on a 2 x 2 grid: the row-block-filtered update and TRSM launches
    take their warp-specialised 128 x 64 tiles; events as the oracle's, factor within 1e-11."""
    n, nb, Pn, prows = 4096, 512, 4, 2
    A = syn.spd_matrix(n, seed=5)
    specs = syn.per_iteration_injections(n, nb, bits=(45, 61))
    specs.append(dict(k=2, hook="RECV", row=3000, col=1100, bit=51, rank=0))
    inj = syn.inj_array(specs)
    ref = oracle.potrf(A, nb, inj=inj, nranks=Pn, prows=prows)
    st, rep, L = run_sim2d(P, A, nb, Pn, prows, inj=inj)
    assert st == ref.status == 0
    assert P.sorted_event_tuples(rep["events"]) == ref.event_tuples()
    assert floor_rel(L, ref.L, A) <= 1e-11


def test_sim2d_abft_off_and_uncorrectable(P):
    n, nb, Pn, prows = 512, 64, 4, 2
    A = syn.spd_matrix(n, seed=2)
    ref = oracle.potrf(A, nb, abft=False)
    st, rep, L = run_sim2d(P, A, nb, Pn, prows, abft=False)
    assert st == 0 and floor_rel(L, ref.L, A) <= 1e-11
    specs = [dict(k=1, hook="REST", row=300, col=150, bit=55), dict(k=1, hook="REST", row=310, col=150, bit=56)]
    inj = syn.inj_array(specs)
    r2 = oracle.potrf(A, nb, inj=inj, nranks=Pn, prows=prows)
    st, rep, _ = run_sim2d(P, A, nb, Pn, prows, inj=inj)
    assert st == 1 == r2.status


def test_sim2d_rejects_bad_grid(P):
    import torch
    n, nb = 512, 64
    A = syn.spd_matrix(n)
    locs = P.block_cyclic_split_2d(A, nb, 6, 3)
    dev = [P.colmajor(L) for L in locs]
    st, _ = P.abft_potrf_dist_sim(n, nb, dev, lda=n, opt=P.options(prows=4))   # 4 does not divide 6
    torch.cuda.synchronize()
    assert st == -11


# ---- separate processes through the peer-memory transport --------------------------------------
def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, prows, port, n, nb, specs, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    import torch
    import torch.distributed as dist
    import paper_conf_ipps_chenlc16_b200 as P
    dist.init_process_group("gloo", rank=rank, world_size=world)
    torch.cuda.set_device(0)
    A = syn.spd_matrix(n)
    At = P.colmajor(P.block_cyclic_split_2d(A, nb, world, prows)[rank])
    comm = P.ipc_comm(n, nb)
    inj = syn.inj_array(specs) if specs else None
    A0 = At.clone()
    # two calls on the same comm (the transport's flags must not leak from one call into the next),
    # a fault-free one first, then the injected one
    st0, rep0 = P.abft_potrf_dist(n, nb, At, comm, rank, world, lda=n, opt=P.options(prows=prows))
    torch.cuda.synchronize()
    At.copy_(A0)
    st, rep = P.abft_potrf_dist(n, nb, At, comm, rank, world, lda=n, inj=inj, opt=P.options(prows=prows))
    torch.cuda.synchronize()
    L = P.to_numpy_colmajor(At)
    dist.barrier()
    P.abft_comm_destroy(comm)
    assert st0 == 0 and rep0["n_events"] == 0, (st0, rep0["n_events"])
    q.put((rank, st, P.sorted_event_tuples(rep["events"]), L))
    dist.destroy_process_group()


@pytest.mark.parametrize("world,prows", [(2, 1), (2, 2), (4, 2)])
def test_processes_ipc_2d_match_oracle(P, world, prows):
    import torch.multiprocessing as mp
    n, nb = 1024, 128
    specs = syn.per_iteration_injections(n, nb, bits=(45, 61))
    specs += [dict(k=1, hook="RECV", row=700, col=150, bit=50, rank=next(r for r in range(world) if P.grid_owner(5, 1, world, prows) != r))]
    A = syn.spd_matrix(n)
    ref = oracle.potrf(A, nb, inj=syn.inj_array(specs), nranks=world, prows=prows)
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, prows, port, n, nb, specs, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = sorted([q.get(timeout=600) for _ in procs], key=lambda t: t[0])
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    assert all(r[1] == 0 for r in res) and ref.status == 0
    assert res[0][2] == ref.event_tuples()
    L = P.block_cyclic_join_2d([r[3] for r in res], nb, n, prows)
    assert floor_rel(L, ref.L, A) <= 1e-11


@pytest.mark.parametrize("n,nb,Pn,prows", [(128, 128, 4, 2), (256, 128, 4, 2), (384, 128, 6, 3), (256, 64, 8, 4),
                                           (512, 128, 4, 1)])
def test_sim2d_small_grids_more_ranks_than_tiles(P, n, nb, Pn, prows):
    """Degenerate 2D cases: one block column (no panel to broadcast), fewer block rows / columns
    than process rows / columns (ranks owning nothing in some iterations), ragged ownership."""
    A = syn.spd_matrix(n)
    specs = [dict(k=0, hook="REST", row=n - 1, col=0, bit=50)] if n > nb else []
    inj = syn.inj_array(specs) if specs else None
    ref = oracle.potrf(A, nb, inj=inj, nranks=Pn, prows=prows)
    st, rep, L = run_sim2d(P, A, nb, Pn, prows, inj=inj)
    assert st == ref.status == 0
    assert P.sorted_event_tuples(rep["events"]) == ref.event_tuples()
    assert floor_rel(L, ref.L, A) <= 1e-11
