"""Host-side logic of the multi-GPU path on CPU: the 1D block-cyclic layout and the NCCL-id
exchange over a world_size-2 gloo process group (127.0.0.1), plus the oracle's P-rank simulation
agreeing with the layout."""
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp

import synthetic as syn


def test_block_cyclic_split_join_roundtrip():
    import paper_conf_ipps_chenlc16_b200 as P
    n, nb = 96, 16
    A = np.asfortranarray(np.arange(n * n, dtype=np.float64).reshape(n, n))
    for Pn in (1, 2, 3, 4, 6, 7):
        loc = P.block_cyclic_split(A, nb, Pn)
        assert sum(L.shape[1] for L in loc) == n
        assert np.array_equal(P.block_cyclic_join(loc, nb, n), A)
        owned = sorted(J for r in range(Pn) for J in P.owned_blocks(n // nb, r, Pn))
        assert owned == list(range(n // nb))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _worker(rank, world, port, q):
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import paper_conf_ipps_chenlc16_b200 as P
    nid = P.nccl_id_exchange()
    N = 13
    mine = P.owned_blocks(N, rank, world)
    import torch
    t = torch.zeros(N, dtype=torch.int64)
    t[mine] = 1
    dist.all_reduce(t)
    ids = [None] * world
    dist.all_gather_object(ids, nid)
    q.put((rank, len(nid), ids[0] == ids[1], t.tolist()))
    dist.destroy_process_group()


def test_gloo_world2_nccl_id_exchange_and_ownership():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = [q.get(timeout=120) for _ in procs]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    for rank, nbytes, same, cover in res:
        assert nbytes == 128 and same
        assert cover == [1] * 13          # every block column owned by exactly one rank


def test_oracle_rank_simulation_owner_schedule():
    """The oracle's P-rank simulation: a RECV error on rank r is seen only by rank r's V4R."""
    import oracle
    n, nb, Pn = 512, 64, 3
    A = syn.spd_matrix(n)
    specs = [dict(k=2, hook="RECV", row=400, col=2 * nb + 3, bit=50, rank=0),
             dict(k=2, hook="RECV", row=300, col=2 * nb + 5, bit=50, rank=1)]
    r = oracle.potrf(A, nb, inj=syn.inj_array(specs), nranks=Pn)
    ev = r.event_tuples()
    assert sorted((e[1], e[7]) for e in ev) == [(7, 0), (7, 1)]    # V4R on receivers 0 and 1 (owner is 2)


def test_block_cyclic_2d_split_join_and_ownership():
    """2D block-cyclic layout (NEXT-3): every tile has exactly one owner, (I mod Pr) * Pc + J mod Pc;
    a rank's local array holds its process column's block columns full height; split/join
    round-trips the matrix."""
    import paper_conf_ipps_chenlc16_b200 as P
    n, nb = 96, 16
    N = n // nb
    A = np.asfortranarray(np.arange(n * n, dtype=np.float64).reshape(n, n))
    for Pn, pr in ((2, 2), (4, 2), (6, 3), (6, 2), (4, 4)):
        loc = P.block_cyclic_split_2d(A, nb, Pn, pr)
        pc = Pn // pr
        for r, L in enumerate(loc):
            assert L.shape == (n, len(range(r % pc, N, pc)) * nb)
        assert np.array_equal(P.block_cyclic_join_2d(loc, nb, n, pr), A)
        owners = [[P.grid_owner(I, J, Pn, pr) for J in range(N)] for I in range(N)]
        for r in range(Pn):
            mine = [(I, J) for I in range(N) for J in range(N) if owners[I][J] == r]
            assert all(I % pr == r // pc and J % pc == r % pc for I, J in mine)
        assert sorted(x for row in owners for x in row) == sorted(
            P.grid_owner(I, J, Pn, pr) for I in range(N) for J in range(N))


def _worker_2d(rank, world, port, q):
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import paper_conf_ipps_chenlc16_b200 as P
    n, nb, prows = 128, 16, 2
    A = syn.spd_matrix(n)
    mine = P.block_cyclic_split_2d(A, nb, world, prows)[rank]
    parts = [None] * world
    dist.all_gather_object(parts, mine)
    q.put((rank, bool(np.array_equal(P.block_cyclic_join_2d(parts, nb, n, prows), A))))
    dist.destroy_process_group()


def test_gloo_world2_2d_layout_exchange():
    """World-2 gloo group on a 2 x 1 process grid: each rank holds only its local 2D array; the
    gathered parts reassemble the matrix from the tile owners."""
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker_2d, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = [q.get(timeout=120) for _ in procs]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    assert all(ok for _, ok in res)
