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
