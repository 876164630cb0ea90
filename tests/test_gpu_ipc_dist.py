"""The multi-GPU path as TWO PROCESSES (one rank each) on the one GPU this box has: NCCL refuses
two ranks on one device, so the ranks talk through the peer-memory (CUDA IPC) transport
(abft_comm_init_ipc / abft_comm_attach_ipc, include/abft.h), which runs the same run_dist driver as
the NCCL path (1D block-cyclic ownership, owner-only panel, panel broadcast, RECV
hook + V4R on the receiver, per-rank trailing updates, merged report). Events and the factor must
equal the oracle's P-rank simulation. The panel broadcast is the fused push (NEXT-3) by default, the
transport's pull collective with ABFT_DIST_PULL=1."""
import os
import socket

import numpy as np
import pytest

import oracle
import synthetic as syn

pytestmark = pytest.mark.gpu


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, n, nb, specs, q, mode="push"):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    if mode == "pull":     # the transport's broadcast collective instead of the fused push
        os.environ["ABFT_DIST_PULL"] = "1"
    import torch
    import torch.distributed as dist
    import paper_conf_ipps_chenlc16_b200 as P
    dist.init_process_group("gloo", rank=rank, world_size=world)
    torch.cuda.set_device(0)
    A = syn.spd_matrix(n)
    loc = P.block_cyclic_split(A, nb, world)[rank]
    At = P.colmajor(loc)
    comm = P.ipc_comm(n, nb)
    inj = syn.inj_array(specs) if specs else None
    st, rep = P.abft_potrf_dist(n, nb, At, comm, rank, world, lda=n, inj=inj)
    torch.cuda.synchronize()
    L = P.to_numpy_colmajor(At)
    dist.barrier()
    P.abft_comm_destroy(comm)
    q.put((rank, st, P.sorted_event_tuples(rep["events"]), L, rep["max_noise_ratio"]))
    dist.destroy_process_group()


def _run(n, nb, world, specs, mode="push"):
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, n, nb, specs, q, mode)) for r in range(world)]
    for p in procs:
        p.start()
    res = sorted([q.get(timeout=600) for _ in procs], key=lambda t: t[0])
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    return res


def floor_rel(L, Lref, A):
    s = np.sqrt(np.diag(A))[:, None]
    return float(np.max(np.abs(np.tril(L) - np.tril(Lref)) / np.maximum(np.abs(np.tril(Lref)), 1e-3 * s)))


@pytest.mark.parametrize("mode", ["push", "pull"])
@pytest.mark.parametrize("specs_kind", ["fault_free", "injected"])
def test_two_processes_ipc_transport_match_oracle(specs_kind, mode):
    """push (default, NEXT-3): the owner's write-back kernel stores the packed panel straight into
    the peer's receive buffer; pull: the transport's broadcast collective copies it out of the
    owner's arena."""
    import paper_conf_ipps_chenlc16_b200 as P
    n, nb, world = 1024, 128, 2
    specs = []
    if specs_kind == "injected":
        specs = syn.per_iteration_injections(n, nb, bits=(45, 61))
        specs += [dict(k=1, hook="RECV", row=700, col=150, bit=50, rank=0),                 # owner of k=1 is 1
                  dict(k=2, hook="RECV", target="CHK", row=2 * 6 + 1, col=2 * nb + 5, bit=50, rank=1)]
    A = syn.spd_matrix(n)
    ref = oracle.potrf(A, nb, inj=syn.inj_array(specs) if specs else None, nranks=world)
    res = _run(n, nb, world, specs, mode)
    # rank 0's report holds every rank's events (gathered through the transport)
    rank0 = res[0]
    assert rank0[1] == ref.status == 0
    assert rank0[2] == ref.event_tuples()
    L = P.block_cyclic_join([r[3] for r in res], nb, n)
    assert floor_rel(L, ref.L, A) <= 1e-11
    assert all(r[1] == 0 for r in res)
