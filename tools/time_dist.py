"""Time the multi-GPU driver (abft_potrf_dist through NCCL, world size 1 on this GPU) against the
single-GPU driver on the same matrix: with look-ahead across ranks the panel of k+1 overlaps
update k in both. Also the one-device P-rank simulation (all ranks share the GPU: a correctness
harness, its time is not a scaling number)."""
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_chenlc16_b200 as P

n = int(sys.argv[1]) if len(sys.argv) > 1 else 16384
nb = int(sys.argv[2]) if len(sys.argv) > 2 else 512
A0 = torch.empty(n, n, dtype=torch.float64, device="cuda").T
P.abft_gen_spd(n, A0)
A = torch.empty_like(A0.T).T
st, nid = P.abft_nccl_id()
st, comm = P.abft_comm_init(1, nid, 0)
s = torch.cuda.current_stream()


def timed(fn, reps=3):
    ts = []
    for i in range(reps + 1):
        A.copy_(A0)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
        e0.record(s)
        st, rep = fn()
        e1.record(s)
        e1.synchronize()
        assert st == 0, st
        if i:
            ts.append(e0.elapsed_time(e1))
    return sorted(ts)[len(ts) // 2]


t1 = timed(lambda: P.abft_potrf_ex(n, nb, A, report=True, cap=16))
t2 = timed(lambda: P.abft_potrf_dist(n, nb, A, comm, 0, 1, report=True, cap=16))
print(f"n={n} nb={nb}: single-GPU driver {t1:.1f} ms ({n**3/3/t1/1e9:.1f} TFLOP/s), "
      f"NCCL driver P=1 {t2:.1f} ms ({n**3/3/t2/1e9:.1f} TFLOP/s)")
P.abft_comm_destroy(comm)
