"""Time the diagonal-block POTRF + inverse alone and a dependent empty-kernel chain (launch latency)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_chenlc16_b200 as P
s = torch.cuda.current_stream()
for nb in (64, 128, 256, 512, 1024):
    A0 = torch.empty(nb, nb, dtype=torch.float64, device="cuda").T
    P.abft_gen_spd(nb, A0)
    A = torch.empty_like(A0.T).T
    Li = torch.empty(nb, nb, dtype=torch.float64, device="cuda").T
    ts = []
    for i in range(6):
        A.copy_(A0); torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
        e0.record(s); st = P.abft_dev_chol_inv(nb, A, Li); e1.record(s); e1.synchronize()
        ts.append(e0.elapsed_time(e1))
    L = torch.tril(A)
    err = (L @ Li - torch.eye(nb, dtype=torch.float64, device="cuda")).abs().max().item()
    print(f"nb={nb}: {sorted(ts)[2]*1e3:.1f} us, launches {P.abft_last_launch_count()}, |L inv(L) - I| {err:.1e}")
# launch latency: chain of tiny dependent kernels
x = torch.zeros(1, device="cuda")
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
e0.record(s)
for _ in range(200):
    x.add_(1)
e1.record(s); e1.synchronize()
print(f"dependent tiny-kernel chain: {e0.elapsed_time(e1)/200*1e3:.2f} us per launch")
