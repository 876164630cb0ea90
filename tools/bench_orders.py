"""Right- vs left-looking order at a given n (ABFT on/off, K)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_chenlc16_b200 as P
n = int(sys.argv[1]) if len(sys.argv) > 1 else 32768
nb = 512
A0 = torch.empty(n, n, dtype=torch.float64, device="cuda").T
P.abft_gen_spd(n, A0)
A = torch.empty_like(A0.T).T
s = torch.cuda.current_stream()
for order in ("right", "left"):
    for abft, K in ((True, 1), (True, 3), (False, 1)):
        ts = []
        for i in range(3):
            A.copy_(A0); torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
            e0.record(s)
            st, r = P.abft_potrf_ex(n, nb, A, opt=P.options(abft_enabled=abft, K=K, order=order), cap=16)
            e1.record(s); e1.synchronize()
            ts.append(e0.elapsed_time(e1))
        t = sorted(ts)[1]
        print(f"order={order} abft={abft} K={K}: {t:.1f} ms  {n**3/3/t/1e9:.1f} GFLOP/s  checks={r['n_checks']}")
