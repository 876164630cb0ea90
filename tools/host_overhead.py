"""Host enqueue time of abft_potrf_ex vs device time (is the host the bottleneck?)."""
import sys, os, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_chenlc16_b200 as P
n = int(sys.argv[1]) if len(sys.argv) > 1 else 32768
nb = 512
A0 = torch.empty(n, n, dtype=torch.float64, device="cuda").T
P.abft_gen_spd(n, A0)
A = torch.empty_like(A0.T).T
s = torch.cuda.current_stream()
for prof in (False, True):
    for rep in range(3):
        A.copy_(A0); torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
        e0.record(s)
        t0 = time.perf_counter()
        st, r = P.abft_potrf_ex(n, nb, A, report=False, opt=P.options(profile=prof))
        t1 = time.perf_counter()
        e1.record(s); e1.synchronize()
        t2 = time.perf_counter()
        print(f"profile={prof} host_enqueue={1e3*(t1-t0):.1f} ms  wall={1e3*(t2-t0):.1f} ms  device={e0.elapsed_time(e1):.1f} ms  launches={P.abft_last_launch_count()}")
