"""Stress (development): repeated fault-free factorisations of the bench workload, profile on/off;
prints status and events of each run (a clean run raises none)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_chenlc16_b200 as P
n, nb, reps = int(sys.argv[1]), int(sys.argv[2]), int(sys.argv[3])
A = torch.empty(n, n, dtype=torch.float64, device="cuda").T
for prof in (True, False):
    for r in range(reps):
        P.abft_gen_spd(n, A)
        st, rep = P.abft_potrf_ex(n, nb, A, opt=P.options(profile=prof))
        torch.cuda.synchronize()
        print("profile", prof, "status", st, "events", rep["n_events"], P.sorted_event_tuples(rep["events"])[:3], flush=True)
