"""Stress repro (development): fault-free factorisations at a given n, nb; prints the events a
run raised (a clean run raises none). Used to find the preemption-induced update errors
(DESIGN.md §5): ABFT_CHOL=tasks ABFT_CHOL_G=1 python tools/stress_v5.py 98304 1024 x"""
import sys, os
sys.path.insert(0, os.getcwd())
import torch
import paper_conf_ipps_chenlc16_b200 as P
import synthetic as syn
n, nb = int(sys.argv[1]), int(sys.argv[2])
specs = [dict(k=0, hook="REST", row=1800, col=900, bit=50),
         dict(k=3, hook="UPDATE_OUT", row=n - 8304, col=n // 2, bit=52)] if len(sys.argv) < 4 else []
print("gpu", torch.cuda.get_device_properties(0).uuid, flush=True)
A = torch.empty(n, n, dtype=torch.float64, device="cuda").T
for it in range(int(os.environ.get("REPS", "2"))):
    P.abft_gen_spd(n, A)
    st, rep = P.abft_potrf_ex(n, nb, A, inj=syn.inj_array(specs) if specs else None,
                              opt=P.options(nchk=int(os.environ.get("ABFT_NCHK", "2"))))
    torch.cuda.synchronize()
    print(it, "status", st, "n_events", rep["n_events"], P.sorted_event_tuples(rep["events"])[:4], flush=True)
    ev = rep["events"]
    for e in ev[:4]:
        print("   ", {k: e[k] for k in ev.dtype.names})
