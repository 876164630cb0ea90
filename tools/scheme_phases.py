"""Why is Online-ABFT slower than Enhanced at C4? Unprofiled step times of
the three schemes on the same input, then one profiled step of each for the phase breakdown.
usage: python tools/scheme_phases.py [n] [nb]"""
import json, os, statistics, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_chenlc16_b200 as P
n = int(sys.argv[1]) if len(sys.argv) > 1 else 32768
nb = int(sys.argv[2]) if len(sys.argv) > 2 else 512
s = torch.cuda.current_stream()
A0 = torch.empty(n, n, dtype=torch.float64, device="cuda").T
P.abft_gen_spd(n, A0)
A = torch.empty_like(A0.T).T
def step(opt):
    A.copy_(A0); torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
    e0.record(s); st, rep = P.abft_potrf_ex(n, nb, A, opt=opt, cap=64); e1.record(s); e1.synchronize()
    assert st == 0 and rep["n_events"] == 0
    return e0.elapsed_time(e1), rep
out = {}
for mode in ("enhanced", "online", "offline"):
    step(P.options(mode=mode))
    ts = [step(P.options(mode=mode))[0] for _ in range(3)]
    _, rep = step(P.options(mode=mode, profile=True))
    out[mode] = {"ms": round(statistics.median(ts), 3), "library_seconds": rep["seconds"],
                 "phases": {k: round(v["ms"], 3) for k, v in P.abft_last_profile().items() if v["ms"] > 0},
                 "launches": P.abft_last_launch_count()}
print(json.dumps(out))
