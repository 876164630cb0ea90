"""Honest ABFT overhead: ABFT on and off timed the same way (unprofiled,
direct launches, interleaved on/off pairs, CUDA events on the launching stream), every fault-free
step asserted event-free; then ONE profiled run of each arm for the phase breakdown.
usage: python tools/time_arms.py [n] [nb] [pairs]"""
import json, os, statistics, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_chenlc16_b200 as P
n = int(sys.argv[1]) if len(sys.argv) > 1 else 32768
nb = int(sys.argv[2]) if len(sys.argv) > 2 else 512
pairs = int(sys.argv[3]) if len(sys.argv) > 3 else 5
s = torch.cuda.current_stream()
A0 = torch.empty(n, n, dtype=torch.float64, device="cuda").T
P.abft_gen_spd(n, A0)
A = torch.empty_like(A0.T).T
def step(opt):
    A.copy_(A0); torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
    e0.record(s); st, rep = P.abft_potrf_ex(n, nb, A, opt=opt, cap=64); e1.record(s); e1.synchronize()
    if not os.environ.get("ABFT_DEV_ABLATE"):   # ablation runs are timing-only (stale checksums)
        assert st == 0 and rep["n_events"] == 0, (st, rep["n_events"], P.sorted_event_tuples(rep["events"])[:4])
    return e0.elapsed_time(e1), rep
on, off = P.options(), P.options(abft_enabled=False)
for _ in range(2):
    step(on); step(off)
t_on, t_off, ratio = [], [], 0.0
for _ in range(pairs):
    t, r = step(on); t_on.append(t); ratio = max(ratio, r["max_noise_ratio"])
    t, _ = step(off); t_off.append(t)
mon, moff = statistics.median(t_on), statistics.median(t_off)
out = {"n": n, "nb": nb, "pairs": pairs, "ablate": os.environ.get("ABFT_DEV_ABLATE", "0"),
       "env": {k: v for k, v in os.environ.items() if k.startswith("ABFT_")}, "on_ms": [round(x, 3) for x in t_on], "off_ms": [round(x, 3) for x in t_off],
       "on_median_ms": round(mon, 3), "off_median_ms": round(moff, 3),
       "on_tflops": round(n**3 / 3 / mon / 1e9, 3), "off_tflops": round(n**3 / 3 / moff / 1e9, 3),
       "overhead_pct": round(100 * (mon - moff) / moff, 3), "max_noise_ratio": ratio,
       "launches_on": None}
for name, opt in (("on", P.options(profile=True)), ("off", P.options(abft_enabled=False, profile=True))):
    step(opt)
    out[f"phases_{name}"] = {k: round(v["ms"], 3) for k, v in P.abft_last_profile().items() if v["ms"] > 0}
    out[f"launches_{name}"] = P.abft_last_launch_count()
print(json.dumps(out), flush=True)
