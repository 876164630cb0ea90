"""Small-n critical-path attribution (VERDICT r1 #4, C2 n=4096 nb=256): median of 30 graph-mode
steps (no report, CUDA events on the stream) for ABFT on and off; run once per ABFT_DEV_ABLATE mask
(1 no checksum rows, 2 no V5, 4 no V1-V4, 8 no fused partials, 16 no encode/V6; timing only).
usage: python tools/c2_ablate.py [n] [nb]  -> one JSON line"""
import json, os, statistics, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_chenlc16_b200 as P
n = int(sys.argv[1]) if len(sys.argv) > 1 else 4096
nb = int(sys.argv[2]) if len(sys.argv) > 2 else 256
s = torch.cuda.current_stream()
A0 = torch.empty(n, n, dtype=torch.float64, device="cuda").T
P.abft_gen_spd(n, A0)
A = torch.empty_like(A0.T).T
out = {"n": n, "nb": nb, "ablate": os.environ.get("ABFT_DEV_ABLATE", "0")}
for name, opt in (("on", P.options()), ("off", P.options(abft_enabled=False))):
    ts = []
    for i in range(40):
        A.copy_(A0)
        e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
        e0.record(s); P.abft_potrf_ex(n, nb, A, opt=opt, report=False); e1.record(s); e1.synchronize()
        if i >= 10: ts.append(e0.elapsed_time(e1))
    out[name + "_ms"] = round(statistics.median(ts), 4)
    out[name + "_tflops"] = round(n ** 3 / 3 / statistics.median(ts) / 1e9, 3)
print(json.dumps(out), flush=True)
