"""One abft_potrf on the device-generated A15 matrix (for ncu captures)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_chenlc16_b200 as P
n = int(sys.argv[1]) if len(sys.argv) > 1 else 16384
nb = int(sys.argv[2]) if len(sys.argv) > 2 else 512
abft = int(sys.argv[3]) if len(sys.argv) > 3 else 1
A = torch.empty(n, n, dtype=torch.float64, device="cuda").T
P.abft_gen_spd(n, A)
st, rep = P.abft_potrf_ex(n, nb, A, opt=P.options(abft_enabled=bool(abft)))
torch.cuda.synchronize()
print("status", st, "seconds", rep["seconds"], "GF/s", n**3/3/rep["seconds"]/1e9)
