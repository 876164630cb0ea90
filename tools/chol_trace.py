"""Per-task timeline of the one-launch diagonal-block kernel (abft_dev_chol_trace)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_chenlc16_b200 as P
NAMES = "PSUZF"
nb = int(sys.argv[1]) if len(sys.argv) > 1 else 512
A = torch.empty(nb, nb, dtype=torch.float64, device="cuda").T
Li = torch.empty(nb, nb, dtype=torch.float64, device="cuda").T
for rep in range(3):
    P.abft_gen_spd(nb, A)
    nt, rows = P.abft_dev_chol_trace(nb, A, Li)
t0 = min(r[6] for r in rows)
print(f"nb={nb} tasks={nt} span={(max(r[8] for r in rows) - t0) / 1e3:.1f} us")
dur = {}
for r in rows:
    dur.setdefault(NAMES[r[0]], []).append((r[8] - r[7]) / 1e3)
for k, v in dur.items():
    print(f"  {k}: n={len(v)} mean {sum(v)/len(v):.2f} us max {max(v):.2f}")
for t, r in enumerate(rows):
    print(f"{t:4d} {NAMES[r[0]]}({r[1]},{r[2]},{r[3]}) cta={r[5]:3d} sm={r[4]:3d} fetch={(r[6]-t0)/1e3:8.2f} "
          f"go={(r[7]-t0)/1e3:8.2f} end={(r[8]-t0)/1e3:8.2f} run={(r[8]-r[7])/1e3:6.2f}")
