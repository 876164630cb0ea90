"""Time the diagonal-block path alone: abft_potrf on a single block (n = nb), per-phase profile."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_chenlc16_b200 as P
for nb in [int(x) for x in (sys.argv[1:] or ["256", "512", "1024"])]:
    A = torch.empty(nb, nb, dtype=torch.float64, device="cuda").T
    for rep in range(3):
        P.abft_gen_spd(nb, A)
        st, r = P.abft_potrf_ex(nb, nb, A, opt=P.options(profile=True))
    pr = P.abft_last_profile()
    print(f"nb={nb} status={st} total={r['seconds']*1e3:.3f} ms potrf_inv={pr['potrf_inv']['ms']:.3f} ms "
          f"launches={P.abft_last_launch_count()}")
