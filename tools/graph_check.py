"""Graph mode vs direct launches: bitwise-identical L, same report, and the per-call time of both."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_chenlc16_b200 as P
for n, nb in [(int(a), int(b)) for a, b in (x.split(":") for x in (sys.argv[1:] or ["4096:256", "16384:512"]))]:
    A = torch.empty(n, n, dtype=torch.float64, device="cuda").T
    res = {}
    for mode in ("0", "1"):
        os.environ["ABFT_GRAPH"] = mode
        ts = []
        for rep in range(4):
            P.abft_gen_spd(n, A)
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
            e0.record()
            st, r = P.abft_potrf_ex(n, nb, A)
            e1.record(); torch.cuda.synchronize()
            ts.append(e0.elapsed_time(e1))
        res[mode] = (st, r["n_events"], r["n_checks"], torch.tril(A).clone(), min(ts[1:]), P.abft_last_launch_count())
    same = torch.equal(res["0"][3], res["1"][3])
    print(f"n={n} nb={nb}: direct {res['0'][4]:.2f} ms  graph {res['1'][4]:.2f} ms  status {res['0'][0]}/{res['1'][0]} "
          f"events {res['0'][1]}/{res['1'][1]} checks {res['0'][2]}/{res['1'][2]} launches {res['0'][5]}/{res['1'][5]} "
          f"bitwise-identical L: {same}  GFLOP/s direct {n**3/3/res['0'][4]/1e6:.0f} graph {n**3/3/res['1'][4]/1e6:.0f}")
    P.abft_graph_release()
