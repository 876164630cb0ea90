import sys, os
sys.path.insert(0, os.getcwd())
import numpy as np, torch
import paper_conf_ipps_chenlc16_b200 as P, synthetic as syn
for (n, nb, graph) in ((1024, 64, None), (1024, 64, "0"), (2048, 256, None)):
    if graph is not None: os.environ["ABFT_GRAPH"] = graph
    A = syn.spd_matrix(n)
    out = {}
    for nc in (2, 3):
        At = P.colmajor(A)
        st, rep = P.abft_potrf_ex(n, nb, At, opt=P.options(nchk=nc))
        torch.cuda.synchronize()
        out[nc] = (st, rep["n_events"], P.to_numpy_colmajor(At))
    L2, L3 = np.tril(out[2][2]), np.tril(out[3][2])
    d = np.argwhere(L2 != L3)
    print(n, nb, graph, out[2][:2], out[3][:2], "ndiff", len(d), "first", d[:3].tolist() if len(d) else None,
          "maxabs", float(np.max(np.abs(L2 - L3))))
