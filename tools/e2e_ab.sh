# e2e (abft_potrf_host on pinned memory) with and without the streamed input, same box
mkdir -p gpurun_out
cat > /tmp/e2e.py <<'PY'
import json, os, statistics, sys, time
sys.path.insert(0, os.getcwd())
import torch
import paper_conf_ipps_chenlc16_b200 as P
n, nb = int(sys.argv[1]), int(sys.argv[2])
A0 = torch.empty(n, n, dtype=torch.float64, device="cuda").T
P.abft_gen_spd(n, A0)
h = torch.empty((n, n), dtype=torch.float64, pin_memory=True)
h0 = torch.empty((n, n), dtype=torch.float64, pin_memory=True)
h0.copy_(A0.T.cpu())
ts = []
for i in range(5):
    h.copy_(h0)
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    st, rep = P.abft_potrf_host(n, nb, h.data_ptr(), lda=n, report=True, cap=16)
    t1 = time.perf_counter()
    assert st == 0 and rep["n_events"] == 0, (st, rep["n_events"])
    if i >= 1: ts.append((t1 - t0) * 1e3)
L = h.T.numpy()
print(json.dumps({"n": n, "stream_in": os.environ.get("ABFT_HOST_STREAM_IN") is None, "ms": round(statistics.median(ts), 2),
                  "tflops": round(n**3 / 3 / statistics.median(ts) / 1e9, 2), "L00": float(L[0, 0]), "Llast": float(L[n - 1, n - 1])}))
PY
for r in 1 2; do
  ABFT_HOST_STREAM_IN=1 timeout 600 python /tmp/e2e.py 32768 512 >> gpurun_out/e2e_ab.jsonl 2>> gpurun_out/e2e_ab.err
  timeout 600 python /tmp/e2e.py 32768 512 >> gpurun_out/e2e_ab.jsonl 2>> gpurun_out/e2e_ab.err
done
