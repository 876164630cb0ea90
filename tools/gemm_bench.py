"""Time the trailing-update GEMM alone: C (M x M lower) -= W W^T with K = nb, as in update k=0."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_chenlc16_b200 as P
M = int(sys.argv[1]) if len(sys.argv) > 1 else 16384
K = int(sys.argv[2]) if len(sys.argv) > 2 else 512
W = torch.randn(K, M, dtype=torch.float64, device="cuda").T          # column-major M x K
C = torch.randn(M, M, dtype=torch.float64, device="cuda").T
for _ in range(3):
    P.abft_dev_gemm_nt(M, M, K, W, W, C)
torch.cuda.synchronize()
ts = []
for _ in range(10):
    e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
    e0.record(); P.abft_dev_gemm_nt(M, M, K, W, W, C); e1.record(); e1.synchronize()
    ts.append(e0.elapsed_time(e1))
ts.sort()
fl = M * (M + 1) * K
print(f"M={M} K={K} lower SYRK: median {ts[5]:.3f} ms  {fl/ts[5]/1e9:.2f} TFLOP/s  best {fl/ts[0]/1e9:.2f}")
# full (non-lower) GEMM for reference
ts = []
for _ in range(5):
    e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
    e0.record(); P.abft_dev_gemm_nt(M, M, K, W, W, C, lower=False); e1.record(); e1.synchronize()
    ts.append(e0.elapsed_time(e1))
ts.sort()
print(f"M={M} K={K} full GEMM: median {ts[2]:.3f} ms  {2*M*M*K/ts[2]/1e9:.2f} TFLOP/s")
