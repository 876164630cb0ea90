"""cuBLAS DGEMM context number (vendor library, not the product): torch.matmul float64 8192^3."""
import torch, time
a = torch.randn(8192, 8192, dtype=torch.float64, device="cuda")
b = torch.randn(8192, 8192, dtype=torch.float64, device="cuda")
for _ in range(3): a @ b
torch.cuda.synchronize()
best = 1e9
for _ in range(10):
    e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
    e0.record(); c = a @ b; e1.record(); torch.cuda.synchronize()
    best = min(best, e0.elapsed_time(e1))
print(f"cuBLAS DGEMM 8192^3 best-of-10: {2*8192**3/best/1e9:.2f} TFLOP/s")
# cuSOLVER potrf context
for n in (16384, 32768):
    x = torch.rand(n, n, dtype=torch.float64, device="cuda"); x = (x + x.T) * 0.5; x.diagonal().add_(n)
    torch.linalg.cholesky(x); torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
    e0.record(); torch.linalg.cholesky(x); e1.record(); torch.cuda.synchronize()
    ms = e0.elapsed_time(e1)
    print(f"cuSOLVER dpotrf n={n}: {ms:.1f} ms = {n**3/3/ms/1e9:.2f} TFLOP/s")
    del x
