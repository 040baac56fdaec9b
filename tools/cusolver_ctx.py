"""Context only (library, not our path): cuSOLVER dpotrf latency/throughput via torch."""
import sys
import torch

for n in [int(x) for x in sys.argv[1:]] or [512, 1024, 2048, 8192, 32768]:
    a = torch.randn(n, min(n, 1024), dtype=torch.float64, device="cuda")
    A = a @ a.T / a.shape[1] + n * torch.eye(n, dtype=torch.float64, device="cuda")
    for _ in range(3):
        torch.linalg.cholesky(A)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    reps = 20 if n <= 8192 else 3
    e0.record()
    for _ in range(reps):
        torch.linalg.cholesky(A)
    e1.record()
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / reps
    print("cusolver dpotrf n=%d: %.3f ms, %.1f GFLOP/s" % (n, ms, n ** 3 / 3 / (ms * 1e-3) / 1e9))
