#!/bin/bash
# Box calibration (run under gpurun): FP64 peaks, layout probes, cuBLAS DGEMM context, host info.
set -u
mkdir -p gpurun_out
nvidia-smi --query-gpu=index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap \
    --format=csv -lms 200 > gpurun_out/calib_clocks.csv &
SMI=$!
./tools/calib_fp64 > gpurun_out/calib_fp64.json 2> gpurun_out/calib_fp64.err
echo "calib rc=$?"
python - <<'EOF' > gpurun_out/calib_dgemm.json
import torch, json, time
r = {}
for n in (4096, 8192, 16384):
    a = torch.randn(n, n, dtype=torch.float64, device="cuda")
    b = torch.randn(n, n, dtype=torch.float64, device="cuda")
    for _ in range(2): a @ b
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    reps = 5 if n < 16384 else 2
    e0.record()
    for _ in range(reps): a @ b
    e1.record(); torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / reps
    r[f"cublas_dgemm_{n}_tflops"] = 2 * n**3 / (ms * 1e-3) / 1e12
# cuSOLVER dpotrf for context (library, not our path)
n = 32768
a = torch.randn(n, 1024, dtype=torch.float64, device="cuda")
A = a @ a.T / 1024 + n * torch.eye(n, dtype=torch.float64, device="cuda")
torch.linalg.cholesky(A[:8192, :8192].contiguous())
for nn in (8192, 32768):
    B = A[:nn, :nn].contiguous()
    torch.cuda.synchronize(); t = time.time()
    torch.linalg.cholesky(B); torch.cuda.synchronize()
    dt = time.time() - t
    r[f"cusolver_potrf_{nn}_gflops"] = nn**3 / 3 / dt / 1e9
print(json.dumps(r, indent=1))
EOF
kill $SMI
nproc > gpurun_out/calib_host.txt; lscpu >> gpurun_out/calib_host.txt; free -g >> gpurun_out/calib_host.txt
cat gpurun_out/calib_fp64.json gpurun_out/calib_dgemm.json
