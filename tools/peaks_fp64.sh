#!/bin/bash
# Measures FP64 peaks on the GPU box; writes gpurun_out/peaks_fp64.txt
set -x
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/peaks_fp64.txt
./tools/peaks_fp64 >> gpurun_out/peaks_fp64.txt 2>&1
python - >> gpurun_out/peaks_fp64.txt 2>&1 << 'PY'
import torch, json
n = 8192
a = torch.randn(n, n, dtype=torch.float64, device="cuda"); b = torch.randn(n, n, dtype=torch.float64, device="cuda")
for _ in range(3): c = a @ b
torch.cuda.synchronize()
e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
best = 1e9
for _ in range(5):
    e0.record(); c = a @ b; e1.record(); torch.cuda.synchronize(); best = min(best, e0.elapsed_time(e1))
print(json.dumps({"kernel": "cublas_dgemm_8192", "tflops": 2 * n**3 / (best * 1e-3) / 1e12}))
PY
