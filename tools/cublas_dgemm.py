"""Context number for the FP64 roofline: cuBLAS DGEMM (torch.matmul on float64 CUDA tensors,
library code, not on the product path) at N = 8192 and 16384 on device-resident data, with the
nvidia-smi clocks sampled during the timed region.  Prints one JSON line."""
import json
import subprocess
import sys
import threading

import torch

out = {"device": torch.cuda.get_device_name(0), "torch": torch.__version__}
samples = []
proc = subprocess.Popen(["nvidia-smi", "--query-gpu=clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active",
                         "--format=csv,noheader", "-lms", "200"], stdout=subprocess.PIPE, text=True)
th = threading.Thread(target=lambda: [samples.append(ln.strip()) for ln in proc.stdout], daemon=True)
th.start()
for N in (8192, 16384):
    g = torch.Generator(device="cuda").manual_seed(0)
    A = torch.rand(N, N, dtype=torch.float64, device="cuda", generator=g)
    B = torch.rand(N, N, dtype=torch.float64, device="cuda", generator=g)
    C = torch.empty(N, N, dtype=torch.float64, device="cuda")
    for _ in range(2):
        torch.matmul(A, B, out=C)
    torch.cuda.synchronize()
    reps = 10 if N == 8192 else 3
    e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
    e0.record()
    for _ in range(reps):
        torch.matmul(A, B, out=C)
    e1.record()
    e1.synchronize()
    ms = e0.elapsed_time(e1) / reps
    out["N%d" % N] = {"ms": round(ms, 3), "tflops": round(2.0 * N ** 3 / (ms * 1e-3) / 1e12, 3)}
    del A, B, C
proc.terminate()
th.join(timeout=2)
out["clocks_samples"] = samples[-20:]
print(json.dumps(out))
