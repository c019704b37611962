"""Hardware probe (not the product path): host/PCIe/cuBLAS context numbers for DESIGN.md."""
import os, time, subprocess, json
import torch
out = {}
out["cores"] = len(os.sched_getaffinity(0))
def sh(c):
    try: return subprocess.run(c, shell=True, capture_output=True, text=True, timeout=60).stdout
    except Exception as e: return str(e)
print(sh("lscpu | head -25; free -g; nvidia-smi; nvidia-smi topo -m; nvidia-smi -q -d CLOCK,POWER | head -60"))
dev = torch.device("cuda:0")
# cuBLAS DGEMM context (library, not product)
for n in (4096, 8192):
    a = torch.randn(n, n, dtype=torch.float64, device=dev); b = torch.randn_like(a)
    for _ in range(3): c = a @ b
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
    e0.record()
    for _ in range(10): c = a @ b
    e1.record(); torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / 10
    print(f"cuBLAS DGEMM n={n}: {ms:.2f} ms {2*n**3/ms/1e9:.2f} TFLOP/s")
# pinned H2D/D2H
for mb in (32, 256, 1024):
    n = mb * 2**20 // 8
    h = torch.empty(n, dtype=torch.float64).pin_memory(); d = torch.empty(n, dtype=torch.float64, device=dev)
    for _ in range(2): d.copy_(h, non_blocking=True)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
    e0.record()
    for _ in range(5): d.copy_(h, non_blocking=True)
    e1.record(); torch.cuda.synchronize()
    h2d = 5 * n * 8 / e0.elapsed_time(e1) / 1e6
    e0.record()
    for _ in range(5): h.copy_(d, non_blocking=True)
    e1.record(); torch.cuda.synchronize()
    d2h = 5 * n * 8 / e0.elapsed_time(e1) / 1e6
    print(f"pinned {mb} MiB: H2D {h2d:.1f} GB/s D2H {d2h:.1f} GB/s")
