"""Standalone tile-kernel driver (ncu target): D = alpha*A*B + beta*C on T x T device tiles."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_sc_gautierl21_b200 as xk

T = int(sys.argv[1]) if len(sys.argv) > 1 else 2048
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 10
ta = sys.argv[3] if len(sys.argv) > 3 else "N"
tb = sys.argv[4] if len(sys.argv) > 4 else "N"
g = torch.Generator(device="cuda").manual_seed(0)
A = torch.rand(T * T, dtype=torch.float64, device="cuda", generator=g) * 2 - 1
B = torch.rand(T * T, dtype=torch.float64, device="cuda", generator=g) * 2 - 1
C = torch.rand(T * T, dtype=torch.float64, device="cuda", generator=g) * 2 - 1
s = torch.cuda.current_stream().cuda_stream
for _ in range(3):
    xk.dgemm_tile_device(ta, tb, T, T, T, 1.5, A, T, B, T, 1.0, C, T, s)
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
e0.record()
for _ in range(reps):
    xk.dgemm_tile_device(ta, tb, T, T, T, 1.5, A, T, B, T, 1.0, C, T, s)
e1.record(); torch.cuda.synchronize()
ms = e0.elapsed_time(e1) / reps
print("tile %s%s T=%d: %.3f ms/launch  %.2f TFLOP/s" % (ta, tb, T, ms, 2 * T ** 3 / ms / 1e9))
