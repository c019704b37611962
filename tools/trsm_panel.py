"""Driver for ncu on the TRSM diagonal-tile ("panel") work: one data-on-device DTRSM
(left, lower, N, non-unit) at N=16384, T=2048 on one GPU."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import inputs
import paper_conf_sc_gautierl21_b200 as xk
N, T = int(os.environ.get("N", 16384)), int(os.environ.get("T", 2048))
L = inputs.tri_dd(4, N, lower=True, fill=0.0)
B = inputs.uniform(2, N, N)
xk.init(ngpus=1, tile=T, probe=False)
xk.register(L); xk.register(B)
for X in (L, B):
    xk.memory_prefetch_async(N, N, X, N)
xk.sync()
xk.dtrsm("L", "L", "N", "N", N, N, 1.0, L, N, B, N, asynchronous=True)
xk.sync()
xk.finalize()
print("trsm panel driver done")
