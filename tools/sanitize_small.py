"""Small end-to-end workload for compute-sanitizer (memcheck / racecheck / synccheck):
tile kernels (TMA and cp.async paths, ragged), grouped launches, SYRK/TRSM diagonal ops and
logical-device forwarding."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import inputs
import paper_conf_sc_gautierl21_b200 as xk

m, n, k = 300, 260, 200
A, B, C0 = inputs.uniform(1, m, k), inputs.uniform(2, k, n), inputs.uniform(3, m, n)
xk.init(ngpus=2, phys=[0, 0], tile=128, probe=False)
C = C0.copy(order="F")
xk.dgemm("N", "N", m, n, k, 1.5, A, m, B, k, -0.75, C, m)
assert np.all(np.isfinite(C))  # numerics are checked by tests/; this drives the kernels
S = inputs.uniform(3, m, m)
xk.dsyrk("L", "N", m, k, 1.0, A, m, 0.5, S, m)
L = inputs.tri_dd(4, m, lower=True, fill=0.0)
X = inputs.uniform(5, m, n)
xk.dtrsm("L", "L", "N", "N", m, n, 1.0, L, m, X, m)
# the base kernel's other paths: right side (vectors = rows, loaded straight into registers),
# the multiply (TRMM), transposed / upper / unit triangles, odd orders (ragged leaves)
U = inputs.tri_dd(6, n, lower=False, fill=0.0)
xk.dtrsm("R", "U", "T", "U", m, n, 0.5, U, n, X, m)
xk.dtrmm("L", "U", "N", "N", m, n, 1.5, L.T.copy(order="F"), m, X, m)
xk.dtrmm("R", "L", "T", "N", m, n, 1.0, U.T.copy(order="F"), n, X, m)
Xo = inputs.uniform(7, 257, 131)
Lo = inputs.tri_dd(8, 257, lower=True, fill=0.0)
xk.dtrsm("L", "L", "N", "N", 257, 131, 1.0, Lo, 257, Xo, 257)
xk.finalize()
print("sanitize workload ok")
