"""Timing fidelity of the planner's virtual-time model (reading Q17).

The planner places every record at an integer-ns virtual time from the link matrix and the
grouped-launch task rate the runtime measures at xk_init.  Its byte counts are pinned exactly
elsewhere; here its makespan is compared with the wall time of the same synchronous
host-resident call on one GPU -- the configuration whose resources (one compute engine, one
H2D and one D2H link) are the model's own.  Measured with the default window W = 4 on a B200:
predicted / measured time 1.01-1.08 over every routine at N = 32768 and DGEMM at N = 16384
(profiles/r02_model_fidelity.jsonl); the bound below leaves room for box-to-box variation.
"""
import time

import pytest
import torch

import inputs
import paper_conf_sc_gautierl21_b200 as xk
from tools.model_fidelity import flops, model_call, user_call

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("name", ["dgemm", "dtrsm"])
def test_model_makespan_matches_one_gpu_call(name):
    N, T = 16384, 2048
    M = [inputs.uniform(1, N, N), inputs.uniform(2, N, N), inputs.uniform(3, N, N),
         inputs.tri_dd(4, N, lower=True, fill=0.0)]
    xk.init(ngpus=1, tile=T, probe=True)
    try:
        for X in M:
            xk.register(X)
        topo = xk.get_topology()
        user_call(name, N, M)  # warm-up
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        for _ in range(2):
            user_call(name, N, M)
        torch.cuda.synchronize()
        meas = (time.perf_counter() - t0) / 2
    finally:
        xk.finalize()
    recs = xk.plan_dump(model_call(name, N, M), topo["bw_MBps"], rate_mflops=topo["task_rate_mflops"],
                        tile=T, cap=1 << 20)
    pred = max(r[12] for r in recs) * 1e-9
    ratio = pred / meas
    print("%s N=%d: measured %.2f, model %.2f TFLOP/s (pred/meas time %.3f)"
          % (name, N, flops(name, N) / meas / 1e12, flops(name, N) / pred / 1e12, ratio))
    assert 0.88 <= ratio <= 1.12, ratio
