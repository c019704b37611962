"""examples/xk_dgemm_example.c run on the GPU: plain C through include/xk.h (sync + composed
async calls, argument error, exact-integer spot checks)."""
import subprocess

import pytest

pytestmark = pytest.mark.gpu


def test_c_example_runs():
    from tools.build_native import build_example
    exe = build_example()
    r = subprocess.run([exe], capture_output=True, text=True, timeout=300)
    assert r.returncode == 0, r.stderr
    assert "xk example ok" in r.stdout
